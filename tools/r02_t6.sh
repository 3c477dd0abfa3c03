set -x
MST_DEBUG_MEMBER=1 python tools/dbg_member.py 2>&1 | grep -v phi | tail -12; rm -f gpurun_out/phi.bin
ENVS="X=0;MST_MEMBER_SCAN=0" WLS="rmat22" REPS=2 bash tools/envab.sh
timeout 1500 python -m pytest tests/test_parity_gpu.py -m gpu -q -k "member or light or config or full_size or dense" 2>&1 | tail -3
