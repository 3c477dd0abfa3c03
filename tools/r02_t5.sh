set -x
python -c "import __graft_entry__ as g; g.build()"
MST_DEBUG_MEMBER=1 python tools/dbg_member.py 2>&1 | grep -v phi | tail -8; rm -f gpurun_out/phi.bin
timeout 1500 python -m pytest tests/test_parity_gpu.py -m gpu -q -k "member or light or config or full_size or dense" 2>&1 | tail -6
ENVS="X=0;MST_MEMBER_SCAN=0" WLS="rmat22 dense" REPS=2 bash tools/envab.sh
