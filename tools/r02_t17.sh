set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
MST_DEBUG_MEMBER=1 timeout 300 python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-oracle --workload rmat22 2>&1 | grep -E "light round|member" | head -30
timeout 1500 python -m pytest tests/test_parity_gpu.py -m gpu -q -x -k "member or light or full_size" 2>&1 | tail -3
ENVS="X=0" WLS="rmat22 uniform" REPS=2 bash tools/envab.sh
