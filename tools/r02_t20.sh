set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
MST_DEBUG_MEMBER=1 timeout 300 python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-oracle --workload rmat22 2>&1 | grep -E "light round|member" | head -4
timeout 1500 python -m pytest tests/test_parity_gpu.py tests/test_dist_procs_gpu.py tests/test_knobs_gpu.py -m gpu -q -x 2>&1 | tail -3
ENVS="X=0;MST_HYBRID=1" WLS="rmat22" REPS=3 bash tools/envab.sh
