set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
timeout 1500 python -m pytest tests/test_parity_gpu.py tests/test_dist_procs_gpu.py -m gpu -q -x -k "member or light or full_size or dist or single" 2>&1 | tail -3
ENVS="X=0;MST_HYBRID=1" WLS="rmat22" REPS=3 bash tools/envab.sh
