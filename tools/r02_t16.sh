set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
timeout 1500 python -m pytest tests/test_parity_gpu.py tests/test_dist_procs_gpu.py -m gpu -q -x -k "member or light or config or full_size or dense or dist" 2>&1 | tail -3
ENVS="X=0" WLS="rmat22 uniform road dense" REPS=2 bash tools/envab.sh
