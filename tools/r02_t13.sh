set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
timeout 1500 python -m pytest tests/test_dist_procs_gpu.py tests/test_parity_gpu.py -m gpu -q -x -k "dist or small or grid64 or random_multigraphs or many_components" 2>&1 | tail -3
LIBS="tr1 tr0" WLS="rmat22 uniform road" REPS=2 bash tools/abrun2.sh
ENVS="X=0" WLS="grid64" REPS=3 bash tools/envab.sh
