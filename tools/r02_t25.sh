python -c "import __graft_entry__ as g; g.build(); g.smoke()"
for w in rmat22 dense uniform road; do
  for e in "X=0" "MST_SOLVE_REORDER=0" "MST_HOST_ZEROCOPY=1"; do
    env $e timeout 300 python tools/e2e_probe.py $w 5 2>&1 | tail -1
  done
  MST_TRACE_BUILD=1 timeout 300 python tools/e2e_probe.py $w 1 2>&1 | grep build | tail -8
done
timeout 1500 python -m pytest tests/test_parity_gpu.py tests/test_abi.py -m gpu -q -x 2>&1 | tail -2
ENVS="X=0" WLS="rmat22 uniform road dense grid64" REPS=1 bash tools/envab.sh
