python -c "import __graft_entry__ as g; g.build(); g.smoke()"
for w in rmat22 dense uniform road grid64; do
  for e in "X=0" "MST_SOLVE_REORDER=0"; do
    env $e timeout 300 python tools/e2e_probe.py $w 5 2>&1 | tail -1
  done
done
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
for w in rmat22 uniform; do timeout 600 python bench.py --workload $w > gpurun_out/t26_bench_$w.json 2> /dev/null; python tools/bsum.py gpurun_out/t26_bench_$w.json | head -3; done
