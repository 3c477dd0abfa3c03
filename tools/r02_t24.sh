python -c "import __graft_entry__ as g; g.build()" > /dev/null
for w in rmat22 dense uniform road; do
  for e in "X=0" "MST_SOLVE_REORDER=1"; do
    env $e timeout 300 python tools/e2e_probe.py $w 5 2>&1 | tail -1
  done
  MST_TRACE_BUILD=1 timeout 300 python tools/e2e_probe.py $w 1 2>&1 | tail -40 | head -20
done
