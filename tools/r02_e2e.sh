python -c "import __graft_entry__ as g; g.build()" > /dev/null
for w in rmat22 dense uniform road; do
  for e in "X=0" "MST_REORDER=1" "MST_REORDER=0" "MST_MEMBER_SCAN=0" "MST_ADJ_DEDUP=0"; do
    env $e timeout 300 python tools/e2e_probe.py $w 3 2>&1 | tail -1
  done
done
