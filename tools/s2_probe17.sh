timeout 1800 python -m pytest tests/test_parity_gpu.py -q -x 2>&1 | tail -2
MST_LIGHT_COMPACT=2 timeout 1800 python -m pytest tests/test_parity_gpu.py -q -x -k "full_size or tie or random or light or member" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_knobs_gpu.py -q -x -k "LIGHT" 2>&1 | tail -2
for wl in rmat22 road uniform dense; do for rep in 1 2 3; do
  for v in head smap smapLC2; do
    lib=build/ab/$v.so; lc=0; [ "$v" = "smapLC2" ] && { lib=build/ab/smap.so; lc=2; }
    MST_LIB=$lib MST_LIGHT_COMPACT=$lc timeout 300 python bench.py --workload $wl --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p17_${v}_${wl}_$rep.json 2>/dev/null
    python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], sys.argv[3], round(d['value']/1e9,3))" gpurun_out/p17_${v}_${wl}_$rep.json $wl $v
  done
done; done | tee gpurun_out/p17_summary.txt
python - <<'PY'
import collections, statistics
d = collections.defaultdict(list)
for l in open("gpurun_out/p17_summary.txt"):
    p = l.split()
    if len(p) == 3: d[(p[0], p[1])].append(float(p[2]))
for k, v in sorted(d.items()): print(k, "median", statistics.median(v), v)
PY
python tools/bsum.py gpurun_out/p17_smapLC2_rmat22_1.json | head -24
