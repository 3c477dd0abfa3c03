# interleaved A/B of build/ab/<variant>.so: VARIANTS="a b" WLS="rmat22 road" REPS=3 bash tools/s2_ab.sh
for wl in ${WLS:-rmat22 road uniform dense}; do
  for rep in $(seq ${REPS:-3}); do
    for v in ${VARIANTS}; do
      lib=build/ab/$v.so; [ "$v" = "." ] && lib=""
      MST_LIB=$lib timeout 300 python bench.py --workload $wl --steps ${STEPS:-10} --e2e-steps 0 --no-oracle > gpurun_out/ab_${v}_${wl}_$rep.json 2>/dev/null
      python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], sys.argv[3], round(d['value']/1e9,3), round(d['ms_per_step'],4))" gpurun_out/ab_${v}_${wl}_$rep.json $wl $v
    done
  done
done 2>&1 | tee gpurun_out/ab_summary.txt
python - <<'PY'
import collections, statistics
d = collections.defaultdict(list)
for l in open("gpurun_out/ab_summary.txt"):
    p = l.split()
    if len(p) == 4: d[(p[0], p[1])].append(float(p[2]))
for k, v in sorted(d.items()): print(k, "median", statistics.median(v), v)
PY
