# NEXT-4 evidence: caller numbering (0) vs hub-first (1) vs BFS order (2): bench lines and the
# label-gather hit rates (ncu L1 / L2 sector hit rates of the A8 passes of one mst_run)
for w in ${WLS:-road uniform rmat22}; do
  for L in 0 1 2; do
    MST_REORDER=$L timeout 600 python bench.py --workload $w --e2e-steps 0 --no-oracle --steps 10 \
        > gpurun_out/layout${L}_$w.json 2> gpurun_out/layout${L}_$w.err
    MST_REORDER=$L timeout 900 ncu --metrics gpu__time_duration.sum,l1tex__t_sector_hit_rate.pct,lts__t_sector_hit_rate.pct,lts__t_requests.sum,dram__bytes_read.sum \
        --clock-control none -k regex:arc_pass --csv --log-file gpurun_out/layout${L}_$w.csv \
        python bench.py --workload $w --e2e-steps 0 --no-oracle --steps 1 --warmup 3 > /dev/null 2>&1
    python - "$L" "$w" <<'PY'
import json, sys, csv
L, w = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/layout{L}_{w}.json"))
    print(f"{w:7s} layout {L}: {d['value']/1e9:8.3f} G/s {d['ms_per_step']:.4f} ms  build {d['config']['build_ms']:.0f} ms  A8 frac {d['roofline_kernels']['A8 filter']['frac'] or 0:.3f}")
except Exception as e:
    print(w, L, "failed", e, open(f"gpurun_out/layout{L}_{w}.err").read()[-400:])
PY
  done
done
