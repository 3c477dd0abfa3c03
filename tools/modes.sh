# NEXT-2 / NEXT-3 / A9 evidence: one bench line per (mode, workload) on this box
for w in ${WLS:-rmat22 uniform road dense grid64}; do
  for mode in ${MODES:-morph sparse keep uf dedup}; do
    timeout 600 python bench.py --workload $w --mode $mode --e2e-steps 0 --no-oracle --steps ${STEPS:-10} \
        > gpurun_out/mode_${mode}_$w.json 2> gpurun_out/mode_${mode}_$w.err
    python - "$mode" "$w" <<'PY'
import json, sys
m, w = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/mode_{m}_{w}.json"))
    print(f"{w:7s} {m:7s} {d['value']/1e9:8.3f} G/s {d['ms_per_step']:.4f} ms  A8 frac {d['roofline_kernels']['A8 filter']['frac'] or 0:.3f}  rounds {d['config']['rounds']}")
except Exception as e:
    print(w, m, "failed", e, open(f"gpurun_out/mode_{m}_{w}.err").read()[-500:])
PY
  done
done
