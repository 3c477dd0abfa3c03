# A/B of prebuilt variants (build/ab/<name>.so) on several workloads, same box, REPS rounds
# usage: LIBS="base v1 v2" WLS="rmat22 road" REPS=2 bash tools/abrun2.sh
for rep in $(seq ${REPS:-2}); do
  for wl in ${WLS:-rmat22}; do
    for v in ${LIBS:-base}; do
      MST_LIB=$(pwd)/build/ab/$v.so timeout 300 python bench.py --steps ${STEPS:-10} --warmup 3 --e2e-steps 0 --no-oracle --workload $wl --mode ${MODE:-morph} ${BARGS} > /tmp/ab_$v.json 2> /tmp/ab_$v.err
      python - "$v" "$wl" <<'PY'
import json, sys
v, wl = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"/tmp/ab_{v}.json"))
    lk = d.get("launch_kinds", {})
    ks = " ".join(f"{k}={x['ms_per_step']*1e3:.0f}" for k, x in lk.items() if x["ms_per_step"] > 0.02)
    print(f"[{v:10s}] {wl:7s} {d['value']/1e9:7.3f} G/s {d['ms_per_step']:.4f} ms  frac {d['roofline']['frac'] or 0:.3f}  {d['parity']}  {ks}")
except Exception as e:
    print(f"[{v}] {wl} failed: {e}", open(f"/tmp/ab_{v}.err").read()[-600:])
PY
    done
  done
done
