# A/B of environment knobs on one library build, same box: ENVS="A=1;B=2" WLS="rmat22" REPS=2
IFS=';' read -ra GROUPS_ <<< "${ENVS:-X=0}"
for rep in $(seq ${REPS:-2}); do
  for wl in ${WLS:-rmat22}; do
    for grp in "${GROUPS_[@]}"; do
      env $grp timeout 300 python bench.py --steps ${STEPS:-10} --warmup 3 --e2e-steps 0 --no-oracle --workload $wl --mode ${MODE:-morph} ${BARGS} > /tmp/eab.json 2> /tmp/eab.err
      python - "$grp" "$wl" <<'PY'
import json, sys
g, wl = sys.argv[1], sys.argv[2]
try:
    d = json.load(open("/tmp/eab.json"))
    lk = d.get("launch_kinds", {})
    ks = " ".join(f"{k}={x['ms_per_step']*1e3:.0f}" for k, x in lk.items() if x["ms_per_step"] > 0.02)
    rs = " ".join(f"r{r['r']}:{r['n_r']}" for r in d["rounds"])
    print(f"[{g:24s}] {wl:7s} {d['value']/1e9:7.3f} G/s {d['ms_per_step']:.4f} ms  frac {d['roofline']['frac'] or 0:.3f}  {ks}  | {rs}")
except Exception as e:
    print(f"[{g}] {wl} failed: {e}", open("/tmp/eab.err").read()[-600:])
PY
    done
  done
done
