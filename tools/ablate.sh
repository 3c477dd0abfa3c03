# usage: ENVS="A=1 B=2;C=3" bash tools/ablate.sh   (each ;-separated group is one run)
IFS=';' read -ra GROUPS_ <<< "${ENVS:-X=0}"
for grp in "${GROUPS_[@]}"; do
  env $grp timeout 300 python bench.py --steps ${STEPS:-5} --warmup 3 --e2e-steps 0 --no-oracle --workload ${WL:-rmat22} --mode ${MODE:-morph} ${BARGS} > /tmp/ab.json 2> /tmp/ab.err
  python -c "
import json,sys
try:
    d=json.load(open('/tmp/ab.json'))
    print('[$grp] ${WL:-rmat22} value %.3f G/s ms/step %.3f frac %.3f'%(d['value']/1e9, d['ms_per_step'], d['roofline']['frac']), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items() if v})
    for r in d['rounds']: print('   r%d %s n=%d A=%d %.3f ms %.0f GB/s comp=%s surv=%s'%(r['r'], r['kind'], r['n_r'], r['A_r'], r['filter_ms'], r['filter_GBps'] or 0, r.get('compacted'), r.get('survival_permille')))
except Exception as e:
    print('[$grp] failed', open('/tmp/ab.err').read()[-400:])
"
done
