for v in ${VARIANTS:-0 9}; do
  MST_FILTER_VARIANT=$v timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-oracle > /tmp/ab_$v.json 2> /tmp/ab_$v.err
  python -c "
import json,sys
try:
    d=json.load(open('/tmp/ab_$v.json'))
    print('variant $v value %.3f G/s ms/step %.3f frac %.3f'%(d['value']/1e9, d['ms_per_step'], d['roofline']['frac']), 'min0 %.3f'%d['kernel_ms_per_step']['min0'])
    for r in d['rounds']: print('   r%d A=%d filter %.3f ms %.0f GB/s'%(r['r'], r['A_r'], r['filter_ms'], r['filter_GBps'] or 0))
except Exception as e:
    print('variant $v failed', open('/tmp/ab_$v.err').read()[-400:])
"
done
