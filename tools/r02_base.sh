# round-2 baseline: every workload's bench line + full ncu capture per workload
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()"
for w in rmat22 uniform road dense grid64; do
  timeout 600 python bench.py --workload $w --e2e-steps 1 > gpurun_out/b0_$w.json 2> gpurun_out/b0_$w.err
  python -c "
import json
d=json.load(open('gpurun_out/b0_$w.json'))
print('$w', 'value %.3f G/s'%(d['value']/1e9), 'ms %.3f'%d['ms_per_step'], 'frac %.3f'%(d['roofline']['frac'] or 0), d['parity'], 'clk', d['clocks']['sm_mhz'], d['clocks']['reasons'])
print({k: round(v,4) for k,v in d['kernel_ms_per_step'].items()})
for r in d['rounds']: print(r['r'], r['kind'], r['n_r'], r['A_r'], r['compacted'], round(r['filter_ms'],4), r['frac'])
" 2>&1 | tail -30
done
for w in rmat22 uniform road; do WL=$w timeout 900 bash tools/profile.sh; done
ls -la gpurun_out
