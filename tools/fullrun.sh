# round-end evidence: GPU tests, every workload's full bench line (oracle parity, cpu_baseline,
# e2e), the launch list and one full ncu capture of the RMAT-22 step (see tools/profile.sh)
set -x
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -3
for w in rmat22 grid64 uniform road dense; do
  timeout 900 python bench.py --workload $w > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
  python -c "
import json
d=json.load(open('gpurun_out/bench_$w.json'))
print('$w', 'value %.3f G/s'%(d['value']/1e9), 'ms %.3f'%d['ms_per_step'], 'frac %.3f'%(d['roofline']['frac'] or 0), d['parity'], 'e2e %.3f G/s'%(d['e2e']['value']/1e9), 'cpu %.2f M/s'%(d['cpu_baseline']['value']/1e6), 'clk', d['clocks']['sm_mhz'], d['clocks']['reasons'])
" 2>&1 | tail -1
done
bash tools/profile.sh
