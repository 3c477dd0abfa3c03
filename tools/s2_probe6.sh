# streamed host-input build: parity, e2e A/B; then a source-level ncu capture of RMAT-22's passes
timeout 1200 python -m pytest tests/test_parity_gpu.py -q -x -k "host" 2>&1 | tail -3
for rep in 1 2; do
for hs in 0 1; do for w in rmat22 road uniform; do MST_HOST_STREAM=$hs timeout 300 python tools/e2e_probe.py $w 3 2>&1 | tail -1; done; done
done
MST_TRACE_BUILD=1 timeout 300 python tools/e2e_probe.py rmat22 1 2>&1 | grep build | tail -9
timeout 300 python bench.py --workload rmat22 --steps 10 --e2e-steps 3 --no-oracle > gpurun_out/p6_rmat22.json 2> gpurun_out/p6_rmat22.err
python -c "import json; d=json.load(open('gpurun_out/p6_rmat22.json')); print(d['value']/1e9, d['e2e'])"
WL=rmat22 RE='arc_pass' timeout 900 bash tools/profile_src.sh
ls -la gpurun_out | tail -5
