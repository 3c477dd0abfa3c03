timeout 1800 python -m pytest tests/test_parity_gpu.py tests/test_knobs_gpu.py -q -x 2>&1 | tail -2
run() { timeout 300 python bench.py --workload $2 --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p15_$1_$2.json 2>/dev/null; python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], sys.argv[3], round(d['value']/1e9,3), d['light_phase'])" gpurun_out/p15_$1_$2.json $2 $1; }
for rep in 1 2 3; do run new rmat22; MST_LIGHT_T=54 run t54 rmat22; run new dense; done
