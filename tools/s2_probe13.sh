timeout 1800 python -m pytest tests/test_parity_gpu.py -q -x 2>&1 | tail -2
run() { timeout 300 python bench.py --workload rmat22 --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p13_$1.json 2>/dev/null; python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], round(d['value']/1e9,3), d['light_phase'])" gpurun_out/p13_$1.json $1; }
for rep in 1 2 3; do run auto; MST_LIGHT_T=36 run t36; MST_LIGHT_T=56 run t56; MST_LIGHT_T=70 run t70; done
