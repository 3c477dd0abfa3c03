run() { timeout 300 python bench.py --workload dense --seed $2 --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p24_$1_$2.json 2>/dev/null; python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], round(d['value']/1e9,2), d['light_phase'])" gpurun_out/p24_$1_$2.json "$1 seed$2"; }
for s in 0 1 2 3 4; do run auto12 $s; done
timeout 1200 python -m pytest tests/test_parity_gpu.py -q -x -k "full_size or dense or light" 2>&1 | tail -1
timeout 300 python bench.py --workload dense --steps 10 --e2e-steps 0 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('dense seed0 parity', d['parity'], round(d['value']/1e9,2))"
