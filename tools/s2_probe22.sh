run() { timeout 300 python bench.py --workload dense --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p22_$1.json 2>/dev/null; python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], round(d['value']/1e9,2), d['light_phase'], d['rounds'][0]['A_r'])" gpurun_out/p22_$1.json $1; }
for rep in 1 2 3; do run auto; for t in 3 4 5 8; do MST_LIGHT_T=$t run t$t; done; done
