timeout 1800 python -m pytest tests/test_parity_gpu.py tests/test_knobs_gpu.py tests/test_dist_procs_gpu.py -q -x 2>&1 | tail -2
run() { timeout 300 python bench.py --workload $2 --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p12_$1_$2.json 2>/dev/null; python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], sys.argv[3], round(d['value']/1e9,3))" gpurun_out/p12_$1_$2.json $2 $1; }
for w in rmat22 road uniform dense; do for rep in 1 2 3; do
  MST_HJ1_MAX=0 run hj0 $w; run hj1 $w
done; done
for rep in 1 2 3; do for t in 0 1 2; do MST_TX_DEDUP=$t run tx$t uniform; done; done
for rep in 1 2; do for t in 1 2; do MST_TX_DEDUP=$t run tx$t rmat22; MST_TX_DEDUP=$t run tx$t road; done; done
python tools/bsum.py gpurun_out/p12_hj1_rmat22.json | head -22
