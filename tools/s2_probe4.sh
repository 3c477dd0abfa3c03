# PASS_YAGG A/B + parity
run() { timeout 300 python bench.py --workload $2 --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p4_$1_$2.json 2> gpurun_out/p4_$1_$2.err; python tools/bsum.py gpurun_out/p4_$1_$2.json | grep -v '^   [a-z]'; }
for w in rmat22 dense; do for rep in 1 2; do for y in 0 1 2; do MST_YAGG=$y run y$y $w; done; done; done
for w in uniform road; do for rep in 1 2; do for y in 0 2; do MST_YAGG=$y run y$y $w; done; done; done
python tools/bsum.py gpurun_out/p4_y1_rmat22.json
timeout 900 python -m pytest tests/test_knobs_gpu.py -q -x -k "YAGG or LIGHT" 2>&1 | tail -3
timeout 1200 python -m pytest tests/test_parity_gpu.py -q -x 2>&1 | tail -3
