# fused light minima in the extraction pass (MST_EXMIN) A/B + parity; e2e build trace
run() { timeout 300 python bench.py --workload $2 --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p5_$1_$2.json 2> gpurun_out/p5_$1_$2.err; python tools/bsum.py gpurun_out/p5_$1_$2.json | grep -v '^   [a-z]'; }
for w in rmat22 dense; do for rep in 1 2 3; do for x in 0 1 2; do MST_EXMIN=$x run x$x $w; done; done; done
python tools/bsum.py gpurun_out/p5_x1_rmat22.json | head -16
timeout 900 python -m pytest tests/test_knobs_gpu.py -q -x -k "EXMIN or LIGHT" 2>&1 | tail -3
timeout 1200 python -m pytest tests/test_parity_gpu.py -q -x 2>&1 | tail -3
MST_TRACE_BUILD=1 timeout 300 python tools/e2e_probe.py rmat22 3 2>&1 | tail -40
