# light-phase compaction knob: parity + A/B on rmat22 / dense
timeout 900 python -m pytest tests/test_knobs_gpu.py -q -x -k LIGHT_COMPACT 2>&1 | tail -3
run() { timeout 300 python bench.py --workload $2 --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p3_$1_$2.json 2> gpurun_out/p3_$1_$2.err; python tools/bsum.py gpurun_out/p3_$1_$2.json | grep -v '^   [a-z]'; }
for rep in 1 2; do
for lc in 0 1 2 3; do MST_LIGHT_COMPACT=$lc run lc$lc rmat22; done
done
python tools/bsum.py gpurun_out/p3_lc2_rmat22.json
for lc in 0 2; do MST_LIGHT_COMPACT=$lc run lc$lc dense; done
