# session-2 re-baseline: smoke, GPU tests, bench lines for every config
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -4 | tee gpurun_out/s2_gpu_tests.log
for w in rmat22 uniform road dense grid64; do
  timeout 600 python bench.py --workload $w --e2e-steps 3 > gpurun_out/s2_bench_$w.json 2> gpurun_out/s2_bench_$w.err
  python tools/bsum.py gpurun_out/s2_bench_$w.json | head -40
done
