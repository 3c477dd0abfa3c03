# round-2 final evidence (session 2): smoke, every GPU test, ncu launch lists + DRAM traffic +
# raw metric exports per workload, full bench lines, the reference arm
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1 | tee gpurun_out/f2_smoke.log
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4 | tee gpurun_out/f2_gpu_tests.log
for w in rmat22 uniform road dense grid64; do WL=$w timeout 900 bash tools/profile.sh; done
for w in rmat22 uniform road dense grid64; do
  timeout 900 python bench.py --workload $w --e2e-steps 3 > gpurun_out/f2_bench_$w.json 2> gpurun_out/f2_bench_$w.err
  python tools/bsum.py gpurun_out/f2_bench_$w.json | head -3
done
timeout 900 python bench.py --impl reference --workload rmat22 --steps 3 --warmup 3 > gpurun_out/f2_reference_rmat22.json 2>&1
ls -la gpurun_out | wc -l
