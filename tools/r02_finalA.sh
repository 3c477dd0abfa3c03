# round-2 final evidence, part A: tests, ncu launch lists + DRAM traffic, full bench lines
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4 | tee gpurun_out/final_gpu_tests.log
for w in rmat22 uniform road dense grid64; do WL=$w timeout 900 bash tools/profile.sh; done
for w in rmat22 uniform road dense grid64; do
  timeout 900 python bench.py --workload $w --e2e-steps 3 > gpurun_out/final_bench_$w.json 2> gpurun_out/final_bench_$w.err
  python tools/bsum.py gpurun_out/final_bench_$w.json | head -30
done
timeout 900 python bench.py --impl reference --workload rmat22 --steps 3 --warmup 1 > gpurun_out/final_reference_rmat22.json 2>&1
ls -la gpurun_out | head -80
