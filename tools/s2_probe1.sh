# hook warp-aggregated forest bits; member-decision trace on RMAT-22
for w in road rmat22 uniform; do
  timeout 600 python bench.py --workload $w --e2e-steps 0 --no-oracle > gpurun_out/p1_$w.json 2> gpurun_out/p1_$w.err
  python tools/bsum.py gpurun_out/p1_$w.json | head -40
done
MST_DEBUG_MEMBER=1 timeout 300 python bench.py --workload rmat22 --steps 1 --warmup 3 --e2e-steps 0 --no-oracle > /dev/null 2> gpurun_out/p1_member.err
grep -v phi gpurun_out/p1_member.err | grep -i 'round' | head -20
