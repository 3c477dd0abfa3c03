# member-scan decision without the 32-hub gate (MST_HUBGATE=0), light threshold sweep
run() { timeout 300 python bench.py --workload rmat22 --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p2_$1.json 2> gpurun_out/p2_$1.err; python tools/bsum.py gpurun_out/p2_$1.json | grep -v '^   [a-z]'; }
run base
MST_HUBGATE=0 run g0
MST_HUBGATE=0 MST_LIGHT_T=30 run g0t30
MST_HUBGATE=0 MST_LIGHT_T=60 run g0t60
MST_HUBGATE=0 MST_LIGHT_T=90 run g0t90
MST_HUBGATE=0 MST_DEBUG_MEMBER=1 timeout 300 python bench.py --workload rmat22 --steps 1 --warmup 3 --e2e-steps 0 --no-oracle > /dev/null 2> gpurun_out/p2_member.err
grep -v phi gpurun_out/p2_member.err | grep round | tail -8
