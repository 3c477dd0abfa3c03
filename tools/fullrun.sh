set -x
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -3
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap --format=csv -lms 200 > gpurun_out/clocks_full.csv &
CPID=$!
timeout 900 python bench.py > gpurun_out/bench_rmat22.json 2> gpurun_out/bench_rmat22.err
kill $CPID
for w in grid64 uniform road dense; do timeout 600 python bench.py --workload $w --no-oracle --e2e-steps 1 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err; done
tail -c 600 gpurun_out/bench_rmat22.json
