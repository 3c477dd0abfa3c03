# launch list (cold-cache, serialised; compare SHARES) + one full capture of the RMAT-22 step
WL=${WL:-rmat22}
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$WL.csv \
    python bench.py --workload $WL --steps 2 --warmup 3 --e2e-steps 0 --no-oracle > /dev/null 2>&1
# warmup 3 + 1 timed step: skip the warmup runs' launches of the captured kernels
ncu --set full --clock-control none --import-source on \
    -k regex:"arc_pass|k_hook|k_jump|k_dense|k_output|k_sample|k_compose" -s 45 -c 15 \
    -o gpurun_out/full_$WL python bench.py --workload $WL --steps 1 --warmup 3 --e2e-steps 0 --no-oracle \
    > gpurun_out/ncu_full_$WL.log 2>&1
tail -1 gpurun_out/ncu_full_$WL.log
