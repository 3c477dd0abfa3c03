# launch list (cold-cache, serialised; compare SHARES) + one full capture of the hot kernels
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-oracle > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"arc_pass|k_hook|k_jump|k_dense_round|k_output" \
    -s 30 -c 10 -o gpurun_out/full python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-oracle > gpurun_out/ncu_full.log 2>&1
tail -1 gpurun_out/ncu_full.log
python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 300 gpurun_out/bench.json
