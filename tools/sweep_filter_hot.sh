#!/bin/bash
# MST_FILTER_HOT re-check on the final code (bench.py --no-oracle, 10 steps each); run under gpurun
# from the repo root: mkdir -p gpurun_out/sweep; bash tools/sweep_filter_hot.sh
mkdir -p gpurun_out/sweep
for wl in uniform road rmat22; do
  for h in def 6144 8192; do
    if [ $h = def ]; then unset MST_FILTER_HOT; else export MST_FILTER_HOT=$h; fi
    timeout 300 python bench.py --workload $wl --no-oracle --e2e-steps 0 > gpurun_out/sweep/${wl}_$h.json 2>/dev/null
    python -c "import json,sys; d=json.load(open('gpurun_out/sweep/${wl}_$h.json')); print('$wl','$h',round(d['ms_per_step'],4), d['kernel_ms_per_step']['filter'])"
  done
done
unset MST_FILTER_HOT
