python -c "import __graft_entry__ as g; g.build(); g.smoke()"
timeout 1500 python -m pytest tests/test_parity_gpu.py tests/test_dist_procs_gpu.py -m gpu -q -x -k "member or light or full_size or dist or single" 2>&1 | tail -2
for w in rmat22 dense uniform road; do timeout 300 python tools/e2e_probe.py $w 5 2>&1 | tail -1; done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_e2e_rmat22.csv python tools/e2e_probe.py rmat22 1 > /dev/null 2>&1
python tools/launch_share.py gpurun_out/launches_e2e_rmat22.csv 5 | head -24
