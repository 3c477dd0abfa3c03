python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -2
for rep in 1 2; do for w in rmat22 road; do timeout 300 python bench.py --workload $w --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/v_$w.json 2>/dev/null; python tools/bsum.py gpurun_out/v_$w.json | head -1; done; done
