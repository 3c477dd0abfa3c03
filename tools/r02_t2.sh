set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
timeout 1500 python -m pytest tests/test_parity_gpu.py -m gpu -q -x -k "small or grid64 or golden or tiny or empty" 2>&1 | tail -5
for w in grid64 rmat22; do
  timeout 600 python bench.py --workload $w --e2e-steps 1 > gpurun_out/b2_$w.json 2> gpurun_out/b2_$w.err
  python tools/bsum.py gpurun_out/b2_$w.json 2>/dev/null | head -14
done
WL=rmat22 timeout 900 bash tools/profile_src.sh
ls -la gpurun_out
