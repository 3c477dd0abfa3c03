set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 2400 python -m pytest tests -m gpu -q -x -p no:randomly 2>&1 | tail -25
for w in rmat22 uniform road dense grid64; do
  timeout 600 python bench.py --workload $w --mode uf --e2e-steps 0 > gpurun_out/uf_$w.json 2> gpurun_out/uf_$w.err
  python tools/bsum.py gpurun_out/uf_$w.json | head -3; tail -3 gpurun_out/uf_$w.err
done
