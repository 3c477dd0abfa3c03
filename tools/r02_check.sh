# build + GPU tests + every workload's bench line + arc-pass profiles of three workloads
set -x
python -c "import __graft_entry__ as g; g.build()"
python -c "import __graft_entry__ as g; g.smoke()"
timeout 1800 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
for w in rmat22 uniform road dense grid64; do
  timeout 600 python bench.py --workload $w --e2e-steps 1 > gpurun_out/b1_$w.json 2> gpurun_out/b1_$w.err
  python tools/bsum.py gpurun_out/b1_$w.json
done
for w in ${PROF_WL:-rmat22 uniform road}; do WL=$w timeout 900 bash tools/profile.sh; done
du -sh gpurun_out; ls -la gpurun_out
