set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
timeout 1200 python -m pytest tests/test_parity_gpu.py -m gpu -q -x -k "small or grid64 or golden or tiny or empty or dense_rounds or transition" 2>&1 | tail -3
ENVS="X=0" WLS="grid64" REPS=3 bash tools/envab.sh
bash tools/modes.sh
bash tools/layouts.sh
