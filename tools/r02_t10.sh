set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4
ENVS="X=0" WLS="rmat22 uniform road dense grid64" REPS=2 bash tools/envab.sh
TOOLS="racecheck" TMO=1500 bash tools/sanitize.sh
