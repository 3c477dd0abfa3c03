set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4
ENVS="X=0;MST_ADJ_DEDUP=0;MST_REORDER=1;MST_REORDER=1 MST_ADJ_DEDUP=0" WLS="road uniform dense rmat22" REPS=2 bash tools/envab.sh
