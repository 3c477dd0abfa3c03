set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()"
timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -8
ENVS="X=0;MST_MEMBER_SCAN=0;MST_LIGHT_SWITCH=4;MST_LIGHT_SWITCH=3" WLS="rmat22" REPS=2 bash tools/envab.sh
ENVS="X=0" WLS="uniform road dense grid64" REPS=1 bash tools/envab.sh
