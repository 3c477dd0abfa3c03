set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -6
ENVS="X=0;MST_LIGHT_T=80;MST_LIGHT_T=100;MST_LIGHT_T=120;MST_LIGHT_T=170;MST_LIGHT_T=220" WLS="rmat22" REPS=1 bash tools/envab.sh
