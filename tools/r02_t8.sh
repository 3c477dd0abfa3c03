set -x
python -c "import __graft_entry__ as g; g.build()"
ENVS="X=0;MST_LIGHT_T=60;MST_LIGHT_ONLY0=1;MST_LIGHT_ONLY0=1 MST_LIGHT_T=100;MST_LIGHT_ONLY0=1 MST_LIGHT_T=120;MST_LIGHT_ONLY0=1 MST_LIGHT_T=170;MST_LIGHT_ONLY0=1 MST_LIGHT_T=220" WLS="rmat22" REPS=2 bash tools/envab.sh
TOOLS="memcheck synccheck" TMO=1200 bash tools/sanitize.sh
