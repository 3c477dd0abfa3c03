set -x
python -c "import __graft_entry__ as g; g.build()"
ENVS="X=0;MST_LIGHT_T=40;MST_LIGHT_T=60;MST_LIGHT_T=80;MST_LIGHT_ONLY0=1 MST_LIGHT_K=2;MST_LIGHT_ONLY0=1 MST_LIGHT_K=2 MST_LIGHT_T=60;MST_LIGHT_ONLY0=1 MST_LIGHT_K=2 MST_LIGHT_T=100;MST_LIGHT_ONLY0=1 MST_LIGHT_K=2 MST_LIGHT_T=160" WLS="rmat22" REPS=2 bash tools/envab.sh
TOOLS="memcheck synccheck racecheck" TMO=1500 bash tools/sanitize.sh
