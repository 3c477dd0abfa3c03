python -c "import __graft_entry__ as g; g.build(); g.smoke()"
ENVS="X=0" WLS="rmat22 uniform road dense" REPS=1 bash tools/envab.sh
TOOLS="racecheck memcheck synccheck" TMO=1500 bash tools/sanitize.sh
bash tools/r02_e2e.sh
