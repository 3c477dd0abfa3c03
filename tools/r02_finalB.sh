# round-2 final evidence, part B: sanitizers and the mode / layout comparisons
set -x
python -c "import __graft_entry__ as g; g.build()"
TOOLS="memcheck synccheck racecheck" TMO=1500 bash tools/sanitize.sh
bash tools/modes.sh
