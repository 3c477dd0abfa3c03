python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/sanitize_cases.py 2>&1 | tail -3
TMO=1200 bash tools/sanitize.sh
