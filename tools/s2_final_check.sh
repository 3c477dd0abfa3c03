python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -1
timeout 300 python bench.py 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['metric'], round(d['value']/1e9,2), d['roofline']['frac'], d['parity'], d['e2e']['value']/1e9)"
