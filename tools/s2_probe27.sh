timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -1
for rep in 1 2 3; do timeout 300 python bench.py 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), d['light_phase'], d['clocks'], round(d['e2e']['value']/1e9,2))"; done
