timeout 900 python -m pytest tests/test_knobs_gpu.py -q -x -k "LIGHT" 2>&1 | tail -2
timeout 1200 python -m pytest tests/test_parity_gpu.py -q -x -k "full_size or member or light" 2>&1 | tail -2
timeout 300 python bench.py --workload rmat22 --steps 10 --e2e-steps 0 --no-oracle 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2))"
