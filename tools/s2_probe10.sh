timeout 1500 python -m pytest tests/test_parity_gpu.py tests/test_knobs_gpu.py -q -x 2>&1 | tail -2
VARIANTS="ilp hubj" WLS="rmat22 dense" REPS=3 bash tools/s2_ab.sh | tail -4
