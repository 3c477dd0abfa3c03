timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "host" 2>&1 | tail -2
VARIANTS="hagg0 hagg1 rd16 rd10" WLS="rmat22 road uniform dense" REPS=3 bash tools/s2_ab.sh | tail -16
