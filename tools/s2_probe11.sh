timeout 1500 python -m pytest tests/test_parity_gpu.py tests/test_knobs_gpu.py tests/test_dist_procs_gpu.py -q -x 2>&1 | tail -2
VARIANTS="hubj fuse" WLS="rmat22 dense" REPS=3 bash tools/s2_ab.sh | tail -4
python tools/bsum.py gpurun_out/ab_fuse_rmat22_1.json | head -20
