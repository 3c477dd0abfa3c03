timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
VARIANTS="nvtx outf" WLS="rmat22 road uniform" REPS=3 bash tools/s2_ab.sh | tail -6
python tools/bsum.py gpurun_out/ab_outf_rmat22_1.json 2>/dev/null | grep output
python tools/bsum.py gpurun_out/ab_nvtx_rmat22_1.json 2>/dev/null | grep output
