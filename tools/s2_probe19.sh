timeout 1800 python -m pytest tests/test_parity_gpu.py -q -x 2>&1 | tail -2
VARIANTS="nvtx sing" WLS="rmat22 dense" REPS=4 bash tools/s2_ab.sh | tail -4
for v in nvtx sing; do python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], round(d['launch_kinds']['min0/singletons']['ms_per_step']*1e3,1))" gpurun_out/ab_${v}_rmat22_2.json $v; done
