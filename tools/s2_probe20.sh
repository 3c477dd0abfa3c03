timeout 1800 python -m pytest tests/test_parity_gpu.py -q -x -k "member or light or full_size or random or host" 2>&1 | tail -2
VARIANTS="nvtx wqs" WLS="rmat22 dense" REPS=4 bash tools/s2_ab.sh | tail -4
for v in nvtx wqs; do python -c "import json,sys; d=json.load(open(sys.argv[1])); lk=d['launch_kinds']; print(sys.argv[2], {k: round(v['ms_per_step']*1e3,1) for k,v in lk.items() if 'member' in k or 'single' in k or 'compose' in k})" gpurun_out/ab_${v}_rmat22_2.json $v; done
