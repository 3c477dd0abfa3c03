timeout 1500 python -m pytest tests/test_parity_gpu.py -q -x 2>&1 | tail -2
VARIANTS="hagg1 ." WLS="rmat22 road uniform dense" REPS=3 bash tools/s2_ab.sh | tail -8
for rep in 1 2 3; do for h in 13312 4096 1024; do
MST_MIN0_HOT=$h timeout 300 python bench.py --workload rmat22 --steps 10 --e2e-steps 0 --no-oracle > gpurun_out/p8_h$h.json 2>/dev/null
python -c "import json,sys; d=json.load(open(sys.argv[1])); lk=d['launch_kinds']; print('hot', sys.argv[2], round(d['value']/1e9,3), {k: round(v['ms_per_step']*1e3,1) for k,v in lk.items() if k.startswith('min0')})" gpurun_out/p8_h$h.json $h
done; done
