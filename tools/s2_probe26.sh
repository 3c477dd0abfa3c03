VARIANTS="base j8 c16" WLS="rmat22 road" REPS=3 bash tools/s2_ab.sh | tail -6
for v in base j8 c16; do python -c "import json,sys; d=json.load(open(sys.argv[1])); lk=d['launch_kinds']; print(sys.argv[2], {k: round(v['ms_per_step']*1e3,1) for k,v in lk.items() if k.startswith(('jump','compose'))})" gpurun_out/ab_${v}_rmat22_2.json $v; done
