VARIANTS="head t62" WLS="rmat22 dense" REPS=4 bash tools/s2_ab.sh | tail -4
