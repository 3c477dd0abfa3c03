# round-2 final evidence (session 2), part B: NEXT-2/NEXT-3/A9 mode lines and NEXT-4 layout lines
bash tools/modes.sh 2>&1 | tee gpurun_out/f3_modes.txt
bash tools/layouts.sh 2>&1 | tee gpurun_out/f3_layouts.txt
