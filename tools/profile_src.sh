# one `ncu --set full` capture of the arc passes of the last mst_run, with the CUDA-line
# correlation exported (source page cuda,sass) before the report is dropped
WL=${WL:-rmat22}
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$WL.csv \
    python bench.py --workload $WL --steps 2 --warmup 3 --e2e-steps 0 --no-oracle > /dev/null 2>&1
RE=${RE:-arc_pass}
SKIP=$(python - "$WL" "$RE" <<'PY'
import csv, re, sys
wl, rx = sys.argv[1], re.compile(sys.argv[2])
rows = [r for r in csv.reader(open(f"gpurun_out/launches_{wl}.csv")) if len(r) > 5]
h = rows[0]; k = h.index("Kernel Name"); idc = h.index("ID")
seen = {}
for r in rows[1:]:
    seen.setdefault(r[idc], r[k])
hits = [n for n in seen.values() if rx.search(n)]
runs = 3 + 2 * 2
per = len(hits) // runs
print((runs - 1) * per, per)
PY
)
set -- $SKIP
ncu --set full --clock-control none --import-source on -k regex:"$RE" -s $1 -c $2 \
    -o gpurun_out/fullsrc_$WL python bench.py --workload $WL --steps 2 --warmup 3 --e2e-steps 0 --no-oracle \
    > gpurun_out/ncu_fullsrc_$WL.log 2>&1
ncu -i gpurun_out/fullsrc_$WL.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | gzip > gpurun_out/srcline_$WL.csv.gz
ncu -i gpurun_out/fullsrc_$WL.ncu-rep --page raw --csv 2>/dev/null | gzip > gpurun_out/rawsrc_$WL.csv.gz
rm -f gpurun_out/fullsrc_$WL.ncu-rep
