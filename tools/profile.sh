# launch list (cold-cache, serialised; compare SHARES) + one `ncu --set full` capture of the
# arc passes (A2/A8) of one mst_run step, exported to text on the box (the .ncu-rep stays
# under gpurun_out/ only when KEEP_REP=1: gpurun brings back <= 64 MiB)
WL=${WL:-rmat22}
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$WL.csv \
    python bench.py --workload $WL --steps 2 --warmup 3 --e2e-steps 0 --no-oracle > /dev/null 2>&1
# the bench runs warmup + 2 x steps mst_run calls: capture the arc passes of the LAST run only
RE=${RE:-arc_pass|k_member_min|k_small_msf}
SKIP=$(python - "$WL" "$RE" <<'PY'
import csv, re, sys
wl, rx = sys.argv[1], re.compile(sys.argv[2])
rows = [r for r in csv.reader(open(f"gpurun_out/launches_{wl}.csv")) if len(r) > 5]
h = rows[0]; k = h.index("Kernel Name"); idc = h.index("ID")
seen = {}
for r in rows[1:]:
    seen.setdefault(r[idc], r[k])
hits = [n for n in seen.values() if rx.search(n)]
runs = 3 + 2 * 2  # warmup + 2 timed + 2 profiled steps (--steps 2 --warmup 3)
per = len(hits) // runs
print((runs - 1) * per, per)
PY
)
set -- $SKIP
ncu --set full --clock-control none --import-source on -k regex:"$RE" -s $1 -c $2 \
    -o gpurun_out/full_$WL python bench.py --workload $WL --steps 2 --warmup 3 --e2e-steps 0 --no-oracle \
    > gpurun_out/ncu_full_$WL.log 2>&1
tail -1 gpurun_out/ncu_full_$WL.log
python tools/ncu_traffic.py gpurun_out/full_$WL.ncu-rep $WL "tools/profile.sh WL=$WL (ncu --set full -k regex:$RE, last mst_run of the bench)" > /dev/null
ncu -i gpurun_out/full_$WL.ncu-rep --page raw --csv 2>/dev/null | gzip > gpurun_out/raw_$WL.csv.gz
ncu -i gpurun_out/full_$WL.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/src_$WL.csv.gz
ncu -i gpurun_out/full_$WL.ncu-rep --page details --csv 2>/dev/null | gzip > gpurun_out/details_$WL.csv.gz
cp profiles/ncu_traffic_$WL.json gpurun_out/ 2>/dev/null
[ "${KEEP_REP:-0}" = "1" ] || rm -f gpurun_out/full_$WL.ncu-rep
