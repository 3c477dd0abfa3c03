# per-kernel launch list (ncu, cold-cache, serialised) of one bench step for each variant dir
ROOT=$(pwd)
for v in ${VARIANTS:-head .}; do
  d=$ROOT; [ "$v" != "." ] && d=$ROOT/build/ab/$v
  (cd $d && ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file /tmp/l_$$.csv \
      python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-oracle --workload ${WL:-rmat22} ${BARGS} > /dev/null 2>&1)
  echo "== $v"
  python3 - /tmp/l_$$.csv <<'PY'
import csv,sys,collections
rows=[r for r in csv.reader(open(sys.argv[1])) if len(r)>10]
h=rows[0]; i={k:j for j,k in enumerate(h)}
data=[r for r in rows[1:] if r[i["Metric Name"]]=="gpu__time_duration.sum"]
# last step: the bench does warmup(3) + steps(1) + profiled(1): take the last 1/5 of run launches
names=[r[i["Kernel Name"]].split("(")[0] for r in data]
vals=[float(r[i["Metric Value"]]) for r in data]
unit=data[0][i["Metric Unit"]]
# find the last occurrence of the min0 pass to delimit the final run
starts=[j for j,n in enumerate(names) if "k_arc_pass<0" in n or "k_arc_pass<(int)0" in n]
s=starts[-1]
for n,v in zip(names[s:],vals[s:]):
    print("%-40s %10.1f %s"%(n[:40],v,unit))
PY
done
