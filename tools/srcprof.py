"""Summarise an exported `ncu --page source --csv --print-source sass` page (gzip): per kernel
section the executed warp instructions and stall samples, and the hottest SASS lines.

    python tools/srcprof.py gpurun_out/src_rmat22.csv.gz [section] [top]
"""
import csv
import gzip
import io
import sys

path = sys.argv[1]
want = int(sys.argv[2]) if len(sys.argv) > 2 else -1
top = int(sys.argv[3]) if len(sys.argv) > 3 else 60
lines = io.TextIOWrapper(gzip.open(path), "utf-8").read().splitlines()
secs, cur = [], None
for l in lines:
    if l.startswith('"Kernel Name"'):
        cur = {"name": l.split('","')[1][:60], "rows": []}
        secs.append(cur)
    elif l.startswith('"Address"'):
        cur["hdr"] = next(csv.reader([l]))
    else:
        cur["rows"].append(next(csv.reader([l])))
for i, s in enumerate(secs):
    h = {k: j for j, k in enumerate(s["hdr"])}
    ie = h["Instructions Executed"]
    ss = h["Warp Stall Sampling (All Samples)"]
    tot = sum(int(r[ie] or 0) for r in s["rows"])
    smp = sum(int(r[ss] or 0) for r in s["rows"])
    print(f"section {i}: {s['name']}  inst {tot/1e6:.1f} M  samples {smp}")
    if i != want:
        continue
    rows = [(int(r[ie] or 0), int(r[ss] or 0), r[h["Address"]][-5:], r[h["Source"]].strip()) for r in s["rows"]]
    print("  -- by address (count>0): inst(M)  samples  sass")
    for c, sm, a, src in rows:
        if c > 0 and (c > tot * 0.002 or sm > smp * 0.004):
            print(f"  {a} {c/1e6:8.2f} {sm:7d}  {src[:90]}")
