"""Per-CUDA-line instruction counts and stall samples from an exported
`ncu --page source --csv --print-source cuda,sass` page (gzip).
    python tools/srcline.py gpurun_out/srcline_rmat22.csv.gz <result index> [min share]
Result index = the n-th profiled kernel launch (0-based) in the export order."""
import csv
import gzip
import io
import sys

path = sys.argv[1]
want = int(sys.argv[2]) if len(sys.argv) > 2 else -1
mins = float(sys.argv[3]) if len(sys.argv) > 3 else 0.004
lines = io.TextIOWrapper(gzip.open(path), "utf-8").read().splitlines()
results = []  # list of dict file -> [(line, src, inst, samples)]
cur_file, cur_fn = None, None
for l in lines:
    if l.startswith('"File Path"'):
        cur_file = next(csv.reader([l]))[1].split("/")[-1]
        continue
    if l.startswith('"Function Name"'):
        fn = next(csv.reader([l]))[1]
        # a new result starts when common.cuh (first file) appears again with a function header
        if cur_file == "common.cuh" and (not results or results[-1]["files_seen"] and "common.cuh" in results[-1]["files_seen"]):
            results.append({"fn": fn[:60], "rows": [], "files_seen": set()})
        results[-1]["files_seen"].add(cur_file)
        continue
    if l.startswith('"Line No"'):
        hdr = next(csv.reader([l]))
        h = {k: j for j, k in enumerate(hdr)}
        continue
    r = next(csv.reader([l]))

    def num(x):
        try:
            return int(float(x))
        except ValueError:
            return 0
    if r[0]:
        results[-1]["rows"].append((cur_file, int(r[0]), r[1].strip(), num(r[h["Instructions Executed"]]),
                                    num(r[h["Warp Stall Sampling (All Samples)"]])))
for i, res in enumerate(results):
    tot = sum(x[3] for x in res["rows"]); smp = sum(x[4] for x in res["rows"])
    print(f"result {i}: {res['fn']} inst {tot/1e6:.1f} M samples {smp}")
    if i != want:
        continue
    for f, ln, src, ie, sm in res["rows"]:
        if ie > tot * mins or sm > smp * mins:
            print(f"  {f[:8]}:{ln:5d} {ie/1e6:7.2f}M {100*ie/tot:5.1f}% smp {100*sm/smp:5.1f}%  {src[:70]}")
