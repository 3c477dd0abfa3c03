"""Kernel shares of one mst_run from an ncu launch list (`--metrics gpu__time_duration.sum`):
per kernel, launches and µs per run and the share of the summed kernel time (cold-cache,
serialised: compare shares, not absolute times).
python tools/launch_share.py launches.csv [runs] [--run-only]  (--run-only: without the
one-time build kernels of mst_create)"""
import csv
import sys
from collections import defaultdict

path = sys.argv[1]
runs = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2].isdigit() else 7
BUILD = ("k_degree", "k_deg_argmax", "k_scan_rows", "k_bucket_count", "k_bucket_scatter",
         "k_apply_perm", "k_owner_degree", "k_scatter", "k_rdeg", "k_rbase", "k_rfill",
         "k_adj_fill", "k_bfs_order", "k_bfs_rest", "k_key_format")
run_only = "--run-only" in sys.argv
rows = [r for r in csv.reader(open(path)) if len(r) > 5]
h = rows[0]
k, mn, mv, mu = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
tot, cnt = defaultdict(float), defaultdict(int)
for r in rows[1:]:
    if r[mn] != "gpu__time_duration.sum":
        continue
    v = float(r[mv].replace(",", "")) * {"ns": 1e-3, "nsecond": 1e-3, "us": 1, "usecond": 1, "ms": 1e3, "msecond": 1e3}.get(r[mu], 1e-3)
    name = r[k].split("(")[0].replace("void ", "").replace("mstk::", "")
    if not name.startswith(("k_", "<")) and "k_" not in name:
        continue
    if run_only and name in BUILD:
        continue
    tot[name] += v
    cnt[name] += 1
S = sum(tot.values())
print(f"| kernel | launches / run | µs / run | share |\n|---|---|---|---|")
for name, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"| `{name[:60]}` | {cnt[name]/runs:.1f} | {v/runs:.1f} | {100*v/S:.1f} % |")
print(f"| **all** | {sum(cnt.values())/runs:.0f} | {S/runs:.1f} | |")
