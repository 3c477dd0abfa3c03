"""e2e breakdown through the C ABI on one workload: mst_solve_host total, and create_host /
run_host / destroy timed apart (pinned host arrays), under the current environment's knobs.
python tools/e2e_probe.py <workload> [reps]"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_ppopp_nasrebp13_b200 as lib  # noqa: E402
from paper_conf_ppopp_nasrebp13_b200 import mst as mstb  # noqa: E402

wl = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
g = graphgen.config(wl, s=0)
n, m = g.n, len(g.src)
pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory().numpy()  # noqa: E731
hs, hd, hw = pin(g.src), pin(g.dst), pin(g.w.view(np.int32)).view(np.uint32)
hout = torch.empty(max(n - 1, 1), dtype=torch.int32).pin_memory().numpy()
mstb.mst_solve_host(n, hs, hd, hw, hout)
tot, tc, tr, td = [], [], [], []
for _ in range(reps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    mstb.mst_solve_host(n, hs, hd, hw, hout)
    tot.append(time.perf_counter() - t0)
    t0 = time.perf_counter()
    h = lib.MSTGraph(n, hs, hd, hw, host=True)
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    h.run_host(hout)
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    h.close()
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    tc.append(t1 - t0); tr.append(t2 - t1); td.append(t3 - t2)
env = " ".join(f"{k}={v}" for k, v in os.environ.items() if k.startswith("MST_"))
print(f"[{env or 'default':28s}] {wl:7s} solve_host {np.median(tot)*1e3:7.2f} ms ({m/np.median(tot)/1e9:.2f} G/s)"
      f"  create {np.median(tc)*1e3:7.2f}  run {np.median(tr)*1e3:6.2f}  destroy {np.median(td)*1e3:6.2f} ms")
