"""Kernel-level microbenchmark of the A8 pass (mst_debug_filter_pass) on a BASELINE workload.

    MST_FILTER_VARIANT=v python tools/kbench.py --workload rmat22 --map 1 --group 43
"""
import argparse, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import graphgen
import paper_conf_ppopp_nasrebp13_b200 as p

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="rmat22")
ap.add_argument("--maps", default="0:1,1:43,2:43,1:4096")
ap.add_argument("--iters", type=int, default=10)
ap.add_argument("--relabel", default="none", choices=["none", "degree"])
a = ap.parse_args()
g = graphgen.config(a.workload)
if a.relabel == "degree":  # hub-first vertex numbering (emulates a locality layout pass)
    deg = np.bincount(g.src, minlength=g.n) + np.bincount(g.dst, minlength=g.n)
    order = np.argsort(-deg, kind="stable")
    newid = np.empty(g.n, np.int32); newid[order] = np.arange(g.n, dtype=np.int32)
    g.src, g.dst = newid[g.src], newid[g.dst]
t = lambda x: torch.from_numpy(np.ascontiguousarray(x).view(np.int32)).cuda()
h = p.MSTGraph(g.n, t(g.src), t(g.dst), t(g.w))
A = h.stats()["arcs0"]
peak = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6650
for spec in a.maps.split(","):
    kind, group = (int(x) for x in spec.split(":"))
    ms, surv = h.debug_filter_pass(kind, group, a.iters)
    byts = 16 * A + 16 * surv
    print(json.dumps({"relabel": a.relabel, "variant": os.environ.get("MST_FILTER_VARIANT", "0"), "map": kind,
                      "group": group, "ms": round(ms, 4), "A": A, "surv": surv,
                      "GBps": round(byts / ms / 1e6, 1), "frac": round(byts / ms / 1e6 / peak, 3)}))
