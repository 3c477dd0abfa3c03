"""Subprocess runner for tests/test_knobs_gpu.py: parity of one ablation-knob setting.

The library reads its ablation knobs (MST_PASSCFG, MST_QFILTER, ... : DESIGN.md, the ablation
table) from the environment once per process, so every setting runs in a fresh interpreter:
    MST_PASSCFG=3 python tests/knob_parity.py
It runs the CUDA path through the C ABI on scaled BASELINE configs plus a dense random
multigraph and compares ids, count and total weight with the oracle bit for bit (SURVEY.md
§8(c)). Prints "ok <cases>" and exits 0, or raises.
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import torch  # noqa: E402

import graphgen  # noqa: E402
import mstcheck as mc  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ppopp_nasrebp13_b200 as lib  # noqa: E402

LF = 5  # MST_OPT_LIGHT_FIRST (include/mst.h)


def dev(a):
    a = np.ascontiguousarray(a)
    if a.dtype == np.uint32:
        a = a.view(np.int32)
    return torch.from_numpy(a.astype(np.int32, copy=False)).to("cuda")


# MST_TEST_OPTIONS="6=1,4=0": run options applied to every case (option=value, include/mst.h)
EXTRA = [tuple(int(x) for x in kv.split("=")) for kv in
         os.environ.get("MST_TEST_OPTIONS", "").split(",") if kv]


def check(name, n, src, dst, w, options=()):
    options = list(options) + EXTRA
    src = np.asarray(src, np.int32)
    dst = np.asarray(dst, np.int32)
    w32 = np.asarray(w, np.uint64).astype(np.uint32)
    with lib.MSTGraph(n, dev(src), dev(dst), dev(w32)) as g:
        for opt, val in options:
            g.set_option(opt, val)
        runs = [g.run() for _ in range(2)]  # re-runnable on one handle
    o_ids, o_tot = oracle.kruskal(n, src, dst, w)
    for ids, cnt, tot in runs:
        ids = ids.cpu().numpy()
        assert cnt == len(o_ids), (name, cnt, len(o_ids))
        assert tot == o_tot, (name, tot, o_tot)
        assert np.array_equal(ids, o_ids), name


def main():
    lib.load()
    oracle.build()
    graphgen.build()
    cases = 0
    # scaled BASELINE configs: grid64, uniform, road-like, RMAT, dense (graphgen recipe)
    for k, sd in [(1, 0), (2, 6), (3, 8), (4, 6), (5, 6), (4, 4)]:
        g = graphgen.config(k, s=2, scale_down=sd)
        check(f"config{k}/sd{sd}", g.n, g.src, g.dst, g.w)
        cases += 1
    # the light-edge phase forced on a sparse input, and off on a dense one
    g = graphgen.config(4, s=3, scale_down=6)
    check("rmat light K=1", g.n, g.src, g.dst, g.w, options=[(LF, 1)])
    g = graphgen.config(5, s=3, scale_down=6)
    check("dense light off", g.n, g.src, g.dst, g.w, options=[(LF, 0)])
    cases += 2
    # dense random multigraph with heavy ties (duplicate pairs, equal weights)
    rng = np.random.default_rng(1234)
    n, m = 3000, 400_000
    src, dst, w = mc.random_multigraph(rng, n, m, 40)
    check("multigraph", n, src, dst, w)
    cases += 1
    print(f"ok {cases}")


if __name__ == "__main__":
    main()
