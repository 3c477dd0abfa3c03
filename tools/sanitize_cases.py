"""Small cases for compute-sanitizer (tools/sanitize.sh): every kernel family of libmst.so on
graphs small enough for memcheck/racecheck/synccheck, each checked against the oracle.

grid64 through the multi-kernel path (device tail on and off, light phase forced, keep-edges,
union-find, sharded simulation) and through the one-CTA path; small random multigraphs with
ties, loops and parallel edges; a scaled RMAT with the dense transition and the hub row (and
the light phase: threshold select in the init launch, member scans, the jump's hub set); the
streamed host-input build.
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import torch  # noqa: E402

import graphgen  # noqa: E402
import mstcheck as mc  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ppopp_nasrebp13_b200 as lib  # noqa: E402

DENSE, KEEP, TAIL, TAU, LF, UF, SMALL = 1, 2, 3, 4, 5, 6, 7


def dev(a):
    a = np.ascontiguousarray(a)
    if a.dtype == np.uint32:
        a = a.view(np.int32)
    return torch.from_numpy(a.astype(np.int32, copy=False)).cuda()


def check(name, n, s, d, w, opts=(), nshards=1):
    s = np.asarray(s, np.int32); d = np.asarray(d, np.int32); w = np.asarray(w, np.uint32)
    with lib.MSTGraph(n, dev(s), dev(d), dev(w), nshards=nshards) as g:
        for o, v in opts:
            g.set_option(o, v)
        ids, cnt, tot = g.run()
        ids = ids.cpu().numpy()
    o_ids, o_tot = oracle.kruskal(n, s, d, w)
    assert cnt == len(o_ids) and tot == o_tot and np.array_equal(ids, o_ids), name
    print("ok", name, flush=True)


def main():
    lib.load(); oracle.build(); graphgen.build()
    g = graphgen.config(1)
    base = [(SMALL, 0)]
    check("grid64 small-path", g.n, g.src, g.dst, g.w)
    check("grid64 tail", g.n, g.src, g.dst, g.w, base)
    check("grid64 no-tail", g.n, g.src, g.dst, g.w, base + [(TAIL, 0)])
    check("grid64 sparse", g.n, g.src, g.dst, g.w, base + [(DENSE, 0)])
    check("grid64 keep", g.n, g.src, g.dst, g.w, base + [(KEEP, 1)])
    check("grid64 uf", g.n, g.src, g.dst, g.w, [(UF, 1)])
    check("grid64 tau1000", g.n, g.src, g.dst, g.w, base + [(TAU, 1000), (DENSE, 0)])
    check("grid64 sim3", g.n, g.src, g.dst, g.w, base, nshards=3)
    rng = np.random.default_rng(5)
    for i in range(3):
        n = int(rng.integers(200, 3000)); m = int(n * rng.integers(10, 40))
        s, d, w = mc.random_multigraph(rng, n, m, [3, 1000, 2**32 - 1][i])
        check(f"multigraph{i} light", n, s, d, w, base + [(LF, 2)])
        check(f"multigraph{i} default", n, s, d, w)
    r = graphgen.config(4, s=1, scale_down=9)  # RMAT 8 K vertices, 131 K edges
    check("rmat-sd9", r.n, r.src, r.dst, r.w, base)
    check("rmat-sd9 no-tail", r.n, r.src, r.dst, r.w, base + [(TAIL, 0), (LF, 0)])
    # streamed host-input build (degree per endpoint chunk, scatter per weight chunk, key format
    # afterwards), one-shot and persistent, in many small chunks
    os.environ["MST_HOST_CHUNK"] = "20011"
    o_ids, o_tot = oracle.kruskal(r.n, r.src, r.dst, r.w)
    ids, cnt, tot = lib.mst_solve_host(r.n, r.src, r.dst, r.w)
    assert cnt == len(o_ids) and tot == o_tot and np.array_equal(ids, o_ids), "host solve"
    with lib.MSTGraph(r.n, r.src, r.dst, r.w, host=True) as h:
        ids, cnt, tot = h.run_host()
    assert cnt == len(o_ids) and tot == o_tot and np.array_equal(ids, o_ids), "host handle"
    print("ok rmat-sd9 host streamed", flush=True)


if __name__ == "__main__":
    main()
