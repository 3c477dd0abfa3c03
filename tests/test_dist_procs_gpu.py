"""The distributed round loop in separate processes (-m gpu).

NCCL takes one rank per device and the GPU box has one GPU, so the ranks here are processes
that SHARE cuda:0 and exchange through mst_create_dist_hostx: the library's distributed
handle (each rank builds only the records of its owner range, decides its own compaction,
agrees on the light-edge threshold, and runs the per-round allreduce-MIN) with the MIN done by
a gloo process group instead of NCCL. Every rank must return the oracle's forest bit for bit.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
LF, TAU, DENSE, TAIL, KEEP = 5, 4, 1, 3, 2  # include/mst.h option ids


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _cases():
    """(name, graph spec, per-rank options). Graph specs are rebuilt in every process."""
    c = []
    for k, sd in [(1, 0), (2, 6), (3, 8), (4, 8), (5, 6)]:
        c.append((f"cfg{k}", ("config", k, sd), {}))
    # rank-divergent compaction: rank 0 never compacts, the others always do
    for k, sd in [(2, 6), (3, 8), (4, 8)]:
        c.append((f"cfg{k}-tau-split", ("config", k, sd),
                  {"per_rank": [[(TAU, 0)], [(TAU, 1000)], [(TAU, 500)]]}))
    c.append(("cfg4-sparse", ("config", 4, 8), {"all": [(DENSE, 0)]}))
    c.append(("cfg5-notail", ("config", 5, 6), {"all": [(TAIL, 0)]}))
    c.append(("cfg3-keep", ("config", 3, 8), {"all": [(KEEP, 1)]}))
    c.append(("cfg4-light4", ("config", 4, 6), {"all": [(LF, 4)]}))
    c.append(("cfg5-light1", ("config", 5, 5), {"all": [(LF, 1)]}))
    c.append(("cfg2-light2", ("config", 2, 4), {"all": [(LF, 2)]}))
    # tiny graphs: shards without any record (one edge, a few edges, no edge)
    c.append(("one-edge", ("edges", 2, [0], [1], [7]), {}))
    c.append(("path4", ("edges", 4, [0, 1, 2], [1, 2, 3], [3, 1, 2]), {}))
    c.append(("no-edges", ("edges", 5, [], [], []), {}))
    c.append(("loops", ("edges", 3, [0, 1, 2, 0], [0, 1, 2, 2], [1, 2, 3, 4]), {}))
    return c


def _graph(spec):
    import graphgen
    if spec[0] == "config":
        g = graphgen.config(spec[1], s=3, scale_down=spec[2])
        return g.n, g.src, g.dst, g.w
    _, n, s, d, w = spec
    return n, np.array(s, np.int32), np.array(d, np.int32), np.array(w, np.uint32)


def _worker(rank, world, port, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        import paper_conf_ppopp_nasrebp13_b200 as p
        from paper_conf_ppopp_nasrebp13_b200 import dist as mdist
        p.load()
        out = {}
        for name, spec, opts in _cases():
            n, s, d, w = _graph(spec)
            t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()  # noqa: E731
            calls = []

            def xchg(words):
                calls.append(len(words))
                mdist.allreduce_min_u64_(words)
            with p.MSTGraph(n, t(s), t(d), t(w), hostx=(rank, world, xchg)) as h:
                for o, v in opts.get("all", []):
                    h.set_option(o, v)
                for o, v in opts.get("per_rank", [[]] * world)[rank % 3]:
                    h.set_option(o, v)
                runs = []
                for _ in range(2):
                    ids, cnt, tot = h.run()
                    runs.append((ids.cpu().numpy().tolist(), cnt, tot))
                st = h.stats()
            out[name] = {"runs": runs, "local": st["local_arcs0"], "arcs0": st["arcs0"],
                         "compacted": st["compacted"], "light_t": st["light_t"],
                         "rounds": st["rounds"], "xcalls": len(calls)}
        results[rank] = out
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_dist_round_loop_processes(world, oracle_mod):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), results), nprocs=world, join=True)
    res = [results[r] for r in range(world)]
    divergent = 0
    for name, spec, _ in _cases():
        n, s, d, w = _graph(spec)
        o_ids, o_tot = oracle_mod.kruskal(n, s, d, w)
        per = [r[name] for r in res]
        for r, x in enumerate(per):
            for ids, cnt, tot in x["runs"]:
                assert cnt == len(o_ids) and tot == o_tot, (name, r, cnt, tot)
                assert ids == o_ids.tolist(), (name, r)
        # the ranks' record windows partition the edge records; every rank made the same
        # number of exchange calls (the protocol is collective)
        assert sum(x["local"] for x in per) == per[0]["arcs0"], name
        assert len({x["xcalls"] for x in per}) == 1, name
        assert len({x["light_t"] for x in per}) == 1, name  # one agreed threshold
        if len({tuple(x["compacted"]) for x in per}) > 1:
            divergent += 1
        if name == "one-edge":
            assert min(x["local"] for x in per) == 0, name  # a shard without records
    assert divergent >= 1  # rank-local compaction decisions really differed somewhere
