"""Multi-GPU host logic on CPU: world-size-2 gloo process group.

Covers what the N > 1 bench path does outside libmst's own NCCL communicator: the NCCL
unique id travels from rank 0 to every rank, timings are reduced as the max over ranks, and
every rank derives the same arc-balanced source-range partition from the CSR row offsets
(mst_shard_ranges, the exact host code mst_create_dist runs).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

WORLD = 2


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, port, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        import paper_conf_ppopp_nasrebp13_b200 as p
        from paper_conf_ppopp_nasrebp13_b200 import dist as mdist

        # 1. unique id: rank 0's bytes reach every rank unchanged
        def make_id():
            try:
                return p.mst_get_unique_id()
            except p.MSTError:  # no usable network interface for NCCL's bootstrap here
                return bytes(range(128))
        uid = mdist.share_unique_id(make_id)
        ids = [None] * WORLD
        dist.all_gather_object(ids, uid)

        # 2. max over ranks
        t = mdist.max_over_ranks(10.0 + rank)

        # 3. partition: each rank computes its own window from the same row offsets
        rng = np.random.default_rng(7)
        deg = rng.integers(0, 50, 1000).astype(np.uint32)
        deg[rng.integers(0, 1000, 5)] = 5000  # a few hubs
        row = np.concatenate([[0], np.cumsum(deg)]).astype(np.uint32)
        lo, hi = p.mst.mst_shard_ranges(row, WORLD)
        mine = (int(lo[rank]), int(hi[rank]))
        wins = [None] * WORLD
        dist.all_gather_object(wins, mine)
        # 4. the host exchange's unsigned MIN (mst_create_dist_hostx): values above 2^63 and
        #    the "no edge" key 2^64 - 1 must order as unsigned
        words = np.array([5, 2**64 - 1, 2**63 + 7, 2**63 - 1, 0], np.uint64)
        if rank == 1:
            words = np.array([9, 2**63 + 3, 2**63 + 9, 2**64 - 2, 1], np.uint64)
        mdist.allreduce_min_u64_(words)
        results[rank] = {"ids": ids, "t": t, "wins": wins, "row_end": int(row[-1]),
                         "lo": lo.tolist(), "hi": hi.tolist(), "words": words.tolist()}
    finally:
        dist.destroy_process_group()


def test_gloo_world2_host_logic():
    pytest.importorskip("torch.distributed")
    import paper_conf_ppopp_nasrebp13_b200 as p
    p.load()
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_worker, args=(_free_port(), results), nprocs=WORLD, join=True)
    r0, r1 = results[0], results[1]
    assert r0["ids"][0] == r0["ids"][1] == r1["ids"][0] and len(r0["ids"][0]) == 128
    assert r0["t"] == r1["t"] == 11.0
    assert r0["words"] == r1["words"] == [5, 2**63 + 3, 2**63 + 7, 2**63 - 1, 0]
    # identical partitions on both ranks; contiguous, disjoint, covering [0, arcs)
    assert r0["wins"] == r1["wins"]
    wins = r0["wins"]
    assert wins[0][0] == 0 and wins[-1][1] == r0["row_end"]
    for a, b in zip(wins, wins[1:]):
        assert a[1] == b[0]


@pytest.mark.parametrize("G", [1, 2, 3, 8, 64])
def test_shard_ranges_partition(G):
    import paper_conf_ppopp_nasrebp13_b200 as p
    rng = np.random.default_rng(G)
    deg = rng.integers(0, 20, 5000).astype(np.uint32)
    row = np.concatenate([[0], np.cumsum(deg)]).astype(np.uint32)
    lo, hi = p.mst.mst_shard_ranges(row, G)
    assert lo[0] == 0 and hi[-1] == row[-1]
    assert np.all(lo[1:] == hi[:-1]) and np.all(hi >= lo)
    # windows start at vertex boundaries (a source's arcs never split across ranks)
    assert set(lo.tolist()) <= set(row.tolist())
    # arc-balanced within one vertex's degree
    target = row[-1] / G
    assert np.all(np.abs((hi - lo) - target) <= deg.max() + 1)
