"""GPU parity: the CUDA path through the C ABI == the oracle, bit for bit (-m gpu).

Compared on the same seeded inputs (graphgen): the ascending forest ids, their count and
the exact uint64 total weight (integer work -> bit-exact, no tolerance).
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import mstcheck as mc

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
LF = 5  # MST_OPT_LIGHT_FIRST (include/mst.h)


@pytest.fixture(scope="module")
def lib():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_nasrebp13_b200 as p
    p.load()
    return p


def dev(a, dt=torch.int32):
    a = np.ascontiguousarray(a)
    if a.dtype == np.uint32:
        a = a.view(np.int32)
    return torch.from_numpy(a.astype(np.int32, copy=False)).to("cuda")


SMALL = 7  # MST_OPT_SMALL (include/mst.h)


def gpu_msf(lib, n, src, dst, w, nshards=1, runs=1, options=(), small=False):
    """small=False (the default here) keeps every test on the multi-kernel path even for
    graphs the one-CTA path (MST_OPT_SMALL) would take; the small-path tests pass True."""
    src = np.asarray(src, np.int32)
    dst = np.asarray(dst, np.int32)
    w = np.asarray(w, np.uint64).astype(np.uint32)
    with lib.MSTGraph(n, dev(src), dev(dst), dev(w), nshards=nshards) as g:
        if not small:
            g.set_option(SMALL, 0)
        for opt, val in options:
            g.set_option(opt, val)
        outs = []
        for _ in range(runs):
            ids, cnt, tot = g.run()
            outs.append((ids.cpu().numpy().copy(), cnt, tot))
        st = g.stats()
    for o in outs[1:]:  # re-runnable: same handle, same output
        assert np.array_equal(o[0], outs[0][0]) and o[1:] == outs[0][1:]
    return outs[0][0], outs[0][1], outs[0][2], st


def assert_parity(lib, oracle_mod, n, src, dst, w, nshards=1, runs=1, options=(), small=False):
    ids, cnt, tot, st = gpu_msf(lib, n, src, dst, w, nshards, runs, options, small)
    o_ids, o_tot = oracle_mod.kruskal(n, src, dst, w)
    assert cnt == len(o_ids), (cnt, len(o_ids))
    assert tot == o_tot, (tot, o_tot)
    assert np.array_equal(ids, o_ids)
    return st


# ------------------------------------------------------------------ fixtures and small graphs
@pytest.mark.parametrize("name", ["hand_small.txt", "hand_forest.txt"])
def test_golden(lib, oracle_mod, name):
    import os
    n, src, dst, w, exp = mc.load_golden(os.path.join(os.path.dirname(__file__), "golden", name))
    ids, cnt, tot, _ = gpu_msf(lib, n, src, dst, w)
    assert list(ids) == exp["expect_ids"] and tot == exp["expect_total"][0]


def test_grid64(lib, oracle_mod, gg):
    g = gg.config(1)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=3)
    assert st["rounds"] >= 3
    assert st["gpu_launches"] >= st["rounds"]  # every kernel of the run is counted


@pytest.mark.parametrize("seed", range(120))
def test_random_multigraphs(lib, oracle_mod, seed):
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(1, 10_000))
    m = int(rng.integers(0, 6 * n))
    wmax = [0, 1, 7, 1000, 2**32 - 1][seed % 5]
    src, dst, w = mc.random_multigraph(rng, n, m, wmax)
    assert_parity(lib, oracle_mod, n, src, dst, w)


@pytest.mark.parametrize("seed", range(20))
def test_tiny_graphs_vs_brute_force(lib, seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 7)); m = int(rng.integers(0, 11))
    src, dst, w = mc.random_multigraph(rng, n, m, 2)
    ids, cnt, tot, _ = gpu_msf(lib, n, src, dst, w)
    bf, bf_w, _ = mc.brute_force_msf(n, src, dst, w)
    assert list(ids) == bf and tot == bf_w


# ------------------------------------------------------------------ edge cases
def test_empty_and_degenerate(lib, oracle_mod):
    for n, src, dst, w in [(0, [], [], []), (1, [], [], []), (5, [], [], []),
                           (3, [0, 1, 2], [0, 1, 2], [1, 2, 3]),   # self-loops only
                           (2, [0], [1], [2**32 - 1]), (2, [1, 0, 1], [0, 1, 0], [3, 3, 3])]:
        assert_parity(lib, oracle_mod, n, src, dst, w)


def test_monotone_path_chain(lib, oracle_mod):
    # every vertex hooks to its left neighbour in round 0: one chain of depth n-1
    n = 1_000_000
    src = np.arange(n - 1, dtype=np.int32)
    st = assert_parity(lib, oracle_mod, n, src, src + 1, np.arange(1, n, dtype=np.uint32))
    assert st["rounds"] <= 2


def test_reverse_monotone_path_chain(lib, oracle_mod):
    n = 300_000
    src = np.arange(n - 1, dtype=np.int32)
    assert_parity(lib, oracle_mod, n, src, src + 1, np.arange(n - 1, 0, -1).astype(np.uint32))


def test_star_huge_degree(lib, oracle_mod):
    # one segment spanning many CTAs (deg 10^6)
    n = 1_000_001
    rng = np.random.default_rng(3)
    src = np.zeros(n - 1, np.int32)
    dst = np.arange(1, n, dtype=np.int32)
    w = rng.integers(0, 1000, n - 1).astype(np.uint32)
    extra = rng.integers(1, n, 200_000).astype(np.int32)  # parallel + cross edges
    src = np.concatenate([src, extra]); dst = np.concatenate([dst, np.roll(extra, 1)])
    w = np.concatenate([w, rng.integers(0, 1000, 200_000).astype(np.uint32)])
    assert_parity(lib, oracle_mod, n, src, dst, w)


@pytest.mark.parametrize("seed", [0, 1])
def test_hub_row_dense_transition(lib, oracle_mod, seed):
    """a hub joined to every vertex by heavy edges, plus light random edges: many components
    keep pairs with the hub's component until the dense transition, which reduces the hub's
    matrix row in shared memory (heavy-tailed degrees switch it on)"""
    rng = np.random.default_rng(seed)
    n = 120_000
    light = 150_000
    s1 = rng.integers(1, n, light).astype(np.int32)
    d1 = rng.integers(1, n, light).astype(np.int32)
    w1 = rng.integers(0, 500, light).astype(np.uint32)
    s2 = np.zeros(n - 1, np.int32)
    d2 = np.arange(1, n, dtype=np.int32)
    w2 = rng.integers(500, 1000, n - 1).astype(np.uint32)
    for parts in ((s1, s2), (s2, s1)):  # hub edges last / first in id order
        src = np.concatenate(parts)
        dst = np.concatenate((d1, d2) if parts[0] is s1 else (d2, d1))
        w = np.concatenate((w1, w2) if parts[0] is s1 else (w2, w1))
        st = assert_parity(lib, oracle_mod, n, src, dst, w, runs=2)
        assert st["dense_round"] >= 0 and st["hub_row"]


def test_all_equal_weights(lib, oracle_mod, gg):
    g = gg.uniform(200_000, 800_000, 1, 2, 3, wlo=7, wmod=1)
    assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w)


def test_max_weights(lib, oracle_mod, gg):
    g = gg.uniform(100_000, 300_000, 4, 5, 6, wlo=2**32 - 4, wmod=4)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w)


def test_many_components_and_isolated(lib, oracle_mod, gg):
    g = gg.uniform(500_000, 200_000, 7, 8, 9)  # m < n: thousands of trees + isolated
    assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w)


def test_parallel_heavy(lib, oracle_mod, gg):
    g = gg.uniform(64, 500_000, 11, 12, 13, wmod=50)
    assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w)


# ------------------------------------------------------------------ scaled configs
@pytest.mark.parametrize("k,sd", [(2, 6), (3, 6), (4, 8), (5, 6), (2, 0)])
def test_config_scaled(lib, oracle_mod, gg, k, sd):
    g = gg.config(k, s=1, scale_down=sd)
    assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=2)


@pytest.mark.parametrize("G", [2, 3, 8])
@pytest.mark.parametrize("k,sd", [(1, 0), (4, 8), (3, 8)])
def test_sim_shards(lib, oracle_mod, gg, G, k, sd):
    g = gg.config(k, scale_down=sd)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, nshards=G)
    assert st["local_arcs0"] == st["arcs0"]


# ------------------------------------------------------------------ API variants, errors
def test_host_paths(lib, oracle_mod, gg):
    g = gg.config(4, scale_down=8)
    o_ids, o_tot = oracle_mod.kruskal(g.n, g.src, g.dst, g.w)
    ids, cnt, tot = lib.mst_solve_host(g.n, g.src, g.dst, g.w)
    assert np.array_equal(ids, o_ids) and tot == o_tot
    with lib.MSTGraph(g.n, g.src, g.dst, g.w, host=True) as h:
        ids, cnt, tot = h.run_host()
        assert np.array_equal(ids, o_ids) and tot == o_tot
    # pinned host arrays: the build reads them zero-copy over PCIe
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).pin_memory().numpy()  # noqa: E731
    ps, pd, pw = pin(g.src), pin(g.dst), pin(g.w).view(np.uint32)
    ids, cnt, tot = lib.mst_solve_host(g.n, ps, pd, pw)
    assert np.array_equal(ids, o_ids) and tot == o_tot
    with lib.MSTGraph(g.n, ps, pd, pw, host=True) as h:
        ids, cnt, tot = h.run_host()
        assert np.array_equal(ids, o_ids) and tot == o_tot


@pytest.mark.parametrize("k,sd", [(4, 0), (3, 0), (2, 2), (5, 4), (1, 0)])
@pytest.mark.parametrize("chunk", [None, "100003"])
def test_host_streamed_build(lib, oracle_mod, gg, k, sd, chunk, monkeypatch):
    """Host-array input: the copies are streamed chunk by chunk under the build (degree per
    endpoint chunk, scatter per weight chunk, key format fixed afterwards) — bit-exact at full
    size, with the default chunks and with many small ragged ones (MST_HOST_CHUNK)."""
    if chunk:
        monkeypatch.setenv("MST_HOST_CHUNK", chunk)
    g = gg.config(k, scale_down=sd)
    o_ids, o_tot = oracle_mod.kruskal(g.n, g.src, g.dst, g.w)
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).pin_memory().numpy()  # noqa: E731
    ps, pd, pw = pin(g.src), pin(g.dst), pin(g.w).view(np.uint32)
    ids, cnt, tot = lib.mst_solve_host(g.n, ps, pd, pw)
    assert cnt == len(o_ids) and tot == o_tot and np.array_equal(ids, o_ids)
    with lib.MSTGraph(g.n, ps, pd, pw, host=True) as h:
        for _ in range(2):
            ids, cnt, tot = h.run_host()
            assert cnt == len(o_ids) and tot == o_tot and np.array_equal(ids, o_ids)


def test_host_streamed_errors(lib, oracle_mod, monkeypatch):
    """An out-of-range endpoint in a later chunk fails the streamed build cleanly (EINVAL),
    with weight copies still in flight; the library stays usable."""
    monkeypatch.setenv("MST_HOST_CHUNK", "1000")
    m = 5000
    src = np.arange(m, dtype=np.int32) % 100
    dst = (np.arange(m, dtype=np.int32) * 7 + 1) % 100
    dst[4321] = 100  # n = 100: out of range, in the fifth chunk
    with pytest.raises(lib.MSTError) as e:
        lib.mst_solve_host(100, src, dst, np.ones(m, np.uint32))
    assert e.value.status == 1
    dst[4321] = 5
    w = (np.arange(m, dtype=np.uint32) * 2654435761 % 1000).astype(np.uint32)
    ids, cnt, tot = lib.mst_solve_host(100, src, dst, w)
    o_ids, o_tot = oracle_mod.kruskal(100, src, dst, w)
    assert cnt == len(o_ids) and tot == o_tot and np.array_equal(ids, o_ids)


def test_errors(lib):
    with pytest.raises(lib.MSTError) as e:
        lib.MSTGraph(3, dev([0, 1]), dev([1, 3]), dev([1, 1]))
    assert e.value.status == 1
    with pytest.raises(lib.MSTError) as e:
        lib.MSTGraph(3, dev([0, -1]), dev([1, 2]), dev([1, 1]))
    assert e.value.status == 1
    with pytest.raises(lib.MSTError) as e:
        lib.mst_solve_host(-1, np.array([], np.int32), np.array([], np.int32), np.array([], np.uint32))
    assert e.value.status == 1
    # a valid handle still works after failed creates (nothing leaked / poisoned)
    ids, cnt, tot = lib.mst_solve_host(3, np.array([0, 1]), np.array([1, 2]), np.array([5, 6]))
    assert list(ids) == [0, 1] and tot == 11


def test_profiling_stats(lib, gg):
    g = gg.config(2, scale_down=4)
    with lib.MSTGraph(g.n, dev(g.src), dev(g.dst), dev(g.w)) as h:
        h.set_profiling(True)
        h.run()
        st = h.stats()
    assert st["profiling"] and st["kernel_ms"]["filter"] > 0
    dr = st["dense_round"]
    # the last round only hooks (<= 1 live component left): filters run in rounds 0..R-2
    assert st["kernel_launches"]["filter"] == (dr if dr >= 0 else st["rounds"] - 1)
    assert st["a_r"][0] == st["arcs0"] and st["n_r"][0] == g.n
    assert all(a >= b for a, b in zip(st["n_r"], st["n_r"][1:]))


# ------------------------------------------------------------------ full-size configs
@pytest.mark.parametrize("k", [1, 2, 3, 4, 5])
def test_full_size_configs(lib, oracle_mod, gg, k):
    g = gg.config(k)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w)
    # |F| = n - c with c from the oracle's own component labelling (not from Kruskal)
    _, c = oracle_mod.components(g.n, g.src, g.dst)
    assert st["num_edges"] == g.n - c


# ------------------------------------------------------------------ sparse-only rounds
@pytest.mark.parametrize("k,sd", [(1, 0), (2, 6), (4, 8), (5, 6)])
def test_sparse_only_rounds(lib, oracle_mod, gg, k, sd):
    """MST_OPT_DENSE = 0 keeps every round on the compaction path (no dense min-matrix)."""
    g = gg.config(k, s=2, scale_down=sd)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w,
                       options=[(lib.mst.MST_OPT_DENSE, 0)], runs=2)
    assert st["dense_round"] == -1


@pytest.mark.parametrize("k,sd", [(1, 0), (2, 6), (3, 8), (4, 8), (5, 6)])
def test_keep_edges_paper_scheme(lib, oracle_mod, gg, k, sd):
    """MST_OPT_KEEP_EDGES = 1: no deletion, original records re-read every round."""
    g = gg.config(k, s=4, scale_down=sd)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w,
                       options=[(lib.mst.MST_OPT_KEEP_EDGES, 1)], runs=2)
    assert st["dense_round"] == -1
    assert all(a == st["arcs0"] for a in st["a_r"])  # nothing is ever deleted


@pytest.mark.parametrize("tau", [0, 300, 900, 1000])
@pytest.mark.parametrize("k,sd", [(1, 0), (2, 6), (3, 8), (4, 8), (5, 6)])
def test_compaction_policy(lib, oracle_mod, gg, k, sd, tau):
    """MST_OPT_COMPACT_TAU: a pass compacts only when its sampled survival is below tau;
    otherwise later passes re-read the same records through the composed label map (row A7).
    Every policy -- never (0), adaptive, always (1000) -- gives the identical forest, also
    with the dense rounds off (long chains of non-compacting sparse passes)."""
    g = gg.config(k, s=7, scale_down=sd)
    for extra in ([], [(lib.mst.MST_OPT_DENSE, 0)]):
        st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=2,
                           options=[(lib.mst.MST_OPT_COMPACT_TAU, tau), (LF, 0)] + extra)
        sparse = [r for r in range(st["rounds"] - 1)
                  if st["dense_round"] < 0 or r + 1 < st["dense_round"]]
        if tau == 0:
            assert not any(st["compacted"])
        if tau == 1000:
            assert all(st["compacted"][r] for r in sparse)
        for r in range(1, st["rounds"]):  # a non-compacting pass keeps every record
            if r - 1 in sparse and r in sparse and not st["compacted"][r - 1]:
                assert st["a_r"][r] == st["a_r"][r - 1]
        for r in sparse:
            sp = st["survival_permille"][r]
            if 0 < tau < 1000:
                assert 0 <= sp <= 1000 and st["compacted"][r] == (sp < tau)
            else:
                assert sp == -1


def test_compaction_policy_sharded(lib, oracle_mod, gg):
    """the sampled decision is taken once per pass for every shard of a simulated split"""
    g = gg.config(4, s=8, scale_down=8)
    for tau in (0, 700, 1000):
        assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, nshards=3, runs=2,
                      options=[(lib.mst.MST_OPT_COMPACT_TAU, tau), (lib.mst.MST_OPT_DENSE, 0)])


def test_compaction_tau_range(lib, gg):
    g = gg.config(1)
    with lib.MSTGraph(g.n, dev(g.src), dev(g.dst), dev(g.w)) as h:
        for bad in (-1, 1001):
            with pytest.raises(lib.MSTError):
                h.set_option(lib.mst.MST_OPT_COMPACT_TAU, bad)


def test_options_switch_on_one_handle(lib, oracle_mod, gg):
    g = gg.config(4, s=5, scale_down=8)
    o_ids, o_tot = oracle_mod.kruskal(g.n, g.src, g.dst, g.w)
    with lib.MSTGraph(g.n, dev(g.src), dev(g.dst), dev(g.w)) as h:
        for opts in ([], [(2, 1)], [(2, 0), (1, 0)], [(1, 1)]):
            for o, v in opts:
                h.set_option(o, v)
            ids, cnt, tot = h.run()
            assert np.array_equal(ids.cpu().numpy(), o_ids) and tot == o_tot
        with pytest.raises(lib.MSTError):
            h.set_option(99, 1)


@pytest.mark.parametrize("tail", [1, 0])
@pytest.mark.parametrize("k,sd", [(1, 0), (4, 6), (5, 6), (3, 6), (2, 4)])
def test_dense_rounds_used(lib, oracle_mod, gg, k, sd, tail):
    """dense rounds both in the cooperative device tail and as per-round launches"""
    g = gg.config(k, s=3, scale_down=sd)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=2,
                       options=[(lib.mst.MST_OPT_DEVICE_TAIL, tail), (LF, 0)])
    assert st["dense_round"] >= 0
    assert st["n_r"][-1] <= 1 or st["rounds"] >= 1


# ------------------------------------------------------------------ distributed path, 1 rank
@pytest.mark.parametrize("k,sd", [(1, 0), (4, 8), (3, 8), (5, 6)])
def test_dist_single_rank_nccl(lib, oracle_mod, gg, k, sd):
    """mst_create_dist with nranks = 1: a real NCCL communicator and the per-round
    ncclAllReduce(MIN) of best (and of the min-matrix at the dense transition) on one GPU."""
    g = gg.config(k, s=6, scale_down=sd)
    try:
        uid = lib.mst_get_unique_id()
    except lib.MSTError as e:
        pytest.skip(f"NCCL unique id unavailable: {e}")
    o_ids, o_tot = oracle_mod.kruskal(g.n, g.src, g.dst, g.w)
    with lib.MSTGraph(g.n, dev(g.src), dev(g.dst), dev(g.w), dist=(uid, 0, 1)) as h:
        h.set_profiling(True)
        for opts in ([], [(lib.mst.MST_OPT_DEVICE_TAIL, 0)], [(lib.mst.MST_OPT_KEEP_EDGES, 1)]):
            for o, v in opts:
                h.set_option(o, v)
            ids, cnt, tot = h.run()
            assert np.array_equal(ids.cpu().numpy(), o_ids) and tot == o_tot
        st = h.stats()
        assert st["nranks"] == 1 and st["kernel_launches"]["comm"] >= 1


# ------------------------------------------------------------------ light-edge phase


@pytest.mark.parametrize("seed", range(24))
def test_light_first_random_dense(lib, oracle_mod, seed):
    """dense random multigraphs (m/n 10..60) with the light-edge phase at several K: ties at
    the threshold (few distinct weights), loops, parallels, several components"""
    rng = np.random.default_rng(7000 + seed)
    K = [1, 2, 4][seed % 3]
    n = int(rng.integers(300, 6000))
    m = int(n * rng.integers(4 * K + 1, 60))
    wmax = [0, 1, 7, 1000, 2**32 - 1, 3][seed % 6]
    src, dst, w = mc.random_multigraph(rng, n, m, wmax)
    if seed % 4 == 3:  # a second part joined to nothing: two big components
        src = np.concatenate([src, src + n]); dst = np.concatenate([dst, dst + n])
        w = np.concatenate([w, w]); n *= 2
    st = assert_parity(lib, oracle_mod, n, src, dst, w, runs=2, options=[(LF, K)])
    assert st["light_t"] != 0xFFFFFFFF


def test_light_first_deferred_components(lib, oracle_mod):
    """a light core plus pendant vertices and a whole second core reachable only through
    heavy edges: components without a light edge are deferred through the light phase and
    merged after the heavy records are re-read"""
    rng = np.random.default_rng(5)
    n1, n2, np_ = 4000, 3000, 2000
    n = n1 + n2 + np_
    m1 = 40 * n1
    s1 = rng.integers(0, n1, m1); d1 = rng.integers(0, n1, m1); w1 = rng.integers(0, 100, m1)
    m2 = 40 * n2
    s2 = n1 + rng.integers(0, n2, m2); d2 = n1 + rng.integers(0, n2, m2)
    w2 = rng.integers(900, 1000, m2)                              # second core: heavy only
    sp = np.arange(n1 + n2, n); dp = rng.integers(0, n1 + n2, np_)
    wp = rng.integers(800, 1000, np_)                              # pendants: heavy only
    sb = rng.integers(0, n1, 50); db = n1 + rng.integers(0, n2, 50)
    wb = rng.integers(950, 1000, 50)                               # bridges: heavy
    src = np.concatenate([s1, s2, sp, sb]).astype(np.int32)
    dst = np.concatenate([d1, d2, dp, db]).astype(np.int32)
    w = np.concatenate([w1, w2, wp, wb]).astype(np.uint32)
    for K in (1, 4):
        st = assert_parity(lib, oracle_mod, n, src, dst, w, runs=2, options=[(LF, K)])
        assert st["light_t"] < 900 and st["light_switch_round"] >= 1


@pytest.mark.parametrize("K", [0, 1, 4, 16])
@pytest.mark.parametrize("k,sd", [(4, 6), (5, 6), (5, 4), (4, 4)])
def test_light_first_configs(lib, oracle_mod, gg, k, sd, K):
    g = gg.config(k, s=2, scale_down=sd)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=2, options=[(LF, K)])
    assert (st["light_t"] == 0xFFFFFFFF) == (K == 0 or st["arcs0"] < 4 * K * g.n)


@pytest.mark.parametrize("opts", [[(1, 0)], [(3, 0)], [(4, 0)], [(4, 1000)], [(1, 0), (4, 0)]])
def test_light_first_with_other_options(lib, oracle_mod, gg, opts):
    g = gg.config(5, s=3, scale_down=5)
    assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=2, options=[(LF, 2)] + opts)


def test_light_first_option_range(lib, gg):
    g = gg.config(1)
    with lib.MSTGraph(g.n, dev(g.src), dev(g.dst), dev(g.w)) as h:
        for bad in (-2, 65):
            with pytest.raises(lib.MSTError):
                h.set_option(LF, bad)
        h.set_option(LF, 64)
        h.set_option(LF, -1)


def test_light_only_round0_deferred(lib, oracle_mod):
    """dense regime (>= 64 records per vertex, auto options): round 0 reads only the light
    records; pendant vertices whose edges are all heavy are deferred from round 0 on and get
    their edge after the switch to all records; isolated vertices finish"""
    rng = np.random.default_rng(11)
    nc, npend, niso = 3000, 500, 50
    n = nc + npend + niso
    mc_ = 100 * nc
    s1 = rng.integers(0, nc, mc_); d1 = rng.integers(0, nc, mc_); w1 = rng.integers(0, 100, mc_)
    sp = np.repeat(np.arange(nc, nc + npend), 2); dp = rng.integers(0, nc, 2 * npend)
    wp = rng.integers(900, 1000, 2 * npend)
    src = np.concatenate([s1, sp]).astype(np.int32)
    dst = np.concatenate([d1, dp]).astype(np.int32)
    w = np.concatenate([w1, wp]).astype(np.uint32)
    st = assert_parity(lib, oracle_mod, n, src, dst, w, runs=2)
    # the pendants got their exact round-0 minimum from their own records (the reverse index
    # exists at >= 8 records per vertex: member_ends[0] = the record ends that scan read), or
    # their edge after the switch to all records
    assert st["light_t"] < 900
    assert st["light_switch_round"] >= 0 or st["member_ends"][0] > 0
    # without the member scans: deferred from round 0 on, the switch re-reads every record
    env = dict(os.environ, MST_MEMBER_SCAN="0")
    code = ("import sys; sys.path.insert(0, 'tests'); import numpy as np, test_parity_gpu as t, "
            "paper_conf_ppopp_nasrebp13_b200 as p, oracle as o; p.load(); o.build(); "
            "t.check_light_only_round0_no_member(p, o)")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                       timeout=600, cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    assert r.returncode == 0, r.stderr[-3000:]


def _light_only_graph():
    rng = np.random.default_rng(11)
    nc, npend, niso = 3000, 500, 50
    n = nc + npend + niso
    mc_ = 100 * nc
    s1 = rng.integers(0, nc, mc_); d1 = rng.integers(0, nc, mc_); w1 = rng.integers(0, 100, mc_)
    sp = np.repeat(np.arange(nc, nc + npend), 2); dp = rng.integers(0, nc, 2 * npend)
    wp = rng.integers(900, 1000, 2 * npend)
    src = np.concatenate([s1, sp]).astype(np.int32)
    dst = np.concatenate([d1, dp]).astype(np.int32)
    w = np.concatenate([w1, wp]).astype(np.uint32)
    return n, src, dst, w


def check_light_only_round0_no_member(lib, oracle_mod):
    n, src, dst, w = _light_only_graph()
    st = assert_parity(lib, oracle_mod, n, src, dst, w, runs=2)
    assert st["light_t"] < 900 and st["light_switch_round"] >= 0


@pytest.mark.parametrize("nclusters", [60, 140, 400, 900])
def test_transition_into_few_components(lib, oracle_mod, nclusters):
    """many records between few components at the dense transition: the whole next matrix in
    shared memory (<= ~157 components), local rows + warp-merged REDs (<= 1024), with and
    without the hub row (a hub joined to everything by heavy edges makes degrees heavy-tailed)"""
    rng = np.random.default_rng(nclusters)
    size = 40
    n = nclusters * size + 1
    base = 1 + np.arange(nclusters) * size
    # light edges inside clusters (each cluster contracts in the first rounds)
    ci = rng.integers(0, nclusters, 60 * nclusters)
    s1 = base[ci] + rng.integers(0, size, ci.size); d1 = base[ci] + rng.integers(0, size, ci.size)
    w1 = rng.integers(0, 100, ci.size)
    # many medium edges between clusters (the records that cross at the transition)
    ca, cb = rng.integers(0, nclusters, 400 * nclusters), rng.integers(0, nclusters, 400 * nclusters)
    s2 = base[ca] + rng.integers(0, size, ca.size); d2 = base[cb] + rng.integers(0, size, cb.size)
    w2 = rng.integers(100, 900, ca.size)
    # the hub: vertex 0 joined to every vertex by heavy edges
    s3 = np.zeros(n - 1, np.int64); d3 = np.arange(1, n); w3 = rng.integers(900, 1000, n - 1)
    src = np.concatenate([s1, s2, s3]).astype(np.int32)
    dst = np.concatenate([d1, d2, d3]).astype(np.int32)
    w = np.concatenate([w1, w2, w3]).astype(np.uint32)
    for opts in ([(LF, 0)], [(LF, 0), (lib.mst.MST_OPT_DEVICE_TAIL, 0)], []):
        st = assert_parity(lib, oracle_mod, n, src, dst, w, runs=2, options=opts)
    assert st["rounds"] >= 2


@pytest.mark.parametrize("seed", range(16))
def test_light_auto_dense_regime_random(lib, oracle_mod, seed):
    """default options on random multigraphs with >= 64 records per vertex: light-only round 0
    (K = 8) with ties at the threshold, loops, parallels, disconnected parts and vertices whose
    edges are all heavy"""
    rng = np.random.default_rng(9100 + seed)
    n = int(rng.integers(200, 3000))
    m = int(n * rng.choice([70, 100, 200]))
    wmax = [0, 2, 9, 1000, 2**32 - 1, 50][seed % 6]
    src, dst, w = mc.random_multigraph(rng, n, m, wmax)
    if seed % 3 == 0:  # a few vertices whose edges are all much heavier
        k = max(1, n // 50)
        hv = rng.choice(n, k, replace=False)
        heavy = np.isin(src, hv) | np.isin(dst, hv)
        w = np.where(heavy, np.uint32(min(2**32 - 1, int(wmax) * 4 + 100)), w).astype(np.uint32)
    if seed % 4 == 1:  # plus a separate small dense part
        src = np.concatenate([src, (src[:m // 8] % 64) + n]); dst = np.concatenate([dst, (dst[:m // 8] % 64) + n])
        w = np.concatenate([w, w[:m // 8]]); n += 64
    assert_parity(lib, oracle_mod, n, src, dst, w, runs=2)


def test_output_dense_forest_tiles(lib, oracle_mod):
    """forest edges packed into the first edge ids (a path listed first, then many heavier
    edges): the output's id staging is sized to the average forest density, so these tiles
    exceed it and take the direct-store path"""
    rng = np.random.default_rng(17)
    n = 300_000
    ps = np.arange(n - 1, dtype=np.int64)
    extra = 4_000_000
    es = rng.integers(0, n, extra); ed = rng.integers(0, n, extra)
    src = np.concatenate([ps, es]).astype(np.int32)
    dst = np.concatenate([ps + 1, ed]).astype(np.int32)
    w = np.concatenate([rng.integers(0, 10, n - 1), rng.integers(10, 1000, extra)]).astype(np.uint32)
    assert_parity(lib, oracle_mod, n, src, dst, w, runs=2)


# ------------------------------------------------------------------ NEXT-3: union-find variant
UF = 6  # MST_OPT_UNION_FIND (include/mst.h)


@pytest.mark.parametrize("seed", range(40))
def test_union_find_random_multigraphs(lib, oracle_mod, seed):
    rng = np.random.default_rng(5000 + seed)
    n = int(rng.integers(1, 20_000))
    m = int(rng.integers(0, 8 * n))
    wmax = [0, 1, 7, 1000, 2**32 - 1][seed % 5]
    src, dst, w = mc.random_multigraph(rng, n, m, wmax)
    st = assert_parity(lib, oracle_mod, n, src, dst, w, runs=2, options=[(UF, 1)])
    assert st["dense_round"] == -1 and st["light_t"] == 0xFFFFFFFF


@pytest.mark.parametrize("tau", [0, 500, 900, 1000])
@pytest.mark.parametrize("k,sd", [(1, 0), (2, 6), (3, 8), (4, 6), (5, 6)])
def test_union_find_configs(lib, oracle_mod, gg, k, sd, tau):
    g = gg.config(k, s=9, scale_down=sd)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=2,
                       options=[(UF, 1), (lib.mst.MST_OPT_COMPACT_TAU, tau)])
    assert not st["compacted"][0]  # round 0: every non-loop record crosses two singletons
    if tau == 0:
        assert all(a == st["arcs0"] for a in st["a_r"])  # the records are never touched
    assert st["n_r"][0] == g.n and all(a >= b for a, b in zip(st["n_r"], st["n_r"][1:]))


@pytest.mark.parametrize("k", [1, 2, 3, 4, 5])
def test_union_find_full_size(lib, oracle_mod, gg, k):
    g = gg.config(k)
    assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, options=[(UF, 1)])


def test_union_find_adversarial(lib, oracle_mod):
    # monotone path: every union links the next vertex, one chain of depth n - 1
    n = 300_000
    src = np.arange(n - 1, dtype=np.int32)
    assert_parity(lib, oracle_mod, n, src, src + 1, np.arange(1, n, dtype=np.uint32),
                  options=[(UF, 1)])
    assert_parity(lib, oracle_mod, n, src, src + 1, np.arange(n - 1, 0, -1).astype(np.uint32),
                  options=[(UF, 1)])
    # star of degree 10^6 with extra cross edges; empty and degenerate inputs
    n = 1_000_001
    rng = np.random.default_rng(4)
    src = np.zeros(n - 1, np.int32)
    dst = np.arange(1, n, dtype=np.int32)
    w = rng.integers(0, 1000, n - 1).astype(np.uint32)
    assert_parity(lib, oracle_mod, n, src, dst, w, options=[(UF, 1)])
    for n, s_, d_, w_ in [(0, [], [], []), (1, [], [], []), (5, [], [], []),
                          (3, [0, 1, 2], [0, 1, 2], [1, 2, 3]), (2, [1, 0, 1], [0, 1, 0], [3, 3, 3])]:
        assert_parity(lib, oracle_mod, n, s_, d_, w_, options=[(UF, 1)])


def test_union_find_single_gpu_only(lib, gg):
    g = gg.config(1)
    with lib.MSTGraph(g.n, dev(g.src), dev(g.dst), dev(g.w), nshards=2) as h:
        h.set_option(UF, 1)
        with pytest.raises(lib.MSTError) as e:
            h.run()
        assert e.value.status == 6  # MST_ENOTSUP


# ------------------------------------------------------------------ A10: the one-CTA path
def _small_used(st):
    return st["kernel_launches"].get("small", 0) > 0 if st["profiling"] else st["gpu_launches"] == 1


@pytest.mark.parametrize("seed", range(60))
def test_small_path_random_multigraphs(lib, oracle_mod, seed):
    """graphs that fit one CTA's shared memory run every round in one launch (the default)"""
    rng = np.random.default_rng(8000 + seed)
    n = int(rng.integers(2, 4000))
    m = int(rng.integers(0, min(9000, 6 * n)))
    wmax = [0, 1, 7, 1000, 2**32 - 1][seed % 5]
    src, dst, w = mc.random_multigraph(rng, n, m, wmax)
    st = assert_parity(lib, oracle_mod, n, src, dst, w, runs=2, small=True)
    assert st["gpu_launches"] == 1  # the whole method in one kernel


@pytest.mark.parametrize("seed", range(20))
def test_small_path_tiny_vs_brute_force(lib, seed):
    rng = np.random.default_rng(300 + seed)
    n = int(rng.integers(1, 7)); m = int(rng.integers(0, 11))
    src, dst, w = mc.random_multigraph(rng, n, m, 2)
    ids, cnt, tot, _ = gpu_msf(lib, n, src, dst, w, small=True)
    bf, bf_w, _ = mc.brute_force_msf(n, src, dst, w)
    assert list(ids) == bf and tot == bf_w


def test_small_path_grid64_and_edges(lib, oracle_mod, gg):
    g = gg.config(1)  # grid64: the BASELINE config the one-CTA path exists for
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=3, small=True)
    assert st["gpu_launches"] == 1 and st["rounds"] >= 3
    assert st["n_r"][0] == g.n and st["a_r"][0] == st["arcs0"]
    for n, s_, d_, w_ in [(1, [], [], []), (5, [], [], []), (3, [0, 1, 2], [0, 1, 2], [1, 2, 3]),
                          (2, [0], [1], [2**32 - 1]), (2, [1, 0, 1], [0, 1, 0], [3, 3, 3])]:
        assert_parity(lib, oracle_mod, n, s_, d_, w_, small=True)
    # a monotone path (every vertex hooks left: one chain of depth n - 1 in one CTA)
    n = 6000
    src = np.arange(n - 1, dtype=np.int32)
    assert_parity(lib, oracle_mod, n, src, src + 1, np.arange(1, n, dtype=np.uint32), small=True)
    # a graph just too large for shared memory takes the multi-kernel path
    g = gg.config(2, scale_down=8)  # n = 16 K, m = 64 K
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, small=True)
    assert st["gpu_launches"] > 1


# ------------------------------------------------------------------ member-scan rounds
@pytest.mark.parametrize("k,sd,seed", [(4, 4, 1), (4, 2, 2), (4, 6, 3), (5, 6, 4)])
def test_member_scan_rounds(lib, oracle_mod, gg, k, sd, seed):
    """after the light-edge phase of a heavy-tailed graph the components outside the top hub's
    take their minima from their members' records (reverse index) instead of a pass over every
    record; the hub's component is deferred; bit-exact, re-runnable"""
    g = gg.config(k, s=seed, scale_down=sd)
    st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=2)
    if k == 4 and st["light_switch_round"] >= 0:
        assert any(x >= 0 for x in st["member_ends"])  # at least one member-scan round


def test_member_scan_two_giants(lib, oracle_mod, gg):
    """two heavy-tailed graphs side by side, joined by one heavy edge: after the light phase a
    second giant lies outside the top hub's component, the member work is large, and the run
    falls back to a pass over every record; bit-exact either way"""
    a = gg.config(4, s=5, scale_down=4)
    b = gg.config(4, s=6, scale_down=4)
    n = a.n + b.n
    src = np.concatenate([a.src, b.src + a.n, [0]]).astype(np.int32)
    dst = np.concatenate([a.dst, b.dst + a.n, [a.n]]).astype(np.int32)
    w = np.concatenate([a.w, b.w, [999]]).astype(np.uint32)
    assert_parity(lib, oracle_mod, n, src, dst, w, runs=2)


# ------------------------------------------------------------------ A9: sort-based dedup
DEDUP = 8  # MST_OPT_DEDUP (include/mst.h)


@pytest.mark.parametrize("k,sd", [(2, 6), (3, 8), (4, 6), (5, 6), (2, 2)])
def test_dedup_configs(lib, oracle_mod, gg, k, sd):
    """after every sparse pass the survivors are sorted by component pair and only each pair's
    minimum record is kept (A9); the forest is unchanged and the records shrink"""
    g = gg.config(k, s=11, scale_down=sd)
    for extra in ([], [(lib.mst.MST_OPT_DENSE, 0), (LF, 0)]):
        st = assert_parity(lib, oracle_mod, g.n, g.src, g.dst, g.w, runs=2,
                           options=[(DEDUP, 1)] + extra)
        for r, din in enumerate(st["dedup_in"]):
            if din >= 0:
                assert st["a_r"][r + 1] <= din  # never more records after the dedup


@pytest.mark.parametrize("seed", range(12))
def test_dedup_random_multigraphs(lib, oracle_mod, seed):
    rng = np.random.default_rng(6100 + seed)
    n = int(rng.integers(2, 30_000))
    m = int(rng.integers(0, 40 * n))
    src, dst, w = mc.random_multigraph(rng, n, m, [1, 7, 1000, 2**32 - 1][seed % 4])
    assert_parity(lib, oracle_mod, n, src, dst, w, runs=2,
                  options=[(DEDUP, 1), (lib.mst.MST_OPT_DENSE, seed % 2)])
