"""Pins for the oracle (CPU only, -m "not gpu").

The oracle (oracle/kruskal.cpp) is checked against things other than itself: hand-worked
golden fixtures, brute force over all spanning forests, an independent Prim, the cut and
cycle optimality certificates, |F| = n - c from BFS, closed forms, and networkx's total
weight. A plausible oracle bug — a dropped tie-break, skipping the wrong edges, an
off-by-one in ids, a 32-bit total, union without find — fails at least one of these.
"""
import glob
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st, HealthCheck

import mstcheck as mc

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ------------------------------------------------------------------ golden (hand-worked)
@pytest.mark.parametrize("path", sorted(glob.glob(os.path.join(GOLDEN, "hand_*.txt"))))
def test_golden_hand_worked(oracle_mod, path):
    n, src, dst, w, exp = mc.load_golden(path)
    ids, total = oracle_mod.kruskal(n, src, dst, w)
    assert list(ids) == exp["expect_ids"]
    assert total == exp["expect_total"][0]
    assert len(ids) == exp["expect_count"][0]


# ------------------------------------------------------------------ brute force, n <= 7
@st.composite
def small_multigraph(draw):
    n = draw(st.integers(1, 7))
    m = draw(st.integers(0, 11))
    wmax = draw(st.sampled_from([0, 1, 3, 2**32 - 1]))
    edges = draw(st.lists(st.tuples(st.integers(0, n - 1), st.integers(0, n - 1),
                                    st.integers(0, wmax)), min_size=m, max_size=m))
    src = np.array([e[0] for e in edges], np.int32)
    dst = np.array([e[1] for e in edges], np.int32)
    w = np.array([e[2] for e in edges], np.uint64).astype(np.uint32)
    return n, src, dst, w


@settings(max_examples=400, deadline=None, suppress_health_check=list(HealthCheck))
@given(small_multigraph())
def test_brute_force(oracle_mod, g):
    n, src, dst, w = g
    ids, total = oracle_mod.kruskal(n, src, dst, w)
    bf_ids, bf_min_w, n_min = mc.brute_force_msf(n, src, dst, w)
    assert n_min == 1, "argmin of sum(w*m+id) must be unique"
    assert list(ids) == bf_ids
    assert total == bf_min_w  # the MSF also minimises plain total weight
    c, _ = mc.bfs_components(n, src, dst)
    assert len(ids) == n - c


# ------------------------------------------------------------------ Prim + certificates
@pytest.mark.parametrize("seed", range(12))
def test_prim_and_certificates(oracle_mod, seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 120))
    m = int(rng.integers(0, 4 * n))
    wmax = [0, 2, 10, 1000, 2**32 - 1][seed % 5]
    src, dst, w = mc.random_multigraph(rng, n, m, wmax)
    ids, total = oracle_mod.kruskal(n, src, dst, w)
    p_ids, p_total = mc.prim_msf(n, src, dst, w)
    assert list(ids) == p_ids and total == p_total
    c, _ = mc.bfs_components(n, src, dst)
    assert len(ids) == n - c
    mc.check_cut_property(n, src, dst, w, ids)
    mc.check_cycle_property(n, src, dst, w, ids)


@pytest.mark.parametrize("seed", range(4))
def test_prim_medium(oracle_mod, seed):
    rng = np.random.default_rng(100 + seed)
    n = 3000
    m = [2000, 6000, 12000, 30000][seed]
    src, dst, w = mc.random_multigraph(rng, n, m, [5, 1000, 2**32 - 1, 1][seed])
    ids, total = oracle_mod.kruskal(n, src, dst, w)
    p_ids, p_total = mc.prim_msf(n, src, dst, w)
    assert list(ids) == p_ids and total == p_total
    mc.check_cycle_property(n, src, dst, w, ids)


def test_networkx_total_weight(oracle_mod):
    nx = pytest.importorskip("networkx")
    rng = np.random.default_rng(7)
    for n, m in [(50, 200), (500, 1500), (2000, 9000)]:
        src, dst, w = mc.random_multigraph(rng, n, m, 100)
        ids, total = oracle_mod.kruskal(n, src, dst, w)
        G = nx.MultiGraph()
        G.add_nodes_from(range(n))
        for i in range(m):
            if src[i] != dst[i]:
                G.add_edge(int(src[i]), int(dst[i]), key=i, weight=int(w[i]))
        nx_total = sum(d["weight"] for _, _, _, d in
                       nx.minimum_spanning_edges(G, algorithm="kruskal", keys=True, data=True))
        assert total == nx_total  # tie-insensitive: only the total is comparable
        assert len(ids) == n - nx.number_connected_components(G)


# ------------------------------------------------------------------ closed forms
def test_tree_input_is_its_own_forest(oracle_mod):
    rng = np.random.default_rng(1)
    n = 500
    parent = np.array([rng.integers(0, v) for v in range(1, n)], np.int32)
    src, dst = np.arange(1, n, dtype=np.int32), parent
    w = rng.integers(0, 50, n - 1).astype(np.uint32)
    ids, total = oracle_mod.kruskal(n, src, dst, w)
    assert list(ids) == list(range(n - 1)) and total == int(w.astype(np.uint64).sum())


def test_monotone_path(oracle_mod):
    # the adversarial chain of SURVEY.md §7 hard part 6: a path is a tree -> all edges
    n = 10000
    src = np.arange(n - 1, dtype=np.int32)
    dst = src + 1
    w = np.arange(1, n, dtype=np.uint32)
    ids, total = oracle_mod.kruskal(n, src, dst, w)
    assert len(ids) == n - 1 and total == (n - 1) * n // 2


@pytest.mark.parametrize("n", [3, 4, 17])
def test_cycle_drops_its_max_edge(oracle_mod, n):
    rng = np.random.default_rng(n)
    src = np.arange(n, dtype=np.int32)
    dst = (src + 1) % n
    w = rng.integers(0, 4, n).astype(np.uint32)  # ties likely
    ids, total = oracle_mod.kruskal(n, src, dst, w)
    worst = max(range(n), key=lambda i: (int(w[i]), i))
    assert list(ids) == [i for i in range(n) if i != worst]
    assert total == int(w.astype(np.uint64).sum()) - int(w[worst])


def test_grid_horizontal_1_vertical_2(oracle_mod):
    W, H = 13, 9
    src, dst, w = [], [], []
    for y in range(H):
        for x in range(W):
            v = y * W + x
            if x < W - 1:
                src.append(v); dst.append(v + 1); w.append(1)
            if y < H - 1:
                src.append(v); dst.append(v + W); w.append(2)
    ids, total = oracle_mod.kruskal(W * H, src, dst, w)
    chosen = set(int(i) for i in ids)
    horiz = {i for i in range(len(src)) if w[i] == 1}
    vert = {i for i in range(len(src)) if w[i] == 2 and src[i] % W == 0}  # x = 0 column
    assert chosen == horiz | vert
    assert total == H * (W - 1) + 2 * (H - 1)


@pytest.mark.parametrize("n", [2, 5, 40])
def test_complete_graph_abs_diff(oracle_mod, n):
    src, dst, w = [], [], []
    for i in range(n):
        for j in range(i + 1, n):
            src.append(j); dst.append(i); w.append(j - i)
    ids, total = oracle_mod.kruskal(n, src, dst, w)
    assert total == n - 1
    assert {(min(src[i], dst[i]), max(src[i], dst[i])) for i in ids} == \
        {(i, i + 1) for i in range(n - 1)}


def test_parallel_copies_lowest_id(oracle_mod):
    k = 9
    ids, total = oracle_mod.kruskal(2, [0, 1] * k, [1, 0] * k, [5] * (2 * k))
    assert list(ids) == [0] and total == 5


def test_disjoint_union(oracle_mod):
    rng = np.random.default_rng(3)
    parts, off = [], 0
    allsrc, alldst, allw, expect, exp_total = [], [], [], [], 0
    for _ in range(5):
        n = int(rng.integers(1, 40)); m = int(rng.integers(0, 80))
        s, d, w = mc.random_multigraph(rng, n, m, 20)
        ids, tot = oracle_mod.kruskal(n, s, d, w)
        base = len(allsrc)
        expect += [base + int(i) for i in ids]
        exp_total += tot
        allsrc += list(s + off); alldst += list(d + off); allw += list(w)
        off += n
    ids, total = oracle_mod.kruskal(off, allsrc, alldst, allw)
    assert list(ids) == expect and total == exp_total


def test_all_equal_weights_is_greedy_by_id(oracle_mod):
    rng = np.random.default_rng(11)
    n, m = 300, 1200
    s, d, _ = mc.random_multigraph(rng, n, m, 0)
    ids, _ = oracle_mod.kruskal(n, s, d, np.full(m, 7, np.uint32))
    par = list(range(n))

    def find(x):
        while par[x] != x:
            x = par[x]
        return x
    greedy = []
    for i in range(m):
        a, b = find(int(s[i])), find(int(d[i]))
        if a != b:
            par[a] = b
            greedy.append(i)
    assert list(ids) == greedy


def test_max_weights_total_is_64bit(oracle_mod):
    n = 1000
    src = np.arange(n - 1, dtype=np.int32)
    ids, total = oracle_mod.kruskal(n, src, src + 1, np.full(n - 1, 2**32 - 1, np.uint32))
    assert total == (n - 1) * (2**32 - 1)


def test_empty_and_invalid(oracle_mod):
    assert oracle_mod.kruskal(0, [], [], [])[0].size == 0
    ids, total = oracle_mod.kruskal(5, [], [], [])
    assert ids.size == 0 and total == 0
    ids, total = oracle_mod.kruskal(3, [1, 2], [1, 2], [4, 4])  # only self-loops
    assert ids.size == 0 and total == 0
    with pytest.raises(ValueError):
        oracle_mod.kruskal(3, [0], [3], [1])
    with pytest.raises(ValueError):
        oracle_mod.kruskal(3, [-1], [0], [1])


def test_components_oracle_vs_bfs(oracle_mod):
    rng = np.random.default_rng(5)
    n, m = 2000, 1500
    s, d, _ = mc.random_multigraph(rng, n, m, 0)
    lab, c = oracle_mod.components(n, s, d)
    c_bfs, comp = mc.bfs_components(n, s, d)
    assert c == c_bfs
    # same partition: label is the min vertex of the BFS class
    mins = {}
    for v in range(n):
        mins.setdefault(comp[v], v)
    assert all(lab[v] == mins[comp[v]] for v in range(n))
