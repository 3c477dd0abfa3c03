"""Independent checkers that pin the oracle (and, transitively, the CUDA path).

None of these call ``oracle/``; each is a different algorithm or a property that the
unique minimum spanning forest F* under the order (w, id) must satisfy (SURVEY.md §8(c)
"What pins each part"):

* ``brute_force_msf``  — enumerate every spanning forest, argmin of sum(w*m + id)
* ``prim_msf``         — Prim with a heap keyed by (w, id), restarted per component
* ``bfs_components``   — connected components by BFS (pins |F| = n - c)
* ``check_cut_property`` / ``check_cycle_property`` — the two optimality certificates
"""
from __future__ import annotations

import heapq
import itertools
from collections import deque

import numpy as np


def _adj(n, src, dst):
    adj = [[] for _ in range(n)]
    for i, (u, v) in enumerate(zip(src, dst)):
        u, v = int(u), int(v)
        if u != v:
            adj[u].append((v, i))
            adj[v].append((u, i))
    return adj


def bfs_components(n, src, dst):
    """Returns (c, comp) with comp[v] = component index in discovery order."""
    adj = _adj(n, src, dst)
    comp = [-1] * n
    c = 0
    for s in range(n):
        if comp[s] >= 0:
            continue
        comp[s] = c
        q = deque([s])
        while q:
            x = q.popleft()
            for y, _ in adj[x]:
                if comp[y] < 0:
                    comp[y] = c
                    q.append(y)
        c += 1
    return c, comp


def _is_acyclic(n, edges, src, dst):
    par = list(range(n))

    def find(x):
        while par[x] != x:
            par[x] = par[par[x]]
            x = par[x]
        return x

    for i in edges:
        a, b = find(int(src[i])), find(int(dst[i]))
        if a == b:
            return False
        par[a] = b
    return True


def brute_force_msf(n, src, dst, w):
    """Exhaustive: every acyclic subset of n-c non-loop edges is a spanning forest; F* is
    the unique argmin of sum(w_e*m + e) (distinct element weights => unique min basis).
    Returns (sorted ids, min total weight over all spanning forests, #minimisers)."""
    m = len(src)
    c, _ = bfs_components(n, src, dst)
    k = n - c
    cand = [i for i in range(m) if int(src[i]) != int(dst[i])]
    best_f, best_set, n_best, min_w = None, None, 0, None
    for sub in itertools.combinations(cand, k):
        if not _is_acyclic(n, sub, src, dst):
            continue
        f = sum(int(w[i]) * m + i for i in sub)
        tw = sum(int(w[i]) for i in sub)
        min_w = tw if min_w is None else min(min_w, tw)
        if best_f is None or f < best_f:
            best_f, best_set, n_best = f, sub, 1
        elif f == best_f:
            n_best += 1
    if best_set is None:  # k == 0
        best_set, min_w, n_best = (), 0, 1
    return sorted(best_set), min_w, n_best


def prim_msf(n, src, dst, w):
    """Prim's algorithm with a heap keyed by (w, id); restarted from each unvisited vertex
    in increasing id order, so it returns a spanning forest. Returns (sorted ids, total)."""
    adj = _adj(n, src, dst)
    seen = [False] * n
    out, total = [], 0
    for root in range(n):
        if seen[root]:
            continue
        seen[root] = True
        h = [(int(w[i]), i, y) for y, i in adj[root]]
        heapq.heapify(h)
        while h:
            wi, i, y = heapq.heappop(h)
            if seen[y]:
                continue
            seen[y] = True
            out.append(i)
            total += wi
            for z, j in adj[y]:
                if not seen[z]:
                    heapq.heappush(h, (int(w[j]), j, z))
    return sorted(out), total


def _forest_adj(n, ids, src, dst):
    fadj = [[] for _ in range(n)]
    for i in ids:
        u, v = int(src[i]), int(dst[i])
        fadj[u].append((v, i))
        fadj[v].append((u, i))
    return fadj


def _reach(fadj, start, banned):
    seen = {start}
    q = deque([start])
    while q:
        x = q.popleft()
        for y, i in fadj[x]:
            if i != banned and y not in seen:
                seen.add(y)
                q.append(y)
    return seen


def check_cut_property(n, src, dst, w, ids):
    """Every forest edge f=(u,v) is the (w,id)-minimum edge crossing the cut between the
    two halves of its tree obtained by deleting f."""
    fadj = _forest_adj(n, ids, src, dst)
    for f in ids:
        f = int(f)
        su = _reach(fadj, int(src[f]), f)
        sv = _reach(fadj, int(dst[f]), f)
        assert not (su & sv), "forest edge closes a cycle"
        kf = (int(w[f]), f)
        for e in range(len(src)):
            a, b = int(src[e]), int(dst[e])
            if (a in su and b in sv) or (a in sv and b in su):
                assert (int(w[e]), e) >= kf, f"cut property violated by edge {e} vs {f}"
    return True


def check_cycle_property(n, src, dst, w, ids):
    """Every non-forest non-loop edge joins two vertices of one tree and is (w,id)-greater
    than every edge on the tree path between them."""
    idset = set(int(i) for i in ids)
    fadj = _forest_adj(n, ids, src, dst)
    # root every tree, record parent edge and depth
    par = [-1] * n
    pedge = [-1] * n
    depth = [-1] * n
    for r in range(n):
        if depth[r] >= 0:
            continue
        depth[r] = 0
        q = deque([r])
        while q:
            x = q.popleft()
            for y, i in fadj[x]:
                if depth[y] < 0:
                    depth[y], par[y], pedge[y] = depth[x] + 1, x, i
                    q.append(y)
    for e in range(len(src)):
        a, b = int(src[e]), int(dst[e])
        if a == b or e in idset:
            continue
        ke = (int(w[e]), e)
        x, y = a, b
        while x != y:
            if depth[x] < depth[y]:
                x, y = y, x
            if par[x] < 0:
                raise AssertionError(f"non-forest edge {e} joins two trees: forest not spanning")
            i = pedge[x]
            assert (int(w[i]), i) < ke, f"cycle property violated: edge {e} vs path edge {i}"
            x = par[x]
    return True


def random_multigraph(rng: np.random.Generator, n, m, wmax):
    src = rng.integers(0, n, m).astype(np.int32)
    dst = rng.integers(0, n, m).astype(np.int32)
    w = rng.integers(0, wmax + 1, m).astype(np.uint64).astype(np.uint32)
    return src, dst, w


def load_golden(path):
    n, edges, exp = None, [], {}
    with open(path) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            tok = line.split()
            if tok[0] == "n":
                n = int(tok[1])
            elif tok[0] == "e":
                edges.append((int(tok[1]), int(tok[2]), int(tok[3])))
            else:
                exp[tok[0]] = [int(t) for t in tok[1:]]
    src = np.array([e[0] for e in edges], np.int32)
    dst = np.array([e[1] for e in edges], np.int32)
    w = np.array([e[2] for e in edges], np.uint64).astype(np.uint32)
    return n, src, dst, w, exp
