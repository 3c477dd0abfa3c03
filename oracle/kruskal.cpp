// oracle/kruskal.cpp — TEST INFRASTRUCTURE ONLY (the parity oracle).
//
// Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
// may load this. The product path (paper_conf_ppopp_nasrebp13_b200/) never links, calls
// or imports it, and it shares no code with the CUDA path.
//
// What it computes (DESIGN.md "Readings" R1-R6): the unique minimum
// spanning FOREST F* of an undirected multigraph under the strict edge order
//     e < f  <=>  (w_e, e) <_lex (w_f, f)            (R1: ties broken by edge id)
// Boruvka's method (§5) reaches exactly this forest; the plain
// definition we write out is Kruskal's "ordered algorithm": contract
// edges in increasing order, skipping those whose endpoints are already in one component.
// Self-loops are never in a forest (R4, "without self-loops"); parallel
// edges compete by (w, id) (R5); a disconnected input yields a spanning forest (R3).
//
// Steps (SURVEY.md §8(c) "Oracle algorithm"):
//   1. validate 0 <= src, dst < n;
//   2. k_i = (uint64(w_i) << 32) | i; sort ascending (library sort; keys are unique);
//   3. union-find over n vertices (union by size, path halving);
//   4. scan in key order: skip src == dst; if find(u) != find(v): union, record i, add w_i;
//   5. sort recorded ids ascending; return (ids, count, total).
//
// Parity pins for this file are in tests/test_oracle_pins.py (brute force, Prim, cut and
// cycle properties, |F| = n - c, closed forms, networkx total weight).
#include <algorithm>
#include <chrono>
#include <cstdint>
#include <vector>

namespace {

struct UnionFind {
    std::vector<int64_t> parent, size;
    explicit UnionFind(int64_t n) : parent(n), size(n, 1) {
        for (int64_t i = 0; i < n; ++i) parent[i] = i;
    }
    int64_t find(int64_t x) {
        while (parent[x] != x) {          // path halving
            parent[x] = parent[parent[x]];
            x = parent[x];
        }
        return x;
    }
    bool unite(int64_t a, int64_t b) {
        a = find(a); b = find(b);
        if (a == b) return false;
        if (size[a] < size[b]) std::swap(a, b);
        parent[b] = a; size[a] += size[b];
        return true;
    }
};

}  // namespace

extern "C" {

// Returns |F*| (= n - #connected components), or -1 if an endpoint is out of range.
// out_ids must hold at least max(n-1, 0) entries. *seconds receives the steady_clock time
// of steps 2-5 (key build, sort, union-find scan, id sort) when non-null.
int64_t oracle_kruskal(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                       const uint32_t* w, int32_t* out_ids, uint64_t* out_total,
                       double* seconds) {
    for (int64_t i = 0; i < m; ++i)
        if (src[i] < 0 || src[i] >= n || dst[i] < 0 || dst[i] >= n) return -1;
    auto t0 = std::chrono::steady_clock::now();

    std::vector<uint64_t> key(m);
    for (int64_t i = 0; i < m; ++i) key[i] = (uint64_t(w[i]) << 32) | uint64_t(i);
    std::sort(key.begin(), key.end());

    UnionFind uf(n);
    std::vector<int32_t> ids;
    ids.reserve(n > 0 ? n - 1 : 0);
    uint64_t total = 0;
    for (int64_t j = 0; j < m; ++j) {
        int64_t i = int64_t(key[j] & 0xffffffffu);
        if (src[i] == dst[i]) continue;
        if (uf.unite(src[i], dst[i])) {
            ids.push_back(int32_t(i));
            total += w[i];
        }
    }
    std::sort(ids.begin(), ids.end());
    auto t1 = std::chrono::steady_clock::now();

    for (size_t j = 0; j < ids.size(); ++j) out_ids[j] = ids[j];
    *out_total = total;
    if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
    return int64_t(ids.size());
}

// Connected-component labels: label[v] = smallest vertex id in v's component (plain
// definition of the partition the forest spans). Its count c gives the forest size n - c
// that the GPU parity tests check independently of Kruskal (pinned against BFS in
// tests/test_oracle_pins.py).
int64_t oracle_components(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                          int32_t* label) {
    for (int64_t i = 0; i < m; ++i)
        if (src[i] < 0 || src[i] >= n || dst[i] < 0 || dst[i] >= n) return -1;
    UnionFind uf(n);
    for (int64_t i = 0; i < m; ++i) uf.unite(src[i], dst[i]);
    std::vector<int32_t> minv(n, INT32_MAX);
    for (int64_t v = 0; v < n; ++v) {
        int64_t r = uf.find(v);
        if (v < minv[r]) minv[r] = int32_t(v);
    }
    int64_t c = 0;
    for (int64_t v = 0; v < n; ++v) {
        label[v] = minv[uf.find(v)];
        c += (label[v] == v);
    }
    return c;
}

}  // extern "C"
