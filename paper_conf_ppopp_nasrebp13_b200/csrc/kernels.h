// kernels.h — host-side launchers of the MST kernels (internal; not part of the C ABI).
#pragma once
#include <algorithm>
#include <cstdint>
#include <cuda_runtime.h>

#define MST_CHAIN_MAX 64
#define ACC_SLOTS 64  // forest weight/size accumulators: 64 (sum, count) pairs summed on the host
#define DENSE_MAX 4096
#define SAMPLES_PER_PASS 4096  // records sampled for a pass's compaction decision  // components: the dense min-matrix then holds <= 8.4 M entries (67 MB)

namespace mstk {
typedef uint32_t u32;
typedef uint64_t u64;

// The node->component map of PAPER.md §6.5, kept as the chain of per-round maps
// M_0..M_{r-1}: label_r(v) = M_{r-1}[...M_0[v]]. Passed by value (≤ 520 B of parameters).
struct MapChain {
    const int* m[MST_CHAIN_MAX];
    int len;
};

// Compaction decision of a sparse pass (MST_OPT_COMPACT_TAU): the pass deletes its dead
// records only if the estimated surviving fraction num/den is below tau/1000, where (num,
// den) is the previous pass's exact count or, for round 0, a sample. num == nullptr: the
// host decided (compact unless `out` is null). Every pass counts its survivors into *surv and
// its records into *seen (the next pass's estimate); block 0 writes the decision to *hword
// (mapped host memory, tagged) for the host's bookkeeping at the next round.
struct CompactCtl {
    const u32* num = nullptr;
    const u32* den = nullptr;
    u32 tau = 1000;
    u32* surv = nullptr;
    u32* seen = nullptr;
    u64* hword = nullptr;
    u32 tag = 0;
};

cudaError_t launch_degree(cudaStream_t st, int nsm, u32 n, u32 m, const int* src, const int* dst,
                          const unsigned* w, u32* eu, u32* ev, u32* deg, u32* err, u32* wmax,
                          u64* span);  // *span += sum over non-loop edges of |u - v|
cudaError_t launch_scan_rows(cudaStream_t st, u32 n, const u32* deg, u32* row, u32* cursor,
                             u64* status, u32 epoch);
cudaError_t launch_reorder(cudaStream_t st, int nsm, u32 n, u32 m, const u32* deg, u32* degn,
                           u32* eu, u32* ev, u32* newid, u32* counts, u64* status, u32 epoch,
                           u32* odeg, int hi_owner);
u64 reorder_scratch(u64 n);
// NEXT-4 BFS layout (MST_REORDER=2): newid = BFS discovery order from vertex `root` (then the
// next unvisited vertex with an edge per component; edgeless vertices last), then the same
// relabelling as launch_reorder. off: n + 1, cursor / q / newid: n, adj: 2 m, stt: 8 words.
cudaError_t launch_reorder_bfs(cudaStream_t st, int nsm, u32 n, u32 m, const u32* deg, u32* degn,
                               u32* eu, u32* ev, u32* off, u32* cursor, u32* adj, u32* q,
                               u32* newid, u32* stt, u64* status, u32 epoch, u32* odeg,
                               int hi_owner, u32 root);
// *out = max (deg[v] << 32 | ~v): the largest degree and the lowest vertex with it
cudaError_t launch_deg_argmax(cudaStream_t st, int nsm, u32 n, const u32* deg, u64* out);
cudaError_t launch_owner_degree(cudaStream_t st, int nsm, u32 m, const u32* eu, const u32* ev,
                                u32* odeg, int hi_owner);
cudaError_t launch_scatter(cudaStream_t st, int nsm, u32 m, const u32* eu, const u32* ev,
                           const unsigned* w, u32* cursor, uint4* arcs, uint2* euv,
                           int hi_owner, u32 kfmt, u32 vlo, u32 vhi, u32 wbase, u32 e0 = 0,
                           u32* wmax = nullptr);
// records written in the (w << 32 | eid) format -> the packed format kfmt (host-input builds)
cudaError_t launch_key_format(cudaStream_t st, int nsm, u64 A, uint4* arcs, u32 kfmt);
// (only the records of owners in [vlo, vhi), at their CSR position minus wbase)
// light_out != nullptr (MST_OPT_LIGHT_FIRST): also append the records of weight <= *light_t
// to light_out; every consumer warp reserves blocks of light_blk records (one atomic each)
// and fills the unused end of its last block with dead records (owner ~0); *light_count =
// records written including that filler (<= light + light_blk * warps of the launch)
cudaError_t launch_min0(cudaStream_t st, int nsm, u64 A, const uint4* arcs, u64* best, u32 nb,
                        u32* tile_ctrs, u32& seq, uint4* light_out = nullptr,
                        const u32* light_t = nullptr, u32* light_count = nullptr,
                        u32 light_blk = 0, u32 kfmt = 0);
// seq: the handle's pass sequence (tile-counter slot parity), consumed only by a launch
// light_blk | 1 << 31: extract only (no minima; light-only round 0)
// round-0 minimum over records whose count is on the device (*a_in <= a_max)
cudaError_t launch_min0_dev(cudaStream_t st, int nsm, const u32* a_in, u64 a_max,
                            const uint4* arcs, u64* best, u32 nb, u32* tile_ctrs, u32& seq,
                            u32 kfmt = 0);
u32 pass_warps(int nsm);  // consumer warps of one pass launch, rounded up (the filler bound)
unsigned long long kernel_launches();  // kernels launched by this process so far
// A1: best = inf (n), msf = 0 (nwords), acc = 0 (nacc), ctr = 0 (nctr), *zero1 = 0,
// ctr2 = 0 (nctr2: every per-shard, per-round record count of the run)
// The light-edge threshold selection (launch_light_threshold) done by the init launch's last
// CTA (on = 0: none)
struct LightSel {
    const uint4* arcs;
    u64 A, target;
    u32* t_out;
    u32 s1;
    int on;
};
cudaError_t launch_init(cudaStream_t st, int nsm, u32 n, u64* best, u32 nwords, u32* msf,
                        u64* acc, u32 nacc, u32* ctr, u32 nctr, u32* zero1, u32* ctr2, u32 nctr2,
                        const struct LightSel* ls = nullptr);
// phi[x] = chain.m[len-1][...chain.m[0][x]] for x < n (-1 stays -1)
cudaError_t launch_chain_compose(cudaStream_t st, int nsm, u32 n, const MapChain& chain, int* phi);
// defer (light-edge phase): a component with no (light) edge left is kept, not finished
cudaError_t launch_hook(cudaStream_t st, u32 nr, const u64* best, u64* best_next, u64* hmap, u32 tag,
                        const uint2* euv, const MapChain& chain, u32* P, int* Mtmp, u32* msf,
                        u64* acc, u32* tcnt, u32* n_next, bool defer = false, u32 kfmt = 0);
// tcnt: 2 * hook_tiles(n) words (tile counts, then their exclusive scan)
// rounds with few hook tiles: the jump also does k_hook_scan's work (n_{r+1} to *nn and to
// the tagged word hmap, which launch_hook then does not launch)
// The hub set of a member-scan decision (the components of internal vertices 0..31 from vertex
// ids through chain and M_r, sorted, + their distinct live count, also to the tagged mapped
// word hword), computed by the jump's last CTA (on = 0: none); done: a counter left at 0
struct HubTask {
    MapChain chain;
    int* hubs;
    u64* hword;
    u32 tag, n;
    u32* done;
    int on;
};
cudaError_t launch_jump(cudaStream_t st, int nsm, u32 nr, u32* P, const int* Mtmp, const u32* tcnt,
                        int* Mr, u32* nn, u64* best_next, const int* hub, int* hub_next,
                        u64* hmap, u32 tag, const HubTask* ht = nullptr);
u64 hook_tiles(u64 n);
cudaError_t launch_filter_min(cudaStream_t st, int nsm, const u32* a_in, u64 a_max,
                              const uint4* in, const int* M, uint4* out, u64* best, u32 nb,
                              u64* status, u32 epoch, u32* a_next, u32* tile_ctrs, u32& seq,
                              u64* mat, const CompactCtl& cc = CompactCtl(),
                              const int* hub = nullptr, u32 kfmt = 0, bool adj = false);
// adj: A8's adjacent-duplicate filter in a compacting pass
// NEXT-3 union-find variant: parent = identity; one pass (K1: roots by find,
// intra-component records dropped, survivors compacted unchanged when the policy says so,
// minima keys (w << s1 | eid) | tag into best[root]); then partner + union (K2a/K2b: forest
// bits, forest weight/size into acc, *unions += unions; K2a first publishes *surv to hmap)
cudaError_t launch_uf_init(cudaStream_t st, int nsm, u32 n, u32* parent);
cudaError_t launch_uf_pass(cudaStream_t st, int nsm, const u32* a_in, u64 a_max, const uint4* in,
                           u32* parent, uint4* out, u64* best, u32 n, u64* status, u32 epoch,
                           u32* a_next, u32* tile_ctrs, u32& seq, const CompactCtl& cc, u32 kfmt,
                           u64 tag, bool adj = false);
cudaError_t launch_uf_hook(cudaStream_t st, int nsm, u32 n, u32* parent, const u64* best, u32 kfmt,
                           bool tagged, u64 tag, const uint2* euv, u32* P, u32* msf, u64* acc,
                           u32* unions, const u32* surv, u64* hmap, u32 htag);
// member-scan rounds (after the light-edge phase): *work += record ends of the vertices outside
// the component of vertex 0 (phi: vertex -> component)
cudaError_t launch_member_work(cudaStream_t st, int nsm, u32 n, const int* phi, const u32* row,
                               const u32* rrow, u32 vlo, u32 vhi, u64* work);
// member minima of the components outside an exclusion set: own records [row[v] - wbase,
// row[v+1] - wbase) for owners in [vlo, vhi), reverse records ridx[rrow[v] .. rrow[v+1]).
// hubs == nullptr: a member-scan round, the set is {phi[0]} and best[phi[0]] = KEY_DEFER;
// else a hybrid round next to a light pass: the set is hubs[0..31] (launch_compose_work's)
cudaError_t launch_member_min(cudaStream_t st, int nsm, u32 n, const int* hubs, const int* phi,
                              const u32* row, const u32* rrow, const u32* ridx, const uint4* arcs,
                              u32 vlo, u32 vhi, u32 wbase, u64* best, u32 kfmt);
// round 0 after a light-only round-0 pass: best[v] = min over all of v's records for every v
// whose best is still inf (no light record); *ends += record ends read
cudaError_t launch_singleton_min(cudaStream_t st, int nsm, u32 n, u64* best, const u32* row,
                                 const u32* rrow, const u32* ridx, const uint4* arcs, u32 vlo,
                                 u32 vhi, u32 wbase, u32 kfmt, u64* ends);
// the reverse index of the A local records (other endpoint -> record indices); rdeg, cursor:
// n-word scratch; rrow: n + 1 words; ridx: A words
u64 reverse_index_scratch(int nsm, u32 n);  // u32 words of launch_reverse_index's pc
cudaError_t launch_reverse_index(cudaStream_t st, int nsm, u32 n, u64 A, const uint4* arcs,
                                 u32* rdeg, u32* rrow, u32* cursor, u32* ridx, u64* status,
                                 u32 epoch, u32* pc);
// A9 (MST_OPT_DEDUP, dedup.cu): sort the A records {s', d', key base} in rec (labels < nlab) by
// their pair (min, max) and keep the minimum key of every pair, in place; *a_count = records
// left (written on the device). scratch: dedup_scratch_bytes(A) bytes; nruns: one device int
size_t dedup_scratch_bytes(u64 A);
cudaError_t launch_dedup(cudaStream_t st, int nsm, u64 A, u32 nlab, u32* a_count, uint4* rec,
                         void* scratch, size_t scratch_bytes, int* nruns);
// kfmt: key format of the minima the pass emits = s1 | pb << 8 (pb = 0: (w << 32) | eid)
cudaError_t launch_dense_best(cudaStream_t st, int nsm, u32 n, const u64* mat, u64* best);
cudaError_t launch_dense_init(cudaStream_t st, int nsm, u32 n, u64* mat);
cudaError_t launch_dense_round(cudaStream_t st, int nsm, u32 n, const u64* mat, const int* M,
                               u32 n_next, u64* mat_next, u64* best_next);
u64 dense_entries(u64 n);
cudaError_t launch_dense_tail(cudaStream_t st, int nsm, u32 n0, u64* best0, u64* best1,
                              u64* mat0, u64* mat1, const uint2* euv, const MapChain& chain,
                              u32* msf, u64* acc, u32* bar, u32* stats, u64* trace = nullptr,
                              int defer = 0, int* map_out = nullptr, u32* n_out = nullptr);
cudaError_t launch_compose(cudaStream_t st, int nsm, u32 nb, const int* src, const int* Mr, int* phi);
// the same over vertex ids, also summing into *work the record ends of the vertices outside
// the hub set's components (the member-scan decision); hubs: 33 ints written first (the
// sorted labels of the components of vertices 0..31 after Mr, then their number of distinct
// live labels)
cudaError_t launch_compose_work(cudaStream_t st, int nsm, u32 nb, const int* src, const int* Mr,
                                int* phi, int* hubs, const u32* row, const u32* rrow,
                                u32 vlo, u32 vhi, u64* work);
cudaError_t launch_sample_survival(cudaStream_t st, const uint4* in, const u32* a_ptr, const int* M,
                                   u32* num, u32* den);
// A10 latency regime: the whole method in one CTA (records, component arrays and forest bits
// in shared memory) when small_smem_bytes(n, E, nwords) <= small_smem_limit() and packed keys
// (w << s1 | eid << pb | partner) fit 64 bits; res (device, small_out_bytes()) receives
// {count, rounds, total, n_r[64], a_r[64], tag} — tag written last
size_t small_smem_bytes(u64 n, u64 E, u64 nwords);
size_t small_smem_limit();
size_t small_out_bytes();
cudaError_t launch_small(cudaStream_t st, u32 n, u32 E, u32 nwords, const uint4* arcs, u32 s1,
                         u32 pb, int* out, void* res, u64 tag);  // res: mapped host memory
// max_ids: an upper bound of the forest size (n - 1) — sizes the staging of the id writes
cudaError_t launch_output(cudaStream_t st, u32 nwords, const u32* msf, int* out, u32* tcnt,
                          u32* out_count, u32 max_ids);
u64 out_tiles(u64 nwords);  // tcnt needs 2 * out_tiles(nwords) words
cudaError_t launch_combine_min(cudaStream_t st, int nsm, u32 nr, int nshards, u64* shard_best,
                               u64 stride, u64* best);
u64 status_slots_needed(u64 n, u64 arcs, u64 nwords);
cudaError_t launch_debug_map(cudaStream_t st, u32 n, int kind, u32 group, int* M, u32* ncomp);
}  // namespace mstk
