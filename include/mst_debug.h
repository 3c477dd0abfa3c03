/*
 * include/mst_debug.h — test/benchmark-only entry points of libmst.so (not the product API).
 *
 * mst_debug_filter_pass: times the A8 kernel alone on the handle's
 * round-0 arcs with a synthetic label map, so kernel variants can be measured in isolation:
 *   map_kind 0: M[v] = v            (identity: every non-loop arc survives)
 *   map_kind 1: M[v] = v / group    (contiguous blocks of `group` vertices per component)
 *   map_kind 2: M[v] = h(v) % ncomp (hashed, ncomp = max(1, n / group) components)
 *   stream     : device work is enqueued here; the call synchronises it.
 *   iters      : timed repetitions (after one warm-up); *out_ms = mean ms per launch (CUDA
 *                events on `stream`); *out_survivors = arcs kept by the last launch.
 * The handle's per-round state is clobbered; run mst_run again before trusting it.
 * Returns MST_EINVAL for bad arguments, MST_ECUDA on launch failure.
 */
#ifndef MST_DEBUG_H_
#define MST_DEBUG_H_
#include "mst.h"
#ifdef __cplusplus
extern "C" {
#endif
mst_status mst_debug_filter_pass(mst_graph* g, mst_stream_t stream, int map_kind, int64_t group,
                                 int iters, double* out_ms, int64_t* out_survivors);

/* mst_shard_ranges: the multi-GPU edge partition of mst_create_dist / mst_create_sim
 * (SURVEY.md §8(e)), pure host code (no device needed):
 *   row_offsets : HOST pointer, uint32[n+1], a CSR row-offset array (row[n] = arcs)
 *   nranks      : 1..64 shards
 *   lo, hi      : HOST int64[nranks]; shard j owns the arc window [lo[j], hi[j]), i.e. the
 *                 sources [v_j, v_{j+1}) with v_j the first vertex whose offset reaches
 *                 j * arcs / nranks. Windows are contiguous, disjoint and cover [0, arcs). */
mst_status mst_shard_ranges(const uint32_t* row_offsets, int64_t n, int nranks, int64_t* lo,
                            int64_t* hi);
/* mst_create_dist_hostx: a distributed handle (as mst_create_dist) whose
 * exchange step is a HOST callback instead of NCCL, so that several processes sharing one
 * GPU (NCCL allows one rank per device) run the real distributed round loop — per-rank
 * record builds, rank-local compaction decisions, the per-round MIN, the agreed light-edge
 * threshold — with the MIN done by their own process group (tests: a gloo all_reduce).
 *   src, dst, w : DEVICE pointers to the identical full input on every rank (as mst_create)
 *   rank, nranks: this process's rank, the number of ranks (1..64)
 *   fn          : called by mst_run (on the calling thread, the run's stream synchronised) with
 *                 a HOST buffer of `count` uint64 words; it must replace every word by the
 *                 minimum of that word over all ranks (unsigned compare) and return 0, or
 *                 non-zero to fail the run with MST_ENCCL. Every rank calls it the same
 *                 number of times with the same counts, in the same order.
 *   ctx         : passed through to fn.
 * MST_EINVAL for a NULL fn or bad rank/nranks; otherwise as mst_create_dist. */
typedef int (*mst_allreduce_min_fn)(uint64_t* host_buf, int64_t count, void* ctx);
mst_status mst_create_dist_hostx(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                                 const uint32_t* w, int rank, int nranks,
                                 mst_allreduce_min_fn fn, void* ctx, mst_graph** out);
#ifdef __cplusplus
}
#endif
#endif
