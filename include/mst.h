/*
 * include/mst.h — C ABI of the B200 Boruvka minimum-spanning-forest hot path (libmst.so).
 *
 * Operation (§5, "Boruvka's Minimum Spanning Tree Algorithm"): given an
 * edge-weighted undirected graph, repeatedly (1) find the minimum edge of each node whose
 * other endpoint is in another component, (2) isolate the minimum inter-component edge of
 * each component, (3) break the cycles of chosen edges at the component with minimum id,
 * (4) merge every cycle/tree into its representative — "the process repeats until there is
 * a single component. The inter-component minimum-weight edges are the MST" (L227).
 * Realised as SURVEY.md §8(a) rows A0-A11; the per-row design is in DESIGN.md.
 *
 * Readings of the paper adopted by this ABI:
 *   R1  ties between equal weights are broken by edge id: e < f <=> (w_e, e) <_lex (w_f, f);
 *       the result is therefore the UNIQUE minimum spanning forest F* (bit-checkable);
 *   R3  disconnected inputs give a spanning FOREST, |F*| = n - c (c = #connected comps);
 *   R4  self-loops are legal input and never selected (L217 assumes none);
 *   R5  parallel edges are legal and compete by (w, id);
 *   R6  weights are uint32 (0 allowed); the total weight is an exact uint64.
 *
 * Conventions shared by every entry point
 *   - Edge id e in [0, m) is the position in the caller's src/dst/w arrays.
 *   - 0 <= n <= 2^31-1 and 0 <= m <= 2^31-1 (edge ids and 2m arcs fit in 32 bits).
 *   - Every endpoint must satisfy 0 <= src[e], dst[e] < n, else MST_EINVAL (checked on the
 *     device during the build, before anything else runs).
 *   - No C++ exception crosses the ABI. All functions are thread-compatible per handle
 *     (one thread at a time per handle; different handles are independent).
 *   - On any non-OK status a message is available from mst_last_error() (thread-local).
 *   - There is no CPU fallback: without a usable CUDA device every call that needs one
 *     returns MST_ECUDA.
 */
#ifndef MST_H_
#define MST_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* mst_stream_t; /* == cudaStream_t; NULL = legacy default stream */

typedef enum {
    MST_OK = 0,
    MST_EINVAL = 1,    /* bad argument: null pointer with m > 0, n/m out of range, endpoint >= n */
    MST_ENOMEM = 2,    /* device allocation failed (nothing leaked)                           */
    MST_ECUDA = 3,     /* CUDA runtime/launch error; handle may only be destroyed afterwards   */
    MST_ENCCL = 4,     /* NCCL error in a distributed handle                                   */
    MST_EINTERNAL = 5, /* an internal invariant failed (e.g. forest size != n - c)             */
    MST_ENOTSUP = 6    /* feature not built into this library                                  */
} mst_status;

typedef struct mst_graph mst_graph; /* opaque; owned by the library */

/* ------------------------------------------------------------------ build (row A0)
 * mst_create — validate the COO input and build the device-resident edge records.
 *   n, m     : vertex and edge counts (see conventions).
 *   src, dst : DEVICE pointers, int32[m], caller-owned, read only during the call.
 *   w        : DEVICE pointer, uint32[m], caller-owned, read only during the call.
 *   out      : receives the handle; *out = NULL on any error (nothing is leaked).
 * The call first synchronises the device (cudaDeviceSynchronize), so inputs still being
 * written by work in flight on any stream are complete before the build reads them.
 * Layout (reading R14): the CSR of PAPER.md §6 L229 stores "each edge twice,
 * once for each direction"; this build stores every non-self-loop edge ONCE, as a 16-byte
 * record {owner, other, eid, w} in the segment of its owner endpoint (the higher internal
 * vertex id under the build's hub-first numbering), records grouped by owner (CSR order).
 * E_0 = the number of non-self-loop edges = the records built (mst_stats.arcs0). Both
 * endpoints' minima are still computed every round, so the result is the same. All per-round
 * buffers are allocated here once, sized for the worst case (§7.1: MST
 * pre-allocation, "the sum of the nodes in all components is constant"); mst_run allocates
 * nothing. Synchronous. */
mst_status mst_create(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                      const uint32_t* w, mst_graph** out);

/* mst_create_host — as mst_create but src/dst/w are HOST pointers (pageable or pinned),
 * read only during the call. The arrays are streamed to stream-ordered device buffers in
 * 8 M-edge chunks (copy engines; pinned arrays reach the bus rate, ~55 GB/s, pageable ones
 * are staged by the driver) WHILE the build consumes them: the degree/validation pass runs
 * per endpoint chunk, the layout while the weights travel, the record scatter per weight
 * chunk (input transferred to the GPU) — the result is the same handle as
 * mst_create's. An endpoint outside [0, n) in any chunk: MST_EINVAL, nothing leaked.
 * (MST_HOST_STREAM=0 copies everything first; MST_HOST_CHUNK sets the chunk, in edges.)
 * The build's small pinned host buffers come from a process-wide free list (no
 * page-locking per handle). */
mst_status mst_create_host(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                           const uint32_t* w, mst_graph** out);

/* ------------------------------------------------------------------ run (rows A1-A11)
 * mst_run — compute the minimum spanning forest F* of the handle's graph.
 *   stream          : all device work is enqueued on this stream (torch's current stream
 *                     when called from the Python binding).
 *   out_edge_ids    : DEVICE pointer, int32, caller-owned, capacity >= max(n-1, 0);
 *                     receives the ids of F* in ASCENDING order.
 *   out_num_edges   : HOST pointer; receives |F*| = n - c.
 *   out_total_weight: HOST pointer; receives sum of w[e] over F* (exact uint64).
 * Blocks until results are valid (per-round sizes come back to the host, §7.1
 * L263 "kernel computes the future size and the host reads it"). Re-runnable: the arcs of
 * the build are never overwritten, so the same handle gives the same output every call.
 * After an error the handle may only be destroyed. */
mst_status mst_run(mst_graph* g, mst_stream_t stream, int32_t* out_edge_ids,
                   int64_t* out_num_edges, uint64_t* out_total_weight);

/* mst_run_host — as mst_run but out_edge_ids is a HOST pointer (capacity >= max(n-1,0));
 * the device->host copy of the ids is part of the call. */
mst_status mst_run_host(mst_graph* g, mst_stream_t stream, int32_t* out_edge_ids_host,
                        int64_t* out_num_edges, uint64_t* out_total_weight);

/* mst_solve_host — one end-to-end call from host arrays to host results:
 * mst_create_host + mst_run_host + mst_destroy. Device memory comes from a stream-ordered
 * pool that the library keeps between calls, so repeated solves do not pay cudaMalloc. The
 * build uses the automatic layout except the BFS order, and lays down no reverse index (the
 * member-scan rounds' ~2 ms build pass, which one run does not repay; the BFS pass costs
 * ~10 ms: those graphs keep the caller's numbering); the result is identical either way. */
mst_status mst_solve_host(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                          const uint32_t* w, int32_t* out_edge_ids_host,
                          int64_t* out_num_edges, uint64_t* out_total_weight);

/* mst_destroy — NULL-safe; frees every library allocation of the handle. */
void mst_destroy(mst_graph* g);

/* thread-local message describing the last non-OK status returned on this thread */
const char* mst_last_error(void);

/* ------------------------------------------------------------------ introspection
 * Per-run statistics of the last mst_run on the handle. Sizes let the caller compute the
 * algorithmic byte model of SURVEY.md §8(d); kernel times are filled only while profiling
 * is enabled (CUDA events recorded on the run's stream around every launch). */
#define MST_MAX_ROUNDS 64
enum {
    MST_K_INIT = 0,    /* A1 run init (best = inf, msf bits = 0, counters)            */
    MST_K_MIN0 = 1,    /* A2 round-0 segmented min                                    */
    MST_K_HOOK = 2,    /* A4 hook + A6 renumber scan                                  */
    MST_K_JUMP = 3,    /* A5 pointer-jump + A6 map compose                            */
    MST_K_FILTER = 4,  /* A8 fused relabel + filter + compaction + next-round min     */
    MST_K_OUTPUT = 5,  /* A11 output compaction                                       */
    MST_K_COMM = 6,    /* A3 cross-GPU MIN (distributed handles)                      */
    MST_K_DENSE = 7,   /* A9 dense rounds over the component min-matrix              */
    MST_K_LIGHT = 8,   /* (unused: the light threshold is selected inside MST_K_INIT)  */
    MST_K_COMPOSE = 9, /* A7 label-map composition (+ the round-0 survival sample)    */
    MST_K_SMALL = 10,  /* A1-A11 in one CTA (MST_OPT_SMALL: graphs that fit smem)      */
    MST_K_DEDUP = 11,  /* A9 sort-based duplicate collapse (MST_OPT_DEDUP)            */
    MST_K_COUNT = 12
};
/* launch sub-kinds (mst_launch_time.sub), so unlike launches of one kind are told apart:
 *   MST_K_MIN0  : MIN_ALL   = minima over every record (+ the light-record write);
 *                 EXTRACT   = light-only round 0: the light-record write alone;
 *                 MIN_LIGHT = minima over the light records; SINGLETONS = the minima of
 *                 the vertices without a light record, from their own records
 *   MST_K_FILTER: SPARSE = a pass over the alive records; LIGHT = a light-edge phase pass;
 *                 SWITCH = the pass that re-reads every record after the light phase;
 *                 TRANSITION = the pass into the dense min-matrix; MEMBER = a member-scan round
 *                 (the minima of the components outside the top hub's from their members'
 *                 records, after the light-edge phase)
 *   MST_K_DENSE : DENSE_ROUND, DENSE_BEST, TAIL (the cooperative device tail) */
enum {
    MST_SUB_MIN_ALL = 0, MST_SUB_EXTRACT = 1, MST_SUB_MIN_LIGHT = 2, MST_SUB_SINGLETONS = 3,
    MST_SUB_SPARSE = 0, MST_SUB_LIGHT = 1, MST_SUB_SWITCH = 2, MST_SUB_TRANSITION = 3,
    MST_SUB_MEMBER = 4,
    MST_SUB_DENSE_ROUND = 0, MST_SUB_DENSE_BEST = 1, MST_SUB_TAIL = 2
};
typedef struct {
    int64_t n, m, arcs0;                  /* vertices, edges, E_0 = #non-loop edges (one
                                             record per edge, all ranks together)         */
    int32_t rounds;                       /* R: rounds executed by the last run          */
    int32_t nranks, rank;                 /* 1/0 for single-GPU handles                  */
    int64_t local_arcs0;                  /* edge records owned by this rank             */
    int64_t n_r[MST_MAX_ROUNDS];          /* live components entering round r            */
    int64_t a_r[MST_MAX_ROUNDS];          /* alive (local) edge records entering round r's
                                             pass (dense rounds: matrix entries)          */
    int64_t num_edges;                    /* |F*| of the last run                        */
    uint64_t total_weight;
    double build_ms;                      /* wall time of the build in mst_create*       */
    int32_t profiling;                    /* 1 if the kernel timers below are valid      */
    double kernel_ms[MST_K_COUNT];        /* summed event time per kernel kind           */
    int64_t kernel_launches[MST_K_COUNT];
    double round_filter_ms[MST_MAX_ROUNDS]; /* A8 (or A9 dense) kernel time per round     */
    int64_t gpu_launches;                 /* kernels launched by the last run            */
    int32_t dense_round;                  /* first round run on the dense min-matrix, -1 */
    int64_t compacted_mask;               /* bit r: round r's pass compacted its records  */
    int32_t survival_permille[MST_MAX_ROUNDS]; /* estimated survivors of pass r that its
                                                  compaction decision used (-1: none)      */
    int32_t hub_row;                      /* 1: the dense transition kept the top hub's
                                             matrix row in shared memory (heavy tail)     */
    int32_t light_switch_round;           /* light-edge phase (MST_OPT_LIGHT_FIRST): round
                                             whose pass re-read every edge record (the
                                             heavy ones), -1 = not reached / phase off    */
    uint32_t light_t;                     /* its weight threshold (light: w <= light_t);
                                             0xffffffff when the phase was off            */
    int64_t member_ends[MST_MAX_ROUNDS];  /* member-scan round r: record ends read (the
                                             members' own + reverse records); -1: not one;
                                             [0]: round 0's singleton scan, if it ran     */
    int64_t dedup_in[MST_MAX_ROUNDS];     /* A9: records entering the dedup after round r's
                                             pass (a_r[r + 1] = after it); -1: none        */
    int32_t layout;                       /* internal vertex numbering of the build: 0 the
                                             caller's, 1 hub-first, 2 BFS order (NEXT-4)   */
    int32_t member_round[MST_MAX_ROUNDS]; /* 1: round r was a member-scan round, 2: a hybrid
                                             round (light pass + member scan), 0: neither */
} mst_stats;

mst_status mst_get_stats(const mst_graph* g, mst_stats* out);

/* Per-launch event times of the last PROFILED run (mst_set_profiling), in launch order:
 * kind (MST_K_*), sub (MST_SUB_*), round, shard (sharded handles), ms. Copies
 * min(cap, *count) records to out (HOST array); *count = the number of launches recorded. */
typedef struct {
    int32_t kind, sub, round, shard;
    double ms;
} mst_launch_time;
mst_status mst_get_launch_times(const mst_graph* g, mst_launch_time* out, int64_t cap,
                                int64_t* count);

/* enable (1) / disable (0) per-launch CUDA-event timing for subsequent runs */
mst_status mst_set_profiling(mst_graph* g, int enable);

/* ------------------------------------------------------------------ run options
 * Options change how later mst_run calls work, never what they return (the forest is the
 * unique F*, reading R1). MST_EINVAL for an unknown option or value.
 *   MST_OPT_DENSE (default 1): once a round has <= 4096 live components, keep the alive
 *       edges as a min-matrix over component pairs (duplicate collapse, SURVEY.md §8(a) A9 /
 *       §8(f) NEXT-1); 0 = every round stays on the compacted edge list.
 *   MST_OPT_KEEP_EDGES (default 0): 1 = the paper's own scheme ("maintains
 *       the original adjacency list for each node and performs edge traversals per node"):
 *       no deletion/compaction; every round re-reads all original edge records and skips
 *       same-component ones through the explicitly maintained vertex->component map
 *       (row A7). Implies MST_OPT_DENSE = 0. Used as an ablation of what the
 *       morph step (deletion) buys.
 *   MST_OPT_DEVICE_TAIL (default 1): once dense, run every remaining round inside one
 *       cooperative kernel (no host round trip per round); 0 = one launch set per round.
 *   MST_OPT_COMPACT_TAU (default 900, permille in [0, 1000]): a sparse pass deletes the dead
 *       edge records (compaction, the morph step) only when the sampled fraction of its
 *       records that survive is below tau/1000; otherwise the next pass re-reads the same
 *       records through the composed label map (row A7). 1000 = always compact, 0 = never
 *       (deletion deferred to the dense transition). Decided on the device per pass from the
 *       previous pass's exact survival (round 0: 4096 sampled records); the passes of the
 *       light-edge phase and the pass that then re-reads every record never compact. Never
 *       changes the result.
 *   MST_OPT_LIGHT_FIRST (default -1 = auto; 0 = off, else K in [1, 64]): light-edge phase
 *       (auto: K = 8 with a light-only round 0 when there are >= 64 records per
 *       vertex, else K = 2; R16). Kruskal
 *       takes the edges in (w, id) order (the "ordered" algorithm), so the
 *       forest restricted to the edges with w <= t is the forest of that light subgraph for
 *       every t. mst_run first picks t so that about K*n edge records are light (a 4096-record
 *       sample, on the device), writes the light records while it computes the round-0
 *       minima, runs the Boruvka rounds over the light records only — a component without a
 *       light edge is deferred, not finished — and once no light edge joins two components
 *       re-reads every record (relabelled; all the light ones are now intra-component and
 *       deleted) and continues as usual. Used when at least 4*K*n records exist (dense and
 *       heavy-tailed inputs) and MST_OPT_KEEP_EDGES is off, on every kind of handle (a
 *       distributed run agrees on one t: the minimum of the ranks' sampled thresholds).
 *       Never changes the result.
 *   MST_OPT_UNION_FIND (default 0): 1 = the union-find variant (
 *       PAPER.md §8.4: a component-based Boruvka with a "fast union-find" that "keeps the
 *       graph unmodified" in a "bulk-synchronous executor"): every round finds both endpoint
 *       roots of the alive edge records by union-find (path halving), drops intra-component
 *       records (the survivors are compacted unchanged, never relabelled, under
 *       MST_OPT_COMPACT_TAU; 0 or MST_OPT_KEEP_EDGES = the unmodified records every round),
 *       min-reduces per root, and unions the two roots of every chosen edge by CAS. No
 *       renumbering, no label maps, no dense rounds, no light-edge phase. Single-GPU handles
 *       only (MST_ENOTSUP from mst_run otherwise). Never changes the result.
 *   MST_OPT_SMALL (default 1): graphs whose edge records (16 B each), per-vertex arrays
 *       (16 B per vertex) and forest bits fit one CTA's shared memory (~220 KB; grid64: 197 KB)
 *       run every round in ONE launch on one SM (kernels.cu k_small_msf: minima with the
 *       partner in packed keys, hook, path-halving jumps, block-scan renumbering, relabel and
 *       deletion, ascending ids): the latency regime of row A10, where the multi-kernel path
 *       pays launches and a host wait per round for microseconds of work. Single-GPU handles
 *       without MST_OPT_KEEP_EDGES / MST_OPT_UNION_FIND; 0 = always the multi-kernel path.
 *   MST_OPT_DEDUP (default 0): 1 = row A9's sort-based duplicate collapse: after every
 *       sparse pass (which then always compacts) the surviving records are sorted by their
 *       component pair (CUB device radix sort) and each pair keeps its minimum key (CUB
 *       reduce-by-key), leaving records grouped by their lower label (reading R13). Setting it
 *       allocates ~32 B per local record of scratch (here, not in mst_run). Single-shard,
 *       non-distributed handles; measured in DESIGN.md §5c. Never changes the result.
 * Keys of the component minima (rows A2/A8): (uint64(w) << 32) | eid, or, when the largest
 * weight, the largest edge id and the largest vertex id fit 63 bits together, the packed
 * (w << s1) | (eid << pb) | partner label — the same (w, eid) order (reading R17).
 */
enum { MST_OPT_DENSE = 1, MST_OPT_KEEP_EDGES = 2, MST_OPT_DEVICE_TAIL = 3, MST_OPT_COMPACT_TAU = 4,
       MST_OPT_LIGHT_FIRST = 5, MST_OPT_UNION_FIND = 6, MST_OPT_SMALL = 7, MST_OPT_DEDUP = 8 };
mst_status mst_set_option(mst_graph* g, int option, int64_t value);

/* ------------------------------------------------------------------ multi-GPU (§8(e))
 * One process per GPU (torchrun). Every rank passes the identical full input; rank g keeps
 * the arcs whose source lies in its vertex range (ranges chosen from the CSR row offsets so
 * that arcs are balanced). Each round ends with an NCCL allreduce-MIN of the component-best
 * array over NVLink; hook/jump/renumber then run replicated, so every rank holds identical
 * labels and returns the identical full forest. The paper is single-GPU;
 * this exchange step is the north star's extension. */
mst_status mst_get_unique_id(uint8_t id[128]); /* wraps ncclGetUniqueId (rank 0 calls) */
mst_status mst_create_dist(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                           const uint32_t* w, const uint8_t id[128], int rank, int nranks,
                           mst_graph** out);

/* mst_create_sim — test aid: a single-GPU handle that splits the arcs into `nshards`
 * source ranges exactly as mst_create_dist would for nranks = nshards, runs every shard's
 * per-round work itself and combines the shard minima with a device MIN in place of the
 * NCCL allreduce. Exercises the sharding/replication logic without a second GPU. */
mst_status mst_create_sim(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                          const uint32_t* w, int nshards, mst_graph** out);

/* library version string, e.g. "mst-b200 0.1 sm_100a" */
const char* mst_version(void);

#ifdef __cplusplus
}
#endif
#endif /* MST_H_ */
