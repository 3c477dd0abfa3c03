// mst_api.cu — the C ABI (include/mst.h) and the round loop that drives the kernels.
//
// Round structure (§5 L227 and the host loop of Fig. 3,
// "the process repeats until there is a single component"):
//
//   A1  init   best_0 = inf, forest bits = 0
//   A2  min0   best_0[v] = min key over v's arcs                        [A3: MIN over ranks]
//   loop r = 0, 1, ...
//     A4/A6 hook   parent, forest edges, keep-scan -> new ids, n_{r+1}, best_{r+1} = inf
//     A5/A6 jump   roots, M_r = new id of root (-1: finished)
//     A8    filter relabel + delete intra-component arcs + dedup + compact + best_{r+1}
//     host reads (n_{r+1}, A_{r+1})      (kernel computes sizes, host reads)
//     A10   stop when n_{r+1} == 0, or (single GPU) A_{r+1} == 0       [A3 before the next]
//   A11 output ascending ids, count, total weight
//
// Nothing is allocated inside mst_run (PAPER.md L259 pre-allocation). All work is enqueued
// on the caller's stream.
#include <nvtx3/nvToolsExt.h>
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "../../include/mst.h"
#include "../../include/mst_debug.h"
#include "kernels.h"

using namespace mstk;

namespace {

thread_local std::string g_err;

mst_status fail(mst_status s, const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return s;
}

#define CK(call)                                                                          \
    do {                                                                                  \
        cudaError_t e_ = (call);                                                          \
        if (e_ != cudaSuccess) {                                                          \
            return fail(e_ == cudaErrorMemoryAllocation ? MST_ENOMEM : MST_ECUDA,         \
                        "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__,        \
                        __LINE__);                                                        \
        }                                                                                 \
    } while (0)

#define CKN(call)                                                                         \
    do {                                                                                  \
        ncclResult_t r_ = (call);                                                         \
        if (r_ != ncclSuccess)                                                            \
            return fail(MST_ENCCL, "%s: %s (%s:%d)", #call, ncclGetErrorString(r_),        \
                        __FILE__, __LINE__);                                              \
    } while (0)

#define CKS(call)                                                                         \
    do {                                                                                  \
        mst_status s_ = (call);                                                           \
        if (s_ != MST_OK) return s_;                                                      \
    } while (0)

u32 bits_of(u64 x) { u32 b = 0; while (x) { ++b; x >>= 1; } return b; }

constexpr int HUBS_N = 32;  // (kernels.cu HUBS: the hub set's size)

// device-counter slots
enum { C_ERR = 0, C_OUT = 1, C_NNEXT = 2, C_TILE = 3, C_AREC = 8 };  // C_TILE: 2 slots
// C_AREC: per shard j and round r, the alive arcs entering round r (written by round r-1's
// filter on the device; read back by the host together with n_{r+1} after the hook)
constexpr int AREC_STRIDE = MST_MAX_ROUNDS + 1;
inline int arec(int j, int r) { return C_AREC + j * AREC_STRIDE + r; }
constexpr int C_BAR = C_AREC + 64 * AREC_STRIDE;  // grid barrier {count, generation}
constexpr int C_TAIL = C_BAR + 2;                   // device tail: rounds, n per round
constexpr int C_SEEN = C_TAIL + 1 + MST_MAX_ROUNDS;  // records entering pass r (all shards)
constexpr int C_SURV = C_SEEN + MST_MAX_ROUNDS;       // survivors of pass r (all shards)
constexpr int C_SAMP = C_SURV + MST_MAX_ROUNDS;       // round-0 sample: {alive, samples}
constexpr int C_HUB = C_SAMP + 2;  // label of internal vertex 0 (the top hub) per round
constexpr int C_LT = C_HUB + MST_MAX_ROUNDS + 1;  // light-edge threshold t
constexpr int C_WMAX = C_LT + 1;                   // largest weight (build)
constexpr int C_TAILN = C_WMAX + 1;                // light-phase tail: labels after it
constexpr u32 LBLK_MIN = 32, LBLK_MAX = 256;      // light write: records per warp reservation
constexpr int C_UFU = C_TAILN + 1;                 // union-find variant: unions per round
constexpr int C_JDONE = C_UFU + MST_MAX_ROUNDS;    // jump CTAs done (hub set: the last one)
constexpr int DCNT_WORDS = C_JDONE + 1;
constexpr int HSURV = MST_MAX_ROUNDS + 1;  // mapped words: [0, HSURV) sizes, [HSURV, 2 HSURV) decisions,
constexpr int HHUB = 2 * HSURV;            // [2 HSURV, 3 HSURV) the hub sets' component counts

struct Shard {
    u64 lo, hi;  // record window [lo, hi) in the handle's arcs0 and in the ping-pong buffers
    u64 llo;     // window start of the shard's light records in abuf[0] (light-edge phase):
                 // lo + j * light slack, so every shard has room for its filler records
    u32 A;       // alive records entering the current round
};

// Exchange of a distributed handle (row A3): NCCL over NVLink in production; a host callback
// (mst_create_dist_hostx, test aid) lets several processes that share one GPU run the same
// round loop with the MIN done by their own process group.
enum XKind { X_NONE = 0, X_NCCL = 1, X_HOST = 2 };

struct ProfRec {
    int kind, round, sub, shard;
    cudaEvent_t a, b;
};

}  // namespace

struct mst_graph {
    int dev = 0, nsm = 148;
    int64_t n = 0, m = 0;
    u64 A0 = 0, nwords = 0;
    cudaStream_t cst = nullptr;  // internal stream (create / destroy)
    std::vector<void*> allocs;

    u32 *eu = nullptr, *ev = nullptr, *row = nullptr;
    uint2* euv = nullptr;  // {eu, ev} interleaved: the hook's partner lookup
    uint4* arcs0 = nullptr;                 // A_0 arcs {s, d, eid, w}, grouped by source
    uint4* abuf[2] = {nullptr, nullptr};    // ping-pong alive arcs of rounds >= 1
    u64 *bestA = nullptr, *bestB = nullptr, *shard_best = nullptr;
    u32* P = nullptr;
    int *Mtmp = nullptr, *maps = nullptr;
    u32* tcnt = nullptr;  // hook tile counts and their scan (renumber offsets)
    u32* msf = nullptr;
    u64* mat[2] = {nullptr, nullptr};  // dense min-matrices over component pairs
    u64* status = nullptr;
    u32 epoch = 1;
    u32 pass_seq = 0;  // TMA arc-pass launches (tile-counter slot parity)
    u32* dcnt = nullptr;
    u64* acc = nullptr;
    void* hblock = nullptr;  // the pinned block (pinned_get) hcnt .. small_host live in
    u32* hcnt = nullptr;  // pinned
    volatile u64* hmap = nullptr;  // pinned + mapped: tagged n_{r+1} written by the hook,
                                   // then (at HSURV + r) the sampled compaction decision
    u64* dmap = nullptr;           // its device alias
    u32 run_seq = 0;
    u64* hacc = nullptr;  // pinned
    u64* hscr = nullptr;  // pinned scratch: [0] member-scan work, [1] round 0's singleton ends
    int* out_tmp = nullptr;  // for mst_run_host

    std::vector<Shard> shards;  // local shards (1, or G in the simulation)
    bool sim = false;
    int rank = 0, nranks = 1;
    ncclComm_t comm = nullptr;
    int xkind = X_NONE;
    mst_allreduce_min_fn xfn = nullptr;  // X_HOST: allreduce-MIN of u64 in host memory
    void* xctx = nullptr;
    u64* xhost = nullptr;                // X_HOST: pinned staging (n + dense matrix entries)
    u64 xcap = 0;
    u64 A0_local = 0;                    // records built on this rank (all shards)
    u32 vlo = 0, vhi = 0, wbase = 0;     // owners of this handle's records, their first record
    u32 *rrow = nullptr, *ridx = nullptr;  // reverse index (member-scan rounds): other -> records
    u64* mwork = nullptr;                // member-scan work estimate (device)
    int* hubs = nullptr;                 // the hub set of a member decision (33 ints, device)

    bool opt_uf = false;     // MST_OPT_UNION_FIND (NEXT-3 variant)
    bool opt_small = true;   // MST_OPT_SMALL (one-CTA path for graphs that fit shared memory)
    bool adj_dedup = true;   // A8's adjacent-duplicate filter in compacting passes (layout rule)
    bool opt_dedup = false;  // MST_OPT_DEDUP (A9: sort-based duplicate collapse after compaction)
    void* dd_scratch = nullptr;  // its scratch (allocated when the option is set)
    size_t dd_bytes = 0;
    int* dd_runs = nullptr;
    void* small_res = nullptr;   // its device result block (SmallOut)
    void* small_host = nullptr;  // pinned copy
    bool opt_dense = true;   // MST_OPT_DENSE
    bool opt_keep = false;   // MST_OPT_KEEP_EDGES (paper-faithful ablation)
    bool opt_tail = true;    // MST_OPT_DEVICE_TAIL
    u32 tau = 900;           // MST_OPT_COMPACT_TAU (permille; measured: uniform 950 -> 900 +2.7 %)
    int light_k = -1;        // MST_OPT_LIGHT_FIRST (-1 auto, 0 off, else light records ~ K n)
    u32 kfmt = 0;            // packed minima keys (w << s1 | eid << pb | partner): s1 | pb << 8
    bool hub_row = false;
    u64* trace = nullptr;    // MST_TAIL_TRACE=1 (tools): phase timestamps of the dense tail    // heavy-tailed input: hub row of the dense transition in smem
    int* phi = nullptr;      // composed label map of the records' label space (row A7)
    int* phi2 = nullptr;     // vertex -> component while phi maps compacted light records

    cudaEvent_t fail_ev = nullptr;  // recorded on the run stream when a run fails: the frees
                                    // of mst_destroy wait for whatever is still in flight
    bool prof = false;
    std::vector<ProfRec> recs;
    std::vector<mst_launch_time> ltimes;  // per launch of the last profiled run
    std::vector<cudaEvent_t> evpool;
    size_t evused = 0;
    mst_stats st{};
    bool broken = false;
};

namespace {

// The handle's small pinned host buffers (counters, the mapped round words, the one-CTA result
// block) live in one mapped block taken from a process-wide free list: pinning and unpinning
// host memory costs milliseconds per handle (measured: 1.4-6 ms of a one-shot solve), and a
// released block is zeroed and reused by the next handle.
struct PinnedBlocks {
    std::mutex mu;
    std::vector<void*> free;
};
PinnedBlocks& pinned_blocks() {
    static PinnedBlocks* p = new PinnedBlocks();  // (never destroyed: outlives every handle)
    return *p;
}
void* pinned_get(size_t bytes) {
    void* q = nullptr;
    {
        PinnedBlocks& pb = pinned_blocks();
        std::lock_guard<std::mutex> lk(pb.mu);
        if (!pb.free.empty()) {
            q = pb.free.back();
            pb.free.pop_back();
        }
    }
    if (!q && cudaHostAlloc(&q, bytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
        (void)cudaGetLastError();
        return nullptr;
    }
    memset(q, 0, bytes);
    return q;
}
void pinned_put(void* q) {
    if (!q) return;
    PinnedBlocks& pb = pinned_blocks();
    std::lock_guard<std::mutex> lk(pb.mu);
    pb.free.push_back(q);
}
constexpr size_t al64(size_t x) { return (x + 63) & ~(size_t)63; }
size_t pinned_block_bytes() {  // hcnt | hacc | hscr | hmap | small_host
    return al64(DCNT_WORDS * sizeof(u32)) + al64(2 * ACC_SLOTS * sizeof(u64)) +
           al64(4 * sizeof(u64)) + al64(3 * HSURV * sizeof(u64)) + al64(small_out_bytes());
}

// keep freed pool memory reserved for the next handle (per device, idempotent, thread-safe)
mst_status configure_pool(int dev) {
    cudaMemPool_t pool;
    CK(cudaDeviceGetDefaultMemPool(&pool, dev));
    uint64_t thr = UINT64_MAX;
    CK(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
    return MST_OK;
}

template <typename T>
mst_status galloc(mst_graph* g, T** p, u64 count) {
    u64 bytes = std::max<u64>(count * sizeof(T), 16);
    void* q = nullptr;
    cudaError_t e = cudaMallocAsync(&q, bytes, g->cst);
    if (e != cudaSuccess) {
        (void)cudaGetLastError();
        return fail(e == cudaErrorMemoryAllocation ? MST_ENOMEM : MST_ECUDA,
                    "device allocation of %llu bytes failed: %s", (unsigned long long)bytes,
                    cudaGetErrorString(e));
    }
    g->allocs.push_back(q);
    *p = reinterpret_cast<T*>(q);
    return MST_OK;
}

void release(mst_graph* g) {
    if (!g) return;
    if (g->comm) ncclCommDestroy(g->comm);
    if (g->cst) {
        if (g->fail_ev) cudaStreamWaitEvent(g->cst, g->fail_ev, 0);
        for (void* p : g->allocs) cudaFreeAsync(p, g->cst);
        cudaStreamSynchronize(g->cst);
    }
    pinned_put(g->hblock);  // (hcnt, hacc, hscr, hmap and small_host live in it)
    if (g->xhost) cudaFreeHost(g->xhost);
    if (g->trace) cudaFree(g->trace);
    for (auto e : g->evpool) cudaEventDestroy(e);
    if (g->fail_ev) cudaEventDestroy(g->fail_ev);
    if (g->cst) cudaStreamDestroy(g->cst);
    delete g;
}

// --------------------------------------------------------------------------- profiling
cudaEvent_t next_event(mst_graph* g) {
    if (g->evused == g->evpool.size()) {
        cudaEvent_t e;
        cudaEventCreate(&e);
        g->evpool.push_back(e);
    }
    return g->evpool[g->evused++];
}

// NVTX ranges: every profiled launch group is also a host range named by its
// kind with the round as payload (nvtx3 is header-only: without an attached tool a push/pop
// is a check of one function pointer)
const char* const kNvtxName[MST_K_COUNT] = {"mst init", "mst min0 (A2)", "mst hook (A4/A6)",
                                            "mst jump (A5/A6)", "mst filter (A8)", "mst output (A11)",
                                            "mst comm (A3)", "mst dense (A9)", "mst light",
                                            "mst compose (A7)", "mst small (A1-A11)", "mst dedup (A9)"};
void nvtx_push(const char* name, int payload) {
    nvtxEventAttributes_t ea{};
    ea.version = NVTX_VERSION;
    ea.size = NVTX_EVENT_ATTRIB_STRUCT_SIZE;
    ea.messageType = NVTX_MESSAGE_TYPE_ASCII;
    ea.message.ascii = name;
    ea.payloadType = NVTX_PAYLOAD_TYPE_INT32;
    ea.payload.iValue = payload;
    nvtxRangePushEx(&ea);
}
struct NvtxRange {
    NvtxRange(const char* name, int payload = 0) { nvtx_push(name, payload); }
    ~NvtxRange() { nvtxRangePop(); }
};

struct Prof {
    mst_graph* g;
    cudaStream_t s;
    int kind, round, sub, shard;
    cudaEvent_t a = nullptr;
    Prof(mst_graph* g_, cudaStream_t s_, int kind_, int round_, int sub_ = 0, int shard_ = 0)
        : g(g_), s(s_), kind(kind_), round(round_), sub(sub_), shard(shard_) {
        nvtx_push(kind >= 0 && kind < MST_K_COUNT ? kNvtxName[kind] : "mst", round);
        if (g->prof) {
            a = next_event(g);
            cudaEventRecord(a, s);
        }
    }
    ~Prof() {
        nvtxRangePop();
        if (g->prof) {
            cudaEvent_t b = next_event(g);
            cudaEventRecord(b, s);
            g->recs.push_back({kind, round, sub, shard, a, b});
        }
    }
};

// --------------------------------------------------------------------------- build (A0)
mst_status check_args(int64_t n, int64_t m, const void* src, const void* dst, const void* w) {
    if (n < 0 || n > INT32_MAX) return fail(MST_EINVAL, "n = %lld out of [0, 2^31-1]", (long long)n);
    if (m < 0 || m > INT32_MAX) return fail(MST_EINVAL, "m = %lld out of [0, 2^31-1]", (long long)m);
    if (m > 0 && (!src || !dst || !w)) return fail(MST_EINVAL, "null input pointer with m > 0");
    if (m > 0 && n == 0) return fail(MST_EINVAL, "m > 0 edges on n = 0 vertices");
    return MST_OK;
}

// Arc-balanced source ranges: shard j owns the sources [v_j, v_{j+1}),
// v_j = the first vertex whose CSR row offset reaches j * A0 / G; returns the arc windows
// [row[v_j], row[v_{j+1}]). Pure host code (exported for tests as mst_shard_ranges).
void compute_shard_ranges(const u32* row, u64 n, int G, u64* lo, u64* hi, u64* vbo = nullptr) {
    const u64 A0 = row[n];
    std::vector<u64> vb(G + 1);
    vb[0] = 0;
    vb[G] = n;
    for (int j = 1; j < G; ++j) {
        const u64 target = A0 * (u64)j / (u64)G;
        vb[j] = (u64)(std::lower_bound(row, row + n + 1, (u32)target) - row);
        vb[j] = std::min<u64>(std::max(vb[j], vb[j - 1]), n);
    }
    for (int j = 0; j < G; ++j) {
        lo[j] = row[vb[j]];
        hi[j] = row[vb[j + 1]];
    }
    if (vbo)
        for (int j = 0; j <= G; ++j) vbo[j] = vb[j];
}

mst_status shard_ranges(mst_graph* g, int G, std::vector<u64>& lo, std::vector<u64>& hi,
                        std::vector<u64>& vb) {
    lo.assign(G, 0);
    hi.assign(G, 0);
    vb.assign(G + 1, 0);
    vb[G] = (u64)g->n;
    if (G == 1) {
        hi[0] = g->A0;
        return MST_OK;
    }
    std::vector<u32> row(g->n + 1);
    CK(cudaMemcpyAsync(row.data(), g->row, (g->n + 1) * sizeof(u32), cudaMemcpyDeviceToHost,
                       g->cst));
    CK(cudaStreamSynchronize(g->cst));
    compute_shard_ranges(row.data(), g->n, G, lo.data(), hi.data(), vb.data());
    return MST_OK;
}

// Host-array input streamed into the build (mst_create_host / mst_solve_host): the device
// arrays src/dst/w of build() are staging buffers filled chunk by chunk on a copy stream; the
// degree pass runs per endpoint chunk as it lands, the weights travel while the layout and row
// offsets are built, and the scatter runs per weight chunk — the PCIe transfer hides the build.
struct HostIn {
    const int32_t *src, *dst;
    const uint32_t* w;
    cudaStream_t cs;
    u64 chunk;                     // edges per chunk
    std::vector<cudaEvent_t> evs;  // one per endpoint chunk, then one per weight chunk
};

mst_status build(mst_graph* g, const int* src, const int* dst, const unsigned* w, int nshards_sim,
                 int rank, int nranks, int reorder, HostIn* hin = nullptr) {
    auto t0 = std::chrono::steady_clock::now();
    const u64 n = g->n, m = g->m;
    // reorder: 0 the caller's numbering, 1 the automatic layout, 2 a one-shot solve's (no BFS
    // order, no reverse index: builds that one run does not repay)
    const bool one_shot = reorder == 2;
    // MST_TRACE_BUILD=1: the build's phases timed on the host (a stream sync at each mark)
    static const bool btrace = getenv("MST_TRACE_BUILD") && getenv("MST_TRACE_BUILD")[0] == '1';
    auto tmark = t0;
    auto mark = [&](const char* what) {
        if (!btrace) return;
        cudaStreamSynchronize(g->cst);
        const auto now = std::chrono::steady_clock::now();
        fprintf(stderr, "build %-22s %8.3f ms\n", what,
                std::chrono::duration<double, std::milli>(now - tmark).count());
        tmark = now;
    };
    g->nwords = (m + 31) / 32;
    CKS(galloc(g, &g->eu, m));
    CKS(galloc(g, &g->ev, m));
    CKS(galloc(g, &g->row, n + 1));
    u32* deg;
    u32* cursor;
    CKS(galloc(g, &deg, n));
    CKS(galloc(g, &cursor, n));
    CKS(galloc(g, &g->dcnt, DCNT_WORDS));
    CKS(galloc(g, &g->acc, 2 * ACC_SLOTS));
    const u64 nslots = status_slots_needed(n, 2 * m, g->nwords);
    CKS(galloc(g, &g->status, nslots));
    CK(cudaMemsetAsync(g->status, 0, nslots * sizeof(u64), g->cst));
    CK(cudaMemsetAsync(deg, 0, std::max<u64>(n, 1) * sizeof(u32), g->cst));
    CK(cudaMemsetAsync(g->dcnt, 0, DCNT_WORDS * sizeof(u32), g->cst));
    {
        char* hb = (char*)pinned_get(pinned_block_bytes());
        if (!hb) return fail(MST_ENOMEM, "pinned host block of %zu bytes", pinned_block_bytes());
        g->hblock = hb;
        g->hcnt = (u32*)hb;
        hb += al64(DCNT_WORDS * sizeof(u32));
        g->hacc = (u64*)hb;
        hb += al64(2 * ACC_SLOTS * sizeof(u64));
        g->hscr = (u64*)hb;
        hb += al64(4 * sizeof(u64));
        g->hmap = (volatile u64*)hb;
        CK(cudaHostGetDevicePointer((void**)&g->dmap, hb, 0));
        hb += al64(3 * HSURV * sizeof(u64));
        g->small_host = hb;
    }

    mark("allocations");
    u64* dspan;  // [0] sum of |u - v|, [1] the degree argmax
    CKS(galloc(g, &dspan, 2));
    CK(cudaMemsetAsync(dspan, 0, sizeof(u64), g->cst));
    u64 nch = 0;  // host input: chunks of both copies
    if (hin) {
        nch = (m + hin->chunk - 1) / hin->chunk;
        for (u64 k = 0; k < nch; ++k) {  // endpoints, chunk by chunk; degree per chunk
            const u64 off = k * hin->chunk, len = std::min<u64>(hin->chunk, m - off);
            CK(cudaMemcpyAsync(const_cast<int*>(src) + off, hin->src + off, len * 4,
                               cudaMemcpyHostToDevice, hin->cs));
            CK(cudaMemcpyAsync(const_cast<int*>(dst) + off, hin->dst + off, len * 4,
                               cudaMemcpyHostToDevice, hin->cs));
            CK(cudaEventRecord(hin->evs[k], hin->cs));
            CK(cudaStreamWaitEvent(g->cst, hin->evs[k], 0));
            CK(launch_degree(g->cst, g->nsm, (u32)n, (u32)len, src + off, dst + off, nullptr,
                             g->eu + off, g->ev + off, deg, g->dcnt + C_ERR, g->dcnt + C_WMAX,
                             dspan));
        }
        for (u64 k = 0; k < nch; ++k) {  // then the weights (the scatter waits per chunk)
            const u64 off = k * hin->chunk, len = std::min<u64>(hin->chunk, m - off);
            CK(cudaMemcpyAsync(const_cast<unsigned*>(w) + off, hin->w + off, len * 4,
                               cudaMemcpyHostToDevice, hin->cs));
            CK(cudaEventRecord(hin->evs[nch + k], hin->cs));
        }
    } else {
        CK(launch_degree(g->cst, g->nsm, (u32)n, (u32)m, src, dst, w, g->eu, g->ev, deg,
                         g->dcnt + C_ERR, g->dcnt + C_WMAX, dspan));
    }
    CK(launch_deg_argmax(g->cst, g->nsm, (u32)n, deg, dspan + 1));
    u64 span = 0, dtop = 0;
    CK(cudaMemcpyAsync(&span, dspan, sizeof(u64), cudaMemcpyDeviceToHost, g->cst));
    CK(cudaMemcpyAsync(&dtop, dspan + 1, sizeof(u64), cudaMemcpyDeviceToHost, g->cst));
    CK(cudaMemcpyAsync(g->hcnt, g->dcnt, sizeof(u32), cudaMemcpyDeviceToHost, g->cst));
    CK(cudaMemcpyAsync(g->hcnt + C_WMAX, g->dcnt + C_WMAX, sizeof(u32), cudaMemcpyDeviceToHost,
                       g->cst));
    CK(cudaStreamSynchronize(g->cst));
    if (g->hcnt[0]) return fail(MST_EINVAL, "an endpoint is outside [0, n) (n = %lld)", (long long)n);
    mark("degree (reads inputs)");
    // packed minima keys when weight, edge id and a label fit in 63 bits (every handle:
    // the keys' order is the (w, eid) order, so the MIN of a distributed run is unchanged);
    // the records carry their key base, so the format is fixed before they are built (host
    // input: after the scatter, which then writes (w << 32 | eid) and takes the largest weight)
    auto key_format = [&]() {
        const u32 wb = bits_of(g->hcnt[C_WMAX]), eb = bits_of(m > 0 ? (u64)m - 1 : 0),
                  pb = bits_of(n > 0 ? (u64)n - 1 : 0);
        static const char* pk = getenv("MST_PACKED_KEYS");  // "0": always (w << 32) | eid
        if (pb > 0 && wb + eb + pb <= 63 && !(pk && pk[0] == '0')) g->kfmt = (eb + pb) | (pb << 8);
    };
    if (!hin) key_format();

    // owner degrees (each non-loop edge once, owned by one endpoint: owner_of())
    // default: the higher internal id (the lower-degree endpoint) owns the record, so the
    // random per-record work lands on the hot hub labels; MST_OWNER_MAX=0 reverts
    const char* op = getenv("MST_OWNER_MAX");
    const int hi_owner = (op && op[0] == '0') ? 0 : 1;
    CK(cudaMemsetAsync(cursor, 0, std::max<u64>(n, 1) * sizeof(u32), g->cst));
    const char* ro = getenv("MST_REORDER");  // "0": the caller's numbering, "1": hub-first, "2": BFS
    const u32 dmax = (u32)(dtop >> 32), droot = ~(u32)dtop;  // (device argmax: no n-word copy)
    bool bfs = ro && ro[0] == '2' && nranks == 1;
    if (n > 0 && reorder && !ro) {
        // auto layout (NEXT-4, measured in DESIGN.md §5d): heavy-tailed degrees -> hub-first;
        // near-regular degrees whose ids carry no locality (mean |u - v| > n / 8: uniform,
        // dense) -> BFS order; near-regular with local ids (road, grids) -> hub-first, i.e.
        // the caller's order within equal degree buckets
        const bool heavy = (double)dmax * (double)n >= 16.0 * 2.0 * (double)m;
        // (not for a distributed handle: the BFS order depends on atomics, and every rank
        // must derive the identical numbering)
        bfs = !heavy && m > 0 && (double)span / (double)m > (double)n / 8.0 && nranks == 1;
        if (bfs && reorder == 2) {  // (a one-shot solve: the BFS build, ~10 ms, does not pay)
            bfs = false;
            reorder = 0;
        }
    }
    g->st.layout = (n > 0 && reorder && !(ro && ro[0] == '0')) ? (bfs ? 2 : 1) : 0;
    mark("layout decision");
    // A8's adjacent-duplicate filter pays where parallel records sit next to each other (road:
    // 2.50 -> 2.19 ms) and costs a little where the ids carry no locality (uniform +2 %)
    {
        static const char* ad = getenv("MST_ADJ_DEDUP");  // "0" / "1": force
        g->adj_dedup = ad ? ad[0] == '1' : !bfs;
    }
    if (n > 0 && reorder && bfs) {
        // NEXT-4 locality layout: BFS order from the highest-degree vertex (§6.1)
        const u32 root = droot;
        u32 *degn, *newid, *off, *bcur, *adj, *q, *stt;
        CKS(galloc(g, &degn, n));
        CKS(galloc(g, &newid, n));
        CKS(galloc(g, &off, n + 1));
        CKS(galloc(g, &bcur, n));
        CKS(galloc(g, &adj, 2 * (u64)m));
        CKS(galloc(g, &q, n));
        CKS(galloc(g, &stt, 16));
        CK(launch_reorder_bfs(g->cst, g->nsm, (u32)n, (u32)m, deg, degn, g->eu, g->ev, off, bcur,
                              adj, q, newid, stt, g->status, g->epoch++, cursor, hi_owner, root));
        u32 d0 = 0;
        CK(cudaMemcpyAsync(&d0, degn, sizeof(u32), cudaMemcpyDeviceToHost, g->cst));
        CK(cudaStreamSynchronize(g->cst));
        g->hub_row = (double)d0 * (double)n >= 16.0 * 2.0 * (double)m;
    } else if (n > 0 && reorder && !(ro && ro[0] == '0')) {
        // A0 locality layout: hub-first internal numbering (stable, by log2 degree); the
        // relabelling pass also counts owner degrees in the new numbering
        u32 *degn, *newid, *counts;
        CKS(galloc(g, &degn, n));
        CKS(galloc(g, &newid, n));
        CKS(galloc(g, &counts, reorder_scratch(n)));
        CK(launch_reorder(g->cst, g->nsm, (u32)n, (u32)m, deg, degn, g->eu, g->ev, newid, counts,
                          g->status, g->epoch++, cursor, hi_owner));
        // heavy-tailed degrees (internal vertex 0 = the top hub far above the mean degree):
        // the dense transition then keeps the hub's matrix row in shared memory
        u32 d0 = 0;
        CK(cudaMemcpyAsync(&d0, degn, sizeof(u32), cudaMemcpyDeviceToHost, g->cst));
        CK(cudaStreamSynchronize(g->cst));
        g->hub_row = (double)d0 * (double)n >= 16.0 * 2.0 * (double)m;
    } else {
        CK(launch_owner_degree(g->cst, g->nsm, (u32)m, g->eu, g->ev, cursor, hi_owner));
    }
    mark("renumbering");
    deg = cursor;
    u32* odeg_scan_out;
    CKS(galloc(g, &odeg_scan_out, n));
    cursor = odeg_scan_out;
    if (n > 0) {
        CK(launch_scan_rows(g->cst, (u32)n, deg, g->row, cursor, g->status, g->epoch++));
    } else {
        CK(cudaMemsetAsync(g->row, 0, sizeof(u32), g->cst));
    }
    u32 A0;
    CK(cudaMemcpyAsync(&A0, g->row + n, sizeof(u32), cudaMemcpyDeviceToHost, g->cst));
    CK(cudaStreamSynchronize(g->cst));
    g->A0 = A0;  // every rank's records together (the global E_0: identical decisions)
    mark("row offsets");

    // shards: owner-vertex ranges balanced by records. The simulation keeps
    // all G ranges in one handle; a distributed rank builds ONLY the records of its own range
    const int G = nshards_sim > 1 ? nshards_sim : nranks;
    std::vector<u64> lo, hi, vb;
    CKS(shard_ranges(g, G, lo, hi, vb));
    u64 wbase = 0, vlo = 0, vhi = n;  // the records this handle builds: owners [vlo, vhi)
    if (nshards_sim <= 1 && G > 1) {
        wbase = lo[rank];
        vlo = vb[rank];
        vhi = vb[rank + 1];
    }
    const u64 A_loc = (nshards_sim <= 1 && G > 1) ? hi[rank] - lo[rank] : (u64)A0;
    g->A0_local = A_loc;
    CKS(galloc(g, &g->arcs0, A_loc));
    CKS(galloc(g, &g->euv, m));
    if (hin) {
        for (u64 k = 0; k < nch; ++k) {
            const u64 off = k * hin->chunk, len = std::min<u64>(hin->chunk, m - off);
            CK(cudaStreamWaitEvent(g->cst, hin->evs[nch + k], 0));
            CK(launch_scatter(g->cst, g->nsm, (u32)len, g->eu, g->ev, w, cursor, g->arcs0, g->euv,
                              hi_owner, 0u, (u32)vlo, (u32)vhi, (u32)wbase, (u32)off,
                              g->dcnt + C_WMAX));
        }
        CK(cudaMemcpyAsync(g->hcnt + C_WMAX, g->dcnt + C_WMAX, sizeof(u32), cudaMemcpyDeviceToHost,
                           g->cst));
        CK(cudaStreamSynchronize(g->cst));
        key_format();
        CK(launch_key_format(g->cst, g->nsm, A_loc, g->arcs0, g->kfmt));
    } else {
        CK(launch_scatter(g->cst, g->nsm, (u32)m, g->eu, g->ev, w, cursor, g->arcs0, g->euv,
                          hi_owner, g->kfmt, (u32)vlo, (u32)vhi, (u32)wbase));
    }
    g->vlo = (u32)vlo;
    g->vhi = (u32)vhi;
    g->wbase = (u32)wbase;
    mark("scatter (reads w)");
    if (n > 0 && (u64)A0 >= 8ull * n && !one_shot) {
        // heavy-tailed / dense inputs (the light-edge phase's regime): the reverse index of the
        // records for the member-scan rounds (other endpoint -> record indices; build time only)
        u32* rdeg;
        CKS(galloc(g, &rdeg, n));
        CKS(galloc(g, &g->rrow, n + 1));
        CKS(galloc(g, &g->ridx, A_loc));
        CKS(galloc(g, &g->mwork, 1));
        CKS(galloc(g, &g->hubs, 64));
        // (the spare vertex map only serves the light-compaction ablation, MST_LIGHT_COMPACT)
        const char* lcv = getenv("MST_LIGHT_COMPACT");
        if (lcv && atoi(lcv) != 0) CKS(galloc(g, &g->phi2, n));
        u32* rpc;  // (per-CTA counts of the hot vertices; build time only)
        CKS(galloc(g, &rpc, reverse_index_scratch(g->nsm, (u32)n)));
        CK(launch_reverse_index(g->cst, g->nsm, (u32)n, A_loc, g->arcs0, rdeg, g->rrow, cursor,
                                g->ridx, g->status, g->epoch++, rpc));
    }
    mark("reverse index");
    g->shards.clear();
    // light-edge phase: each shard's light records and their dead filler records (at most
    // LBLK_MAX per consumer warp of the pass) get their own window in abuf[0]
    const u64 slack = (u64)pass_warps(g->nsm) * LBLK_MAX;
    for (int j = 0; j < G; ++j) {
        if (nshards_sim <= 1 && j != rank) continue;
        const u64 l = lo[j] - wbase, h = hi[j] - wbase, k = g->shards.size();
        g->shards.push_back({l, h, l + k * slack, (u32)(h - l)});
    }
    // ping-pong record buffers: a shard's records keep their [lo, hi) window in every buffer
    CKS(galloc(g, &g->abuf[0], A_loc + g->shards.size() * slack));
    CKS(galloc(g, &g->abuf[1], A_loc));
    CKS(galloc(g, &g->bestA, n));
    CKS(galloc(g, &g->bestB, n));
    if (g->sim) CKS(galloc(g, &g->shard_best, n * (u64)g->shards.size()));
    CKS(galloc(g, &g->P, n));
    CKS(galloc(g, &g->Mtmp, n));
    CKS(galloc(g, &g->tcnt, 2 * std::max(hook_tiles(n), out_tiles(g->nwords)) + 2));
    // sum_r n_r <= 2n when every live component merges each round; the light-edge phase
    // defers components (no merge) and switches to all edges before 3n + 1 is reached
    CKS(galloc(g, &g->maps, 3 * n + 1));
    CKS(galloc(g, &g->msf, g->nwords));
    // the one-CTA path's result block lives in mapped pinned memory: the kernel writes it and
    // publishes a tag; the host spins on the tag (no copy, no stream synchronisation)
    CK(cudaHostGetDevicePointer(&g->small_res, g->small_host, 0));  // (zeroed with the block)
    CKS(galloc(g, &g->phi, n));
    if (n >= 2) {  // dense min-matrices (A9 / NEXT-1), <= 67 MB each
        CKS(galloc(g, &g->mat[0], dense_entries(n)));
        CKS(galloc(g, &g->mat[1], dense_entries(n)));
    }
    CK(cudaStreamSynchronize(g->cst));
    mark("rest");
    g->st.n = g->n;
    g->st.m = g->m;
    g->st.arcs0 = (int64_t)g->A0;
    g->st.nranks = nranks;
    g->st.rank = rank;
    g->st.local_arcs0 = (int64_t)g->A0_local;
    g->st.build_ms =
        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return MST_OK;
}

mst_status create_common(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                         const uint32_t* w, int nshards_sim, const uint8_t* id, int rank,
                         int nranks, mst_graph** out, int reorder = 1,
                         mst_allreduce_min_fn xfn = nullptr, void* xctx = nullptr,
                         HostIn* hin = nullptr) {
    if (!out) return fail(MST_EINVAL, "out is NULL");
    *out = nullptr;
    CKS(check_args(n, m, src, dst, w));
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(MST_EINVAL, "bad rank/nranks");
    if (nshards_sim < 1 || nshards_sim > 64) return fail(MST_EINVAL, "nshards must be in [1, 64]");
    int dev;
    CK(cudaGetDevice(&dev));
    CKS(configure_pool(dev));
    mst_graph* g = new (std::nothrow) mst_graph();
    if (!g) return fail(MST_ENOMEM, "host allocation failed");
    g->dev = dev;
    g->n = n;
    g->m = m;
    g->sim = nshards_sim > 1;
    g->rank = rank;
    g->nranks = nranks;
    cudaError_t e = cudaDeviceGetAttribute(&g->nsm, cudaDevAttrMultiProcessorCount, dev);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&g->cst, cudaStreamNonBlocking);
    if (e != cudaSuccess) {
        release(g);
        return fail(MST_ECUDA, "device setup: %s", cudaGetErrorString(e));
    }
    // the inputs may still be written by work in flight on any of the caller's streams (the
    // build reads them on the handle's own non-blocking stream): wait for the device first
    // (a one-time cost of the build)
    if (cudaDeviceSynchronize() != cudaSuccess) {
        const cudaError_t e2 = cudaGetLastError();
        release(g);
        return fail(MST_ECUDA, "device synchronisation before the build: %s", cudaGetErrorString(e2));
    }
    mst_status s;
    {
        NvtxRange range("mst_create (A0 build)", (int)std::min<int64_t>(m, INT32_MAX));
        s = build(g, src, dst, (const unsigned*)w, nshards_sim, rank, nranks, reorder, hin);
    }
    if (s == MST_OK && id != nullptr) {  // mst_create_dist: NCCL communicator (also 1 rank)
        ncclUniqueId uid;
        memcpy(&uid, id, sizeof uid);
        ncclResult_t r = ncclCommInitRank(&g->comm, nranks, uid, rank);
        if (r != ncclSuccess) s = fail(MST_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
        else g->xkind = X_NCCL;
    }
    if (s == MST_OK && xfn != nullptr) {  // host-callback exchange (test aid)
        g->xkind = X_HOST;
        g->xfn = xfn;
        g->xctx = xctx;
        g->xcap = std::max<u64>((u64)n, dense_entries((u64)n)) + 1;
        const cudaError_t e2 = cudaMallocHost(&g->xhost, g->xcap * sizeof(u64));
        if (e2 != cudaSuccess) {
            g->xhost = nullptr;
            s = fail(MST_ENOMEM, "pinned exchange staging: %s", cudaGetErrorString(e2));
        }
    }
    if (s != MST_OK) {
        std::string keep = g_err;
        (void)cudaGetLastError();
        release(g);
        g_err = keep;
        return s;
    }
    *out = g;
    return MST_OK;
}

// --------------------------------------------------------------------------- run
// Spin on the tagged word the hook writes to mapped host memory (no memcpy, no stream sync);
// a failing kernel never writes it, so the stream is queried now and then for errors.
mst_status wait_word(mst_graph* g, cudaStream_t s, int idx, u32 tag, u32* val) {
    const auto t0 = std::chrono::steady_clock::now();
    for (u64 spin = 0;; ++spin) {
        const u64 v = g->hmap[idx];
        if ((u32)(v >> 32) == tag) {
            *val = (u32)v;
            return MST_OK;
        }
        if ((spin & 1023) == 1023) {
            const cudaError_t e = cudaStreamQuery(s);
            if (e != cudaSuccess && e != cudaErrorNotReady)
                return fail(MST_ECUDA, "word %d: %s", idx, cudaGetErrorString(e));
            if (e == cudaSuccess) {  // stream drained: the word must be visible now
                const u64 w = g->hmap[idx];
                if ((u32)(w >> 32) == tag) {
                    *val = (u32)w;
                    return MST_OK;
                }
                return fail(MST_EINTERNAL, "word %d: not written", idx);
            }
            if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(120))
                return fail(MST_EINTERNAL, "word %d: timed out waiting for the device", idx);
        }
    }
}
// Spin on the tagged word the hook writes to mapped host memory (no memcpy, no stream sync);
// a failing kernel never writes it, so the stream is queried now and then for errors.
mst_status wait_round(mst_graph* g, cudaStream_t s, int r, u32 tag, u32* nn) {
    return wait_word(g, s, r, tag, nn);
}

// A3: allreduce-MIN over the ranks of a distributed handle, in place on the device (u64
// minima keys, or u32 for the light-edge threshold). NCCL: one ncclAllReduce on the run's
// stream. Host exchange (test aid): device -> pinned host, the caller's callback reduces across
// its processes, host -> device; the stream is synchronised around it.
mst_status xchg_min(mst_graph* g, cudaStream_t s, void* buf, u64 count, bool u32w) {
    if (count == 0 || g->xkind == X_NONE) return MST_OK;
    if (g->xkind == X_NCCL) {
        CKN(ncclAllReduce(buf, buf, count, u32w ? ncclUint32 : ncclUint64, ncclMin, g->comm, s));
        return MST_OK;
    }
    if (count > g->xcap) return fail(MST_EINTERNAL, "exchange of %llu words > staging", (unsigned long long)count);
    const size_t es = u32w ? 4 : 8;
    CK(cudaMemcpyAsync(g->xhost, buf, count * es, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    u32* x32 = reinterpret_cast<u32*>(g->xhost);
    if (u32w)  // widen in place (downwards: entry i is read before bytes [8i, 8i + 8) are written)
        for (u64 i = count; i-- > 0;) g->xhost[i] = (u64)x32[i];
    if (g->xfn(g->xhost, (int64_t)count, g->xctx) != 0)
        return fail(MST_ENCCL, "host exchange callback failed (rank %d)", g->rank);
    if (u32w)
        for (u64 i = 0; i < count; ++i) x32[i] = (u32)g->xhost[i];
    CK(cudaMemcpyAsync(buf, g->xhost, count * es, cudaMemcpyHostToDevice, s));
    CK(cudaStreamSynchronize(s));
    return MST_OK;
}

bool use_hub_row(const mst_graph* g) {
    static const char* e = getenv("MST_HUB_ROW");  // "0" / "1": override (ablation)
    if (e && (e[0] == '0' || e[0] == '1')) return e[0] == '1';
    return g->hub_row;
}

// per-launch event times of a profiled run -> kernel_ms / kernel_launches / round times
void collect_profile(mst_graph* g) {
    g->ltimes.clear();
    if (g->prof) {
        for (auto& rc : g->recs) {
            float ms = 0;
            cudaEventElapsedTime(&ms, rc.a, rc.b);
            g->ltimes.push_back({rc.kind, rc.sub, rc.round, rc.shard, (double)ms});
            g->st.kernel_ms[rc.kind] += ms;
            g->st.kernel_launches[rc.kind] += 1;
            if ((rc.kind == MST_K_FILTER || rc.kind == MST_K_DENSE) && rc.round < MST_MAX_ROUNDS)
                g->st.round_filter_ms[rc.round] += ms;
        }
    }
    g->st.profiling = g->prof ? 1 : 0;
}

// ---------------------------------------------------------------- A10: the one-CTA path
// Graphs whose records, per-component arrays and forest bits fit one CTA's shared memory run
// the whole method in one launch (kernels.cu k_small_msf): no per-round launches, no host
// round trips (grid64: ~10 launches and a host wait per round for microseconds of work).
bool small_ok(const mst_graph* g) {
    static const char* e = getenv("MST_SMALL");  // "0": never (ablation)
    if (!g->opt_small || (e && e[0] == '0') || g->opt_keep || g->shards.size() != 1 ||
        g->xkind != X_NONE || g->n < 2)
        return false;
    const u64 E = g->shards[0].hi - g->shards[0].lo;
    return g->kfmt != 0 &&  // (packed keys: the partner's label travels in the key)
           small_smem_bytes((u64)g->n, E, g->nwords) <= small_smem_limit();
}
struct SmallHost {  // (the layout of kernels.cu SmallOut)
    u32 count, rounds;
    u64 total;
    u32 n_r[64], a_r[64];
    u64 tag;
};
mst_status run_small(mst_graph* g, cudaStream_t s, int32_t* out_ids, int64_t* out_num,
                     uint64_t* out_total, unsigned long long kl0) {
    static_assert(sizeof(SmallHost) == 8 + 8 + 512 + 8, "SmallOut layout");
    const u64 n = g->n, E = g->shards[0].hi - g->shards[0].lo;
    const u64 tag = ((u64)(++g->run_seq) << 1) | 1u;  // (never 0: the initial value)
    {
        Prof p(g, s, MST_K_SMALL, 0);
        CK(launch_small(s, (u32)n, (u32)E, (u32)g->nwords, g->arcs0 + g->shards[0].lo,
                        g->kfmt & 0xffu, g->kfmt >> 8, out_ids, g->small_res, tag));
    }
    volatile SmallHost* vh = reinterpret_cast<volatile SmallHost*>(g->small_host);
    for (u64 spin = 0; vh->tag != tag; ++spin) {  // (the stream is checked now and then)
        if ((spin & 4095) == 4095) {
            const cudaError_t e = cudaStreamQuery(s);
            if (e != cudaSuccess && e != cudaErrorNotReady)
                return fail(MST_ECUDA, "one-CTA path: %s", cudaGetErrorString(e));
            if (e == cudaSuccess && vh->tag != tag) return fail(MST_EINTERNAL, "one-CTA path: no result");
        }
    }
    if (g->prof) CK(cudaStreamSynchronize(s));  // (the profiling events)
    const SmallHost* h = const_cast<const SmallHost*>(reinterpret_cast<volatile SmallHost*>(g->small_host));
    g->st.rounds = (int32_t)std::min<u32>(h->rounds, MST_MAX_ROUNDS);
    for (int r = 0; r < g->st.rounds; ++r) {
        g->st.n_r[r] = h->n_r[r];
        g->st.a_r[r] = h->a_r[r];
    }
    g->st.dense_round = -1;
    g->st.light_switch_round = -1;
    g->st.light_t = 0xffffffffu;
    g->st.compacted_mask = 0;
    g->st.hub_row = 0;
    for (int i = 0; i < MST_MAX_ROUNDS; ++i) g->st.survival_permille[i] = -1;
    if ((u64)h->count >= n) return fail(MST_EINTERNAL, "forest has >= n edges");
    *out_num = (int64_t)h->count;
    *out_total = h->total;
    g->st.num_edges = *out_num;
    g->st.total_weight = *out_total;
    collect_profile(g);
    g->st.gpu_launches = (int64_t)(kernel_launches() - kl0);
    return MST_OK;
}

// ---------------------------------------------------------------- NEXT-3: union-find variant
// Bulk-synchronous Boruvka over the unmodified edge records with a union-find (§8.4
// L389; kernels in kernels.cu "NEXT-3"). Per round r: K1 = k_arc_pass<MODE_UF>
// (roots by find, intra-component records dropped, survivors compacted unchanged when the
// policy says so, tagged minima into best[root]); K2a/K2b = partner roots, then forest bits
// and CAS unions. One host round trip per round: K1's survivor count (zero: done).
mst_status run_uf(mst_graph* g, cudaStream_t s, int32_t* out_ids, int64_t* out_num,
                  uint64_t* out_total, unsigned long long kl0) {
    const u64 n = g->n;
    if (g->shards.size() != 1 || g->xkind != X_NONE)
        return fail(MST_ENOTSUP, "MST_OPT_UNION_FIND: single-GPU handles only");
    Shard& sh = g->shards[0];
    u32* parent = reinterpret_cast<u32*>(g->Mtmp);  // (the morph path's scratch, n words)
    {
        Prof p(g, s, MST_K_INIT, 0);
        CK(launch_init(s, g->nsm, (u32)n, g->bestA, (u32)std::max<u64>(g->nwords, 1), g->msf,
                       g->acc, 2 * ACC_SLOTS, g->dcnt + C_SEEN, 2 * MST_MAX_ROUNDS,
                       g->dcnt + C_UFU, g->dcnt + C_AREC, AREC_STRIDE));
        CK(launch_uf_init(s, g->nsm, (u32)n, parent));
        CK(cudaMemsetAsync(g->dcnt + C_UFU, 0, MST_MAX_ROUNDS * sizeof(u32), s));
    }
    // key format: tagged when weight and edge-id bits fit below the 6-bit round tag
    const u32 wb = bits_of(g->hcnt[C_WMAX]);
    const u32 s1 = (g->kfmt >> 8) ? (g->kfmt & 0xffu) : 32u;  // the records' key format
    static const char* te = getenv("MST_UF_TAG");  // "0": untagged keys + a reset per round
    const bool tagged = wb + s1 <= 58 && !(te && te[0] == '0');
    g->hcnt[arec(0, 0)] = sh.A = (u32)(sh.hi - sh.lo);
    CK(cudaMemcpyAsync(g->dcnt + arec(0, 0), g->hcnt + arec(0, 0), sizeof(u32),
                       cudaMemcpyHostToDevice, s));
    const u32 tag_base = ((++g->run_seq) & 0xffffffu) << 8;
    const uint4* cur = g->arcs0;
    g->st.compacted_mask = 0;
    g->st.dense_round = -1;
    g->st.light_switch_round = -1;
    g->st.light_t = 0xffffffffu;
    g->st.hub_row = 0;
    for (int i = 0; i < MST_MAX_ROUNDS; ++i) g->st.survival_permille[i] = -1;
    int r = 0;
    while (true) {
        if (r >= 63) return fail(MST_EINTERNAL, "union-find variant: round limit exceeded");
        const u64 tag = tagged ? (u64)(62 - r) << 58 : 0ull;
        if (!tagged && r > 0) CK(cudaMemsetAsync(g->bestA, 0xff, n * sizeof(u64), s));
        // compaction of the survivors (unchanged records): never in round 0 (every non-loop
        // record crosses two singletons), else as the morph passes (MST_OPT_COMPACT_TAU)
        const bool never = r == 0 || g->tau == 0 || g->opt_keep;
        const bool adaptive = !never && g->tau < 1000;
        const uint4* outbuf = (cur == g->abuf[0]) ? g->abuf[1] : g->abuf[0];
        CompactCtl cc;
        cc.surv = g->dcnt + C_SURV + r;
        cc.seen = g->dcnt + C_SEEN + r;
        if (adaptive) {
            cc.tau = g->tau;
            cc.num = g->dcnt + C_SURV + (r - 1);
            cc.den = g->dcnt + C_SEEN + (r - 1);
            cc.hword = g->dmap + HSURV + r;
            cc.tag = tag_base | (u32)r;
        }
        {
            Prof p(g, s, MST_K_FILTER, r, MST_SUB_SPARSE);
            CK(launch_uf_pass(s, g->nsm, g->dcnt + arec(0, r), sh.hi - sh.lo, cur, parent,
                              never ? nullptr : const_cast<uint4*>(outbuf), g->bestA, (u32)n,
                              g->status, g->epoch++, g->dcnt + arec(0, r + 1), g->dcnt + C_TILE,
                              g->pass_seq, cc, g->kfmt, tag, g->adj_dedup));
        }
        {
            Prof p(g, s, MST_K_HOOK, r);
            CK(launch_uf_hook(s, g->nsm, (u32)n, parent, g->bestA, g->kfmt, tagged, tag, g->euv, g->P,
                              g->msf, g->acc, g->dcnt + C_UFU + r, g->dcnt + C_SURV + r,
                              g->dmap + r, tag_base | (u32)r));
        }
        u32 surv;
        CKS(wait_round(g, s, r, tag_base | (u32)r, &surv));
        if (!never) {
            u32 word = 1;  // (always compacting: tau >= 1000)
            if (adaptive) {
                CKS(wait_word(g, s, HSURV + r, tag_base | (u32)r, &word));
                g->st.survival_permille[r] = (int32_t)(word >> 1);
            }
            if (word & 1u) {
                cur = outbuf;
                g->st.compacted_mask |= 1ll << r;
            }
        }
        ++r;
        if (surv == 0) break;  // no record joins two components: the forest is complete
    }
    g->st.rounds = r;
    CK(cudaMemcpyAsync(g->hcnt + C_AREC, g->dcnt + C_AREC, AREC_STRIDE * sizeof(u32),
                       cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(g->hcnt + C_UFU, g->dcnt + C_UFU, MST_MAX_ROUNDS * sizeof(u32),
                       cudaMemcpyDeviceToHost, s));
    {
        Prof p(g, s, MST_K_OUTPUT, r);
        if (g->nwords) {
            CK(launch_output(s, (u32)g->nwords, g->msf, out_ids, g->tcnt, g->dcnt + C_OUT,
                             (u32)std::max<int64_t>(n - 1, 1)));
        } else {
            CK(cudaMemsetAsync(g->dcnt + C_OUT, 0, sizeof(u32), s));
        }
    }
    CK(cudaMemcpyAsync(g->hcnt, g->dcnt, 2 * sizeof(u32), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(g->hacc, g->acc, 2 * ACC_SLOTS * sizeof(u64), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    for (int i = 1; i < ACC_SLOTS; ++i) {
        g->hacc[0] += g->hacc[2 * i];
        g->hacc[1] += g->hacc[2 * i + 1];
    }
    int64_t comps = (int64_t)n;  // components (incl. isolated vertices) entering each round
    for (int rr = 0; rr < r; ++rr) {
        g->st.n_r[rr] = comps;
        g->st.a_r[rr] = g->hcnt[arec(0, rr)];
        comps -= g->hcnt[C_UFU + rr];
    }
    if ((u64)g->hcnt[C_OUT] != g->hacc[1])
        return fail(MST_EINTERNAL, "forest size mismatch: %u ids vs %llu unions", g->hcnt[C_OUT],
                    (unsigned long long)g->hacc[1]);
    if (g->hacc[1] >= n) return fail(MST_EINTERNAL, "forest has >= n edges");
    *out_num = (int64_t)g->hacc[1];
    *out_total = g->hacc[0];
    g->st.num_edges = *out_num;
    g->st.total_weight = *out_total;
    collect_profile(g);
    g->st.gpu_launches = (int64_t)(kernel_launches() - kl0);
    return MST_OK;
}

mst_status run_impl(mst_graph* g, cudaStream_t s, int32_t* out_ids, int64_t* out_num,
                    uint64_t* out_total) {
    const u64 n = g->n;
    g->recs.clear();
    g->evused = 0;
    g->st.gpu_launches = 0;
    const unsigned long long kl0 = kernel_launches();  // kernels of this run (set at the end)
    g->st.rounds = 0;
    for (int j = 0; j < MST_K_COUNT; ++j) {
        g->st.kernel_ms[j] = 0;
        g->st.kernel_launches[j] = 0;
    }
    for (int r = 0; r < MST_MAX_ROUNDS; ++r) {
        g->st.n_r[r] = g->st.a_r[r] = 0;
        g->st.round_filter_ms[r] = 0;
        g->st.member_ends[r] = -1;
        g->st.member_round[r] = 0;
        g->st.dedup_in[r] = -1;
    }
    if (n == 0) {
        *out_num = 0;
        *out_total = 0;
        g->st.num_edges = 0;
        g->st.total_weight = 0;
        return MST_OK;
    }
    if (g->opt_uf) return run_uf(g, s, out_ids, out_num, out_total, kl0);
    if (small_ok(g)) return run_small(g, s, out_ids, out_num, out_total, kl0);
    const int G = (int)g->shards.size();
    // light-edge phase (MST_OPT_LIGHT_FIRST): single handle, enough records to pay
    static const u32 lk_env = getenv("MST_LIGHT_K") ? (u32)atoi(getenv("MST_LIGHT_K")) : 0xffffffffu;
    // auto: the light subgraph of a dense near-regular graph must be connected to finish
    // in the light phase (light degree ~ 2K >= ln n); a heavy-tailed sparse one never is
    // (low-degree vertices), where fewer light records cost less (measured: dense K = 4,
    // RMAT-22 K = 2)
    // light-only round 0 (auto, >= 64 records per vertex): the round-0 pass only extracts
    // the light records (no minima over the full stream); the round-0 minima come from the
    // light records and vertices without one are deferred. K = 8 makes that a ~e^-16 event
    // per vertex on near-regular graphs (light degree ~ Poisson(2K)); it stays exact anyway.
    // (with the reverse index, >= 8 records per vertex, round 0 stays exact for the vertices
    // without a light record: their minima come from their own records, k_singleton_min, so
    // the round-0 pass is a pure extraction there too — RMAT-22: 357 -> ~200 us)
    static const char* lo_env = getenv("MST_LIGHT_ONLY0");
    static const char* me_env = getenv("MST_MEMBER_SCAN");  // "0": never (ablation)
    const bool member_ok = g->ridx && !(me_env && me_env[0] == '0');
    const bool dense_regime = g->A0 >= 64ull * (u64)n;
    const bool lo0_want = lo_env ? lo_env[0] == '1' : (g->light_k < 0 && (dense_regime || member_ok));
    const u32 lk = lk_env != 0xffffffffu ? lk_env
                 : g->light_k >= 0 ? (u32)g->light_k : (dense_regime ? 8u : 2u);
    // (decided on the global record count E_0: every rank of a distributed run agrees)
    int phase = (lk > 0 && !g->opt_keep && g->A0 >= 4096 &&
                 g->A0 >= 4ull * lk * n) ? 1 : 0;  // light records <= a quarter
    const bool dist = g->xkind != X_NONE;
    const bool light_only0 = lo0_want && phase;
    // round-0 minima of the vertices without a light record from their own records
    const bool singletons = light_only0 && member_ok;
    g->st.light_switch_round = -1;
    g->st.light_t = 0xffffffffu;
    // the light threshold t: selected by the init launch's last CTA (no launch of its own)
    LightSel lsel{};
    static const char* tf = getenv("MST_LIGHT_T");  // ablation: a fixed threshold
    if (phase && !tf && g->A0_local > 0) {
        // auto K = 2 aims a little above 2 n: below t ~ 119 RMAT-22 leaves a small part
        // uncontracted after the all-records pass (one more full pass: 52.7 -> 44.4 G
        // edges/s) while t 120-150 is flat; the 4096-record sample puts t within ~+-5
        // (dense regime, K = 8: aimed at 10 n so that t <= 2 — light degree ~8, a few
        // vertices without a light edge and one more all-records pass — stays unlikely)
        // (with member-scan rounds, fewer light records pay: the components the light
        // phase leaves are finished by member scans, not by a pass over every record;
        // measured on RMAT-22: t 139 -> 60, 62.8 -> 66.1 G edges/s; t 40: 64.9; with the
        // light-only round 0: t 60 / 50 / 40 -> 69.2 / 70.8 / 69.1; round 2, session 2, with
        // cheaper light passes, medians of 3: t 20 / 26 / 31 / 36 / 42 / ~54 (0.85 n) ->
        // 78.5 / 80.6 / 81.1 / 82.2 / 82.3 / 79.3: aimed at 0.62 n, t ~ 39; dense: t = 3 has a
        // cliff on some seeds (113 vs 216 G edges/s) and t <= 2 everywhere, so its target is
        // 12 n — t 5 +- 1 from the 4096-record sample — rather than 10 n, where t = 3 came out
        // of the sample ~8 % of the time)
        const bool auto_k = lk_env == 0xffffffffu && g->light_k < 0;
        const u64 target = !auto_k ? (u64)lk * n : dense_regime ? (u64)12 * n
                         : member_ok ? (u64)n * 62 / 100 : (u64)23 * n / 10;
        // a rank samples its own records, aimed at the same fraction of them; every rank
        // must use the SAME t (a mixed threshold is not a prefix of the (w, id) order),
        // so the ranks agree on the smallest sampled t
        const u64 Al = g->A0_local;
        lsel = LightSel{g->arcs0, Al, (u64)((double)target * Al / g->A0), g->dcnt + C_LT,
                        (g->kfmt >> 8) ? (g->kfmt & 0xffu) : 32u, 1};
    }
    // ---- A1 init
    {
        Prof p(g, s, MST_K_INIT, 0);
        // best_0 = inf, forest bits, accumulators, per-pass counters (C_SEEN, C_SURV), the
        // hub label (round 0: vertex 0 itself) and every shard's per-round record counts (a
        // pass that meets no record must not read a count an earlier run left)
        static_assert(C_SURV == C_SEEN + MST_MAX_ROUNDS, "counter layout");
        CK(launch_init(s, g->nsm, (u32)n, g->bestA, (u32)std::max<u64>(g->nwords, 1), g->msf,
                       g->acc, 2 * ACC_SLOTS, g->dcnt + C_SEEN, 2 * MST_MAX_ROUNDS,
                       g->dcnt + C_HUB, g->dcnt + C_AREC, (u32)G * AREC_STRIDE, &lsel));
        if (g->sim) CK(cudaMemsetAsync(g->shard_best, 0xff, n * G * sizeof(u64), s));
    }
    if (phase) {
        if (tf) {
            g->hcnt[C_LT] = (u32)strtoul(tf, nullptr, 10);
            CK(cudaMemcpyAsync(g->dcnt + C_LT, g->hcnt + C_LT, sizeof(u32), cudaMemcpyHostToDevice, s));
        } else if (g->A0_local == 0) {
            CK(cudaMemsetAsync(g->dcnt + C_LT, 0xff, sizeof(u32), s));
        }
        if (dist) {
            Prof p(g, s, MST_K_COMM, 0);
            CKS(xchg_min(g, s, g->dcnt + C_LT, 1, true));
        }
    }
    // ---- A2 round-0 minimum (+ A3); with the light phase it also writes the light records
    for (int j = 0; j < G; ++j) {
        Shard& sh = g->shards[j];
        sh.A = (u32)(sh.hi - sh.lo);
        u64* tgt = g->sim ? g->shard_best + (u64)j * n : g->bestA;
        if (sh.A == 0) continue;
        if (phase) {
            // a quarter of a warp's expected light records per reservation: few atomics on
            // the counter, filler <= a quarter of them (the shard's share of ~K n records)
            const u64 per_warp = (u64)((double)lk * n * sh.A / g->A0) / ((u64)g->nsm * 30);
            const u32 blk = (u32)std::min<u64>(LBLK_MAX, std::max<u64>(LBLK_MIN, per_warp / 4));
            {
                Prof p(g, s, MST_K_MIN0, 0, light_only0 ? MST_SUB_EXTRACT : MST_SUB_MIN_ALL, j);
                CK(launch_min0(s, g->nsm, sh.A, g->arcs0 + sh.lo, tgt, (u32)n, g->dcnt + C_TILE,
                               g->pass_seq, g->abuf[0] + sh.llo, g->dcnt + C_LT,
                               g->dcnt + arec(j, 0), blk | (light_only0 ? 1u << 31 : 0u), g->kfmt));
            }
            if (light_only0) {
                Prof p(g, s, MST_K_MIN0, 0, MST_SUB_MIN_LIGHT, j);
                CK(launch_min0_dev(s, g->nsm, g->dcnt + arec(j, 0),
                                   sh.A + (u64)pass_warps(g->nsm) * LBLK_MAX, g->abuf[0] + sh.llo,
                                   tgt, (u32)n, g->dcnt + C_TILE, g->pass_seq, g->kfmt));
            }
        } else {
            Prof p(g, s, MST_K_MIN0, 0, MST_SUB_MIN_ALL, j);
            CK(launch_min0(s, g->nsm, sh.A, g->arcs0 + sh.lo, tgt, (u32)n, g->dcnt + C_TILE,
                           g->pass_seq, nullptr, nullptr, nullptr, 0, g->kfmt));
        }
    }
    if (g->sim) {
        Prof p(g, s, MST_K_COMM, 0);
        CK(launch_combine_min(s, g->nsm, (u32)n, G, g->shard_best, n, g->bestA));
    }
    if (singletons) {
        // (a rank scans its own records for the vertices without a LOCAL light key: a vertex
        // with a light record elsewhere keeps it through the MIN, light keys < heavy keys)
        Prof p(g, s, MST_K_MIN0, 0, MST_SUB_SINGLETONS);
        CK(cudaMemsetAsync(g->mwork, 0, sizeof(u64), s));
        CK(launch_singleton_min(s, g->nsm, (u32)n, g->bestA, g->row, g->rrow, g->ridx, g->arcs0,
                                g->vlo, g->vhi, g->wbase, g->kfmt, g->mwork));
        // (stream-ordered before the member scans reuse the counter; read at the run's end)
        CK(cudaMemcpyAsync(&g->hscr[1], g->mwork, sizeof(u64), cudaMemcpyDeviceToHost, s));
    }
    if (dist) {
        // edge-once records: a vertex's round-0 minimum has contributions from every rank
        // that owns one of its edges (the other endpoint's side), so round 0 needs a
        // reduction too, not an allgather of rank-local minima
        Prof p(g, s, MST_K_COMM, 0);
        CKS(xchg_min(g, s, g->bestA, n, false));
    }

    // round-0 arc counts (host-known) into the per-round record
    for (int j = 0; j < G && !phase; ++j) g->hcnt[arec(j, 0)] = g->shards[j].A;
    for (int j = 0; j < G && !phase; ++j)
        CK(cudaMemcpyAsync(g->dcnt + arec(j, 0), g->hcnt + arec(j, 0), sizeof(u32),
                           cudaMemcpyHostToDevice, s));
    const u32 tag_base = ((++g->run_seq) & 0xffffffu) << 8;  // run-unique tags for hmap
    MapChain chain;
    chain.len = 0;
    u64 moff = 0;
    u32 nr = (u32)n;
    u64* bcur = g->bestA;
    u64* bnxt = g->bestB;
    int r = 0;
    // where the alive records live: buffer `cur` (per-shard windows), labels of round `brnd`
    // (n_b = nb_sz labels); a pass whose compaction was decided on the device (sampled) is
    // resolved at the next round's wait (pend)
    const uint4* cur = phase ? g->abuf[0] : g->arcs0;  // light phase: the light records
    bool cur_light = phase != 0;  // cur holds light records at the shards' llo windows
    auto off = [&](const Shard& sh) { return cur_light ? sh.llo : sh.lo; };
    int brnd = 0;
    u32 nb_sz = (u32)n;
    int pend = -1;
    const uint4* pend_out = nullptr;
    g->st.compacted_mask = 0;
    g->st.hub_row = 0;
    for (int i = 0; i < MST_MAX_ROUNDS; ++i) g->st.survival_permille[i] = -1;
    auto resolve = [&](u32 word) {  // outcome of round pend's sampled decision
        g->st.survival_permille[pend] = (int32_t)(word >> 1);  // the estimate the pass used
        if (word & 1u) {
            cur = pend_out;
            cur_light = false;
            brnd = pend + 1;
            nb_sz = (u32)g->st.n_r[pend + 1];
            g->st.compacted_mask |= 1ll << pend;
        }
        pend = -1;
    };
    // member-scan rounds (after the light-edge phase, kernels.cu "member-scan"): Ψ = vertex ->
    // round r+1 label composed (if not yet) together with the record ends outside the top hub's
    // component; the busiest rank's count decides for every rank
    // nbig: the distinct components among the top hubs' (1: only the giant is big)
    // (records still in vertex ids, brnd = 0: Ψ itself, ready for the pass too; compacted
    // light records, brnd > 0: the spare map g->phi2 from the whole chain — it becomes Ψ only
    // when the member round is taken, phi keeps the records' pass map otherwise)
    auto member_work = [&](int rr, const int* Mrr, bool hubk, bool& ready, u64& work,
                           u32& nbig) -> mst_status {
        CK(cudaMemsetAsync(g->mwork, 0, sizeof(u64), s));
        const bool vs = brnd == 0;
        int* vphi = vs ? g->phi : g->phi2;
        const int* vsrc = rr >= 1 && chain.len ? (brnd == rr - 1 ? chain.m[chain.len - 1] : g->phi) : nullptr;
        if (!vs) {
            Prof p(g, s, MST_K_COMPOSE, rr);
            CK(launch_chain_compose(s, g->nsm, (u32)n, chain, g->phi2));
            vsrc = g->phi2;
            ready = false;
        }
        if (!ready && hubk) {  // one pass: compose + count (the hub's label is tracked)
            Prof p(g, s, MST_K_COMPOSE, rr, 2);
            CK(launch_compose_work(s, g->nsm, (u32)n, vsrc, Mrr, vphi, g->hubs, g->row,
                                   g->rrow, g->vlo, g->vhi, g->mwork));
            CK(cudaMemcpyAsync(&g->hscr[2], g->hubs + HUBS_N, sizeof(int), cudaMemcpyDeviceToHost, s));
        } else {
            if (!ready) {
                Prof p(g, s, MST_K_COMPOSE, rr);
                CK(launch_compose(s, g->nsm, (u32)n, vsrc, Mrr, vphi));
            }
            Prof p(g, s, MST_K_COMPOSE, rr, 2);
            CK(launch_member_work(s, g->nsm, (u32)n, vphi, g->row, g->rrow, g->vlo, g->vhi,
                                  g->mwork));
        }
        const bool hubset = !ready && hubk;
        ready = vs;
        CK(cudaMemcpyAsync(&g->hscr[0], g->mwork, sizeof(u64), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        work = g->hscr[0];
        nbig = hubset ? (u32)*reinterpret_cast<int*>(&g->hscr[2]) : 1u;
        if (dist) {  // MAX over ranks = ~MIN(~x) (nbig is replicated: the labels are)
            u64 nx = ~work;
            CK(cudaMemcpyAsync(g->mwork, &nx, sizeof(u64), cudaMemcpyHostToDevice, s));
            CKS(xchg_min(g, s, g->mwork, 1, false));
            CK(cudaMemcpyAsync(&nx, g->mwork, sizeof(u64), cudaMemcpyDeviceToHost, s));
            CK(cudaStreamSynchronize(s));
            work = ~nx;
        }
        return MST_OK;
    };
    // record ends to touch against the 2 E_0 of a pass over every record (random 16-B reads:
    // worth it below ~1/16 of the streamed bytes)
    auto member_cheap = [&](u64 work) { return work * 16 < 2 * g->A0 / (u64)std::max(1, g->nranks); };
    bool member_next = false;  // the phase-1 check chose a member-scan round for this round
    int last_member_r = -2;    // the last member-scan round and its work (an upper bound after)
    u64 last_member_w = 0;
    bool hybrid_next = false;  // ... a hybrid round: light pass + member scan of the small ones
    bool hub_pending = false;  // the jump's hub set count is on its way to the host
    u64 member_w = 0;
    u32 member_nbig = 1;
    bool dense = false;  // this round's alive arcs live in the min-matrix g->mat[mc]
    int mc = 0;
    g->st.dense_round = -1;
    int tail_r0 = -1;  // first round run by the device-resident dense tail
    // a light-phase tail that stopped on deferred components hands over a virtual round: its
    // composite map (tail-start labels -> labels after it) and size, with no hook to run
    bool vround = false, hub_ok = true, phi_ready = false;
    u32 v_nn = 0;
    while (true) {
        if (r >= MST_MAX_ROUNDS || chain.len >= MST_CHAIN_MAX)
            return fail(MST_EINTERNAL, "round limit exceeded (r = %d)", r);
        if (dense && g->opt_tail) {
            // every remaining round in one cooperative launch (A4/A5/A6/A9 on the device)
            Prof p(g, s, MST_K_DENSE, r, MST_SUB_TAIL);
            static const bool tr = getenv("MST_TAIL_TRACE") && getenv("MST_TAIL_TRACE")[0] == '1';
            if (tr && !g->trace) {
                CK(cudaMalloc(&g->trace, 64 * sizeof(u64)));
                CK(cudaMemsetAsync(g->trace, 0, 64 * sizeof(u64), s));
            }
            const bool lp = phase == 1;
            if (lp && moff + nr > 3 * n + 1) return fail(MST_EINTERNAL, "label-map storage overflow");
            CK(launch_dense_tail(s, g->nsm, nr, bcur, bnxt, g->mat[mc], g->mat[mc ^ 1], g->euv,
                                 chain, g->msf, g->acc, g->dcnt + C_BAR, g->dcnt + C_TAIL,
                                 tr ? g->trace : nullptr, lp ? 1 : 0,
                                 lp ? g->maps + moff : nullptr, lp ? g->dcnt + C_TAILN : nullptr));
            if (tr) {
                u64 h[64];
                CK(cudaMemcpyAsync(h, g->trace, sizeof h, cudaMemcpyDeviceToHost, s));
                CK(cudaStreamSynchronize(s));
                for (int k = 0; k < 8 && h[k * 8]; ++k) {
                    fprintf(stderr, "tail round %d:", k);
                    for (int q = 1; q < 8; ++q)
                        fprintf(stderr, " %+.1f", h[k * 8 + q] ? (double)(h[k * 8 + q] - h[k * 8]) / 1e3 : -1.0);
                    fprintf(stderr, " us\n");
                }
                CK(cudaMemsetAsync(g->trace, 0, 64 * sizeof(u64), s));
            }
            if (lp) {  // did the light phase finish inside the tail?
                CK(cudaMemcpyAsync(g->hcnt + C_TAIL, g->dcnt + C_TAIL,
                                   (1 + MST_MAX_ROUNDS) * sizeof(u32), cudaMemcpyDeviceToHost, s));
                CK(cudaMemcpyAsync(g->hcnt + C_TAILN, g->dcnt + C_TAILN, sizeof(u32),
                                   cudaMemcpyDeviceToHost, s));
                CK(cudaStreamSynchronize(s));
                const u32 k = g->hcnt[C_TAIL];
                const u32 nf = g->hcnt[C_TAILN];
                if (k >= 1 && nf > 1 && r + (int)k < MST_MAX_ROUNDS) {
                    for (u32 i = 0; i < k; ++i) {
                        g->st.n_r[r + i] = g->hcnt[C_TAIL + 1 + i];
                        g->st.a_r[r + i] = (int64_t)dense_entries(g->hcnt[C_TAIL + 1 + i]);
                    }
                    r += (int)k - 1;  // this iteration stands for the tail's last round
                    vround = true;
                    v_nn = nf;
                    hub_ok = false;  // (the hub's label is not tracked through the tail)
                    CK(cudaMemsetAsync(bnxt, 0xff, (size_t)nf * sizeof(u64), s));
                }
            }
            if (!vround) {
                tail_r0 = r;
                break;
            }
        }
        int* Mr = g->maps + moff;
        u32 nn;
        const bool was_v = vround;
        hub_pending = false;
        if (vround) {
            vround = false;
            nn = v_nn;
        } else {
        // (the member-scan decision below first asks whether it can pay: the hub set, computed
        // by the jump's last CTA)
        hub_pending = phase == 1 && member_ok && r >= 1 && !dense && chain.len < MST_CHAIN_MAX;
        const bool hdefer = phase == 1 && (r > 0 || (light_only0 && !singletons));  // (else
                                                  // round 0's minima cover every edge)
        const u32 hkfmt = dense ? 0u : g->kfmt;  // dense rounds: matrix keys (w << 32 | eid)
        HubTask ht{chain, g->hubs, g->dmap + HHUB + r, tag_base | (u32)r, (u32)n,
                   g->dcnt + C_JDONE, hub_pending ? 1 : 0};
        {
            {
                Prof p(g, s, MST_K_HOOK, r);
                CK(launch_hook(s, nr, bcur, bnxt, g->dmap + r, tag_base | (u32)r, g->euv, chain,
                               g->P, g->Mtmp, g->msf, g->acc, g->tcnt, g->dcnt + C_NNEXT, hdefer,
                               hkfmt));
            }
            // the jump does not need the host: it reads n_{r+1} on the device and runs while
            // the counts travel to the host
            Prof p(g, s, MST_K_JUMP, r);
            CK(launch_jump(s, g->nsm, nr, g->P, g->Mtmp, g->tcnt, Mr, g->dcnt + C_NNEXT, bnxt,
                           (const int*)g->dcnt + C_HUB + r, (int*)g->dcnt + C_HUB + r + 1,
                           g->dmap + r, tag_base | (u32)r, &ht));
        }
        // one host round trip per round: n_{r+1} (sizes round r's filter),
        // read zero-copy from the word the hook's last tile writes to mapped host memory
        CKS(wait_round(g, s, r, tag_base | (u32)r, &nn));
        g->st.n_r[r] = nr;
        g->st.a_r[r] = dense ? (int64_t)dense_entries(nr) : -1;  // sparse: filled at the end
        if (pend >= 0) {  // the previous pass decided on the device whether it compacted
            u32 word;
            CKS(wait_word(g, s, HSURV + pend, tag_base | (u32)pend, &word));
            resolve(word);
        }
        }
        if (nn <= 1) {  // <= 1 live component left: no inter-component edge remains
            ++r;
            break;
        }
        // switch to all records when < 1/sw_den of the components merged: 1/8, or — when the
        // member-scan rounds can take over (reverse index) — only once the light rounds stop
        // merging: RMAT-22 merges 1.2 % in round 3 and 0.1 % in round 4, but those last merges
        // join the big pieces of its giant (then the member scan finishes cheaply)
        static const char* sw_env = getenv("MST_LIGHT_SWITCH");
        const u64 sw_den = sw_env ? (u64)atoi(sw_env) : (member_ok ? (u64)n + 1 : 8);
        member_next = false;
        hybrid_next = false;
        static const char* hy_env = getenv("MST_HYBRID");
        const bool hy = hy_env ? atoi(hy_env) != 0 : false;
        u32 hub_comps = 0;
        if (hub_pending && !was_v) CKS(wait_word(g, s, HHUB + r, tag_base | (u32)r, &hub_comps));
        if (phase == 1 && member_ok && r >= 1 && !was_v && !dense && hub_pending &&
            ((hy && brnd == 0) || hub_comps <= 1) &&
            nn > 1 && (u64)(nr - nn) * 4 < 3 * nr && moff + nr + 3ull * nn <= 3 * n) {
            // light phase: once the components outside the top hubs' own few record ends, the
            // member scan gives them their exact minima: next to a light pass while the hubs
            // are still in several big pieces (a hybrid round: the pieces merge by their light
            // minima), alone — replacing both the light pass and the pass over every record —
            // once one giant is left (RMAT-22: ~10 K small components, 2.37 M vertices in it)
            CKS(member_work(r, Mr, true, phi_ready, member_w, member_nbig));
            const bool cheap = member_cheap(member_w);
            member_next = cheap && member_nbig <= 1;
            hybrid_next = hy && brnd == 0 && cheap && member_nbig > 1;
            if (member_next && brnd != 0) {  // the vertex map becomes Ψ (records: arcs0 next)
                std::swap(g->phi, g->phi2);
                phi_ready = true;
            }
            static const bool dbg1 = getenv("MST_DEBUG_MEMBER") != nullptr;
            if (dbg1) fprintf(stderr, "light round %d: nr %u nn %u member work %llu hub comps %u -> %d %d\n",
                              r, nr, nn, (unsigned long long)member_w, member_nbig, (int)member_next,
                              (int)hybrid_next);
        }
        if (phase == 1 && (member_next || was_v || nn == nr || (u64)(nr - nn) * sw_den < nr ||
                           moff + nr + 3ull * nn > 3 * n)) {
            // no light edge joins two components any more (every component would otherwise
            // have merged or absorbed one), or < 1/8 merged (most components are deferred:
            // no light edge), or the label-map storage asks for it: this round's pass
            // re-reads every edge record in vertex ids through the composed map. Switching
            // at any round is exact: every merge so far took a component's minimum edge.
            phase = 2;
            dense = false;  // the records are read again (a dense phase-1 matrix is dropped)
            g->st.light_switch_round = r;
            if (!phi_ready && r >= 1 && chain.len + 1 < MST_CHAIN_MAX) {  // Ψ = Mr ∘ chain in one kernel
                Prof p(g, s, MST_K_COMPOSE, r);
                MapChain full = chain;
                full.m[full.len++] = Mr;
                CK(launch_chain_compose(s, g->nsm, (u32)n, full, g->phi));
                phi_ready = true;
            }
            cur = g->arcs0;
            cur_light = false;
            brnd = 0;
            nb_sz = (u32)n;
            for (int j = 0; j < G; ++j) {  // every shard re-reads all its records
                g->hcnt[arec(j, r)] = (u32)(g->shards[j].hi - g->shards[j].lo);
                CK(cudaMemcpyAsync(g->dcnt + arec(j, r), g->hcnt + arec(j, r), sizeof(u32),
                                   cudaMemcpyHostToDevice, s));
            }
        }
        if (moff + nr + nn > 3 * n + 1) return fail(MST_EINTERNAL, "label-map storage overflow");
        bool to_dense = false;
        if (dense) {
            // A9/NEXT-1 dense round: scan the matrix, collapse into the next (smaller) one
            Prof p(g, s, MST_K_DENSE, r, MST_SUB_DENSE_ROUND);
            CK(launch_dense_init(s, g->nsm, nn, g->mat[mc ^ 1]));
            CK(launch_dense_round(s, g->nsm, nr, g->mat[mc], Mr, nn, g->mat[mc ^ 1], bnxt));
        } else {
            // member-scan round (after the light-edge phase): the records are read in vertex ids
            // through Ψ; when the vertices outside the top hub's component own few record ends,
            // their components' minima come from their members' records alone (kernels.cu)
            bool member = false;
            u64 mwork = member_w;
            if (member_next) {
                member = true;  // (decided by the phase-1 check of this round)
            } else if (phase == 2 && member_ok && cur == g->arcs0 && brnd == 0 &&
                       (phi_ready || brnd < r) && last_member_r == r - 1) {
                // right after a member round: the vertices outside the hub's component only
                // ever join it, so the work cannot have grown — no count, no host round trip
                if (!phi_ready) {
                    Prof p(g, s, MST_K_COMPOSE, r);
                    CK(launch_compose(s, g->nsm, (u32)n, brnd == r - 1 ? chain.m[chain.len - 1] : g->phi,
                                      Mr, g->phi));
                    phi_ready = true;
                }
                member = true;
                mwork = last_member_w;
            } else if (phase == 2 && member_ok && cur == g->arcs0 && brnd == 0 &&
                       (phi_ready || brnd < r)) {
                u32 nbig = 1;
                CKS(member_work(r, Mr, false, phi_ready, mwork, nbig));
                member = member_cheap(mwork);
                static const bool dbg = getenv("MST_DEBUG_MEMBER") != nullptr;
                if (dbg) {
                    fprintf(stderr, "member round %d: nn %u work %llu A0 %llu -> %d\n", r, nn,
                            (unsigned long long)mwork, (unsigned long long)g->A0, (int)member);
                    std::vector<int> ph(n);
                    std::vector<u32> rw(n + 1), rr(n + 1);
                    CK(cudaMemcpy(ph.data(), g->phi, n * 4, cudaMemcpyDeviceToHost));
                    CK(cudaMemcpy(rw.data(), g->row, (n + 1) * 4, cudaMemcpyDeviceToHost));
                    CK(cudaMemcpy(rr.data(), g->rrow, (n + 1) * 4, cudaMemcpyDeviceToHost));
                    std::vector<u64> sz(nn + 1, 0), dg(nn + 1, 0);
                    u64 fin = 0;
                    for (u64 v = 0; v < n; ++v) {
                        if (ph[v] < 0) { ++fin; continue; }
                        sz[ph[v]]++;
                        dg[ph[v]] += (rw[v + 1] - rw[v]) + (rr[v + 1] - rr[v]);
                    }
                    u64 big = 0;
                    for (u32 c = 0; c < nn; ++c) if (sz[c] > sz[big]) big = c;
                    if (FILE* f = fopen("gpurun_out/phi.bin", "wb")) {
                        fwrite(ph.data(), 4, n, f);
                        fclose(f);
                    }
                    fprintf(stderr, "  phi[0] = %d (size %llu, ends %llu); largest comp %llu size %llu ends %llu; finished vertices %llu; rrow[n] %u row[n] %u\n",
                            ph[0], ph[0] >= 0 ? (unsigned long long)sz[ph[0]] : 0ull,
                            ph[0] >= 0 ? (unsigned long long)dg[ph[0]] : 0ull, (unsigned long long)big,
                            (unsigned long long)sz[big], (unsigned long long)dg[big], (unsigned long long)fin,
                            rr[n], rw[n]);
                }
            }
            // (light phase: only when its ~K n records outnumber the matrix cells — measured
            // on dense: 0.76 M light records against 5.7 M cells made the tail 2x slower)
            to_dense = !member && g->mat[0] && g->opt_dense && !g->opt_keep && nn <= (u32)DENSE_MAX &&
                       (phase != 1 || (u64)lk * n >= dense_entries(nn));
            if (to_dense) CK(launch_dense_init(s, g->nsm, nn, g->mat[0]));
            // A7: the map of this round's pass, from the records' label space (round brnd)
            // to round r+1: M_r itself, or composed over the rounds that did not compact
            const int* Mpass = Mr;
            if (phi_ready) {  // (the switch or the member decision composed Ψ with M_r already)
                Mpass = g->phi;
                phi_ready = false;
            } else if (brnd < r) {
                Prof p(g, s, MST_K_COMPOSE, r);
                const int* src = (brnd == r - 1) ? chain.m[chain.len - 1] : g->phi;
                CK(launch_compose(s, g->nsm, nb_sz, src, Mr, g->phi));
                Mpass = g->phi;
            }
            // compaction policy: never (keep-edges: the paper's scheme, or tau = 0), always
            // (tau >= 1000), or decided on the device from the estimated survival (CompactCtl)
            // the pass that re-reads every record after the light phase never compacts:
            // measured on RMAT-22, ~70 % of the records still join two components there, but
            // one more hook round usually finishes (writing them back cost 0.3 ms)
            // (nor do the light-phase passes: their records are read only a couple more
            // times; measured on RMAT-22 with ~80 % surviving: 49.2 -> 51.1 G edges/s)
            // light-phase passes (MST_LIGHT_COMPACT): 0 never, 1 adaptive from round 1, 2 always
            // from round 1, 3 adaptive from round 0
            static const int lcm = getenv("MST_LIGHT_COMPACT") ? atoi(getenv("MST_LIGHT_COMPACT")) : 0;
            const bool light_never = phase == 1 && (lcm == 0 || r < (lcm == 3 ? 0 : 1) ||
                                                    (member_ok && !g->phi2));
            const bool never = g->opt_keep || g->tau == 0 || r == g->st.light_switch_round ||
                               light_never;
            int dsh = -1;  // the shard whose pass reports the device-side decision
            for (int j = 0; j < G && dsh < 0; ++j)
                if (g->shards[j].hi > g->shards[j].lo) dsh = j;
            // (A9 dedup needs the survivors compacted: it always compacts then)
            const bool dedup = g->opt_dedup && g->dd_scratch && G == 1 && !dist && !to_dense &&
                               !never && !member && phase != 1;
            const bool adaptive = !to_dense && !never && g->tau < 1000 && dsh >= 0 && !dedup &&
                                  !(phase == 1 && lcm == 2);
            const uint4* outbuf = (cur == g->abuf[0]) ? g->abuf[1] : g->abuf[0];
            CompactCtl cc;
            cc.surv = g->dcnt + C_SURV + r;
            cc.seen = g->dcnt + C_SEEN + r;
            if (adaptive) {
                cc.tau = g->tau;
                if (r == 0) {  // no previous pass: sample this pass's records
                    Prof p(g, s, MST_K_COMPOSE, r, 1);
                    const Shard& sh = g->shards[dsh];
                    CK(launch_sample_survival(s, cur + off(sh), g->dcnt + arec(dsh, r), Mpass,
                                              g->dcnt + C_SAMP, g->dcnt + C_SAMP + 1));
                    cc.num = g->dcnt + C_SAMP;
                    cc.den = g->dcnt + C_SAMP + 1;
                } else {
                    cc.num = g->dcnt + C_SURV + (r - 1);
                    cc.den = g->dcnt + C_SEEN + (r - 1);
                }
            }
            if (hybrid_next && phase == 1 && !to_dense) {
                // hybrid round: the small components' exact minima next to the light pass below
                Prof p(g, s, MST_K_FILTER, r, MST_SUB_MEMBER);
                CK(launch_member_min(s, g->nsm, (u32)n, g->hubs, g->phi, g->row, g->rrow, g->ridx,
                                     g->arcs0, g->vlo, g->vhi, g->wbase,
                                     g->sim ? g->shard_best : bnxt, g->kfmt));
                g->st.member_ends[r] = (int64_t)member_w;
                g->st.member_round[r] = 2;
            }
            if (member) {
                // the members' records of every component but the top hub's (deferred); the
                // records themselves are untouched: the next full pass reads all of them
                Prof p(g, s, MST_K_FILTER, r, MST_SUB_MEMBER);
                CK(launch_member_min(s, g->nsm, (u32)n, nullptr, g->phi, g->row, g->rrow, g->ridx,
                                     g->arcs0, g->vlo, g->vhi, g->wbase,
                                     g->sim ? g->shard_best : bnxt, g->kfmt));
                for (int j = 0; j < G; ++j) {
                    g->hcnt[arec(j, r + 1)] = (u32)(g->shards[j].hi - g->shards[j].lo);
                    CK(cudaMemcpyAsync(g->dcnt + arec(j, r + 1), g->hcnt + arec(j, r + 1),
                                       sizeof(u32), cudaMemcpyHostToDevice, s));
                }
                g->st.member_ends[r] = (int64_t)mwork;
                g->st.member_round[r] = 1;
                last_member_r = r;
                last_member_w = mwork;
            }
            for (int j = 0; j < G && !member; ++j) {
                Shard& sh = g->shards[j];
                u64* tgt = g->sim ? g->shard_best + (u64)j * n : bnxt;
                Prof p(g, s, MST_K_FILTER, r,
                       to_dense ? MST_SUB_TRANSITION
                       : cur_light ? MST_SUB_LIGHT
                       : (r == g->st.light_switch_round ? MST_SUB_SWITCH : MST_SUB_SPARSE), j);
                uint4* out = (never || to_dense) ? nullptr : const_cast<uint4*>(outbuf) + sh.lo;
                CompactCtl ccj = cc;
                if (adaptive && j == dsh) {
                    ccj.hword = g->dmap + HSURV + r;
                    ccj.tag = tag_base | (u32)r;
                }
                // (a light window holds <= the shard's records + its filler)
                const u64 amax = (sh.hi - sh.lo) + (cur_light ? (u64)pass_warps(g->nsm) * LBLK_MAX : 0);
                CK(launch_filter_min(s, g->nsm, g->dcnt + arec(j, r), amax, cur + off(sh),
                                     Mpass, out, tgt, nn, g->status, g->epoch++,
                                     g->dcnt + arec(j, r + 1), g->dcnt + C_TILE, g->pass_seq,
                                     to_dense ? g->mat[0] : nullptr, ccj,
                                     (to_dense && use_hub_row(g) && hub_ok)
                                         ? (const int*)g->dcnt + C_HUB + r + 1 : nullptr,
                                     g->kfmt, g->adj_dedup));
            }
            if (to_dense && use_hub_row(g) && hub_ok) g->st.hub_row = 1;
            if (member) {
                // (nothing compacted: the records stay in vertex ids, read through Ψ)
            } else if (adaptive) {
                pend = r;
                pend_out = outbuf;
            } else if (!never && !to_dense) {
                if (dedup) {  // A9: sort the survivors by component pair, keep each pair's minimum
                    u32 acnt = 0;
                    CK(cudaMemcpyAsync(&acnt, g->dcnt + arec(0, r + 1), sizeof(u32),
                                       cudaMemcpyDeviceToHost, s));
                    CK(cudaStreamSynchronize(s));
                    g->st.dedup_in[r] = acnt;
                    Prof p(g, s, MST_K_DEDUP, r);
                    CK(launch_dedup(s, g->nsm, acnt, nn, g->dcnt + arec(0, r + 1),
                                    const_cast<uint4*>(outbuf) + g->shards[0].lo, g->dd_scratch,
                                    g->dd_bytes, g->dd_runs));
                }
                cur = outbuf;
                cur_light = false;
                brnd = r + 1;
                nb_sz = nn;
                g->st.compacted_mask |= 1ll << r;
            }
        }
        chain.m[chain.len++] = Mr;
        moff += nr;
        ++r;
        if (to_dense) {
            // the transition pass filled only the matrix: every rank needs all of it for the
            // replicated dense rounds, and the first dense round's minima come from it
            if (dist) {
                Prof p(g, s, MST_K_COMM, r);
                CKS(xchg_min(g, s, g->mat[0], dense_entries(nn), false));
            }
            Prof p(g, s, MST_K_DENSE, r, MST_SUB_DENSE_BEST);
            CK(launch_dense_best(s, g->nsm, nn, g->mat[0], bnxt));
        } else if (g->sim && !dense) {
            Prof p(g, s, MST_K_COMM, r);
            CK(launch_combine_min(s, g->nsm, nn, G, g->shard_best, n, bnxt));
        } else if (dist && !dense) {
            Prof p(g, s, MST_K_COMM, r);
            CKS(xchg_min(g, s, bnxt, nn, false));
        }
        if (to_dense) {
            dense = true;
            mc = 0;
            g->st.dense_round = r;
        } else if (dense) {
            mc ^= 1;
        }
        std::swap(bcur, bnxt);
        nr = nn;
    }
    if (tail_r0 >= 0)
        CK(cudaMemcpyAsync(g->hcnt + C_TAIL, g->dcnt + C_TAIL, (1 + MST_MAX_ROUNDS) * sizeof(u32),
                           cudaMemcpyDeviceToHost, s));
    g->st.rounds = r;
    // per-round alive records (device-side counters, fetched once per run for the stats)
    CK(cudaMemcpyAsync(g->hcnt + C_AREC, g->dcnt + C_AREC, (size_t)G * AREC_STRIDE * sizeof(u32),
                       cudaMemcpyDeviceToHost, s));
    // ---- A11 output
    {
        Prof p(g, s, MST_K_OUTPUT, r);
        if (g->nwords) {
            CK(launch_output(s, (u32)g->nwords, g->msf, out_ids, g->tcnt, g->dcnt + C_OUT,
                             (u32)std::max<int64_t>(n - 1, 1)));
        } else {
            CK(cudaMemsetAsync(g->dcnt + C_OUT, 0, sizeof(u32), s));
        }
    }
    CK(cudaMemcpyAsync(g->hcnt, g->dcnt, 2 * sizeof(u32), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(g->hacc, g->acc, 2 * ACC_SLOTS * sizeof(u64), cudaMemcpyDeviceToHost, s));
    if (phase) CK(cudaMemcpyAsync(g->hcnt + C_LT, g->dcnt + C_LT, sizeof(u32), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (phase) g->st.light_t = g->hcnt[C_LT];
    if (pend >= 0) {  // the last sampled decision (stats only)
        u32 word;
        CKS(wait_word(g, s, HSURV + pend, tag_base | (u32)pend, &word));
        resolve(word);
    }
    if (singletons) g->st.member_ends[0] = (int64_t)g->hscr[1];
    for (int i = 1; i < ACC_SLOTS; ++i) {  // sum the spread accumulators
        g->hacc[0] += g->hacc[2 * i];
        g->hacc[1] += g->hacc[2 * i + 1];
    }
    if (tail_r0 >= 0) {  // rounds run by the device tail
        const u32 k = g->hcnt[C_TAIL];
        for (u32 i = 0; i < k && tail_r0 + (int)i < MST_MAX_ROUNDS; ++i) {
            g->st.n_r[tail_r0 + i] = g->hcnt[C_TAIL + 1 + i];
            g->st.a_r[tail_r0 + i] = (int64_t)dense_entries(g->hcnt[C_TAIL + 1 + i]);
        }
        r = tail_r0 + (int)k;
        g->st.rounds = r;
    }
    for (int rr = 0; rr < r; ++rr) {
        if (g->st.a_r[rr] >= 0) continue;
        int64_t a = 0;
        for (int j = 0; j < G; ++j) a += g->hcnt[arec(j, rr)];
        g->st.a_r[rr] = a;
    }
    if ((u64)g->hcnt[C_OUT] != g->hacc[1])
        return fail(MST_EINTERNAL, "forest size mismatch: %u ids vs %llu hooks", g->hcnt[C_OUT],
                    (unsigned long long)g->hacc[1]);
    if (g->hacc[1] >= n) return fail(MST_EINTERNAL, "forest has >= n edges");
    *out_num = (int64_t)g->hacc[1];
    *out_total = g->hacc[0];
    g->st.num_edges = *out_num;
    g->st.total_weight = *out_total;
    collect_profile(g);
    g->st.gpu_launches = (int64_t)(kernel_launches() - kl0);
    return MST_OK;
}

template <typename F>
mst_status guarded(F&& f) {
    try {
        return f();
    } catch (const std::bad_alloc&) {
        return fail(MST_ENOMEM, "host allocation failed");
    } catch (...) {
        return fail(MST_EINTERNAL, "unexpected C++ exception");
    }
}

}  // namespace

// =========================================================================== C ABI
extern "C" {

const char* mst_version(void) { return "mst-b200 0.1 sm_100a"; }

const char* mst_last_error(void) { return g_err.c_str(); }

mst_status mst_create(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                      const uint32_t* w, mst_graph** out) {
    return guarded([&] { return create_common(n, m, src, dst, w, 1, nullptr, 0, 1, out); });
}

mst_status mst_create_sim(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                          const uint32_t* w, int nshards, mst_graph** out) {
    return guarded([&] { return create_common(n, m, src, dst, w, nshards, nullptr, 0, 1, out); });
}

mst_status mst_get_unique_id(uint8_t id[128]) {
    return guarded([&]() -> mst_status {
        if (!id) return fail(MST_EINVAL, "id is NULL");
        ncclUniqueId uid;
        CKN(ncclGetUniqueId(&uid));
        static_assert(sizeof(uid) == 128, "ncclUniqueId is 128 bytes");
        memcpy(id, &uid, 128);
        return MST_OK;
    });
}

mst_status mst_create_dist(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                           const uint32_t* w, const uint8_t id[128], int rank, int nranks,
                           mst_graph** out) {
    return guarded([&]() -> mst_status {
        if (nranks > 1 && !id) return fail(MST_EINVAL, "id is NULL");
        return create_common(n, m, src, dst, w, 1, id, rank, nranks, out);
    });
}

mst_status mst_create_dist_hostx(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                                 const uint32_t* w, int rank, int nranks,
                                 mst_allreduce_min_fn fn, void* ctx, mst_graph** out) {
    return guarded([&]() -> mst_status {
        if (!fn) return fail(MST_EINVAL, "exchange callback is NULL");
        return create_common(n, m, src, dst, w, 1, nullptr, rank, nranks, out, true, fn, ctx);
    });
}

// Host-array input. Pinned (page-locked) arrays are device-addressable under UVA: the build
// kernels then read them straight over PCIe (zero-copy), so the transfer overlaps the
// validation/degree and scatter passes instead of preceding them. Pageable arrays are staged
// through a device copy first.
static const void* device_alias(const void* p) {
    cudaPointerAttributes a;
    if (!p || cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        (void)cudaGetLastError();
        return nullptr;
    }
    if (a.type == cudaMemoryTypeHost && a.devicePointer) return a.devicePointer;
    if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) return p;
    return nullptr;
}

static mst_status create_host_impl(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                                   const uint32_t* w, mst_graph** out, int reorder) {
    if (!out) return fail(MST_EINVAL, "out is NULL");
    *out = nullptr;
    CKS(check_args(n, m, src, dst, w));
    int dev;
    CK(cudaGetDevice(&dev));
    CKS(configure_pool(dev));
    // (pinned host arrays are copied by DMA too: the build kernels reading them in place over
    // the bus reached ~34 GB/s — measured 15.8 + 5.3 ms for RMAT-22's 805 MB — the copy
    // engines ~55 GB/s)
    static const char* zc = getenv("MST_HOST_ZEROCOPY");  // "1": read pinned inputs in place
    if (m > 0 && zc && zc[0] == '1') {
        const void *as = device_alias(src), *ad = device_alias(dst), *aw = device_alias(w);
        if (as && ad && aw)
            return create_common(n, m, (const int32_t*)as, (const int32_t*)ad,
                                 (const uint32_t*)aw, 1, nullptr, 0, 1, out, reorder);
    }
    cudaStream_t st;
    CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    void *ds = nullptr, *dd = nullptr, *dw = nullptr;
    const size_t b = std::max<size_t>((size_t)m * 4, 16);
    cudaError_t e = cudaMallocAsync(&ds, b, st);
    if (e == cudaSuccess) e = cudaMallocAsync(&dd, b, st);
    if (e == cudaSuccess) e = cudaMallocAsync(&dw, b, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);  // (the staging exists before the build)
    // streamed build (HostIn): the copies overlap the degree pass, layout and scatter;
    // MST_HOST_STREAM=0: copy everything first, then build
    static const char* hsv = getenv("MST_HOST_STREAM");
    const bool stream_in = !(hsv && hsv[0] == '0') && m > 0;
    // (MST_HOST_CHUNK: edges per chunk, read per call — tests cover many small chunks)
    const char* hcv = getenv("MST_HOST_CHUNK");
    const u64 hchunk = hcv && atoll(hcv) > 0 ? (u64)atoll(hcv) : (u64)8 << 20;
    HostIn hin{src, dst, w, st, hchunk, {}};
    if (e == cudaSuccess && stream_in) {
        const u64 nch = ((u64)m + hin.chunk - 1) / hin.chunk;
        for (u64 k = 0; k < 2 * nch && e == cudaSuccess; ++k) {
            cudaEvent_t ev;
            e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
            if (e == cudaSuccess) hin.evs.push_back(ev);
        }
    } else if (e == cudaSuccess && m > 0) {
        e = cudaMemcpyAsync(ds, src, (size_t)m * 4, cudaMemcpyHostToDevice, st);
        if (e == cudaSuccess) e = cudaMemcpyAsync(dd, dst, (size_t)m * 4, cudaMemcpyHostToDevice, st);
        if (e == cudaSuccess) e = cudaMemcpyAsync(dw, w, (size_t)m * 4, cudaMemcpyHostToDevice, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    }
    mst_status s = MST_OK;
    if (e != cudaSuccess)
        s = fail(e == cudaErrorMemoryAllocation ? MST_ENOMEM : MST_ECUDA, "host->device input copy: %s",
                 cudaGetErrorString(e));
    else
        s = create_common(n, m, (const int32_t*)ds, (const int32_t*)dd, (const uint32_t*)dw, 1,
                          nullptr, 0, 1, out, reorder, nullptr, nullptr, stream_in ? &hin : nullptr);
    cudaStreamSynchronize(st);  // (copies still queued after a failed build finish first)
    if (ds) cudaFreeAsync(ds, st);
    if (dd) cudaFreeAsync(dd, st);
    if (dw) cudaFreeAsync(dw, st);
    cudaStreamSynchronize(st);
    for (cudaEvent_t ev : hin.evs) cudaEventDestroy(ev);
    cudaStreamDestroy(st);
    return s;
}

mst_status mst_create_host(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                           const uint32_t* w, mst_graph** out) {
    return guarded([&]() { return create_host_impl(n, m, src, dst, w, out, 1); });
}

mst_status mst_run(mst_graph* g, mst_stream_t stream, int32_t* out_edge_ids,
                   int64_t* out_num_edges, uint64_t* out_total_weight) {
    return guarded([&]() -> mst_status {
        if (!g) return fail(MST_EINVAL, "handle is NULL");
        if (g->broken) return fail(MST_EINVAL, "handle is unusable after an earlier error");
        if (!out_num_edges || !out_total_weight) return fail(MST_EINVAL, "null output pointer");
        if (!out_edge_ids && g->n > 1) return fail(MST_EINVAL, "out_edge_ids is NULL");
        NvtxRange range("mst_run", (int)std::min<int64_t>(g->n, INT32_MAX));
        mst_status s = run_impl(g, (cudaStream_t)stream, out_edge_ids, out_num_edges, out_total_weight);
        if (s != MST_OK) {
            g->broken = true;
            // kernels of the failed run may still be queued or running on `stream`: the
            // handle's frees are ordered after them (release waits on this event)
            (void)cudaGetLastError();
            if (!g->fail_ev && cudaEventCreateWithFlags(&g->fail_ev, cudaEventDisableTiming) != cudaSuccess)
                g->fail_ev = nullptr;
            if (g->fail_ev) cudaEventRecord(g->fail_ev, (cudaStream_t)stream);
            (void)cudaGetLastError();
        }
        return s;
    });
}

mst_status mst_run_host(mst_graph* g, mst_stream_t stream, int32_t* out_ids_host,
                        int64_t* out_num_edges, uint64_t* out_total_weight) {
    return guarded([&]() -> mst_status {
        if (!g) return fail(MST_EINVAL, "handle is NULL");
        if (!out_ids_host && g->n > 1) return fail(MST_EINVAL, "out_edge_ids_host is NULL");
        if (!g->out_tmp) CKS(galloc(g, &g->out_tmp, std::max<int64_t>(g->n - 1, 1)));
        CK(cudaStreamSynchronize(g->cst));
        CKS(mst_run(g, stream, g->out_tmp, out_num_edges, out_total_weight));
        if (*out_num_edges > 0) {
            CK(cudaMemcpyAsync(out_ids_host, g->out_tmp, (size_t)*out_num_edges * sizeof(int32_t),
                               cudaMemcpyDeviceToHost, (cudaStream_t)stream));
            CK(cudaStreamSynchronize((cudaStream_t)stream));
        }
        return MST_OK;
    });
}

mst_status mst_solve_host(int64_t n, int64_t m, const int32_t* src, const int32_t* dst,
                          const uint32_t* w, int32_t* out_ids_host, int64_t* out_num_edges,
                          uint64_t* out_total_weight) {
    mst_graph* g = nullptr;
    // one-shot: the automatic layout too (hub-first costs ~1 ms of build and saves RMAT-22's
    // member scans ~8 ms of run; MST_SOLVE_REORDER=0: the caller's numbering)
    static const char* sr = getenv("MST_SOLVE_REORDER");
    const int reorder = (sr && sr[0] == '0') ? 0 : 2;
    mst_status s = guarded([&]() { return create_host_impl(n, m, src, dst, w, &g, reorder); });
    if (s != MST_OK) return s;
    s = mst_run_host(g, g->cst, out_ids_host, out_num_edges, out_total_weight);
    std::string keep = g_err;
    mst_destroy(g);
    g_err = keep;
    return s;
}

void mst_destroy(mst_graph* g) { release(g); }

mst_status mst_get_stats(const mst_graph* g, mst_stats* out) {
    if (!g || !out) return fail(MST_EINVAL, "null argument");
    *out = g->st;
    return MST_OK;
}

mst_status mst_set_option(mst_graph* g, int option, int64_t value) {
    return guarded([&]() -> mst_status {
        if (!g) return fail(MST_EINVAL, "handle is NULL");
        if (option == MST_OPT_COMPACT_TAU) {
            if (value < 0 || value > 1000)
                return fail(MST_EINVAL, "MST_OPT_COMPACT_TAU must be in [0, 1000] (permille)");
            g->tau = (u32)value;
            return MST_OK;
        }
        if (option == MST_OPT_LIGHT_FIRST) {
            if (value < -1 || value > 64)
                return fail(MST_EINVAL, "MST_OPT_LIGHT_FIRST must be -1 (auto) or in [0, 64]");
            g->light_k = (int)value;
            return MST_OK;
        }
        if (value != 0 && value != 1) return fail(MST_EINVAL, "option value must be 0 or 1");
        if (option == MST_OPT_DENSE) {
            g->opt_dense = value != 0;
        } else if (option == MST_OPT_DEVICE_TAIL) {
            g->opt_tail = value != 0;
        } else if (option == MST_OPT_KEEP_EDGES) {
            g->opt_keep = value != 0;
        } else if (option == MST_OPT_UNION_FIND) {
            g->opt_uf = value != 0;
        } else if (option == MST_OPT_SMALL) {
            g->opt_small = value != 0;
        } else if (option == MST_OPT_DEDUP) {
            g->opt_dedup = value != 0;
            if (g->opt_dedup && !g->dd_scratch) {  // (allocated here: mst_run allocates nothing)
                const u64 A = std::max<u64>(g->A0_local, 1);
                g->dd_bytes = dedup_scratch_bytes(A);
                CKS(galloc(g, reinterpret_cast<unsigned char**>(&g->dd_scratch), g->dd_bytes));
                CKS(galloc(g, &g->dd_runs, 2));
                CK(cudaStreamSynchronize(g->cst));
            }
        } else {
            return fail(MST_EINVAL, "unknown option %d", option);
        }
        return MST_OK;
    });
}

mst_status mst_get_launch_times(const mst_graph* g, mst_launch_time* out, int64_t cap,
                                int64_t* count) {
    if (!g || !count || cap < 0 || (cap > 0 && !out)) return fail(MST_EINVAL, "bad argument");
    const int64_t k = (int64_t)g->ltimes.size();
    *count = k;
    for (int64_t i = 0; i < std::min(k, cap); ++i) out[i] = g->ltimes[i];
    return MST_OK;
}

mst_status mst_set_profiling(mst_graph* g, int enable) {
    if (!g) return fail(MST_EINVAL, "handle is NULL");
    g->prof = enable != 0;
    return MST_OK;
}

mst_status mst_debug_filter_pass(mst_graph* g, mst_stream_t stream, int map_kind, int64_t group,
                                 int iters, double* out_ms, int64_t* out_survivors) {
    return guarded([&]() -> mst_status {
        if (!g || !out_ms || iters < 1 || g->n == 0 || g->shards.empty())
            return fail(MST_EINVAL, "bad argument");
        if (group < 1) group = 1;
        cudaStream_t s = (cudaStream_t)stream;
        const u64 n = g->n;
        u32 ncomp = 0;
        CK(launch_debug_map(s, (u32)n, map_kind, (u32)group, g->maps, &ncomp));
        const Shard& sh = g->shards[0];
        const u32 A = (u32)(sh.hi - sh.lo);
        cudaEvent_t e0, e1;
        CK(cudaEventCreate(&e0));
        CK(cudaEventCreate(&e1));
        for (int it = -1; it < iters; ++it) {
            if (it == 0) CK(cudaEventRecord(e0, s));
            CK(cudaMemsetAsync(g->bestB, 0xff, n * sizeof(u64), s));
            CK(launch_filter_min(s, g->nsm, nullptr, A, g->arcs0 + sh.lo, g->maps,
                                 g->abuf[0] + sh.lo, g->bestB, ncomp, g->status, g->epoch++,
                                 g->dcnt + arec(0, 1), g->dcnt + C_TILE, g->pass_seq, nullptr));
        }
        CK(cudaEventRecord(e1, s));
        CK(cudaEventSynchronize(e1));
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        cudaEventDestroy(e0);
        cudaEventDestroy(e1);
        u32 surv = 0;
        CK(cudaMemcpy(&surv, g->dcnt + arec(0, 1), sizeof(u32), cudaMemcpyDeviceToHost));
        *out_ms = ms / iters;
        if (out_survivors) *out_survivors = surv;
        return MST_OK;
    });
}

mst_status mst_shard_ranges(const uint32_t* row_offsets, int64_t n, int nranks, int64_t* lo,
                            int64_t* hi) {
    return guarded([&]() -> mst_status {
        if (!row_offsets || !lo || !hi || n < 0 || nranks < 1 || nranks > 64)
            return fail(MST_EINVAL, "bad argument");
        std::vector<u64> l(nranks), h(nranks);
        compute_shard_ranges(row_offsets, (u64)n, nranks, l.data(), h.data());
        for (int j = 0; j < nranks; ++j) {
            lo[j] = (int64_t)l[j];
            hi[j] = (int64_t)h[j];
        }
        return MST_OK;
    });
}

}  // extern "C"
