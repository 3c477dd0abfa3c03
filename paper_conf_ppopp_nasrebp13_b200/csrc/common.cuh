// common.cuh — device helpers shared by the MST kernels (sm_100a).
//
// Nothing here is MST arithmetic; it is the plumbing the kernels share: cache-hinted
// loads/stores, warp segmented minimum, and the decoupled look-back tile-status protocol
// used for every single-pass stream compaction / scan (rows A0, A4/A6, A8, A11 of
// SURVEY.md §8(a); the paper's "explicit deletion" of PAPER.md §7.2 L273 done as a
// single-pass scan instead of a global re-layout).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace mstk {

typedef uint32_t u32;
typedef uint64_t u64;

constexpr u64 KEY_INF = ~0ull;          // "no edge" (SURVEY.md §8 notation: ∞ = UINT64_MAX)
// "not looked at this round" (the member-scan rounds defer the component of the top hub): no
// real key takes this value (packed keys use < 64 bits; (w << 32 | eid) has eid < 2^31)
constexpr u64 KEY_DEFER = ~1ull;
constexpr u32 FULL = 0xffffffffu;

// ------------------------------------------------------------------ memory access
// L2 eviction-priority policies (createpolicy): the arc streams are read once and marked
// evict-first so the small, hot label maps (evict-last) stay resident in the 126 MB L2.
__device__ __forceinline__ u64 pol_evict_first() {
    u64 p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ u64 pol_evict_last() {
    u64 p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// Streamed once: no L1 allocation, L2 evict-first.
__device__ __forceinline__ u32 ld_stream_u32(const u32* p, u64 pol) {
    u32 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;"
                 : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ u64 ld_stream_u64(const u64* p, u64 pol) {
    u64 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;"
                 : "=l"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ void st_stream_u32(u32* p, u32 v, u64 pol) {
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.u32 [%0], %1, %2;"
                 :: "l"(p), "r"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_stream_u64(u64* p, u64 v, u64 pol) {
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.u64 [%0], %1, %2;"
                 :: "l"(p), "l"(v), "l"(pol) : "memory");
}
// One arc record = 16 B {s, d, eid, w}: one LDG.128 / STG.128 per arc, coalesced.
__device__ __forceinline__ uint4 ld_arc(const uint4* p, u64 pol) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ void st_arc(uint4* p, uint4 v, u64 pol) {
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.u32 [%0], {%1,%2,%3,%4}, %5;"
                 :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "l"(pol) : "memory");
}
// Gathers from the label maps: read-only in-kernel, keep in L2 (evict-last).
__device__ __forceinline__ int ld_map(const int* p, u64 pol) {
    int v;
    asm volatile("ld.global.nc.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
// Coherent (L2) read of a word other CTAs may be updating in this kernel.
__device__ __forceinline__ u64 ld_relaxed_u64(const u64* p) {
    u64 v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_u64(u64* p, u64 v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ u32 ld_relaxed_u32(const u32* p) {
    u32 v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
// Plain (weak, L1-cacheable) load of a word other threads may update in this kernel: only
// for monotone data where a stale value is still correct (pointer-jumping ancestors).
__device__ __forceinline__ u32 ld_weak_u32(const u32* p) {
    u32 v;
    asm volatile("ld.global.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ void st_relaxed_u32(u32* p, u32 v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}

// Monotone minimum with a stale-read pre-check: values only ever decrease, so any earlier
// (stale) value is >= the current one and a key that does not beat it cannot win; this
// keeps losing candidates off the L2 atomic units. Returns true if the atomic was issued.
__device__ __forceinline__ bool min_update(u64* p, u64 key) {
    u64 cur = __ldcg(p);
    if (key < cur) {
        atomicMin(reinterpret_cast<unsigned long long*>(p), (unsigned long long)key);
        return true;
    }
    return false;
}

// Fire-and-forget minimum (RED, no return value, no pre-check load on the critical path).
__device__ __forceinline__ void red_min_global(u64* p, u64 key) {
    asm volatile("red.relaxed.gpu.global.min.u64 [%0], %1;" :: "l"(p), "l"(key) : "memory");
}
// (No native 64-bit shared min on sm_100a: this lowers to ATOMS.CAST.SPIN.64, measured faster
// than an explicit read-then-CAS loop.)
__device__ __forceinline__ void red_min_shared(u64* p, u64 key) {
    asm volatile("red.shared.min.u64 [%0], %1;" :: "r"((u32)__cvta_generic_to_shared(p)), "l"(key)
                 : "memory");
}
// the same on a 32-bit shared-window address (no generic -> shared conversion per call)
__device__ __forceinline__ void red_min_shared_a(u32 addr, u64 key) {
    asm volatile("red.shared.min.u64 [%0], %1;" :: "r"(addr), "l"(key) : "memory");
}

__device__ __forceinline__ u32 lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ u32 lanemask_lt() {
    u32 r;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
    return r;
}

__device__ __forceinline__ u64 shfl_up_u64(u64 v, int off) {
    return __shfl_up_sync(FULL, v, off);
}

// Inclusive segmented minimum over contiguous runs of a warp. `heads` is the ballot of
// run-head flags (bit 0 must be set). After the call a run's TAIL lane holds the min over
// its whole run; every lane holds the min over [its run head .. itself].
__device__ __forceinline__ u64 warp_seg_min(u64 v, u32 heads, u32 lane) {
    const u32 below = heads & (FULL >> (31 - lane));
    const int head = 31 - __clz(below);
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        u64 o = shfl_up_u64(v, off);
        if ((int)lane - off >= head) v = o < v ? o : v;
    }
    return v;
}

// Minimum key of my run of equal `s` among the 32 lanes (contiguous runs), computed with
// two redux.sync over the run's lane mask: first the weight (hi word), then the edge id (lo
// word) among the lanes holding that weight. Invalid lanes contribute (~0, ~0) = inf.
// Returns the run min in (mh, ml) on every lane of the run and the run's first/last lane.
__device__ __forceinline__ void run_min(u32 s, u32 hi, u32 lo, bool valid, u32 lane,
                                        u32& mh, u32& ml, u32& head, u32& tail) {
    const u32 ps = __shfl_up_sync(FULL, s, 1);
    const u32 heads = __ballot_sync(FULL, lane == 0 || ps != s);
    const u32 le = FULL >> (31 - lane);
    head = 31 - __clz(heads & le);
    const u32 above = heads & ~le;
    tail = above ? (u32)(__ffs(above) - 2) : 31u;
    const u32 mask = (FULL >> (31 - tail)) & (FULL << head);
    const u32 v1 = valid ? hi : FULL;
    mh = __reduce_min_sync(mask, v1);
    const u32 v2 = (valid && hi == mh) ? lo : FULL;
    ml = __reduce_min_sync(mask, v2);
}

// Warp-level duplicate collapse before an L2 min: lanes holding the same `cell` are grouped
// with match.any, their keys are min-reduced through a per-warp shared scratch (32 x u64),
// and only each group's leader issues the RED. Turns W identical-cell REDs into one.
__device__ __forceinline__ void warp_dedup_red_min(u64* __restrict__ gbase, u32 cell, u64 key,
                                                   bool active, u64* wslot, u32 lane) {
    const u32 peers = __match_any_sync(FULL, active ? cell : 0xffffffffu);
    const u32 leader = __ffs(peers) - 1;
    if (lane == leader) wslot[lane] = KEY_INF;
    __syncwarp();
    if (active) red_min_shared(wslot + leader, key);
    __syncwarp();
    if (active && lane == leader) red_min_global(gbase + cell, wslot[lane]);
    __syncwarp();
}

// tails of contiguous runs given their heads: lane l is a tail iff l == 31 or l+1 is a head
__device__ __forceinline__ u32 run_tails(u32 heads) { return (heads >> 1) | 0x80000000u; }

// ------------------------------------------------------------------ TMA bulk copy + mbarrier
// The producer warp streams arc tiles global -> shared with cp.async.bulk (SASS UBLKCP),
// completion tracked by mbarrier transaction counts; consumers wait on the barrier's phase.
__device__ __forceinline__ u32 smem_addr(const void* p) {
    return (u32)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(u64* bar, u32 count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(u64* bar, u32 bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;"
                 :: "r"(smem_addr(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(u64* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_addr(bar)) : "memory");
}
// MST_WAIT_HINT > 0: try_wait with a suspend-time hint (ns): a waiting warp sleeps until the
// phase completes (or the hint expires) instead of spinning on issue slots the working warps
// need (the passes issue on ~68 % of cycles; polling was ~15 % of MIN0's instructions)
// (measured on RMAT-22: 20 us hint -> switch pass 371 -> 356 us, round-0 pass 391 -> 387 us;
// uniform / road / dense neutral; 1 ms the same)
#ifndef MST_WAIT_HINT
#define MST_WAIT_HINT 20000
#endif
__device__ __forceinline__ void mbar_wait(u64* bar, u32 parity) {
    const u32 a = smem_addr(bar);
#if MST_WAIT_HINT > 0
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" :: "r"(a), "r"(parity), "r"((u32)MST_WAIT_HINT) : "memory");
#else
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" :: "r"(a), "r"(parity) : "memory");
#endif
}
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, u32 bytes, u64* bar,
                                            u64 pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1], %2, [%3], %4;"
        :: "r"(smem_addr(dst)), "l"(src), "r"(bytes), "r"(smem_addr(bar)), "l"(pol) : "memory");
}
// TMA bulk store shared -> global (survivor tiles); bulk-group completion tracking.
__device__ __forceinline__ void tma_store_1d(void* dst, const void* src, u32 bytes, u64 pol) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;"
                 :: "l"(dst), "r"(smem_addr(src)), "r"(bytes), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_commit() {
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read0() {
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait0() {
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
// generic-proxy shared-memory writes -> visible to the async proxy (TMA store)
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void named_arrive(u32 id, u32 nthreads) {
    asm volatile("bar.arrive %0, %1;" :: "r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ void sts_arc(uint4* p, uint4 v) {
    asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};"
                 :: "r"(smem_addr(p)), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
// named barrier among the consumer warps only (the producer warp never joins)
__device__ __forceinline__ void named_sync(u32 id, u32 nthreads) {
    asm volatile("bar.sync %0, %1;" :: "r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ uint4 lds_arc(const uint4* p) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(smem_addr(p)));
    return v;
}

// ------------------------------------------------------------------ decoupled look-back
// Tile status word: [63:62] flag (0 = not ready, 1 = aggregate, 2 = inclusive prefix),
// [61:32] epoch (30 bits, unique per launch so the status array is never cleared),
// [31:0] value (counts < 2^32: arcs A_r <= 2m <= 2^32-2).
constexpr u32 ST_AGG = 1, ST_PRE = 2;

__device__ __forceinline__ u64 st_pack(u32 flag, u32 epoch, u32 value) {
    return ((u64)flag << 62) | ((u64)(epoch & 0x3fffffffu) << 32) | (u64)value;
}

__device__ __forceinline__ void publish(u64* status, u32 tile, u32 flag, u32 epoch, u32 value) {
    st_relaxed_u64(status + tile, st_pack(flag, epoch, value));
}

// Called by ONE full warp: returns the exclusive prefix of `tile` (sum of the values of all
// tiles < tile). Deadlock-free when tiles are dispatched in increasing order (one CTA per
// tile in blockIdx order, or a co-resident persistent grid walking tiles in order).
__device__ __forceinline__ u32 lookback(const u64* status, u32 tile, u32 epoch) {
    const u32 lane = lane_id();
    const u32 ep = epoch & 0x3fffffffu;
    u32 excl = 0;
    long long base = (long long)tile - 32;
    while (true) {
        long long idx = base + lane;
        u32 flag, val;
        if (idx >= 0) {
            u64 s;
            do {
                s = ld_relaxed_u64(status + idx);
                flag = (u32)(s >> 62);
                if ((u32)((s >> 32) & 0x3fffffffu) != ep) flag = 0;
            } while (flag == 0);
            val = (u32)s;
        } else {
            flag = ST_PRE;  // virtual tiles before 0: prefix 0
            val = 0;
        }
        const u32 pmask = __ballot_sync(FULL, flag == ST_PRE);
        if (pmask) {
            const u32 hi = 31 - __clz(pmask);
            excl += __reduce_add_sync(FULL, lane >= hi ? val : 0u);
            return excl;
        }
        excl += __reduce_add_sync(FULL, val);
        base -= 32;
    }
}

}  // namespace mstk
