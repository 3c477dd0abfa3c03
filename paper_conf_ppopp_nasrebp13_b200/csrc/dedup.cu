// dedup.cu — row A9's optional supervertex re-CSR / duplicate collapse by a sort (SURVEY.md
// §8(a) A9; §5: Boruvka codes "switch algorithms as the graph becomes dense").
//
// After a compacting pass the surviving records {s', d', key base} are sorted by their
// component pair (lo, hi) = (min(s', d'), max(s', d')) and every run of equal pairs keeps its
// minimum key: parallel records between two components can never be a component minimum
// except the smallest one (reading R13; SURVEY.md §8(c) "dedup may drop arcs"), and the records
// come out grouped by their lower label (long owner runs for the next pass). The sort and the
// run reduction are CUB's device radix sort and reduce-by-key (library primitives, like a
// cuBLAS GEMM); the record <-> (pair, key) conversions are ours. MST_OPT_DEDUP; measured in
// DESIGN.md §5c.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_reduce.cuh>

#include "common.cuh"
#include "kernels.h"

namespace mstk {

namespace {
// pair key (lo << b) | hi over 2b bits (b = bits of the label count); dead records take the
// all-ones key (lo == hi == 2^b - 1 never occurs for a live record): they sort last
__global__ void k_rec_to_pairs(u32 A, const uint4* __restrict__ rec, u32 b, u64* __restrict__ pk,
                               u64* __restrict__ kv) {
    const u64 dead = (b >= 32) ? ~0ull : ((1ull << (2 * b)) - 1);
    for (u32 i = blockIdx.x * blockDim.x + threadIdx.x; i < A; i += gridDim.x * blockDim.x) {
        const uint4 a = rec[i];
        if (a.x == FULL || a.x == a.y) {
            pk[i] = dead;
            kv[i] = KEY_INF;
            continue;
        }
        const u32 lo = min(a.x, a.y), hi = max(a.x, a.y);
        pk[i] = ((u64)lo << b) | hi;
        kv[i] = ((u64)a.z << 32) | a.w;
    }
}
struct MinOp {
    __device__ __forceinline__ u64 operator()(const u64& x, const u64& y) const { return x < y ? x : y; }
};
__global__ void k_pairs_to_rec(const int* __restrict__ nruns, const u64* __restrict__ pk,
                               const u64* __restrict__ kv, u32 b, uint4* __restrict__ rec,
                               u32* __restrict__ a_out) {
    const u64 dead = (b >= 32) ? ~0ull : ((1ull << (2 * b)) - 1);
    const u32 R = (u32)*nruns;
    const u32 K = (R > 0 && pk[R - 1] == dead) ? R - 1 : R;  // (drop the dead run)
    __syncthreads();
    if (blockIdx.x == 0 && threadIdx.x == 0) *a_out = K;
    const u64 hm = (b >= 32) ? ~0ull : ((1ull << b) - 1);
    for (u32 i = blockIdx.x * blockDim.x + threadIdx.x; i < K; i += gridDim.x * blockDim.x) {
        const u64 p = pk[i], k = kv[i];
        rec[i] = make_uint4((u32)(p >> b), (u32)(p & hm), (u32)(k >> 32), (u32)k);
    }
}
u32 bits_needed(u64 x) { u32 b = 0; while (x) { ++b; x >>= 1; } return b; }
}  // namespace

size_t dedup_scratch_bytes(u64 A) {
    size_t t1 = 0, t2 = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, t1, (u64*)nullptr, (u64*)nullptr, (u64*)nullptr,
                                    (u64*)nullptr, (int)std::max<u64>(A, 1));
    cub::DeviceReduce::ReduceByKey(nullptr, t2, (u64*)nullptr, (u64*)nullptr, (u64*)nullptr,
                                   (u64*)nullptr, (int*)nullptr, MinOp(), (int)std::max<u64>(A, 1));
    return 4 * A * sizeof(u64) + std::max(t1, t2) + 256;
}

cudaError_t launch_dedup(cudaStream_t st, int nsm, u64 A, u32 nlab, u32* a_count, uint4* rec,
                         void* scratch, size_t scratch_bytes, int* nruns) {
    if (A == 0) return cudaSuccess;
    const u32 b = std::max<u32>(1, bits_needed(nlab));
    u64* pk0 = reinterpret_cast<u64*>(scratch);
    u64* pk1 = pk0 + A;
    u64* kv0 = pk1 + A;
    u64* kv1 = kv0 + A;
    void* tmp = kv1 + A;
    size_t tb = scratch_bytes - 4 * A * sizeof(u64);
    const u32 grid = std::min<u32>((u32)((A + 255) / 256), (u32)nsm * 8);
    k_rec_to_pairs<<<grid, 256, 0, st>>>((u32)A, rec, b, pk0, kv0);
    const int end_bit = (int)std::min<u32>(64, 2 * b);
    cudaError_t e = cub::DeviceRadixSort::SortPairs(tmp, tb, pk0, pk1, kv0, kv1, (int)A, 0, end_bit, st);
    if (e != cudaSuccess) return e;
    e = cub::DeviceReduce::ReduceByKey(tmp, tb, pk1, pk0, kv1, kv0, nruns, MinOp(), (int)A, st);
    if (e != cudaSuccess) return e;
    k_pairs_to_rec<<<grid, 256, 0, st>>>(nruns, pk0, kv0, b, rec, a_count);
    return cudaGetLastError();
}

}  // namespace mstk
