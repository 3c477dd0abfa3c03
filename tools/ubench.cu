// tools/ubench.cu — micro-benchmarks that size the A8 design (not part of the library).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubench tools/ubench.cu && /tmp/ubench
// 1. random RED.MIN.u64 throughput into tables of N entries (the min-into-best / matrix cost)
// 2. random 4-byte gather throughput from maps of N entries (the label gather cost),
//    with and without a streaming read alongside.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t x) {
    x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 27; x *= 0x94D049BB133111EBull; x ^= x >> 31;
    return x;
}

__global__ void k_red(uint64_t* tab, uint32_t n, uint64_t ops, uint64_t seed) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < ops; i += stride) {
        const uint64_t h = mix(seed + i);
        asm volatile("red.relaxed.gpu.global.min.u64 [%0], %1;" :: "l"(tab + (h % n)), "l"(h) : "memory");
    }
}

// the same REDs, but every CTA into its own private copy of the table (cta * n + h % n)
__global__ void k_red_private(uint64_t* tab, uint32_t n, uint64_t ops, uint64_t seed) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint64_t* mine = tab + (uint64_t)blockIdx.x * n;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < ops; i += stride) {
        const uint64_t h = mix(seed + i);
        asm volatile("red.relaxed.gpu.global.min.u64 [%0], %1;" :: "l"(mine + (h % n)), "l"(h) : "memory");
    }
}

template <int ILP>
__global__ void k_gather(const int* map, uint32_t n, uint64_t ops, uint64_t seed, int* sink) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x * ILP;
    int acc = 0;
    for (uint64_t i = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) * ILP; i < ops; i += stride) {
        int v[ILP];
#pragma unroll
        for (int k = 0; k < ILP; ++k) v[k] = __ldg(map + (mix(seed + i + k) % n));
#pragma unroll
        for (int k = 0; k < ILP; ++k) acc += v[k];
    }
    if (acc == 0x7fffffff) *sink = acc;
}

__global__ void k_stream(const uint4* a, uint64_t n, uint4* out) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint32_t acc = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
        uint4 v = a[i];
        acc ^= v.x ^ v.y ^ v.z ^ v.w;
    }
    if (acc == 0x12345678u) out[0] = make_uint4(acc, 0, 0, 0);
}

int main() {
    int nsm;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float ms;
    uint64_t* tab;
    cudaMalloc(&tab, (size_t)(1 << 24) * 8);
    const uint64_t ops = 1ull << 28;
    for (uint32_t n : {4096u, 1u << 17, 1u << 22, 1u << 24}) {
        cudaMemset(tab, 0xff, (size_t)n * 8);
        k_red<<<nsm * 16, 256>>>(tab, n, ops, 1);
        cudaEventRecord(e0);
        k_red<<<nsm * 16, 256>>>(tab, n, ops, 7);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        printf("RED.MIN.u64 random  table %9u entries: %7.1f G ops/s\n", n, ops / ms / 1e6);
    }
    {
        uint64_t* ptab;
        const uint32_t n = 1u << 16;
        cudaMalloc(&ptab, (size_t)n * 8 * nsm * 4);
        for (int cpsm : {1, 4}) {
            cudaMemset(ptab, 0xff, (size_t)n * 8 * nsm * cpsm);
            k_red_private<<<nsm * cpsm, 1024 / cpsm>>>(ptab, n, ops, 1);
            cudaEventRecord(e0);
            k_red_private<<<nsm * cpsm, 1024 / cpsm>>>(ptab, n, ops, 7);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&ms, e0, e1);
            printf("RED.MIN.u64 random, per-CTA private table of %u (%d CTAs): %7.1f G ops/s\n", n,
                   nsm * cpsm, ops / ms / 1e6);
        }
        for (uint32_t n2 : {1u << 16}) {
            cudaMemset(tab, 0xff, (size_t)n2 * 8);
            k_red<<<nsm * 16, 256>>>(tab, n2, ops, 1);
            cudaEventRecord(e0);
            k_red<<<nsm * 16, 256>>>(tab, n2, ops, 7);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&ms, e0, e1);
            printf("RED.MIN.u64 random  table %9u entries: %7.1f G ops/s\n", n2, ops / ms / 1e6);
        }
        cudaFree(ptab);
    }
    int *map, *sink;
    cudaMalloc(&map, (size_t)(1 << 24) * 4);
    cudaMalloc(&sink, 4);
    cudaMemset(map, 1, (size_t)(1 << 24) * 4);
    for (uint32_t n : {4096u, 97u * 1024, 1u << 22}) {
        for (int blocks : {nsm * 4, nsm * 8, nsm * 16}) {
            k_gather<8><<<blocks, 256>>>(map, n, ops, 1, sink);
            cudaEventRecord(e0);
            k_gather<8><<<blocks, 256>>>(map, n, ops, 3, sink);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&ms, e0, e1);
            printf("gather 4B random map %9u entries, %5d CTAs x 256 (ILP 8): %7.1f G loads/s\n", n,
                   blocks, ops / ms / 1e6);
        }
    }
    // streaming read bandwidth reference
    uint4* big;
    const uint64_t nb = 1ull << 27;  // 2 GiB
    cudaMalloc(&big, nb * 16);
    cudaMemset(big, 0, nb * 16);
    k_stream<<<nsm * 8, 512>>>(big, nb, big);
    cudaEventRecord(e0);
    k_stream<<<nsm * 8, 512>>>(big, nb, big);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("stream read 2 GiB: %7.1f GB/s\n", nb * 16 / ms / 1e6);
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
