// rand_gather_bench.cu — what HBM3e delivers to a traversal's access pattern on this B200: dependent-free
// random 4-byte gathers (one 32-byte sector each) over a 4 GiB array, random 4-byte atomicOr, and a
// sequential stream for reference.  The engine's per-arc status gather and per-hit atomics are exactly
// these patterns, so their rates bound what traffic reduction vs latency hiding can buy.
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/rgb tools/rand_gather_bench.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t mix(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
    return x;
}

template <int U>
__global__ void k_gather(const uint32_t *__restrict__ a, uint64_t mask, int64_t n_per_thread, uint32_t *out) {
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    uint32_t acc = 0;
    for (int64_t i = 0; i < n_per_thread; i += U) {
        uint32_t v[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
            const uint64_t h = ((uint64_t)mix((uint32_t)(t * 2654435761u + (i + k) * 97u)) << 20) ^ mix((uint32_t)(t + (i + k) * 131u));
            v[k] = __ldcg(a + (h & mask));
        }
#pragma unroll
        for (int k = 0; k < U; ++k) acc += v[k];
    }
    if (acc == 0x12345678u) out[0] = acc;
}

__global__ void k_atomic(uint32_t *a, uint64_t mask, int64_t n_per_thread) {
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    for (int64_t i = 0; i < n_per_thread; ++i) {
        const uint64_t h = ((uint64_t)mix((uint32_t)(t * 2654435761u + i * 97u)) << 20) ^ mix((uint32_t)(t + i * 131u));
        asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(a + (h & mask)), "r"(1u << (i & 31)) : "memory");
    }
}

__global__ void k_stream(const uint4 *__restrict__ a, int64_t n, uint32_t *out) {
    uint32_t acc = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const uint4 x = __ldcs(a + i);
        acc += x.x ^ x.y ^ x.z ^ x.w;
    }
    if (acc == 0x12345678u) out[0] = acc;
}

int main(int argc, char **argv) {
    // optional argument: cudaLimitMaxL2FetchGranularity in bytes (0 = leave the driver default)
    const int gran = argc > 1 ? atoi(argv[1]) : 0;
    if (gran > 0) {
        cudaError_t e = cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, (size_t)gran);
        size_t got = 0;
        cudaDeviceGetLimit(&got, cudaLimitMaxL2FetchGranularity);
        printf("cudaLimitMaxL2FetchGranularity set %d -> %s, now %zu\n", gran, cudaGetErrorString(e), got);
    } else {
        size_t got = 0;
        cudaDeviceGetLimit(&got, cudaLimitMaxL2FetchGranularity);
        printf("cudaLimitMaxL2FetchGranularity default %zu\n", got);
    }
    const uint64_t words = 1ull << 30;   // 4 GiB
    uint32_t *a, *out;
    cudaMalloc(&a, words * 4);
    cudaMalloc(&out, 4);
    cudaMemset(a, 1, words * 4);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int block = 512;
    for (int bpsm : {2, 4}) {
        const int grid = sms * bpsm;
        const int64_t per = 256;
        const double gathers = (double)grid * block * per;
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(e0);
            k_gather<8><<<grid, block>>>(a, words - 1, per, out);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (rep) printf("random 4B gathers, %d CTAs/SM x %d, unroll 8: %.1f G gathers/s = %.0f GB/s of 32-B sectors\n",
                            bpsm, block, gathers / ms / 1e6, gathers * 32 / ms / 1e6);
        }
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(e0);
            k_atomic<<<grid, block>>>(a, words - 1, per);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (rep) printf("random red.or, %d CTAs/SM: %.1f G atomics/s\n", bpsm, gathers / ms / 1e6);
        }
    }
    for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(e0);
        k_stream<<<sms * 4, block>>>(reinterpret_cast<const uint4 *>(a), (int64_t)(words / 4), out);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep) printf("sequential read: %.0f GB/s\n", words * 4.0 / ms / 1e6);
    }
    return 0;
}
