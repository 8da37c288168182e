// Microbenchmark of the engine's group barrier (engine.cu group_sync) on the whole grid:
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/bar_bench tools/bar_bench.cu && /tmp/bar_bench
// Variants: 0 = arrive and generation in one cache line (engine r01), 1 = separate lines,
// 2 = monotonic counter (no reset; wait until the count reaches the episode's target),
// 3 = two-level monotonic (leaves of kLeaf CTAs; the last arriver of a leaf arrives at the root and then
//     releases its leaf).
#include <cstdio>
#include <cuda_runtime.h>

struct Bar { unsigned arrive; unsigned gen; unsigned pad[30]; unsigned gen2; unsigned pad2[31]; };

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

constexpr int kLeaf = 16;
struct Leaf { unsigned arrive; unsigned done; unsigned pad[30]; };
__device__ Leaf g_leaves[64 * 64];

template <int V>
__device__ __forceinline__ void gsync(Bar *b, int gcount, unsigned &episode, int grank = 0, int g = 0) {
    __syncthreads();
    if (threadIdx.x == 0) {
        if (V == 3) {
            ++episode;
            const int leaf = grank / kLeaf, nleaf = (gcount + kLeaf - 1) / kLeaf;
            const int lsz = gcount - leaf * kLeaf < kLeaf ? gcount - leaf * kLeaf : kLeaf;
            Leaf *L = g_leaves + g * 64 + leaf;
            unsigned prev;
            asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(prev) : "l"(&L->arrive) : "memory");
            if (prev == episode * (unsigned)lsz - 1) {
                asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&b->arrive) : "memory");
                const unsigned target = episode * (unsigned)nleaf;
                while ((int)(ld_acquire(&b->arrive) - target) < 0) { }
                asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(&L->done), "r"(episode) : "memory");
            } else {
                while ((int)(ld_acquire(&L->done) - episode) < 0) { }
            }
        } else if (V == 2) {
            ++episode;
            asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&b->arrive) : "memory");
            const unsigned target = episode * (unsigned)gcount;
            while ((int)(ld_acquire(&b->arrive) - target) < 0) { }
        } else {
            unsigned *g = V == 0 ? &b->gen : &b->gen2;
            const unsigned gen = ld_acquire(g);
            unsigned prev;
            asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(prev) : "l"(&b->arrive) : "memory");
            if (prev == (unsigned)gcount - 1) {
                asm volatile("st.relaxed.gpu.global.u32 [%0], 0;" ::"l"(&b->arrive) : "memory");
                asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(g) : "memory");
            } else {
                while (ld_acquire(g) == gen) { }
            }
        }
    }
    __syncthreads();
}

template <int V>
__global__ void k_bar(Bar *bars, int groups, int iters, unsigned long long *out) {
    const int gsz = gridDim.x / groups;
    const int g = blockIdx.x / gsz;
    if (g >= groups) return;
    unsigned episode = 0;
    unsigned long long t0 = 0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    for (int i = 0; i < iters; ++i) gsync<V>(bars + g, gsz, episode, blockIdx.x % gsz, g);
    unsigned long long t1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
    if (threadIdx.x == 0 && blockIdx.x % gsz == 0) out[g] = t1 - t0;
}

template <int V>
void run(int grid, int groups, int iters) {
    Bar *bars;
    unsigned long long *out, h[64];
    cudaMalloc(&bars, sizeof(Bar) * 64);
    cudaMemset(bars, 0, sizeof(Bar) * 64);
    cudaMalloc(&out, sizeof(h));
    void *args[] = {&bars, &groups, &iters, &out};
    void *lv = nullptr;
    cudaGetSymbolAddress(&lv, g_leaves);
    for (int rep = 0; rep < 2; ++rep) {
        cudaMemset(bars, 0, sizeof(Bar) * 64);
        cudaMemset(lv, 0, sizeof(Leaf) * 64 * 64);
        cudaLaunchCooperativeKernel((const void *)k_bar<V>, dim3(grid), dim3(512), args, 0, 0);
        cudaDeviceSynchronize();
    }
    cudaMemcpy(h, out, sizeof(unsigned long long) * groups, cudaMemcpyDeviceToHost);
    double mx = 0;
    for (int g = 0; g < groups; ++g) mx = h[g] > mx ? h[g] : mx;
    printf("variant %d grid %d groups %d: %.3f us per barrier (%s)\n", V, grid, groups, mx / iters / 1e3,
           cudaGetErrorString(cudaGetLastError()));
    cudaFree(bars);
    cudaFree(out);
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int groups : {1, 8}) {
        run<0>(2 * sms, groups, 20000);
        run<1>(2 * sms, groups, 20000);
        run<2>(2 * sms, groups, 20000);
        run<3>(2 * sms, groups, 20000);
    }
    run<0>(sms, 1, 20000);
    run<2>(sms, 1, 20000);
    return 0;
}
