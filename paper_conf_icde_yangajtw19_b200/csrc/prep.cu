// prep.cu — load-time and per-alpha kernels of libkgs (product CUDA path; shares nothing with oracle/).
//
//   k_activation   Eqs. 3-5: w, alpha, A -> uint8 activation level a, cached per alpha.
//   k_degree_class light / big node classes for the engine's load balance.
//   k_snap         weights onto the 2^-24 grid (reading R15).
//   k_validate     CSR / index / weight checks of kgs_load_graph.
#include <atomic>

#include "kgs_internal.h"

namespace kgs {

int device_sm_count() {
    static std::atomic<int> cache[64];
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) dev = 0;
    const int slot = dev >= 0 && dev < 64 ? dev : -1;
    if (slot >= 0) {
        const int c = cache[slot].load(std::memory_order_relaxed);
        if (c > 0) return c;
    }
    int sms = 0;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms < 1) sms = 1;
    if (slot >= 0) cache[slot].store(sms, std::memory_order_relaxed);
    return sms;
}

__global__ void k_activation(const float *__restrict__ w, int64_t n, double A, double alpha,
                             uint8_t *__restrict__ act, uint32_t *amax) {
    uint32_t local = 0;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const double wv = (double)w[v];
        double x;
        if (wv < alpha) {            // Eq. 4 reward, Eq. 5 first case
            const double reward = __ddiv_rn(__dmul_rn(A, __dsub_rn(alpha, wv)), alpha);
            x = __dsub_rn(A, reward);
        } else if (wv == alpha) {    // Eq. 5 second case
            x = A;
        } else {                     // Eq. 3 penalty, Eq. 5 third case
            const double penalty = __ddiv_rn(__dmul_rn(A, __dsub_rn(wv, alpha)), __dsub_rn(1.0, alpha));
            x = __dadd_rn(A, penalty);
        }
        double r = floor(__dadd_rn(x, 0.5));   // nearest integer, halves up (R4)
        r = r < 0.0 ? 0.0 : (r > 254.0 ? 254.0 : r);
        const uint8_t a = (uint8_t)r;
        act[v] = a;
        local = local > a ? local : a;
    }
    local = __reduce_max_sync(0xffffffffu, local);
    if ((threadIdx.x & 31) == 0) atomicMax(amax, local);
}

cudaError_t launch_activation(const float *w, int64_t n, double A, double alpha, uint8_t *act, uint32_t *amax,
                              cudaStream_t s) {
    cudaMemsetAsync(amax, 0, sizeof(uint32_t), s);
    if (n > 0) {
        int grid = (int)((n + 255) / 256);
        if (grid > device_sm_count() * 16) grid = device_sm_count() * 16;
        k_activation<<<grid, 256, 0, s>>>(w, n, A, alpha, act, amax);
    }
    return cudaGetLastError();
}

__global__ void k_degree_class(const int64_t *__restrict__ rp, int64_t n, uint8_t *__restrict__ cls) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    {
        const int64_t d = rp[v + 1] - rp[v];
        const int lg = d == 0 ? 0 : 1 + (d == 1 ? 0 : 64 - __clzll((unsigned long long)(d - 1)));   // 2^(lg-1) >= d
        cls[v] = (uint8_t)((d > kBigDeg ? CLS_BIG : CLS_LIGHT) | (lg << 1));
    }
}
cudaError_t launch_degree_class(const int64_t *row_ptr, int64_t n, uint8_t *cls, cudaStream_t s) {
    if (n > 0) {
        int grid = (int)((n + 255) / 256);
        if (grid > device_sm_count() * 16) grid = device_sm_count() * 16;
        k_degree_class<<<grid, 256, 0, s>>>(row_ptr, n, cls);
    }
    return cudaGetLastError();
}

__global__ void k_snap(float *w, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const double x = (double)w[v] * 16777216.0;
        w[v] = (float)(floor(x + 0.5) * (1.0 / 16777216.0));
    }
}
cudaError_t launch_snap_weights(float *w, int64_t n, cudaStream_t s) {
    if (n > 0) {
        int grid = (int)((n + 255) / 256);
        if (grid > device_sm_count() * 16) grid = device_sm_count() * 16;
        k_snap<<<grid, 256, 0, s>>>(w, n);
    }
    return cudaGetLastError();
}

// One thread per node (row_ptr, weight), per arc (col_idx range) and per posting (kw_nodes range and
// strict increase inside each keyword, using a binary search of the posting's keyword).
__global__ void k_validate(DevGraph g, int32_t *err) {
    const int64_t gt = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = gt; v < g.n; v += gs) {
        if (g.row_ptr[v + 1] < g.row_ptr[v]) atomicOr(err, 1);
        const float w = g.weight[v];
        if (!(w >= 0.0f && w <= 1.0f)) atomicOr(err, 4);
    }
    for (int64_t j = gt; j < g.m; j += gs) {
        const int32_t x = g.col_idx[j];
        if (x < 0 || x >= g.n) atomicOr(err, 2);
    }
    const int64_t P = g.kw_ptr[g.n_kw];
    for (int64_t j = gt; j < P; j += gs) {
        const int32_t v = g.kw_nodes[j];
        if (v < 0 || v >= g.n) { atomicOr(err, 16); continue; }
        if (j == 0) continue;
        int64_t lo = 0, hi = g.n_kw;   // keyword t with kw_ptr[t] <= j < kw_ptr[t+1]
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) >> 1;
            if (g.kw_ptr[mid] <= j) lo = mid; else hi = mid;
        }
        if (j > g.kw_ptr[lo] && v <= g.kw_nodes[j - 1]) atomicOr(err, 16);
    }
}
cudaError_t launch_validate(const DevGraph &g, int32_t *err, cudaStream_t s) {
    k_validate<<<device_sm_count() * 8, 256, 0, s>>>(g, err);
    return cudaGetLastError();
}

}  // namespace kgs
