// relabel.cu — load-time vertex reordering of libkgs (product CUDA path; shares nothing with oracle/).
//
// The search gathers the 2-byte status of the TARGET of every inspected arc; on a power-law graph the
// targets concentrate on the high-degree nodes, but the input ids scatter them over the whole status
// array, so every gather is a fresh 32-byte sector.  kgs_load_graph therefore renumbers the nodes
// internally by non-increasing degree (ties by input id), dealt into 8 stripes: the hubs' status, hit-mask,
// M-row and bitmap words then share a few MB that stay resident in L2, and the isolated nodes (58% at C3)
// move to the end of each stripe.
//
// The reordering is invisible at the ABI: every id that leaves the library (central ids, answer node
// and arc lists, the parity view's M / activation / central list) is mapped back to the input id, and
// ranking ties break on input ids (kgs.h).  Only the internal traversal order changes, which the
// method's results do not depend on (Thm. V.2, reading R10).
#include <cub/cub.cuh>

#include "kgs_internal.h"

namespace kgs {

namespace {

__global__ void k_degree_key(const int64_t *__restrict__ rp, int64_t n, uint32_t *__restrict__ deg,
                             int32_t *__restrict__ iota) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int64_t d = rp[v + 1] - rp[v];
        deg[v] = d > 0xFFFFFFFFll ? 0xFFFFFFFFu : (uint32_t)d;
        iota[v] = (int32_t)v;
    }
}

// The j-th node in degree order gets internal id start[j % S] + j / S: the order is dealt into S = 8
// stripes of (almost) equal size, so every stripe starts with its share of the hubs.  The hot set stays
// in S compact regions (L2 locality) and the equal slices of the vertex partition (vpart.cu) at 1, 2, 4
// or 8 ranks own equal shares of the arcs.
constexpr int kStripes = 8;
__device__ __forceinline__ int64_t striped_id(int64_t j, int64_t n) {
    const int64_t s = j % kStripes, t = j / kStripes;
    // stripe s' holds the ranks j' = s' (mod S): (n - s' + S - 1) / S of them
    int64_t start = 0;
    for (int64_t r = 0; r < s; ++r) start += (n - r + kStripes - 1) / kStripes;
    return start + t;
}

// orig[u] = the input id of internal id u, perm = its inverse; new degrees (int64, for the offsets scan);
// permuted weights
__global__ void k_inverse(const int32_t *__restrict__ sorted, const uint32_t *__restrict__ deg_sorted,
                          const float *__restrict__ w, int64_t n, int32_t *__restrict__ orig,
                          int32_t *__restrict__ perm, int64_t *__restrict__ deg64, float *__restrict__ w_new) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
        const int32_t v = sorted[j];
        const int64_t u = striped_id(j, n);
        orig[u] = v;
        perm[v] = (int32_t)u;
        deg64[u] = (int64_t)deg_sorted[j];
        w_new[u] = w[v];
    }
}

// one warp per new row: copy the input row of orig[u], targets renamed through perm
__global__ void k_rows(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, const int64_t *__restrict__ rp_new,
                       const int32_t *__restrict__ orig, const int32_t *__restrict__ perm, int64_t n,
                       int32_t *__restrict__ ci_new) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; u < n; u += warps) {
        const int32_t v = orig[u];
        const int64_t s = rp[v], d = rp[v + 1] - s, o = rp_new[u];
        for (int64_t j = lane; j < d; j += 32) ci_new[o + j] = perm[ci[s + j]];
    }
}

__global__ void k_map(int32_t *__restrict__ ids, int64_t cnt, const int32_t *__restrict__ perm) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < cnt; j += (int64_t)gridDim.x * blockDim.x)
        ids[j] = perm[ids[j]];
}

int grid_for(int64_t n) {
    int64_t g = (n + 255) / 256;
    if (g > device_sm_count() * 16) g = device_sm_count() * 16;
    return g < 1 ? 1 : (int)g;
}

}  // namespace

#define RL_TRY(expr)                                  \
    do {                                              \
        const cudaError_t _e = (expr);                \
        if (_e != cudaSuccess) { cleanup(); return _e; } \
    } while (0)

cudaError_t relabel_by_degree(int64_t n, int64_t m, int64_t P, int64_t **row_ptr, int32_t **col_idx, float **weight,
                              int32_t *kw_nodes, int32_t **orig_out, int32_t **perm_out, cudaStream_t s) {
    *orig_out = nullptr;
    *perm_out = nullptr;
    uint32_t *deg = nullptr, *deg_sorted = nullptr;
    int32_t *iota = nullptr, *orig = nullptr, *perm = nullptr, *ci_new = nullptr;
    int64_t *deg64 = nullptr, *rp_new = nullptr;
    float *w_new = nullptr;
    void *tmp = nullptr;
    auto cleanup = [&]() {
        void *p[] = {deg, deg_sorted, iota, orig, perm, ci_new, deg64, rp_new, w_new, tmp};
        for (void *x : p) if (x) cudaFree(x);
    };
    const size_t nn = (size_t)(n > 0 ? n : 1);
    RL_TRY(cudaMalloc(&deg, nn * sizeof(uint32_t)));
    RL_TRY(cudaMalloc(&deg_sorted, nn * sizeof(uint32_t)));
    RL_TRY(cudaMalloc(&iota, nn * sizeof(int32_t)));
    RL_TRY(cudaMalloc(&orig, nn * sizeof(int32_t)));
    RL_TRY(cudaMalloc(&perm, nn * sizeof(int32_t)));
    RL_TRY(cudaMalloc(&deg64, nn * sizeof(int64_t)));
    RL_TRY(cudaMalloc(&rp_new, (nn + 1) * sizeof(int64_t)));
    RL_TRY(cudaMalloc(&w_new, nn * sizeof(float)));
    RL_TRY(cudaMalloc(&ci_new, (size_t)(m > 0 ? m : 1) * sizeof(int32_t)));
    if (n > 0) {
        k_degree_key<<<grid_for(n), 256, 0, s>>>(*row_ptr, n, deg, iota);
        RL_TRY(cudaGetLastError());
        // stable radix sort: non-increasing degree, ties keep the input order
        size_t tb_sort = 0, tb_scan = 0;
        RL_TRY(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb_sort, deg, deg_sorted, iota, orig, (int)n, 0, 32, s));
        RL_TRY(cub::DeviceScan::InclusiveSum(nullptr, tb_scan, deg64, rp_new + 1, (int)n, s));
        RL_TRY(cudaMalloc(&tmp, std::max(tb_sort, tb_scan)));
        RL_TRY(cub::DeviceRadixSort::SortPairsDescending(tmp, tb_sort, deg, deg_sorted, iota, orig, (int)n, 0, 32, s));
        std::swap(iota, orig);   // iota: the input ids in degree order
        k_inverse<<<grid_for(n), 256, 0, s>>>(iota, deg_sorted, *weight, n, orig, perm, deg64, w_new);
        RL_TRY(cudaGetLastError());
        RL_TRY(cudaMemsetAsync(rp_new, 0, sizeof(int64_t), s));
        RL_TRY(cub::DeviceScan::InclusiveSum(tmp, tb_scan, deg64, rp_new + 1, (int)n, s));
        k_rows<<<device_sm_count() * 16, 256, 0, s>>>(*row_ptr, *col_idx, rp_new, orig, perm, n, ci_new);
        RL_TRY(cudaGetLastError());
        if (P > 0) {
            k_map<<<grid_for(P), 256, 0, s>>>(kw_nodes, P, perm);
            RL_TRY(cudaGetLastError());
        }
    } else {
        RL_TRY(cudaMemsetAsync(rp_new, 0, sizeof(int64_t), s));
    }
    RL_TRY(cudaStreamSynchronize(s));
    // swap in the renumbered arrays
    cudaFree(*row_ptr); *row_ptr = rp_new; rp_new = nullptr;
    cudaFree(*col_idx); *col_idx = ci_new; ci_new = nullptr;
    cudaFree(*weight); *weight = w_new; w_new = nullptr;
    *orig_out = orig; orig = nullptr;
    *perm_out = perm; perm = nullptr;
    cleanup();
    return cudaSuccess;
}

// ---- the parity view in input ids
__global__ void k_levels_out_perm(const uint32_t *st, const uint8_t *M, const int32_t *perm, int64_t n, int q,
                                  uint8_t *out) {
    const int64_t gt = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = gt; v < n; v += gs) {
        const int64_t u = perm ? perm[v] : v;
        const uint32_t hm = st[u] & 0xFFu;
        for (int i = 0; i < q; ++i) out[v * q + i] = ((hm >> i) & 1u) ? M[u * 8 + i] : (uint8_t)KGS_INF_LEVEL;
    }
}
__global__ void k_gather_u8(const uint8_t *src, const int32_t *perm, int64_t n, uint8_t *out) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        out[v] = src[perm ? perm[v] : v];
}
__global__ void k_gather_i32(const int32_t *ids, const int32_t *orig, int64_t cnt, int32_t *out) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < cnt; j += (int64_t)gridDim.x * blockDim.x)
        out[j] = orig ? orig[ids[j]] : ids[j];
}

cudaError_t launch_levels_out(const uint32_t *st, const uint8_t *M, const int32_t *perm, int64_t n, int q,
                              uint8_t *out, cudaStream_t s) {
    k_levels_out_perm<<<device_sm_count() * 8, 256, 0, s>>>(st, M, perm, n, q, out);
    return cudaGetLastError();
}
cudaError_t launch_gather_u8(const uint8_t *src, const int32_t *perm, int64_t n, uint8_t *out, cudaStream_t s) {
    if (n > 0) k_gather_u8<<<grid_for(n), 256, 0, s>>>(src, perm, n, out);
    return cudaGetLastError();
}
cudaError_t launch_to_input_ids(const int32_t *ids, const int32_t *orig, int64_t cnt, int32_t *out, cudaStream_t s) {
    if (cnt > 0) k_gather_i32<<<grid_for(cnt), 256, 0, s>>>(ids, orig, cnt, out);
    return cudaGetLastError();
}

}  // namespace kgs
