// load.cu — load-time preprocessing of libkgs (product CUDA path, shares nothing
// with oracle/).  Produces the inputs kgs_load_graph takes: the normalised node weight w' (Eq. 2 and
// min-max) and the sampled average distance A (Table II).
//
//   k_dist_push / k_dist_update   bit-parallel BFS: 128 (src, dst) pairs per pass, one bit per pair
//                                 in a node's visited / next words (one 32-byte sector per node).
//   k_summary                     Eq. 2 per node over its in-arc labels sorted per row (cub segmented
//                                 sort), one warp per node, runs of equal labels found by ballots.
//   k_normalise                   w' = (w - min) / (max - min) over the nodes with in-arcs, on the 2^-24 grid.
#include <cub/device/device_segmented_sort.cuh>

#include <cmath>
#include <string>
#include <vector>

#include "kgs_internal.h"

namespace kgs {
kgs_status set_error(kgs_status s, const std::string &msg);
}

using namespace kgs;

namespace {

#define LD_TRY(expr)                                                                                   \
    do {                                                                                               \
        cudaError_t _e = (expr);                                                                       \
        if (_e != cudaSuccess) {                                                                       \
            st = set_error(_e == cudaErrorMemoryAllocation ? KGS_ENOMEM : KGS_ECUDA,                   \
                           std::string(#expr) + ": " + cudaGetErrorString(_e));                        \
            goto done;                                                                                 \
        }                                                                                              \
    } while (0)

// ---------------------------------------------------------------- pair distances (A by sampling)

// Node state of a pass: one 32-byte sector per node, {visited[2], next[2]} (128 pair bits each), so
// the per-arc gather of the push touches one sector; the frontier words cur[2] are read sequentially.
struct alignas(32) PairState {
    unsigned long long vis0, vis1, nxt0, nxt1;
};

// Push one level: every node u with frontier bits f = cur[u] ORs f & ~vis[x] into nxt[x] for each
// out-arc u -> x.  A warp takes 32 consecutive nodes and scans the arcs of each active one together
// (coalesced col_idx reads; hubs do not serialise a thread).
__global__ void k_dist_push(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, int64_t n,
                            const ulonglong2 *__restrict__ cur, PairState *__restrict__ st) {
    const int lane = threadIdx.x & 31;
    const int64_t warp0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp0 * 32; base < n; base += nwarps * 32) {
        const int64_t v = base + lane;
        const ulonglong2 f = v < n ? cur[v] : make_ulonglong2(0ull, 0ull);
        unsigned act = __ballot_sync(0xffffffffu, (f.x | f.y) != 0ull);
        while (act) {
            const int src = __ffs(act) - 1;
            act &= act - 1;
            const unsigned long long f0 = __shfl_sync(0xffffffffu, f.x, src);
            const unsigned long long f1 = __shfl_sync(0xffffffffu, f.y, src);
            const int64_t u = base + src;
            const int64_t b = rp[u], e = rp[u + 1];
            for (int64_t j = b + lane; j < e; j += 32) {
                PairState *px = st + ci[j];
                const ulonglong2 vn = *reinterpret_cast<const ulonglong2 *>(&px->vis0);
                const ulonglong2 nx = *reinterpret_cast<const ulonglong2 *>(&px->nxt0);
                const unsigned long long m0 = f0 & ~vn.x, m1 = f1 & ~vn.y;
                if (m0 && (nx.x & m0) != m0) atomicOr(&px->nxt0, m0);
                if (m1 && (nx.y & m1) != m1) atomicOr(&px->nxt1, m1);
            }
        }
    }
}

// New frontier = next & ~visited; visited |= it; next cleared.  any = 1 if some bit is new.
__global__ void k_dist_update(int64_t n, ulonglong2 *__restrict__ cur, PairState *__restrict__ st, int32_t *any) {
    int found = 0;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        PairState p = st[v];
        const unsigned long long n0 = p.nxt0 & ~p.vis0, n1 = p.nxt1 & ~p.vis1;
        cur[v] = make_ulonglong2(n0, n1);
        if (p.nxt0 | p.nxt1) {
            p.vis0 |= n0;
            p.vis1 |= n1;
            p.nxt0 = p.nxt1 = 0ull;
            st[v] = p;
            found |= (n0 | n1) != 0ull;
        }
    }
    if (__syncthreads_or(found) && threadIdx.x == 0) *any = 1;
}

__device__ __forceinline__ bool pair_bit(const PairState &p, int j) {
    return j < 64 ? ((p.vis0 >> j) & 1ull) : ((p.vis1 >> (j - 64)) & 1ull);
}

// Pair j of the batch (bit j): when its target's visited word first shows bit j, its distance is l.
// done counts the resolved pairs.
__global__ void k_dist_check(const int32_t *__restrict__ dst, int32_t cnt, int32_t level,
                             const PairState *__restrict__ st, int32_t *__restrict__ dist, int32_t *done) {
    const int j = threadIdx.x;
    if (j < cnt && dist[j] < 0 && pair_bit(st[dst[j]], j)) {
        dist[j] = level;
        atomicAdd(done, 1);
    }
}

__global__ void k_dist_seed(const int32_t *__restrict__ src, int32_t cnt, ulonglong2 *cur, PairState *st) {
    const int j = threadIdx.x;
    if (j < cnt) {
        const unsigned long long bit = 1ull << (j & 63);
        unsigned long long *c = j < 64 ? &cur[src[j]].x : &cur[src[j]].y;
        unsigned long long *vz = j < 64 ? &st[src[j]].vis0 : &st[src[j]].vis1;
        atomicOr(c, bit);
        atomicOr(vz, bit);
    }
}

__global__ void k_check_ids(const int32_t *__restrict__ ids, int64_t cnt, int64_t n, int32_t *err) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < cnt; j += (int64_t)gridDim.x * blockDim.x)
        if (ids[j] < 0 || ids[j] >= n) atomicOr(err, 1);
}

__global__ void k_check_rows(const int64_t *__restrict__ rp, int64_t n, int64_t m, int32_t *err) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= n; v += (int64_t)gridDim.x * blockDim.x) {
        if (v == 0 && rp[0] != 0) atomicOr(err, 1);
        if (v == n && rp[n] != m) atomicOr(err, 1);
        if (v < n && rp[v + 1] < rp[v]) atomicOr(err, 1);
    }
}

constexpr int kPairs = 128;   // pairs per bit-parallel BFS pass

int grid_for(int64_t items, int block) {
    int64_t g = (items + block - 1) / block;
    if (g > device_sm_count() * 16) g = device_sm_count() * 16;
    return g < 1 ? 1 : (int)g;
}

template <class T>
cudaError_t stage(const T *p, int64_t cnt, bool dev, cudaStream_t s, T **out, T **owned) {
    *owned = nullptr;
    if (dev || cnt == 0) { *out = const_cast<T *>(p); return cudaSuccess; }
    cudaError_t e = cudaMallocAsync((void **)owned, sizeof(T) * (size_t)cnt, s);
    if (e != cudaSuccess) return e;
    *out = *owned;
    return cudaMemcpyAsync(*owned, p, sizeof(T) * (size_t)cnt, cudaMemcpyHostToDevice, s);
}

// ---------------------------------------------------------------- Eq. 2 degree of summary

// One warp per node over its sorted labels: a run of equal labels r has n_r entries and adds
// n_r log2(1 + n_r); w = that sum / deg.  Run starts inside a 32-label chunk come from
// a ballot; a run that started in an earlier chunk carries its start.  The terms are added in label
// order (the run ends of a chunk, lowest lane first, chunk after chunk), the order Eq. 2's sum is
// written in.  Also min/max of w over the nodes with in-arcs (reading R6; w >= 0, so the IEEE bit
// patterns order like the values).
__global__ void k_summary(const int64_t *__restrict__ rp, const int32_t *__restrict__ lab, int64_t n,
                          double *__restrict__ w, unsigned long long *wmin, unsigned long long *wmax) {
    const int lane = threadIdx.x & 31;
    const int64_t warp0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long lmin = ~0ull, lmax = 0ull;
    for (int64_t v = warp0; v < n; v += nwarps) {
        const int64_t b = rp[v], e = rp[v + 1];
        double acc = 0.0;    // the same value in every lane
        int64_t carry = b;   // start of the run open at the chunk boundary
        for (int64_t c = b; c < e; c += 32) {
            const int64_t j = c + lane;
            const bool in = j < e;
            const int32_t l = in ? lab[j] : 0;
            const bool start = in && (j == b || lab[j - 1] != l);
            const bool end = in && (j + 1 == e || lab[j + 1] != l);
            const unsigned starts = __ballot_sync(0xffffffffu, start);
            double term = 0.0;
            if (end) {
                const unsigned upto = starts & (0xffffffffu >> (31 - lane));
                const int64_t s0 = upto ? c + (31 - __clz(upto)) : carry;
                const double nr = (double)(j - s0 + 1);
                term = nr * log2(1.0 + nr);
            }
            for (unsigned ends = __ballot_sync(0xffffffffu, end); ends; ends &= ends - 1)
                acc += __shfl_sync(0xffffffffu, term, __ffs(ends) - 1);
            if (starts) carry = c + (31 - __clz(starts));
        }
        if (e > b) {
            const double wv = acc / (double)(e - b);
            if (lane == 0) {
                w[v] = wv;
                const unsigned long long bits = (unsigned long long)__double_as_longlong(wv);
                lmin = bits < lmin ? bits : lmin;
                lmax = bits > lmax ? bits : lmax;
            }
        } else if (lane == 0) {
            w[v] = 0.0;   // no in-arcs: summarises nothing, out of the min / max (R6)
        }
    }
    if (lane == 0) {
        if (lmin != ~0ull) atomicMin(wmin, lmin);
        atomicMax(wmax, lmax);
    }
}

// w' = (w - min) / (max - min) over the nodes with in-arcs, 0 for the others (R6) and for every node when
// max = min (R26); produced on the 2^-24 grid, nearest point of the fp64 value, ties up (R27).
__global__ void k_normalise(const double *__restrict__ w, const int64_t *__restrict__ rp, int64_t n,
                            const unsigned long long *wmin, const unsigned long long *wmax, float *__restrict__ out) {
    const unsigned long long bmin = *wmin, bmax = *wmax;
    const bool any = bmin != ~0ull;
    const double lo = __longlong_as_double((long long)bmin), hi = __longlong_as_double((long long)bmax);
    const double span = hi - lo;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const double x = (any && span > 0.0 && rp[v + 1] > rp[v]) ? (w[v] - lo) / span : 0.0;
        out[v] = (float)(floor(x * 16777216.0 + 0.5) * (1.0 / 16777216.0));
    }
}

}  // namespace

extern "C" {

kgs_status kgs_prep_pair_distances(int64_t n, int64_t m, const int64_t *row_ptr, const int32_t *col_idx,
                                   int32_t n_pairs, const int32_t *src, const int32_t *dst, int32_t max_hops,
                                   int32_t device, int32_t flags, void *cuda_stream, int32_t *dist, double *mean) {
    if (n < 0 || n >= (int64_t)1 << 31 || m < 0 || n_pairs < 0 || (n_pairs > 0 && (!dist || !src || !dst)) ||
        !row_ptr || (m > 0 && !col_idx) || max_hops < 1 || max_hops > 254)
        return set_error(KGS_EINVAL, "kgs_prep_pair_distances: bad sizes, null pointer or max_hops outside 1..254");
    if (n_pairs > 0 && n == 0) return set_error(KGS_EINVAL, "kgs_prep_pair_distances: pairs on an empty graph");
    kgs_status st = KGS_OK;
    const bool dev = (flags & KGS_INPUT_DEVICE_PTRS) != 0;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    int64_t *d_rp = nullptr, *o_rp = nullptr;
    int32_t *d_ci = nullptr, *o_ci = nullptr, *d_src = nullptr, *o_src = nullptr, *d_dst = nullptr, *o_dst = nullptr;
    ulonglong2 *cur = nullptr;
    PairState *pst = nullptr;
    int32_t *ctl = nullptr, *h_ctl = nullptr, *d_dist = nullptr;   // ctl: [0] err, [1] any, [2] done
    std::vector<int32_t> out((size_t)n_pairs, -1);
    double sum = 0.0;
    int64_t reach = 0;
    LD_TRY(cudaSetDevice(device));
    LD_TRY(stage(row_ptr, n + 1, dev, s, &d_rp, &o_rp));
    LD_TRY(stage(col_idx, m, dev, s, &d_ci, &o_ci));
    LD_TRY(stage(src, (int64_t)n_pairs, dev, s, &d_src, &o_src));
    LD_TRY(stage(dst, (int64_t)n_pairs, dev, s, &d_dst, &o_dst));
    LD_TRY(cudaMallocAsync((void **)&ctl, 4 * sizeof(int32_t), s));
    LD_TRY(cudaMallocHost((void **)&h_ctl, 4 * sizeof(int32_t)));
    LD_TRY(cudaMallocAsync((void **)&d_dist, kPairs * sizeof(int32_t), s));
    LD_TRY(cudaMemsetAsync(ctl, 0, 4 * sizeof(int32_t), s));
    k_check_rows<<<grid_for(n + 1, 256), 256, 0, s>>>(d_rp, n, m, ctl);
    if (m > 0) k_check_ids<<<grid_for(m, 256), 256, 0, s>>>(d_ci, m, n, ctl);
    if (n_pairs > 0) {
        k_check_ids<<<grid_for(n_pairs, 256), 256, 0, s>>>(d_src, n_pairs, n, ctl);
        k_check_ids<<<grid_for(n_pairs, 256), 256, 0, s>>>(d_dst, n_pairs, n, ctl);
    }
    LD_TRY(cudaGetLastError());
    LD_TRY(cudaMemcpyAsync(h_ctl, ctl, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    LD_TRY(cudaStreamSynchronize(s));
    if (h_ctl[0]) { st = set_error(KGS_EINVAL, "kgs_prep_pair_distances: malformed row_ptr or id out of range"); goto done; }
    if (n_pairs > 0) {
        LD_TRY(cudaMallocAsync((void **)&cur, sizeof(ulonglong2) * (size_t)n, s));
        LD_TRY(cudaMallocAsync((void **)&pst, sizeof(PairState) * (size_t)n, s));
    }
    for (int32_t p0 = 0; p0 < n_pairs; p0 += kPairs) {
        const int32_t cnt = n_pairs - p0 < kPairs ? n_pairs - p0 : kPairs;
        LD_TRY(cudaMemsetAsync(cur, 0, sizeof(ulonglong2) * (size_t)n, s));
        LD_TRY(cudaMemsetAsync(pst, 0, sizeof(PairState) * (size_t)n, s));
        LD_TRY(cudaMemsetAsync(d_dist, 0xFF, kPairs * sizeof(int32_t), s));
        LD_TRY(cudaMemsetAsync(ctl + 2, 0, sizeof(int32_t), s));
        k_dist_seed<<<1, kPairs, 0, s>>>(d_src + p0, cnt, cur, pst);
        k_dist_check<<<1, kPairs, 0, s>>>(d_dst + p0, cnt, 0, pst, d_dist, ctl + 2);
        for (int32_t l = 1; l <= max_hops; ++l) {
            LD_TRY(cudaMemsetAsync(ctl + 1, 0, sizeof(int32_t), s));
            k_dist_push<<<grid_for(n, 256), 256, 0, s>>>(d_rp, d_ci, n, cur, pst);
            k_dist_update<<<grid_for(n, 256), 256, 0, s>>>(n, cur, pst, ctl + 1);
            k_dist_check<<<1, kPairs, 0, s>>>(d_dst + p0, cnt, l, pst, d_dist, ctl + 2);
            LD_TRY(cudaGetLastError());
            LD_TRY(cudaMemcpyAsync(h_ctl + 1, ctl + 1, 2 * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
            LD_TRY(cudaStreamSynchronize(s));
            if (!h_ctl[1] || h_ctl[2] == cnt) break;   // frontier empty or every pair of the batch answered
        }
        // every pass starts from zeroed cur / state (reset above)
        LD_TRY(cudaMemcpyAsync(out.data() + p0, d_dist, sizeof(int32_t) * (size_t)cnt, cudaMemcpyDeviceToHost, s));
        LD_TRY(cudaStreamSynchronize(s));
    }
    for (int32_t j = 0; j < n_pairs; ++j) {
        dist[j] = out[(size_t)j];
        if (out[(size_t)j] >= 0) { sum += (double)out[(size_t)j]; ++reach; }
    }
    if (mean) *mean = reach ? sum / (double)reach : NAN;
done:
    if (cur) cudaFreeAsync(cur, s);
    if (pst) cudaFreeAsync(pst, s);
    if (ctl) cudaFreeAsync(ctl, s);
    if (d_dist) cudaFreeAsync(d_dist, s);
    if (o_rp) cudaFreeAsync(o_rp, s);
    if (o_ci) cudaFreeAsync(o_ci, s);
    if (o_src) cudaFreeAsync(o_src, s);
    if (o_dst) cudaFreeAsync(o_dst, s);
    cudaStreamSynchronize(s);
    if (h_ctl) cudaFreeHost(h_ctl);
    return st;
}

kgs_status kgs_prep_summary_weights(int64_t n, int64_t m, const int64_t *in_row_ptr, const int32_t *in_label,
                                    int32_t device, int32_t flags, void *cuda_stream, float *w_norm, double *w_raw) {
    if (n < 0 || n >= (int64_t)1 << 31 || m < 0 || m >= (int64_t)1 << 31 || !in_row_ptr || (m > 0 && !in_label) ||
        (n > 0 && !w_norm))
        return set_error(KGS_EINVAL, "kgs_prep_summary_weights: bad sizes or null pointer");
    if (n == 0) return KGS_OK;
    kgs_status st = KGS_OK;
    const bool dev = (flags & KGS_INPUT_DEVICE_PTRS) != 0;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    int64_t *d_rp = nullptr, *o_rp = nullptr;
    int32_t *d_lab = nullptr, *o_lab = nullptr, *sorted = nullptr, *ctl = nullptr, h_err = 0;
    double *w = nullptr;
    unsigned long long *mm = nullptr;
    float *d_out = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    LD_TRY(cudaSetDevice(device));
    LD_TRY(stage(in_row_ptr, n + 1, dev, s, &d_rp, &o_rp));
    LD_TRY(stage(in_label, m, dev, s, &d_lab, &o_lab));
    LD_TRY(cudaMallocAsync((void **)&ctl, sizeof(int32_t), s));
    LD_TRY(cudaMemsetAsync(ctl, 0, sizeof(int32_t), s));
    k_check_rows<<<grid_for(n + 1, 256), 256, 0, s>>>(d_rp, n, m, ctl);
    LD_TRY(cudaGetLastError());
    LD_TRY(cudaMemcpyAsync(&h_err, ctl, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    LD_TRY(cudaStreamSynchronize(s));
    if (h_err) { st = set_error(KGS_EINVAL, "kgs_prep_summary_weights: malformed in_row_ptr"); goto done; }
    if (m > 0) {
        LD_TRY(cudaMallocAsync((void **)&sorted, sizeof(int32_t) * (size_t)m, s));
        LD_TRY(cub::DeviceSegmentedSort::SortKeys(nullptr, tmp_bytes, d_lab, sorted, (int)m, (int)n, d_rp, d_rp + 1, s));
        LD_TRY(cudaMallocAsync(&tmp, tmp_bytes ? tmp_bytes : 1, s));
        LD_TRY(cub::DeviceSegmentedSort::SortKeys(tmp, tmp_bytes, d_lab, sorted, (int)m, (int)n, d_rp, d_rp + 1, s));
    }
    LD_TRY(cudaMallocAsync((void **)&w, sizeof(double) * (size_t)n, s));
    LD_TRY(cudaMallocAsync((void **)&mm, 2 * sizeof(unsigned long long), s));
    LD_TRY(cudaMallocAsync((void **)&d_out, sizeof(float) * (size_t)n, s));
    LD_TRY(cudaMemsetAsync(mm, 0xFF, sizeof(unsigned long long), s));
    LD_TRY(cudaMemsetAsync(mm + 1, 0, sizeof(unsigned long long), s));
    k_summary<<<grid_for(n * 32, 256), 256, 0, s>>>(d_rp, sorted, n, w, mm, mm + 1);
    k_normalise<<<grid_for(n, 256), 256, 0, s>>>(w, d_rp, n, mm, mm + 1, d_out);
    LD_TRY(cudaGetLastError());
    LD_TRY(cudaMemcpyAsync(w_norm, d_out, sizeof(float) * (size_t)n, cudaMemcpyDeviceToHost, s));
    if (w_raw) LD_TRY(cudaMemcpyAsync(w_raw, w, sizeof(double) * (size_t)n, cudaMemcpyDeviceToHost, s));
    LD_TRY(cudaStreamSynchronize(s));
done:
    if (sorted) cudaFreeAsync(sorted, s);
    if (tmp) cudaFreeAsync(tmp, s);
    if (w) cudaFreeAsync(w, s);
    if (mm) cudaFreeAsync(mm, s);
    if (d_out) cudaFreeAsync(d_out, s);
    if (ctl) cudaFreeAsync(ctl, s);
    if (o_rp) cudaFreeAsync(o_rp, s);
    if (o_lab) cudaFreeAsync(o_lab, s);
    cudaStreamSynchronize(s);
    return st;
}

}  // extern "C"
