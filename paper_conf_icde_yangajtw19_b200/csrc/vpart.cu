// vpart.cu — the vertex-partitioned search of ONE query over P ranks (SURVEY.md §8(e) "a single
// query").  Product CUDA path; shares nothing with oracle/.
//
// The CSR and the per-node hit masks hm are replicated; rank r owns the node rows [lo, hi) of one equal
// slice.  Level l (the level rule of Alg. 2, with the snapshot semantics of reading R10):
//   k_vp_expmask   X[u] = hm[u] if u expands at l (a_u <= l, not a blocked central), else 0 — all u.
//   k_vp_pull      every owned x: new = (OR over in-arcs u->x of X[u]) & ~hm[x], if gate(x) <= l+1;
//                  M[x][i] = l+1 for the new bits (owned rows), hm_slice[x-lo] = hm[x] | new; owned
//                  nodes that become all-hit join the owned central list with depth l+1 (Lemma V.1).
//   k_vp_pull_big  the same for owned nodes of more than kVpBig in-arcs, one CTA per node.
//   k_vp_waiting   when a level made no mark: owned hit nodes that still wait for a gated neighbour
//                  (the work-list of Alg. 2 ln 19 is not empty yet, so the search is not exhausted).
// Between levels the host all-gathers hm_slice into hm and all-reduces {marks, new centrals}.  After
// the search the owned M rows and central lists are all-gathered and the engine's top-down runs on the
// replicated state (k_engine, td_only).
#include "kgs_internal.h"

namespace kgs {

constexpr int kVpBlock = 256;

__global__ void k_vp_init(const int64_t *__restrict__ kw_ptr, const int32_t *__restrict__ kw_nodes, VpQuery qd,
                          uint8_t *__restrict__ hm, uint8_t *__restrict__ gate, uint8_t *__restrict__ M) {
    // sources of every keyword (all ranks, replicated): hm bit i, M[v][i] = 0, no gate
    int64_t base[kMaxQ + 1];
    base[0] = 0;
    for (int i = 0; i < qd.q; ++i) base[i + 1] = base[i] + (kw_ptr[qd.kw[i] + 1] - kw_ptr[qd.kw[i]]);
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < base[qd.q];
         j += (int64_t)gridDim.x * blockDim.x) {
        int i = 0;
        while (j >= base[i + 1]) ++i;
        const int32_t v = kw_nodes[kw_ptr[qd.kw[i]] + (j - base[i])];
        atomicOr(reinterpret_cast<unsigned *>(hm + (v & ~3)), (1u << i) << ((v & 3) * 8));
        gate[v] = 0;
        M[(int64_t)v * 8 + i] = 0;
    }
}

// level-0 identification of the owned rows: nodes that contain every keyword (depth 0)
__global__ void k_vp_ident0(const uint8_t *__restrict__ hm, int64_t lo, int64_t hi, uint32_t full,
                            int32_t *cent, uint8_t *cdep, int32_t *cent_n, unsigned long long *counts) {
    for (int64_t x = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < hi; x += (int64_t)gridDim.x * blockDim.x)
        if (hm[x] == full) {
            const int p = atomicAdd(cent_n, 1);
            cent[p] = (int32_t)x;
            cdep[p] = 0;
            atomicAdd(counts + 1, 1ull);
        }
}

// X[u] for every node: the keywords u pushes at level l (Alg. 2 ln 2-11; 16 nodes per thread step)
__global__ void k_vp_expmask(const uint8_t *__restrict__ hm, const uint8_t *__restrict__ act, int64_t n_pad,
                             int64_t n, int l, uint32_t full, int block_central, uint8_t *__restrict__ X) {
    const int64_t n16 = n_pad / 16;
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n16; j += (int64_t)gridDim.x * blockDim.x) {
        const uint4 h = reinterpret_cast<const uint4 *>(hm)[j];
        uint8_t hb[16], out[16];
        *reinterpret_cast<uint4 *>(hb) = h;
        for (int t = 0; t < 16; ++t) {
            const int64_t u = j * 16 + t;
            const uint32_t hu = hb[t];
            const bool expands = u < n && hu && act[u] <= l && !(block_central && hu == full);
            out[t] = expands ? (uint8_t)hu : 0;
        }
        reinterpret_cast<uint4 *>(X)[j] = *reinterpret_cast<uint4 *>(out);
    }
}

__device__ __forceinline__ void vp_finish_node(int64_t x, int64_t lo, uint32_t h, uint32_t nb, int l, uint32_t full,
                                               uint8_t *hm_slice, uint8_t *M, int32_t *cent, uint8_t *cdep,
                                               int32_t *cent_n, unsigned &marks, unsigned &newc,
                                               unsigned long long *counts, long long *chg) {
    hm_slice[x - lo] = (uint8_t)(h | nb);
    if (!nb) return;
    // a changed owned node: counted (counts[3]) and listed (id << 8 | new mask) for the sparse exchange
    const unsigned long long p = atomicAdd(counts + 3, 1ull);
    if (chg) chg[p] = ((long long)x << 8) | (long long)(h | nb);
    for (int i = 0; i < kMaxQ; ++i)
        if ((nb >> i) & 1u) M[x * 8 + i] = (uint8_t)(l + 1);   // m_xi <- l+1 (Alg. 2 ln 21)
    marks += __popc(nb);
    if ((h | nb) == full) {                                     // all-hit at l+1: central, depth l+1
        const int p = atomicAdd(cent_n, 1);
        cent[p] = (int32_t)x;
        cdep[p] = (uint8_t)(l + 1);
        ++newc;
    }
}

__device__ __forceinline__ void vp_count(unsigned marks, unsigned newc, unsigned wait, unsigned long long *counts) {
    marks = __reduce_add_sync(0xffffffffu, marks);
    newc = __reduce_add_sync(0xffffffffu, newc);
    wait = __reduce_add_sync(0xffffffffu, wait);
    if ((threadIdx.x & 31) == 0) {
        if (marks) atomicAdd(counts, (unsigned long long)marks);
        if (newc) atomicAdd(counts + 1, (unsigned long long)newc);
        if (wait) atomicAdd(counts + 2, (unsigned long long)wait);
    }
}

// one warp per owned node of at most kVpBig in-arcs; early exit once every missing keyword is found
__global__ void __launch_bounds__(kVpBlock) k_vp_pull(const int64_t *__restrict__ in_ptr, const int32_t *__restrict__ in_idx,
                                                      const uint8_t *__restrict__ hm, const uint8_t *__restrict__ X,
                                                      const uint8_t *__restrict__ gate, const uint8_t *__restrict__ act,
                                                      int block_central, int64_t lo, int64_t hi, int l,
                                                      uint32_t full, uint8_t *hm_slice, uint8_t *M, int32_t *cent,
                                                      uint8_t *cdep, int32_t *cent_n, unsigned long long *counts,
                                                      long long *chg) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    unsigned marks = 0, newc = 0, wait = 0;
    for (int64_t x = lo + blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); x < hi; x += warps) {
        const uint32_t h = hm[x];
        // a hit node not active yet stays on the work-list (Alg. 2 ln 4-7)
        if (lane == 0 && h && !(block_central && h == full) && act[x] > l) ++wait;
        const uint32_t need = (gate[x] <= (uint32_t)(l + 1)) ? (full & ~h) : 0u;   // ln 13-18
        const int64_t s0 = in_ptr[x], s1 = in_ptr[x + 1];
        if (need && s1 - s0 > kVpBig) continue;                 // k_vp_pull_big
        uint32_t acc = 0;
        if (need)
            for (int64_t e = s0; e < s1; e += 32) {
                if (e + lane < s1) acc |= X[__ldg(in_idx + e + lane)];
                acc = __reduce_or_sync(0xffffffffu, acc);
                if ((acc & need) == need) break;
            }
        if (lane == 0)
            vp_finish_node(x, lo, h, acc & need, l, full, hm_slice, M, cent, cdep, cent_n, marks, newc, counts, chg);
    }
    vp_count(marks, newc, wait, counts);
}

// one CTA per owned node of more than kVpBig in-arcs (the list is built once per graph and range)
__global__ void __launch_bounds__(kVpBlock) k_vp_pull_big(const int64_t *__restrict__ in_ptr, const int32_t *__restrict__ in_idx,
                                                          const uint8_t *__restrict__ hm, const uint8_t *__restrict__ X,
                                                          const uint8_t *__restrict__ gate, const int32_t *__restrict__ big,
                                                          int nbig, int64_t lo, int l, uint32_t full, uint8_t *hm_slice,
                                                          uint8_t *M, int32_t *cent, uint8_t *cdep, int32_t *cent_n,
                                                          unsigned long long *counts, long long *chg) {
    __shared__ uint32_t s_acc;
    unsigned marks = 0, newc = 0;
    for (int b = blockIdx.x; b < nbig; b += gridDim.x) {
        const int64_t x = big[b];
        const uint32_t h = hm[x];
        const uint32_t need = (gate[x] <= (uint32_t)(l + 1)) ? (full & ~h) : 0u;
        if (!need) continue;                                     // written by k_vp_pull
        if (threadIdx.x == 0) s_acc = 0;
        __syncthreads();
        const int64_t s0 = in_ptr[x], s1 = in_ptr[x + 1];
        uint32_t acc = 0;
        for (int64_t e0 = s0; e0 < s1; e0 += 8 * blockDim.x) {
            for (int t = 0; t < 8; ++t) {
                const int64_t e = e0 + t * blockDim.x + threadIdx.x;
                if (e < s1) acc |= X[__ldg(in_idx + e)];
            }
            acc = __reduce_or_sync(0xffffffffu, acc);
            if ((threadIdx.x & 31) == 0 && (acc & ~s_acc)) atomicOr(&s_acc, acc);
            __syncthreads();
            const uint32_t all = s_acc;
            __syncthreads();
            if ((all & need) == need) break;
            acc = all;
        }
        if (threadIdx.x == 0)
            vp_finish_node(x, lo, h, s_acc & need, l, full, hm_slice, M, cent, cdep, cent_n, marks, newc, counts, chg);
        __syncthreads();
    }
    vp_count(marks, newc, 0u, counts);
}

// Owned active hit nodes f (not blocked) with an out-neighbour vn that is gated at l+1 (vn not in K,
// a_vn > l+1) and lacks one of f's keywords: f retries (Alg. 2 ln 17-19), the work-list is not empty.
// hm is the state after level l; only called when level l made no mark, so it equals the state before.
__global__ void __launch_bounds__(kVpBlock) k_vp_waiting(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ col_idx,
                                                         const uint8_t *__restrict__ hm, const uint8_t *__restrict__ gate,
                                                         const uint8_t *__restrict__ act, int block_central, int64_t lo,
                                                         int64_t hi, int l, uint32_t full, unsigned long long *counts) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    unsigned wait = 0;
    for (int64_t f = lo + blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); f < hi; f += warps) {
        const uint32_t h = hm[f];
        if (!h || (block_central && h == full) || act[f] > l) continue;
        bool any = false;
        for (int64_t e = row_ptr[f] + lane; e < row_ptr[f + 1] && !any; e += 32) {
            const int32_t vn = __ldg(col_idx + e);
            any = gate[vn] > (uint32_t)(l + 1) && (h & ~(uint32_t)hm[vn]);
            any = __any_sync(__activemask(), any);
        }
        any = __any_sync(0xffffffffu, any);
        if (lane == 0 && any) ++wait;
    }
    wait = __reduce_add_sync(0xffffffffu, wait);
    if (lane == 0 && wait) atomicAdd(counts + 2, (unsigned long long)wait);
}

// owned nodes with more than kVpBig in-arcs
__global__ void k_vp_biglist(const int64_t *__restrict__ in_ptr, int64_t lo, int64_t hi, int32_t *big, int32_t *nbig) {
    for (int64_t x = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < hi; x += (int64_t)gridDim.x * blockDim.x)
        if (in_ptr[x + 1] - in_ptr[x] > kVpBig) big[atomicAdd(nbig, 1)] = (int32_t)x;
}

// engine status word of the replicated final state: hm | K << 8 | (nm = 0) | a << 24 (DevWork::st); the
// engine's gate is 0 when K is set, else a: K = (gate == 0) gives the same gate for every node
__global__ void k_vp_pack_st(const uint8_t *__restrict__ hm, const uint8_t *__restrict__ gate,
                             const uint8_t *__restrict__ act, int64_t n, uint32_t *__restrict__ st) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        st[v] = (uint32_t)hm[v] | (gate[v] == 0 ? 0x100u : 0u) | ((uint32_t)act[v] << 24);
}

// sparse exchange: the gathered (id << 8 | mask) lists of every rank into the replicated hit masks
__global__ void k_vp_apply(const long long *__restrict__ list, int64_t cnt, uint8_t *__restrict__ hm) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < cnt; j += (int64_t)gridDim.x * blockDim.x) {
        const long long e = list[j];
        if (e >= 0) hm[e >> 8] = (uint8_t)(e & 0xFF);
    }
}

static int vp_grid(int64_t items, int per_block) {
    int64_t g = (items + per_block - 1) / per_block;
    if (g > device_sm_count() * 16) g = device_sm_count() * 16;
    return g < 1 ? 1 : (int)g;
}

cudaError_t launch_vp_begin(const DevGraph &g, const VpQuery &qd, const uint8_t *act, const VpBufs &b, uint8_t *gate,
                            cudaStream_t s) {
    cudaMemsetAsync(b.hm, 0, (size_t)b.n_pad, s);
    cudaMemcpyAsync(gate, act, (size_t)g.n, cudaMemcpyDeviceToDevice, s);
    cudaMemsetAsync(b.counts, 0, 4 * sizeof(unsigned long long), s);
    cudaMemsetAsync(b.cent_n, 0, sizeof(int32_t), s);
    k_vp_init<<<device_sm_count() * 4, kVpBlock, 0, s>>>(g.kw_ptr, g.kw_nodes, qd, b.hm, gate, b.M);
    k_vp_ident0<<<vp_grid(b.hi - b.lo, kVpBlock), kVpBlock, 0, s>>>(b.hm, b.lo, b.hi, qd.full, b.cent, b.cdep,
                                                                       b.cent_n, b.counts);
    return cudaGetLastError();
}

cudaError_t launch_vp_biglist(const DevGraph &g, int64_t lo, int64_t hi, int32_t *big, int32_t *nbig, cudaStream_t s) {
    cudaMemsetAsync(nbig, 0, sizeof(int32_t), s);
    if (hi > lo) k_vp_biglist<<<vp_grid(hi - lo, kVpBlock), kVpBlock, 0, s>>>(g.in_ptr, lo, hi, big, nbig);
    return cudaGetLastError();
}

cudaError_t launch_vp_level(const DevGraph &g, const VpQuery &qd, const uint8_t *act, const VpBufs &b,
                            const uint8_t *gate, uint8_t *X, const int32_t *big, int nbig, int l, int block_central,
                            cudaStream_t s) {
    cudaMemsetAsync(b.counts, 0, 4 * sizeof(unsigned long long), s);
    k_vp_expmask<<<vp_grid(b.n_pad / 16, kVpBlock), kVpBlock, 0, s>>>(b.hm, act, b.n_pad, g.n, l, qd.full,
                                                                        block_central, X);
    if (b.hi > b.lo)
        k_vp_pull<<<vp_grid(b.hi - b.lo, kVpBlock / 32), kVpBlock, 0, s>>>(
            g.in_ptr, g.in_idx, b.hm, X, gate, act, block_central, b.lo, b.hi, l, qd.full, b.hm_slice, b.M, b.cent,
            b.cdep, b.cent_n, b.counts, b.chg);
    if (nbig)
        k_vp_pull_big<<<nbig < device_sm_count() * 4 ? nbig : device_sm_count() * 4, kVpBlock, 0, s>>>(
            g.in_ptr, g.in_idx, b.hm, X, gate, big, nbig, b.lo, l, qd.full, b.hm_slice, b.M, b.cent, b.cdep, b.cent_n,
            b.counts, b.chg);
    return cudaGetLastError();
}

cudaError_t launch_vp_waiting(const DevGraph &g, const VpQuery &qd, const uint8_t *act, const VpBufs &b,
                              const uint8_t *gate, int l, int block_central, cudaStream_t s) {
    cudaMemsetAsync(b.counts, 0, 4 * sizeof(unsigned long long), s);
    if (b.hi > b.lo)
        k_vp_waiting<<<vp_grid(b.hi - b.lo, kVpBlock / 32), kVpBlock, 0, s>>>(g.row_ptr, g.col_idx, b.hm, gate, act,
                                                                             block_central, b.lo, b.hi, l, qd.full,
                                                                             b.counts);
    return cudaGetLastError();
}

cudaError_t launch_vp_apply(const long long *list, int64_t cnt, uint8_t *hm, cudaStream_t s) {
    if (cnt > 0) k_vp_apply<<<vp_grid(cnt, kVpBlock), kVpBlock, 0, s>>>(list, cnt, hm);
    return cudaGetLastError();
}

cudaError_t launch_vp_pack_st(const uint8_t *hm, const uint8_t *gate, const uint8_t *act, int64_t n, uint32_t *st,
                              cudaStream_t s) {
    if (n > 0) k_vp_pack_st<<<vp_grid(n, kVpBlock), kVpBlock, 0, s>>>(hm, gate, act, n, st);
    return cudaGetLastError();
}

}  // namespace kgs
