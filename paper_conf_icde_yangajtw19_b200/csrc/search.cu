// search.cu — bottom-up search of the Central Graph method on sm_100a (product CUDA path).
//
//   k_activation   Eqs. 3-5: w, alpha, A -> uint8 activation level a, cached per alpha.
//   k_search       Alg. 1 ln 1-7 + Alg. 2 (L244-284) as ONE persistent cooperative kernel:
//                  reset -> initialise M / sources (L254) -> per level { merge new hits + identify
//                  central nodes (L262-266, Lemma V.1) -> termination (Def. 4, Thm. V.3) -> expansion
//                  (Alg. 2, gated by a, L210) } with two grid barriers per level and no host round trip.
//
// Data layout:
//   st[v]   uint16: low byte = hit mask hm (bit i <=> M[v][i] finite, snapshot at the start of the level),
//           high byte = gate (0 if v contains a query keyword, else a_v).  One 2-byte load per inspected arc.
//   nm[v]   uint8 (packed in 32-bit words for atomicOr): bits newly hit during the current level.
//   M[v*8+i] uint8 hitting level, written once per (v, i) by the thread that set the bit; never reset.
//   Frontier: three degree-class rings (light / heavy / huge) of R = amax+2 level slots, deduplicated by
//   a bitmap per slot.  A node is re-queued exactly at the level where it can make progress again:
//   a_v if it is not yet active (Alg. 2 ln 5-7), gate(n)-1 if a neighbour n is still gated (ln 18-19).
//
// Snapshot semantics (reading R10): expansion at level l reads hm as of the start of the level; new hits
// accumulate in nm and are merged in the next merge phase, so the result equals the sequential Alg. 2
// (Thm. V.2).  All writes are idempotent (bits OR-ed, level l+1 written once).
#include <cooperative_groups.h>

#include "kgs_internal.h"

namespace cg = cooperative_groups;

namespace kgs {

// ------------------------------------------------------------------------------------------ activation
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
        if (grid > 148 * 16) grid = 148 * 16;
        k_activation<<<grid, 256, 0, s>>>(w, n, A, alpha, act, amax);
    }
    return cudaGetLastError();
}

__global__ void k_degree_class(const int64_t *__restrict__ rp, int64_t n, uint8_t *__restrict__ cls) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int64_t d = rp[v + 1] - rp[v];
        cls[v] = d > kHugeDeg ? CLS_HUGE : (d > kHeavyDeg ? CLS_HEAVY : CLS_LIGHT);
    }
}
cudaError_t launch_degree_class(const int64_t *row_ptr, int64_t n, uint8_t *cls, cudaStream_t s) {
    if (n > 0) {
        int grid = (int)((n + 255) / 256);
        if (grid > 148 * 16) grid = 148 * 16;
        k_degree_class<<<grid, 256, 0, s>>>(row_ptr, n, cls);
    }
    return cudaGetLastError();
}

// Reading R15: weights on the 2^-24 grid make every fp64 sum of Eq. 6 exact and order-independent.
__global__ void k_snap(float *w, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const double x = (double)w[v] * 16777216.0;
        w[v] = (float)(floor(x + 0.5) * (1.0 / 16777216.0));
    }
}
cudaError_t launch_snap_weights(float *w, int64_t n, cudaStream_t s) {
    if (n > 0) {
        int grid = (int)((n + 255) / 256);
        if (grid > 148 * 16) grid = 148 * 16;
        k_snap<<<grid, 256, 0, s>>>(w, n);
    }
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------ helpers
__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31u; }
__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned r;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
    return r;
}

// Append to a list with one atomic per group of converged lanes sharing the same counter.
__device__ __forceinline__ uint32_t agg_slot(uint32_t *counter, unsigned key) {
    const unsigned mask = __activemask();
    const unsigned peers = __match_any_sync(mask, key);
    const int leader = __ffs(peers) - 1;
    const int rank = __popc(peers & lanemask_lt());
    uint32_t base = 0;
    if ((int)lane_id() == leader) base = atomicAdd(counter, (uint32_t)__popc(peers));
    base = __shfl_sync(peers, base, leader);
    return base + rank;
}

// phase timestamp by the grid's first thread (read back into kgs_stats-like debug output)
#define KGS_STAMP(tag)                                                                            \
    do {                                                                                          \
        if (gtid == 0) {                                                                          \
            const int _i = ctl->n_stamp;                                                          \
            if (_i < 64) { ctl->stamp[_i] = globaltimer_ns(); ctl->stamp_tag[_i] = (tag); ctl->n_stamp = _i + 1; } \
        }                                                                                         \
    } while (0)

// Schedule node v for the joint frontier of level L (FIdentifier[v] <- 1 for level L).
__device__ __forceinline__ void push(const QueryArgs &a, int R, int32_t v, int L) {
    const int s = L % R;
    uint32_t *word = a.w.fbits + (int64_t)s * a.w.W + (v >> 5);
    const uint32_t bit = 1u << (v & 31);
    if (__ldcg(word) & bit) return;
    if (atomicOr(word, bit) & bit) return;
    const int c = a.g.cls[v];
    const uint32_t pos = agg_slot(&a.w.ctl->qcount[c][s], (unsigned)((c << 8) | s));
    a.w.ring[c][(int64_t)s * a.w.cap[c] + pos] = v;
}

// One inspected arc v -> x of Alg. 2 ln 12-22, for all keywords of v at once (hmv = v's snapshot mask).
__device__ __forceinline__ void visit_arc(const QueryArgs &a, int R, int l, int32_t v, uint32_t hmv, int32_t x,
                                          unsigned long long &hits) {
    const uint32_t sx = __ldcg(a.w.st + x);
    const uint32_t bits = hmv & ~sx & 0xFFu;            // ln 13-15: only instances where x is unhit
    if (!bits) return;
    const uint32_t gate = sx >> 8;
    if (gate <= (uint32_t)(l + 1)) {                     // ln 16-18: keyword node or a_x <= l+1
        const uint32_t sh = (uint32_t)(x & 3) << 3;
        uint32_t *nw = a.w.nm + (x >> 2);
        const uint32_t cur = (__ldcg(nw) >> sh) & 0xFFu;
        if (!(bits & ~cur)) return;
        const uint32_t old = (atomicOr(nw, bits << sh) >> sh) & 0xFFu;
        const uint32_t nb = bits & ~old;
        if (nb) {
            hits += __popc(nb);
            uint8_t *row = a.w.M + (int64_t)x * 8;
            const uint8_t lv = (uint8_t)(l + 1);
#pragma unroll
            for (int i = 0; i < kMaxQ; ++i)
                if (nb & (1u << i)) row[i] = lv;          // ln 21: m_xi <- l+1
            if (old == 0) push(a, R, x, l + 1);           // ln 22: FIdentifier[x] <- 1 (first new bit)
        }
    } else {
        push(a, R, v, (int)gate - 1);                     // ln 19: v must retry when x opens
    }
}

// Alg. 2 ln 2-7 for node v at level l: returns its expansion mask (0 = does not expand now).
__device__ __forceinline__ uint32_t prepare(const QueryArgs &a, int R, int l, uint32_t full, int32_t v, bool leader) {
    const uint32_t hm = __ldcg(a.w.st + v) & 0xFFu;
    if (a.block_central && hm == full) return 0;          // ln 2-3: central nodes do not expand
    const int av = a.w.act[v];
    if (av > l) {                                          // ln 5-7: not yet active
        if (leader) push(a, R, v, av);
        return 0;
    }
    return hm;                                             // ln 8-11: every hit instance has m <= l
}

// ------------------------------------------------------------------------------------------ load balance
// Frontier nodes above kHeavyDeg (heavy and huge classes) are expanded in tiles of blockDim entries:
// every CTA computes the same tile prefix of degrees in shared memory, then the tile's arcs form one
// index space that all threads of the grid stride over (owner found by binary search).  A hub's arcs
// are thus spread over the whole GPU instead of one warp or one CTA.
__device__ __forceinline__ long long block_excl_scan64(long long x, long long *total, long long *sh) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
    long long incl = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const long long t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    __syncthreads();
    if (lane == 31) sh[wid] = incl;
    __syncthreads();
    if (threadIdx.x == 0) {
        long long acc = 0;
        for (int w = 0; w < nw; ++w) { const long long t = sh[w]; sh[w] = acc; acc += t; }
        sh[32] = acc;
    }
    __syncthreads();
    const long long r = sh[wid] + incl - x;
    *total = sh[32];
    __syncthreads();
    return r;
}

constexpr int kTileMax = 512;   // == blockDim of the persistent kernel

struct FwdNode {
    int32_t v;
    uint32_t hm;
};

template <class NodeT>
struct BigTile {
    long long incl[kTileMax];
    long long start[kTileMax];
    NodeT node[kTileMax];
    long long scan[40];
};

template <class NodeT, class Prep, class Visit>
__device__ __forceinline__ void expand_big(const int32_t *ring1, uint32_t c1, const int32_t *ring2, uint32_t c2,
                                           const int64_t *ptr, const int32_t *idx, BigTile<NodeT> &S, int64_t gtid,
                                           int64_t gsz, Prep prep, Visit visit, unsigned long long &arcs) {
    const uint32_t cb = c1 + c2;
    for (uint32_t t0 = 0; t0 < cb; t0 += blockDim.x) {
        const int nt = (int)min((uint32_t)blockDim.x, cb - t0);
        const int j = threadIdx.x;
        long long deg = 0, st = 0;
        if (j < nt) {
            const uint32_t e = t0 + j;
            const int32_t v = e < c1 ? ring1[e] : ring2[e - c1];
            NodeT nd;
            if (prep(v, blockIdx.x == 0, nd)) { st = ptr[v]; deg = ptr[v + 1] - st; }
            S.node[j] = nd;
            S.start[j] = st;
        }
        long long T;
        const long long ex = block_excl_scan64(deg, &T, S.scan);
        S.incl[j] = ex + deg;
        __syncthreads();
        if (gtid == 0) arcs += (unsigned long long)T;
        for (long long e = gtid; e < T; e += gsz) {
            int lo = 0, hi = nt - 1;
            while (lo < hi) {
                const int mid = (lo + hi) >> 1;
                if (S.incl[mid] > e) hi = mid; else lo = mid + 1;
            }
            const long long exo = lo ? S.incl[lo - 1] : 0;
            visit(S.node[lo], __ldcs(idx + S.start[lo] + (e - exo)));
        }
        __syncthreads();
    }
}

// light-batch size: 32 frontier nodes per warp when the frontier is large, fewer (down to 1) when it
// is small, so that every warp of the grid gets work
__device__ __forceinline__ uint32_t light_batch(uint32_t c0, int64_t gsz) {
    const uint32_t warps = (uint32_t)(gsz >> 5);
    uint32_t b = (c0 + 2 * warps - 1) / (2 * warps);
    return b < 1 ? 1u : (b > 32 ? 32u : b);
}

// ------------------------------------------------------------------------------------------ pre-pass
// Shared predecessor DAG (top-down): whether u -> x is a B_i-predecessor arc
// (Thm. V.4 + reading R12) depends only on M, a and K, never on the central node whose graph is being
// extracted.  So the backward closure of ALL central nodes is computed once, level by level, with the
// same degree-balanced scheme as the expansion, and every arc that passes the test is stored in a CSR
// keyed by its successor.  Each Central Graph is then a walk over these short lists (topdown.cu).
__device__ __forceinline__ void pd_push(const QueryArgs &a, int slot, int32_t u) {
    const int c = a.g.cls_in[u];
    const uint32_t pos = agg_slot(&a.w.ctl->pd_qcount[c][slot], (unsigned)((c << 8) | slot));
    a.w.pd_ring[c][(int64_t)slot * a.w.pd_cap[c] + pos] = u;
}

// Thm. V.4 test of in-arc u -> x for the keyword bits P of x (hx = M row of x, gx = gate(x) - 1).
__device__ __forceinline__ uint32_t pred_test(const QueryArgs &a, uint32_t full, bool exact_block, uint32_t P,
                                              uint64_t hx, int gx, int32_t u, uint32_t &zbu) {
    const uint32_t hmu = __ldcg(a.w.st + u) & 0xFFu;
    const uint32_t cand = P & hmu;
    if (!cand) return 0;
    const int au = a.w.act[u];
    const uint64_t Mu = __ldcg(reinterpret_cast<const unsigned long long *>(a.w.M) + u);
    uint32_t pb = 0, zb = 0;
    int maxrow = 0;
#pragma unroll
    for (int i = 0; i < kMaxQ; ++i) {
        if (!((hmu >> i) & 1u)) continue;
        const int mu = (int)((Mu >> (8 * i)) & 0xFF);
        maxrow = maxrow > mu ? maxrow : mu;
        if (mu == 0) zb |= 1u << i;
        if (!((cand >> i) & 1u)) continue;
        int need = au > mu ? au : mu;
        need = need > gx ? need : gx;
        if ((int)((hx >> (8 * i)) & 0xFF) == need + 1) pb |= 1u << i;   // m_xi = 1 + max{a_u, m_ui, g_x}
    }
    if (pb && exact_block && hmu == full) {
#pragma unroll
        for (int i = 0; i < kMaxQ; ++i)   // u central at depth maxrow: it only expanded at levels < maxrow
            if (((pb >> i) & 1u) && maxrow <= (int)((hx >> (8 * i)) & 0xFF) - 1) pb &= ~(1u << i);
    }
    zbu = zb;
    return pb;
}

__device__ __forceinline__ void pd_visit(const QueryArgs &a, uint32_t full, bool exact_block, uint32_t P, uint64_t hx,
                                         int gx, int32_t cidx, int32_t u, int nslot) {
    uint32_t zbu = 0;
    const uint32_t pb = pred_test(a, full, exact_block, P, hx, gx, u, zbu);
    if (!pb) return;
    const uint32_t pos = agg_slot(reinterpret_cast<uint32_t *>(a.w.pcnt + cidx), (unsigned)cidx);
    const uint32_t ai = agg_slot(&a.w.ctl->n_parcs, 0xFFFFFFFFu);
    if ((int64_t)ai < a.w.pcap) {
        a.w.pa_u[ai] = u;
        a.w.pa_x[ai] = cidx;
        a.w.pa_b[ai] = (uint16_t)(pb | (zbu << 8));
        a.w.pa_slot[ai] = (int32_t)pos;
    } else {
        atomicExch(&a.w.ctl->fatal, 5);
    }
    const uint32_t nb = pb & ~zbu;        // sources (m = 0) have no predecessors
    if (nb) {
        const uint32_t old = atomicOr(a.w.pd_state + u, nb << 8);
        if (((old >> 8) & 0xFFu) == 0) pd_push(a, nslot, u);
    }
}

struct PdNode {
    uint32_t P;
    uint64_t hx;
    int gx;
    int32_t cidx;
};

__device__ __forceinline__ PdNode pd_prepare(const QueryArgs &a, int32_t x) {
    PdNode nd;
    nd.P = __ldcg(a.w.pd_state + x) & 0xFFu;
    nd.hx = __ldcg(reinterpret_cast<const unsigned long long *>(a.w.M) + x);
    nd.gx = (int)(__ldcg(a.w.st + x) >> 8) - 1;
    nd.cidx = __ldcg(a.w.pd_cid + x);
    return nd;
}

__device__ __forceinline__ int block_excl_scan(int x, int *total, int *sh) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
    int incl = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    __syncthreads();
    if (lane == 31) sh[wid] = incl;
    __syncthreads();
    if (threadIdx.x == 0) {
        int acc = 0;
        for (int w = 0; w < nw; ++w) { const int t = sh[w]; sh[w] = acc; acc += t; }
        sh[32] = acc;
    }
    __syncthreads();
    const int r = sh[wid] + incl - x;
    *total = sh[32];
    __syncthreads();
    return r;
}

__device__ void pred_dag(const QueryArgs &a, cg::grid_group &grid, int64_t gtid, int64_t gsz, uint32_t full) {
    Ctl *ctl = a.w.ctl;
    const bool exact_block = a.extract_mode == KGS_EXTRACT_EXACT && a.block_central;
    const uint32_t nc = __ldcg(&ctl->n_central);
    __shared__ BigTile<PdNode> s_bigb;
    // seeds: every central node, for every keyword it did not contain itself
    for (int64_t j = gtid; j < nc; j += gsz) {
        const int32_t c = a.w.centrals[j];
        const uint64_t Mc = __ldcg(reinterpret_cast<const unsigned long long *>(a.w.M) + c);
        uint32_t zbc = 0;
        for (int i = 0; i < a.q; ++i) if (((Mc >> (8 * i)) & 0xFF) == 0) zbc |= 1u << i;
        const uint32_t bits = full & ~zbc;
        if (bits) { atomicOr(a.w.pd_state + c, bits << 8); pd_push(a, 0, c); }
    }
    grid.sync();
    KGS_STAMP(TS_PD_SEED);
    unsigned long long my_arcs = 0;
    int r = 0;
    for (;; ++r) {
        const int slot = r & 1;
        const uint32_t c0 = __ldcg(&ctl->pd_qcount[0][slot]), c1 = __ldcg(&ctl->pd_qcount[1][slot]),
                       c2 = __ldcg(&ctl->pd_qcount[2][slot]);
        const int64_t total = (int64_t)c0 + c1 + c2;
        if (total == 0) break;
        if (gtid == 0) { ctl->pd_qcount[0][slot ^ 1] = 0; ctl->pd_qcount[1][slot ^ 1] = 0; ctl->pd_qcount[2][slot ^ 1] = 0; }
        // merge: bits to expand this round = newly requested bits not expanded before
        for (int64_t j = gtid; j < total; j += gsz) {
            int32_t u;
            if (j < c0) u = a.w.pd_ring[0][(int64_t)slot * a.w.pd_cap[0] + j];
            else if (j < (int64_t)c0 + c1) u = a.w.pd_ring[1][(int64_t)slot * a.w.pd_cap[1] + (j - c0)];
            else u = a.w.pd_ring[2][(int64_t)slot * a.w.pd_cap[2] + (j - c0 - c1)];
            const uint32_t s = __ldcg(a.w.pd_state + u);
            const uint32_t nx = (s >> 8) & 0xFFu, dn = (s >> 16) & 0xFFu;
            const uint32_t bits = nx & ~dn;
            a.w.pd_state[u] = bits | ((dn | bits) << 16);
            if (bits && __ldcg(a.w.pd_cid + u) < 0) {
                const uint32_t cid = agg_slot(&ctl->n_cid, 1u);
                a.w.pd_cid[u] = (int32_t)cid;
                a.w.pd_touched[cid] = u;
            }
        }
        grid.sync();
        KGS_STAMP(TS_PD_MERGE);
        const int ns = slot ^ 1;
        // heavy and huge nodes: tiles spread over the whole grid
        expand_big(a.w.pd_ring[1] + (int64_t)slot * a.w.pd_cap[1], c1, a.w.pd_ring[2] + (int64_t)slot * a.w.pd_cap[2],
                   c2, a.g.in_ptr, a.g.in_idx, s_bigb, gtid, gsz,
                   [&](int32_t x, bool, PdNode &nd) {
                       nd = pd_prepare(a, x);
                       return nd.P != 0;
                   },
                   [&](const PdNode &nd, int32_t u) { pd_visit(a, full, exact_block, nd.P, nd.hx, nd.gx, nd.cidx, u, ns); },
                   my_arcs);
        const unsigned lane = lane_id();
        const uint32_t B = light_batch(c0, gsz);
        for (;;) {                                                 // light: warp batches
            uint32_t base = 0;
            if (lane == 0) base = atomicAdd(&ctl->pd_work[r & 255], B);
            base = __shfl_sync(0xffffffffu, base, 0);
            if (base >= c0) break;
            const uint32_t idx = base + lane;
            PdNode nd{0, 0, 0, -1};
            int64_t start = 0;
            int deg = 0;
            if (lane < B && idx < c0) {
                const int32_t x = a.w.pd_ring[0][(int64_t)slot * a.w.pd_cap[0] + idx];
                nd = pd_prepare(a, x);
                if (nd.P) { start = a.g.in_ptr[x]; deg = (int)(a.g.in_ptr[x + 1] - start); }
            }
            int incl = deg;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int t = __shfl_up_sync(0xffffffffu, incl, o);
                if ((int)lane >= o) incl += t;
            }
            const int tot = __shfl_sync(0xffffffffu, incl, 31);
            if (lane == 0) my_arcs += (unsigned long long)tot;
            const int excl = incl - deg;
            for (int e0 = 0; e0 < tot; e0 += 32) {
                const int e = e0 + (int)lane;
                int pos = 0;
#pragma unroll
                for (int bb = 16; bb > 0; bb >>= 1) {
                    const int val = __shfl_sync(0xffffffffu, incl, pos + bb - 1);
                    if (val <= e) pos += bb;
                }
                const int64_t st_o = __shfl_sync(0xffffffffu, start, pos);
                const int ex_o = __shfl_sync(0xffffffffu, excl, pos);
                const uint32_t P_o = __shfl_sync(0xffffffffu, nd.P, pos);
                const uint64_t hx_o = __shfl_sync(0xffffffffu, (unsigned long long)nd.hx, pos);
                const int gx_o = __shfl_sync(0xffffffffu, nd.gx, pos);
                const int32_t cid_o = __shfl_sync(0xffffffffu, nd.cidx, pos);
                if (e < tot)
                    pd_visit(a, full, exact_block, P_o, hx_o, gx_o, cid_o, __ldcs(a.g.in_idx + st_o + (e - ex_o)), ns);
            }
        }
        grid.sync();
        KGS_STAMP(TS_PD_EXPAND);
    }
    if (my_arcs) atomicAdd(&ctl->td_arcs, my_arcs);
    if (gtid == 0) ctl->pd_rounds = r;
    // CSR of the predecessor lists: exclusive scan of pcnt over compact ids, then scatter
    __shared__ int sh[40];
    const int64_t ncid = (int64_t)__ldcg(&ctl->n_cid);
    const int64_t chunk = (ncid + gridDim.x - 1) / gridDim.x;
    const int64_t lo = (int64_t)blockIdx.x * chunk, hi = lo + chunk < ncid ? lo + chunk : ncid;
    int run = 0;
    for (int64_t t0 = lo; t0 < hi; t0 += blockDim.x) {
        const int64_t j = t0 + threadIdx.x;
        const int v = j < hi ? __ldcg(a.w.pcnt + j) : 0;
        int tot;
        const int ex = block_excl_scan(v, &tot, sh);
        if (j < hi) a.w.pred_ptr[j] = run + ex;
        run += tot;
    }
    if (threadIdx.x == 0) a.w.scan_tmp[blockIdx.x] = run;
    grid.sync();
    if (blockIdx.x == 0) {   // exclusive scan of the per-CTA sums (gridDim <= a few blockDim)
        int carry = 0;
        for (unsigned b0 = 0; b0 < gridDim.x; b0 += blockDim.x) {
            const unsigned b = b0 + threadIdx.x;
            const int v = b < gridDim.x ? __ldcg(a.w.scan_tmp + b) : 0;
            int tot;
            const int ex = block_excl_scan(v, &tot, sh);
            if (b < gridDim.x) a.w.scan_tmp[b] = carry + ex;
            carry += tot;
        }
        if (threadIdx.x == 0) a.w.pred_ptr[ncid] = carry;
    }
    grid.sync();
    const int off = __ldcg(a.w.scan_tmp + blockIdx.x);
    for (int64_t j = lo + threadIdx.x; j < hi; j += blockDim.x) a.w.pred_ptr[j] += off;
    grid.sync();
    KGS_STAMP(TS_PD_CSR);
    const int64_t np = (int64_t)__ldcg(&ctl->n_parcs) < a.w.pcap ? (int64_t)__ldcg(&ctl->n_parcs) : a.w.pcap;
    for (int64_t ai = gtid; ai < np; ai += gsz) {
        const int64_t pos = (int64_t)__ldcg(a.w.pred_ptr + a.w.pa_x[ai]) + a.w.pa_slot[ai];
        a.w.pred_u[pos] = a.w.pa_u[ai];
        a.w.pred_b[pos] = a.w.pa_b[ai];
    }
}

// ------------------------------------------------------------------------------------------ search
__global__ void __launch_bounds__(512, 2) k_search(QueryArgs a) {
    cg::grid_group grid = cg::this_grid();
    const int64_t gtid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t gsz = (int64_t)gridDim.x * blockDim.x;
    const int64_t n = a.g.n;
    const int R = a.w.R;
    const int amax = R - 2;
    const uint32_t full = (1u << a.q) - 1u;
    Ctl *ctl = a.w.ctl;
    uint8_t *st8 = reinterpret_cast<uint8_t *>(a.w.st);
    uint8_t *nm8 = reinterpret_cast<uint8_t *>(a.w.nm);
    __shared__ BigTile<FwdNode> s_big;
    KGS_STAMP(TS_START);

    // ---- reset the state the previous query left behind
    if (a.full_reset) {
        for (int64_t v = gtid; v < n; v += gsz) a.w.st[v] = (uint16_t)((uint16_t)a.w.act[v] << 8);
        for (int64_t v = gtid; v < (n + 3) / 4; v += gsz) a.w.nm[v] = 0u;
        for (int64_t j = gtid; j < (int64_t)R * a.w.W; j += gsz) a.w.fbits[j] = 0u;
        for (int64_t v = gtid; v < n; v += gsz) { a.w.pd_state[v] = 0u; a.w.pd_cid[v] = -1; a.w.pcnt[v] = 0; }
    } else {
        for (int64_t j = gtid; j < (int64_t)a.w.prev->n_cid; j += gsz) {
            const int32_t v = a.w.pd_touched[j];
            a.w.pd_state[v] = 0u; a.w.pd_cid[v] = -1; a.w.pcnt[j] = 0;
        }
        const Ctl *pv = a.w.prev;
        const int64_t pt = (int64_t)pv->n_touched;
        if (pt > n / 16) {   // many touched rows: a dense sweep beats scattered 2-byte writes
            for (int64_t v = gtid; v < n; v += gsz) a.w.st[v] = (uint16_t)((uint16_t)a.w.act[v] << 8);
        } else
        for (int64_t j = gtid; j < pt; j += gsz) {
            const int32_t v = a.w.touched[j];
            a.w.st[v] = (uint16_t)((uint16_t)a.w.act[v] << 8);
        }
        for (int c = 0; c < 3; ++c)
            for (int s = 0; s < a.prev_R; ++s) {
                const uint32_t cnt = pv->qcount[c][s];
                for (int64_t j = gtid; j < (int64_t)cnt; j += gsz) {
                    const int32_t v = a.w.ring[c][(int64_t)s * a.w.cap[c] + j];
                    a.w.fbits[(int64_t)s * a.w.W + (v >> 5)] = 0u;
                }
            }
    }
    // ---- initialisation: M = 0 on T_i, keyword nodes ungated, F_0 = K
    bool empty = false;
    for (int i = 0; i < a.q; ++i) {
        const int32_t t = a.w.kw_dev[i];
        if (a.g.kw_ptr[t + 1] == a.g.kw_ptr[t]) empty = true;
    }
    grid.sync();
    KGS_STAMP(TS_RESET);
    for (int i = 0; i < a.q; ++i) {
        const int32_t t = a.w.kw_dev[i];
        const int64_t b = a.g.kw_ptr[t], e = a.g.kw_ptr[t + 1];
        for (int64_t j = b + gtid; j < e; j += gsz) {
            const int32_t v = a.g.kw_nodes[j];
            a.w.M[(int64_t)v * 8 + i] = 0;
            st8[2 * (int64_t)v + 1] = 0;                                  // keyword node: no gate (L210)
            atomicOr(a.w.nm + (v >> 2), (1u << i) << ((v & 3) * 8));      // hit in B_i at level 0
            push(a, R, v, 0);
        }
    }
    grid.sync();
    KGS_STAMP(TS_SCATTER);

    unsigned long long my_arcs = 0, my_hits = 0;
    for (int l = 0;; ++l) {
        // ---- enqueue frontiers: anything pending at this or a later level?
        uint32_t pend = 0;
        const int top = l > amax ? l : amax;
        for (int L = l; L <= top; ++L) {
            const int s = L % R;
            pend += __ldcg(&ctl->qcount[0][s]) + __ldcg(&ctl->qcount[1][s]) + __ldcg(&ctl->qcount[2][s]);
        }
        if (pend == 0) {
            if (gtid == 0) { ctl->stop_reason = empty ? KGS_STOP_EMPTY_KEYWORD : KGS_STOP_EXHAUSTED; ctl->levels = l; }
            break;
        }
        const int s = l % R;
        const uint32_t c0 = __ldcg(&ctl->qcount[0][s]), c1 = __ldcg(&ctl->qcount[1][s]),
                       c2 = __ldcg(&ctl->qcount[2][s]);
        const int64_t total = (int64_t)c0 + c1 + c2;
        // ---- merge new hits into hm and identify central nodes (only frontiers can change, L262)
        for (int64_t j = gtid; j < total; j += gsz) {
            int32_t v;
            if (j < c0) v = a.w.ring[0][(int64_t)s * a.w.cap[0] + j];
            else if (j < (int64_t)c0 + c1) v = a.w.ring[1][(int64_t)s * a.w.cap[1] + (j - c0)];
            else v = a.w.ring[2][(int64_t)s * a.w.cap[2] + (j - c0 - c1)];
            a.w.fbits[(int64_t)s * a.w.W + (v >> 5)] = 0u;
            const uint32_t b = nm8[v];
            if (b) {
                nm8[v] = 0;
                const uint32_t old = st8[2 * (int64_t)v];
                const uint32_t nw = old | b;
                st8[2 * (int64_t)v] = (uint8_t)nw;
                if (old == 0) a.w.touched[agg_slot(&ctl->n_touched, 0u)] = v;
                if (nw == full && old != full) {                            // Lemma V.1: depth = l
                    const uint32_t ci = agg_slot(&ctl->n_central, 1u);
                    a.w.centrals[ci] = v;
                    a.w.cdepth[ci] = (uint8_t)l;
                }
            }
        }
        if (gtid == 0) ctl->frontier_total += (unsigned long long)total;
        grid.sync();
        KGS_STAMP(TS_MERGE);
        if (gtid == 0 && l > 0) {
            const int sp = (l - 1) % R;
            ctl->qcount[0][sp] = 0; ctl->qcount[1][sp] = 0; ctl->qcount[2][sp] = 0;
        }
        // ---- termination (Def. 4 / Thm. V.3; reading R9: no expansion at d)
        if (empty) {   // some T_i is empty: M holds the initialisation, nothing can be central (R17)
            if (gtid == 0) { ctl->stop_reason = KGS_STOP_EMPTY_KEYWORD; ctl->levels = 0; ctl->empty_keyword = 1; }
            break;
        }
        const uint32_t nc = __ldcg(&ctl->n_central);
        if (nc >= (uint32_t)a.k) {
            if (gtid == 0) { ctl->stop_reason = KGS_STOP_K; ctl->levels = l; }
            break;
        }
        if (l == a.max_depth) {
            if (gtid == 0) { ctl->stop_reason = KGS_STOP_MAX_DEPTH; ctl->levels = l; }
            break;
        }
        // ---- expansion (Alg. 2)
        // heavy and huge nodes: tiles whose arcs are spread over the whole grid
        expand_big(a.w.ring[1] + (int64_t)s * a.w.cap[1], c1, a.w.ring[2] + (int64_t)s * a.w.cap[2], c2,
                   a.g.row_ptr, a.g.col_idx, s_big, gtid, gsz,
                   [&](int32_t v, bool leader, FwdNode &nd) {
                       nd.v = v;
                       nd.hm = prepare(a, R, l, full, v, leader);
                       return nd.hm != 0;
                   },
                   [&](const FwdNode &nd, int32_t x) { visit_arc(a, R, l, nd.v, nd.hm, x, my_hits); }, my_arcs);
        // light nodes: dynamic batches of frontier nodes per warp, arcs balanced across the lanes
        const unsigned lane = lane_id();
        const uint32_t B = light_batch(c0, gsz);
        for (;;) {
            uint32_t base = 0;
            if (lane == 0) base = atomicAdd(&ctl->work[l], B);
            base = __shfl_sync(0xffffffffu, base, 0);
            if (base >= c0) break;
            const uint32_t idx = base + lane;
            int32_t v = -1;
            uint32_t hm = 0;
            int64_t start = 0;
            int deg = 0;
            if (lane < B && idx < c0) {
                v = a.w.ring[0][(int64_t)s * a.w.cap[0] + idx];
                hm = prepare(a, R, l, full, v, true);
                if (hm) {
                    start = a.g.row_ptr[v];
                    deg = (int)(a.g.row_ptr[v + 1] - start);
                }
            }
            int incl = deg;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int t = __shfl_up_sync(0xffffffffu, incl, o);
                if ((int)lane >= o) incl += t;
            }
            const int tot = __shfl_sync(0xffffffffu, incl, 31);
            if (lane == 0) my_arcs += (unsigned long long)tot;
            const int excl = incl - deg;
            for (int e0 = 0; e0 < tot; e0 += 32) {
                const int e = e0 + (int)lane;
                int pos = 0;
#pragma unroll
                for (int b = 16; b > 0; b >>= 1) {
                    const int val = __shfl_sync(0xffffffffu, incl, pos + b - 1);
                    if (val <= e) pos += b;
                }
                const int64_t st_o = __shfl_sync(0xffffffffu, start, pos);
                const int ex_o = __shfl_sync(0xffffffffu, excl, pos);
                const uint32_t hm_o = __shfl_sync(0xffffffffu, hm, pos);
                const int32_t v_o = __shfl_sync(0xffffffffu, v, pos);
                if (e < tot) visit_arc(a, R, l, v_o, hm_o, __ldcs(a.g.col_idx + st_o + (e - ex_o)), my_hits);
            }
        }
        grid.sync();
        KGS_STAMP(TS_EXPAND);
    }
    my_arcs = __reduce_add_sync(0xffffffffu, (unsigned)my_arcs) + 0ull;   // per-warp totals fit 32 bits
    my_hits = __reduce_add_sync(0xffffffffu, (unsigned)my_hits) + 0ull;
    if ((threadIdx.x & 31) == 0) {
        if (my_arcs) atomicAdd(&ctl->arcs_scanned, my_arcs);
        if (my_hits) atomicAdd(&ctl->hits, my_hits);
    }
    grid.sync();
    KGS_STAMP(TS_END);
    pred_dag(a, grid, gtid, gsz, full);
}

int search_max_grid(int device, int block) {
    int per_sm = 0, sms = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_search, block, 0);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    return per_sm * sms;
}

cudaError_t launch_search(const QueryArgs &a, int grid, int block, cudaStream_t s) {
    void *args[] = {(void *)&a};
    return cudaLaunchCooperativeKernel((const void *)k_search, dim3(grid), dim3(block), args, 0, s);
}

}  // namespace kgs
