// search.cu — bottom-up search of the Central Graph method on sm_100a (product CUDA path).
//
//   k_activation   Eqs. 3-5: w, alpha, A -> uint8 activation level a, cached per alpha.
//   k_search       Alg. 1 ln 1-7 + Alg. 2 (L244-284) as ONE persistent cooperative kernel:
//                  reset -> initialise M / sources (L254) -> per level { enqueue frontiers = compact the
//                  level's bitmap, merge new hits, identify central nodes (L256-266, Lemma V.1) ->
//                  termination (Def. 4, Thm. V.3) -> expansion (Alg. 2, gated by a, L210) }, then the
//                  top-down pre-pass (shared predecessor DAG, see pred_dag), with two grid barriers per
//                  level and no host round trip.
//
// Data layout:
//   st[v]   uint16: low byte = hit mask hm (bit i <=> M[v][i] finite, snapshot at the start of the level),
//           high byte = gate (0 if v contains a query keyword, else a_v).  One 2-byte load per inspected arc.
//   nm[v]   uint8 (packed in 32-bit words for atomicOr): bits newly hit during the current level.
//   M[v*8+i] uint8 hitting level, written once per (v, i) by the thread that set the bit; never reset.
//   fbits   one frontier bitmap per level slot (R = amax+2 slots): "FIdentifier[v] <- 1 for level L" is one
//           atomicOr on a bitmap word, so pushes never contend on a queue counter.  A node is re-queued
//           exactly at the level where it can make progress again: a_v if it is not yet active (Alg. 2
//           ln 5-7), gate(n)-1 if a neighbour n is still gated (ln 18-19).
//   Each level starts by compacting its bitmap into light / big queues (block-aggregated appends, node
//   ids ascending within a CTA's word range); big nodes (> kBigDeg arcs) are expanded in tiles whose arcs
//   are spread over the whole grid, light ones by warp batches.
//
// Snapshot semantics (reading R10): expansion at level l reads hm as of the start of the level; new hits
// accumulate in nm and are merged when the next level is compacted, so the result equals the sequential
// Alg. 2 (Thm. V.2).  All writes are idempotent (bits OR-ed, level l+1 written once).
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
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        cls[v] = (rp[v + 1] - rp[v]) > kBigDeg ? CLS_BIG : CLS_LIGHT;
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

// phase timestamp by the grid's first thread (kgs_result_phases)
#define KGS_STAMP(tag)                                                                            \
    do {                                                                                          \
        if (gtid == 0) {                                                                          \
            const int _i = ctl->n_stamp;                                                          \
            if (_i < 64) { ctl->stamp[_i] = globaltimer_ns(); ctl->stamp_tag[_i] = (tag); ctl->n_stamp = _i + 1; } \
        }                                                                                         \
    } while (0)

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

// ------------------------------------------------------------------------------------------ frontier
// Set v's bit in bitmap `bits` (one level slot); `flag` records that the slot is non-empty.  The bit is
// set with a reduction (no return value: one round trip less); the flag is stored once per group of
// converged lanes.
__device__ __forceinline__ void set_bit(uint32_t *bits, uint32_t *flag, int32_t v) {
    uint32_t *word = bits + (v >> 5);
    const uint32_t bit = 1u << (v & 31);
    if (__ldcg(word) & bit) return;
    asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(word), "r"(bit) : "memory");
    const unsigned mask = __activemask();
    if ((int)lane_id() == __ffs(mask) - 1 && !__ldcg(flag)) *flag = 1u;   // stores to one line contend
}

// Schedule node v for the joint frontier of level L (FIdentifier[v] <- 1).
__device__ __forceinline__ void push(const QueryArgs &a, int R, int32_t v, int L) {
    const int s = L % R;
    set_bit(a.w.fbits + (int64_t)s * a.w.W, &a.w.ctl->slot_flag[s], v);
}

// Enqueue frontiers: compact a bitmap (which is cleared) into the light / big queues.
// on_node(v) runs once per set bit and returns whether v goes to the aux list; on_aux(v, pos) runs
// when v is written there.  Light and aux appends cost one atomic per CTA per tile of blockDim words.
constexpr int kWpt = 8;   // bitmap words per thread per compaction step (two 16-byte loads)

template <class OnNode, class OnAux>
__device__ __forceinline__ void compact(uint32_t *bits, int64_t W, const uint8_t *cls, int32_t *ql, uint32_t *nl,
                                        int32_t *qb, uint32_t *nb, int32_t *aux, uint32_t *naux, long long *sh,
                                        OnNode on_node, OnAux on_aux) {
    const int64_t step = (int64_t)blockDim.x * kWpt;                  // words per CTA iteration
    const int64_t cw = ((W + gridDim.x - 1) / gridDim.x + kWpt - 1) / kWpt * kWpt;
    const int64_t w0 = (int64_t)blockIdx.x * cw, w1 = w0 + cw < W ? w0 + cw : W;
    for (int64_t base = w0; base < w1; base += step) {
        const int64_t wi = base + (int64_t)threadIdx.x * kWpt;         // multiple of kWpt: 16-byte aligned
        uint32_t word[kWpt];
        if (wi + kWpt <= w1) {
            const uint4 x0 = __ldcg(reinterpret_cast<const uint4 *>(bits + wi));
            const uint4 x1 = __ldcg(reinterpret_cast<const uint4 *>(bits + wi + 4));
            word[0] = x0.x; word[1] = x0.y; word[2] = x0.z; word[3] = x0.w;
            word[4] = x1.x; word[5] = x1.y; word[6] = x1.z; word[7] = x1.w;
            if ((x0.x | x0.y | x0.z | x0.w) != 0u) *reinterpret_cast<uint4 *>(bits + wi) = make_uint4(0, 0, 0, 0);
            if ((x1.x | x1.y | x1.z | x1.w) != 0u) *reinterpret_cast<uint4 *>(bits + wi + 4) = make_uint4(0, 0, 0, 0);
        } else {
#pragma unroll
            for (int k = 0; k < kWpt; ++k) {
                word[k] = (wi + k < w1) ? __ldcg(bits + wi + k) : 0u;
                if (word[k]) bits[wi + k] = 0u;
            }
        }
        // (A) node ids of the set bits -> the CTA's segment of the frontier queue (stores only)
        int cnt = 0;
#pragma unroll
        for (int k = 0; k < kWpt; ++k) cnt += __popc(word[k]);
        long long tot;
        const long long ex = block_excl_scan64(cnt, &tot, sh);
        if (threadIdx.x == 0) sh[34] = tot ? (long long)atomicAdd(nl, (uint32_t)tot) : 0;
        __syncthreads();
        const uint32_t seg0 = (uint32_t)sh[34];
        uint32_t p = seg0 + (uint32_t)ex;
#pragma unroll
        for (int k = 0; k < kWpt; ++k)
            for (uint32_t m = word[k]; m; m &= m - 1) ql[p++] = (int32_t)((wi + k) * 32 + __ffs(m) - 1);
        __syncthreads();   // the segment is visible to the whole CTA
        // (B) one node per thread: on_node (merge / identify), big nodes moved to qb, aux appends
        for (long long c0 = 0; c0 < tot; c0 += blockDim.x) {
            const long long j = c0 + threadIdx.x;
            int32_t v = -1;
            int flag = 0;
            if (j < tot) {
                v = ql[seg0 + j];
                flag = on_node(v) ? 1 : 0;
                if (cls[v] != CLS_LIGHT) { qb[atomicAdd(nb, 1u)] = v; ql[seg0 + j] = -1; }
            }
            long long atot;
            const long long aex = block_excl_scan64(flag, &atot, sh);
            if (threadIdx.x == 0) sh[35] = atot ? (long long)atomicAdd(naux, (uint32_t)atot) : 0;
            __syncthreads();
            if (flag) {
                const uint32_t pos = (uint32_t)sh[35] + (uint32_t)aex;
                aux[pos] = v;
                on_aux(v, pos);
            }
        }
    }
}

// st[v] = a_v << 8 (hit mask 0, gate = a) for v in [0, n), 8 nodes per thread-step
__device__ __forceinline__ void reset_st_dense(uint16_t *st, const uint8_t *act, int64_t n, int64_t gtid, int64_t gsz) {
    const int64_t n8 = n / 8;
    for (int64_t j = gtid; j < n8; j += gsz) {
        const uint2 av = *reinterpret_cast<const uint2 *>(act + j * 8);
        uint4 o;
        o.x = ((av.x & 0xFFu) << 8) | ((av.x & 0xFF00u) << 16);
        o.y = ((av.x >> 8) & 0xFF00u) | ((av.x >> 24) << 24);
        o.z = ((av.y & 0xFFu) << 8) | ((av.y & 0xFF00u) << 16);
        o.w = ((av.y >> 8) & 0xFF00u) | ((av.y >> 24) << 24);
        *reinterpret_cast<uint4 *>(st + j * 8) = o;
    }
    for (int64_t v = n8 * 8 + gtid; v < n; v += gsz) st[v] = (uint16_t)((uint16_t)act[v] << 8);
}

// One inspected arc v -> x of Alg. 2 ln 12-22, for all keywords of v at once (hmv = v's snapshot mask).
// sx = st[x], gathered by the caller.
__device__ __forceinline__ void visit_arc(const QueryArgs &a, int R, int l, int32_t v, uint32_t hmv, int32_t x,
                                          uint32_t sx, unsigned &hits) {
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
// Big frontier nodes are expanded in tiles of blockDim entries: every CTA computes the same tile prefix of
// degrees in shared memory, then the tile's arcs form one index space that all threads of the grid stride
// over (owner found by binary search).  A hub's arcs are spread over the whole GPU.
constexpr int kTileMax = 512;   // == blockDim of the persistent kernel

struct FwdNode {
    int32_t v;
    uint32_t hm;
};

struct PdNode {
    uint32_t P;      // keyword bits to expand backwards
    uint64_t hx;     // M row of the node
    int gx;          // gate - 1
    int32_t cidx;    // compact id
};

template <class NodeT>
struct BigTile {
    long long incl[kTileMax];
    long long start[kTileMax];
    NodeT node[kTileMax];
};

constexpr int kBigUnroll = 4;
constexpr int kLightUnroll = 2;

template <class NodeT, class Prep, class Visit>
__device__ __forceinline__ void expand_big(const int32_t *qb, uint32_t cb, const int64_t *ptr, const int32_t *idx,
                                           const uint16_t *st, BigTile<NodeT> &S, long long *sh, int64_t gtid,
                                           int64_t gsz, Prep prep, Visit visit, unsigned long long &arcs) {
    for (uint32_t t0 = 0; t0 < cb; t0 += blockDim.x) {
        const int nt = (int)min((uint32_t)blockDim.x, cb - t0);
        const int j = threadIdx.x;
        long long deg = 0, s0 = 0;
        if (j < nt) {
            const int32_t v = __ldcg(qb + t0 + j);
            NodeT nd;
            if (prep(v, blockIdx.x == 0, nd)) { s0 = ptr[v]; deg = ptr[v + 1] - s0; }
            S.node[j] = nd;
            S.start[j] = s0;
        }
        long long T;
        const long long ex = block_excl_scan64(deg, &T, sh);
        S.incl[j] = ex + deg;
        __syncthreads();
        if (gtid == 0) arcs += (unsigned long long)T;
        // kBigUnroll arcs per thread per step: the index and status gathers of all of them are issued
        // before any of them is processed (memory-level parallelism for a latency-bound loop)
        for (long long e = gtid; e < T; e += kBigUnroll * gsz) {
            int own[kBigUnroll];
            int32_t x[kBigUnroll];
#pragma unroll
            for (int k = 0; k < kBigUnroll; ++k) {
                const long long ek = e + k * gsz;
                own[k] = -1;
                x[k] = 0;
                if (ek < T) {
                    int lo = 0, hi = nt - 1;
                    while (lo < hi) {
                        const int mid = (lo + hi) >> 1;
                        if (S.incl[mid] > ek) hi = mid; else lo = mid + 1;
                    }
                    const long long exo = lo ? S.incl[lo - 1] : 0;
                    own[k] = lo;
                    x[k] = __ldcs(idx + S.start[lo] + (ek - exo));
                }
            }
            uint32_t sx[kBigUnroll];
#pragma unroll
            for (int k = 0; k < kBigUnroll; ++k) sx[k] = own[k] >= 0 ? (uint32_t)__ldcg(st + x[k]) : 0u;
#pragma unroll
            for (int k = 0; k < kBigUnroll; ++k)
                if (own[k] >= 0) visit(S.node[own[k]], x[k], sx[k]);
        }
        __syncthreads();
    }
}

// Light frontier nodes: warp w takes batches w, w + #warps, ... of B nodes each (no shared counter);
// the batch's arcs are balanced over the 32 lanes by a warp scan and a shuffle binary search.
// B = 32 when the frontier is large, fewer (down to 1) when it is small so that every warp gets work.
template <class NodeT, class Prep, class Visit>
__device__ __forceinline__ void expand_light(const int32_t *ql, uint32_t c0, const int64_t *ptr, const int32_t *idx,
                                             const uint16_t *st, int64_t gtid, int64_t gsz, Prep prep, Visit visit,
                                             unsigned long long &arcs) {
    const uint32_t warps = (uint32_t)(gsz >> 5);
    uint32_t B = (c0 + 2 * warps - 1) / (2 * warps);
    B = B < 1 ? 1u : (B > 32 ? 32u : B);
    const uint32_t nbatch = (c0 + B - 1) / B;
    const unsigned lane = lane_id();
    for (uint32_t bi = (uint32_t)(gtid >> 5); bi < nbatch; bi += warps) {
        const uint32_t i = bi * B + lane;
        NodeT nd{};
        int64_t start = 0;
        int deg = 0;
        if (lane < B && i < c0) {
            const int32_t v = __ldcg(ql + i);   // -1: a big node, expanded by expand_big
            if (v >= 0 && prep(v, true, nd)) { start = ptr[v]; deg = (int)(ptr[v + 1] - start); }
        }
        int incl = deg;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, incl, o);
            if ((int)lane >= o) incl += t;
        }
        const int tot = __shfl_sync(0xffffffffu, incl, 31);
        if (lane == 0) arcs += (unsigned long long)tot;
        const int excl = incl - deg;
        for (int e0 = 0; e0 < tot; e0 += 32 * kLightUnroll) {
            NodeT no[kLightUnroll];
            int32_t x[kLightUnroll];
#pragma unroll
            for (int k = 0; k < kLightUnroll; ++k) {
                const int e = e0 + 32 * k + (int)lane;
                int pos = 0;
#pragma unroll
                for (int bb = 16; bb > 0; bb >>= 1) {
                    const int val = __shfl_sync(0xffffffffu, incl, pos + bb - 1);
                    if (val <= e) pos += bb;
                }
                const int64_t st_o = __shfl_sync(0xffffffffu, start, pos);
                const int ex_o = __shfl_sync(0xffffffffu, excl, pos);
                const uint32_t *src = reinterpret_cast<const uint32_t *>(&nd);
                uint32_t *dst = reinterpret_cast<uint32_t *>(&no[k]);
#pragma unroll
                for (int w = 0; w < (int)(sizeof(NodeT) / 4); ++w) dst[w] = __shfl_sync(0xffffffffu, src[w], pos);
                x[k] = e < tot ? __ldcs(idx + st_o + (e - ex_o)) : -1;
            }
            uint32_t sx[kLightUnroll];
#pragma unroll
            for (int k = 0; k < kLightUnroll; ++k) sx[k] = x[k] >= 0 ? (uint32_t)__ldcg(st + x[k]) : 0u;
#pragma unroll
            for (int k = 0; k < kLightUnroll; ++k)
                if (x[k] >= 0) visit(no[k], x[k], sx[k]);
        }
    }
}

// ------------------------------------------------------------------------------------------ pre-pass
// Shared predecessor DAG (top-down): whether u -> x is a B_i-predecessor arc
// (Thm. V.4 + reading R12) depends only on M, a and K, never on the central node whose graph is being
// extracted.  So the backward closure of ALL central nodes is computed once, round by round, with the
// same load balancing as the expansion, and every arc that passes the test is stored in a CSR keyed by
// its successor.  Each Central Graph is then a walk over these short lists (topdown.cu).

// Thm. V.4 test of in-arc u -> x for the keyword bits P of x (hx = M row of x, gx = gate(x) - 1).
__device__ __forceinline__ uint32_t pred_test(const QueryArgs &a, uint32_t full, bool exact_block, uint32_t P,
                                              uint64_t hx, int gx, int32_t u, uint32_t su, uint32_t &zbu) {
    const uint32_t hmu = su & 0xFFu;   // su = st[u], gathered by the caller
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

__device__ __forceinline__ void pd_visit(const QueryArgs &a, uint32_t full, bool exact_block, const PdNode &nd,
                                         int32_t u, uint32_t su, uint32_t *nbits, uint32_t *nflag) {
    uint32_t zbu = 0;
    const uint32_t pb = pred_test(a, full, exact_block, nd.P, nd.hx, nd.gx, u, su, zbu);
    if (!pb) return;
    const uint32_t pos = agg_slot(reinterpret_cast<uint32_t *>(a.w.pcnt + nd.cidx), (unsigned)nd.cidx);
    const uint32_t ai = agg_slot(&a.w.ctl->n_parcs, 0xFFFFFFFFu);
    if ((int64_t)ai < a.w.pcap) {
        a.w.pa_u[ai] = u;
        a.w.pa_x[ai] = nd.cidx;
        a.w.pa_b[ai] = (uint16_t)(pb | (zbu << 8));
        a.w.pa_slot[ai] = (int32_t)pos;
    } else {
        atomicExch(&a.w.ctl->fatal, 5);
    }
    const uint32_t nb = pb & ~zbu;        // sources (m = 0) have no predecessors
    if (nb) {
        const uint32_t old = atomicOr(a.w.pd_state + u, nb << 8);
        if (((old >> 8) & 0xFFu) == 0) set_bit(nbits, nflag, u);
    }
}

__device__ __forceinline__ bool pd_prepare(const QueryArgs &a, int32_t x, PdNode &nd) {
    nd.P = __ldcg(a.w.pd_state + x) & 0xFFu;
    nd.hx = __ldcg(reinterpret_cast<const unsigned long long *>(a.w.M) + x);
    nd.gx = (int)(__ldcg(a.w.st + x) >> 8) - 1;
    nd.cidx = __ldcg(a.w.pd_cid + x);
    return nd.P != 0;
}

__device__ __forceinline__ int block_excl_scan(int x, int *total, long long *sh) {
    long long t;
    const long long r = block_excl_scan64((long long)x, &t, sh);
    *total = (int)t;
    return (int)r;
}

__device__ void pred_dag(const QueryArgs &a, cg::grid_group &grid, int64_t gtid, int64_t gsz, uint32_t full,
                         long long *sh) {
    Ctl *ctl = a.w.ctl;
    const bool exact_block = a.extract_mode == KGS_EXTRACT_EXACT && a.block_central;
    const int64_t W = a.w.W;
    __shared__ BigTile<PdNode> s_bigb;
    // seeds (every central node, for every keyword it did not contain itself) were set when each
    // central was identified (k_search merge step): round 0 starts from them.
    unsigned long long my_arcs = 0;
    int r = 0;
    for (;; ++r) {
        const int slot = r & 1;
        if (!__ldcg(&ctl->pd_flag[slot])) break;
        uint32_t *qn = ctl->pd_qn[slot];
        if (gtid == 0) { ctl->pd_qn[slot ^ 1][0] = 0u; ctl->pd_qn[slot ^ 1][1] = 0u; }
        // merge: bits to expand this round = newly requested bits not expanded before
        compact(a.w.pd_bits + (int64_t)slot * W, W, a.g.cls_in, a.w.pd_qlight, &qn[0], a.w.pd_qbig, &qn[1],
                a.w.pd_touched, &ctl->n_cid, sh,
                [&](int32_t u) {
                    const uint32_t s = __ldcg(a.w.pd_state + u);
                    const uint32_t nx = (s >> 8) & 0xFFu, dn = (s >> 16) & 0xFFu;
                    const uint32_t bits = nx & ~dn;
                    a.w.pd_state[u] = bits | ((dn | bits) << 16);
                    return bits != 0 && __ldcg(a.w.pd_cid + u) < 0;
                },
                [&](int32_t u, uint32_t pos) { a.w.pd_cid[u] = (int32_t)pos; });
        grid.sync();
        KGS_STAMP(TS_PD_MERGE);
        const uint32_t c0 = __ldcg(&qn[0]), c1 = __ldcg(&qn[1]);
        if (gtid == 0) ctl->pd_flag[slot] = 0u;   // read by every thread before the barrier above
        uint32_t *nbits = a.w.pd_bits + (int64_t)(slot ^ 1) * W;
        uint32_t *nflag = &ctl->pd_flag[slot ^ 1];
        auto prep = [&](int32_t x, bool, PdNode &nd) { return pd_prepare(a, x, nd); };
        auto visit = [&](const PdNode &nd, int32_t u, uint32_t su) {
            pd_visit(a, full, exact_block, nd, u, su, nbits, nflag);
        };
        expand_big(a.w.pd_qbig, c1, a.g.in_ptr, a.g.in_idx, a.w.st, s_bigb, sh, gtid, gsz, prep, visit, my_arcs);
        expand_light<PdNode>(a.w.pd_qlight, c0, a.g.in_ptr, a.g.in_idx, a.w.st, gtid, gsz, prep, visit, my_arcs);
        grid.sync();
        KGS_STAMP(TS_PD_EXPAND);
    }
    if (my_arcs) atomicAdd(&ctl->td_arcs, my_arcs);
    if (gtid == 0) ctl->pd_rounds = r;
    // CSR of the predecessor lists: exclusive scan of pcnt over compact ids, then scatter
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
    if (blockIdx.x == 0) {   // exclusive scan of the per-CTA sums
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
    const int64_t W = a.w.W;
    const int R = a.w.R;
    const int amax = R - 2;
    const uint32_t full = (1u << a.q) - 1u;
    Ctl *ctl = a.w.ctl;
    uint8_t *st8 = reinterpret_cast<uint8_t *>(a.w.st);
    uint8_t *nm8 = reinterpret_cast<uint8_t *>(a.w.nm);
    __shared__ BigTile<FwdNode> s_big;
    __shared__ long long sh[40];
    KGS_STAMP(TS_START);

    // ---- reset the state the previous query left behind
    if (a.full_reset) {
        reset_st_dense(a.w.st, a.w.act, n, gtid, gsz);
        for (int64_t v = gtid; v < (n + 3) / 4; v += gsz) a.w.nm[v] = 0u;
        for (int64_t j = gtid; j < (int64_t)R * W; j += gsz) a.w.fbits[j] = 0u;
        for (int64_t j = gtid; j < 2 * W; j += gsz) a.w.pd_bits[j] = 0u;
        for (int64_t v = gtid; v < n; v += gsz) { a.w.pd_state[v] = 0u; a.w.pd_cid[v] = -1; a.w.pcnt[v] = 0; }
    } else {
        const Ctl *pv = a.w.prev;
        for (int64_t j = gtid; j < (int64_t)pv->n_cid; j += gsz) {
            const int32_t v = a.w.pd_touched[j];
            a.w.pd_state[v] = 0u; a.w.pd_cid[v] = -1; a.w.pcnt[j] = 0;
        }
        const int64_t pt = (int64_t)pv->n_touched;
        if (pt > n / 16) {   // many touched rows: a dense sweep beats scattered 2-byte writes
            reset_st_dense(a.w.st, a.w.act, n, gtid, gsz);
        } else {
            for (int64_t j = gtid; j < pt; j += gsz) {
                const int32_t v = a.w.touched[j];
                a.w.st[v] = (uint16_t)((uint16_t)a.w.act[v] << 8);
            }
        }
        for (int s = 0; s < a.prev_R; ++s)   // level slots still pending when the previous query stopped
            if (pv->slot_flag[s])
                for (int64_t j = gtid; j < W; j += gsz) a.w.fbits[(int64_t)s * W + j] = 0u;
    }
    bool empty = false;
    for (int i = 0; i < a.q; ++i) {
        const int32_t t = a.w.kw_dev[i];
        if (a.g.kw_ptr[t + 1] == a.g.kw_ptr[t]) empty = true;
    }
    grid.sync();
    KGS_STAMP(TS_RESET);
    // ---- initialisation: M = 0 on T_i, keyword nodes ungated, F_0 = K
    {   // one flat grid-stride loop over the concatenation T_0 | T_1 | ... | T_{q-1}
        int64_t kb[kMaxQ], ko[kMaxQ + 1];
        ko[0] = 0;
        for (int i = 0; i < a.q; ++i) {
            const int32_t t = a.w.kw_dev[i];
            kb[i] = a.g.kw_ptr[t];
            ko[i + 1] = ko[i] + (a.g.kw_ptr[t + 1] - kb[i]);
        }
        for (int64_t j = gtid; j < ko[a.q]; j += gsz) {
            int i = 0;
            while (j >= ko[i + 1]) ++i;
            const int32_t v = a.g.kw_nodes[kb[i] + (j - ko[i])];
            a.w.M[(int64_t)v * 8 + i] = 0;
            st8[2 * (int64_t)v + 1] = 0;                                  // keyword node: no gate (L210)
            atomicOr(a.w.nm + (v >> 2), (1u << i) << ((v & 3) * 8));      // hit in B_i at level 0
            push(a, R, v, 0);
        }
    }
    grid.sync();
    KGS_STAMP(TS_SCATTER);

    unsigned long long my_arcs = 0;
    unsigned my_hits = 0;
    for (int l = 0;; ++l) {
        // ---- enqueue frontiers: anything pending at this or a later level?
        bool pend = false;
        const int top = l > amax ? l : amax;
        for (int L = l; L <= top; ++L) pend |= __ldcg(&ctl->slot_flag[L % R]) != 0u;
        if (!pend) {
            if (gtid == 0) { ctl->stop_reason = empty ? KGS_STOP_EMPTY_KEYWORD : KGS_STOP_EXHAUSTED; ctl->levels = l; }
            break;
        }
        const int s = l % R;
        uint32_t *qn = ctl->qn[l & 1];
        if (gtid == 0) { ctl->qn[(l + 1) & 1][0] = 0u; ctl->qn[(l + 1) & 1][1] = 0u; }
        // compact the level's bitmap; merge new hits into hm and identify central nodes (L262-266)
        compact(a.w.fbits + (int64_t)s * W, W, a.g.cls, a.w.qlight, &qn[0], a.w.qbig, &qn[1], a.w.touched,
                &ctl->n_touched, sh,
                [&](int32_t v) {
                    const uint32_t b = nm8[v];
                    if (!b) return false;
                    nm8[v] = 0;
                    const uint32_t old = st8[2 * (int64_t)v];
                    const uint32_t nw = old | b;
                    st8[2 * (int64_t)v] = (uint8_t)nw;
                    if (nw == full && old != full) {                        // Lemma V.1: depth = l
                        const uint32_t ci = agg_slot(&ctl->n_central, 1u);
                        a.w.centrals[ci] = v;
                        a.w.cdepth[ci] = (uint8_t)l;
                        // seed of the top-down pre-pass: expand backwards every keyword v does not contain
                        const uint64_t Mv = __ldcg(reinterpret_cast<const unsigned long long *>(a.w.M) + v);
                        uint32_t zb = 0;
                        for (int i = 0; i < a.q; ++i) if (((Mv >> (8 * i)) & 0xFF) == 0) zb |= 1u << i;
                        if (full & ~zb) {
                            a.w.pd_state[v] = (full & ~zb) << 8;
                            set_bit(a.w.pd_bits, &ctl->pd_flag[0], v);
                        }
                    }
                    return old == 0;
                },
                [&](int32_t, uint32_t) {});
        grid.sync();
        KGS_STAMP(TS_MERGE);
        const uint32_t c0 = __ldcg(&qn[0]), c1 = __ldcg(&qn[1]);
        if (gtid == 0) ctl->frontier_total += (unsigned long long)c0 + c1;
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
        // slot s is consumed; nothing pushes to level l + R during this level (pushes reach <= max(l+1, amax))
        if (gtid == 0) ctl->slot_flag[s] = 0u;
        auto prep = [&](int32_t v, bool leader, FwdNode &nd) {
            nd.v = v;
            nd.hm = prepare(a, R, l, full, v, leader);
            return nd.hm != 0;
        };
        auto visit = [&](const FwdNode &nd, int32_t x, uint32_t sx) { visit_arc(a, R, l, nd.v, nd.hm, x, sx, my_hits); };
        expand_big(a.w.qbig, c1, a.g.row_ptr, a.g.col_idx, a.w.st, s_big, sh, gtid, gsz, prep, visit, my_arcs);
        expand_light<FwdNode>(a.w.qlight, c0, a.g.row_ptr, a.g.col_idx, a.w.st, gtid, gsz, prep, visit, my_arcs);
        grid.sync();
        KGS_STAMP(TS_EXPAND);
    }
    const unsigned wa = __reduce_add_sync(0xffffffffu, (unsigned)my_arcs);   // per-warp totals fit 32 bits
    const unsigned wh = __reduce_add_sync(0xffffffffu, my_hits);
    __shared__ unsigned long long s_sum[2];
    if (threadIdx.x < 2) s_sum[threadIdx.x] = 0ull;
    __syncthreads();
    if ((threadIdx.x & 31) == 0) {
        if (wa) atomicAdd(&s_sum[0], (unsigned long long)wa);
        if (wh) atomicAdd(&s_sum[1], (unsigned long long)wh);
    }
    __syncthreads();
    if (threadIdx.x == 0) {      // one global atomic per CTA
        if (s_sum[0]) atomicAdd(&ctl->arcs_scanned, s_sum[0]);
        if (s_sum[1]) atomicAdd(&ctl->hits, s_sum[1]);
    }
    grid.sync();
    KGS_STAMP(TS_END);
    pred_dag(a, grid, gtid, gsz, full, sh);
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
