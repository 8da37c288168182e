// topdown.cu — top-down processing of the Central Graph method on sm_100a (product CUDA path).
//
// For every central node c (all depths <= d, Alg. 3):
//   extract   per keyword i the backward closure from (c, i) under Thm. V.4 (L472-476): u -> x is a
//             B_i-predecessor arc iff m_ui finite and m_xi = 1 + max{a_u, m_ui, a_x - 1 (x outside K)},
//             plus, in exact mode (reading R12), u was not central yet at level m_xi - 1.  Per-keyword
//             masks make it "q independent BFSes" in one pass (L478, reading R11).
//   cover     level-cover pruning (L454, Ex. 5): keyword nodes grouped by how many keywords they
//             contribute, cumulative cover from the top level (central node included, reading R13),
//             hitting paths of the pruned sources removed.
//   score     Eq. 6 (L464): key = pow(d, lambda) * sum of w over the pruned graph, fp64, exact on the
//             2^-24 weight grid (reading R15); smaller is better (reading R14).
// Then a radix select over the 96-bit composite (key bits, id) picks the k best deterministically
// (L478, L496 heap), and the winners' graphs are emitted as sorted node / arc lists.
//
// The paper ran this phase on the CPU because of dynamic allocation and divergence (L452).  Here each
// candidate is one warp with a bounded shared-memory arena (hash table, node / arc lists, FIFO); a
// candidate that outgrows it is re-run by a whole CTA over a per-CTA global-memory arena.
#include <cooperative_groups.h>

#include "kgs_internal.h"

namespace cg = cooperative_groups;

namespace kgs {

// ------------------------------------------------------------------------------------------ teams
struct WarpTeam {
    __device__ __forceinline__ int rank() const { return threadIdx.x & 31; }
    __device__ __forceinline__ int size() const { return 32; }
    __device__ __forceinline__ void sync() const { __syncwarp(); }
    // exclusive scan of x over the team; *total = sum
    __device__ __forceinline__ int scan_excl(int x, int *total) const {
        int incl = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, incl, o);
            if (rank() >= o) incl += t;
        }
        *total = __shfl_sync(0xffffffffu, incl, 31);
        return incl - x;
    }
};

struct BlockTeam {
    int *scratch;  // >= 33 ints of shared memory
    __device__ __forceinline__ int rank() const { return threadIdx.x; }
    __device__ __forceinline__ int size() const { return blockDim.x; }
    __device__ __forceinline__ void sync() const { __syncthreads(); }
    __device__ __forceinline__ int scan_excl(int x, int *total) const {
        const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
        int incl = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += t;
        }
        __syncthreads();
        if (lane == 31) scratch[wid] = incl;
        __syncthreads();
        if (threadIdx.x == 0) {
            int acc = 0;
            for (int w = 0; w < nw; ++w) { const int t = scratch[w]; scratch[w] = acc; acc += t; }
            scratch[32] = acc;
        }
        __syncthreads();
        const int r = scratch[wid] + incl - x;
        *total = scratch[32];
        __syncthreads();
        return r;
    }
};

// ------------------------------------------------------------------------------------------ arena
enum { SC_NODES = 0, SC_ARCS, SC_HEAD, SC_TAIL, SC_OVF, SC_CHANGED, SC_COV, SC_SSTAR, SC_NOUT, SC_AOUT, SC_N };

struct Arena {
    int32_t *hkey;      // [hcap] node id or -1
    int32_t *hval;      // [hcap] node index or -1
    int32_t *id;        // [ncap]
    uint32_t *inmask;   // [ncap] bit i: node in DAG_i(c)
    uint32_t *zb;       // [ncap] bit i: m_vi == 0 (source of B_i)
    uint32_t *pending;  // [ncap] bits still to expand backwards
    uint32_t *keep;     // [ncap] bit i: kept in DAG_i after level-cover
    int32_t *fifo;      // [ncap] ring of node indices with pending bits
    int32_t *au, *ax;   // [acap] arc endpoints (node indices)
    uint32_t *ab;       // [acap] keyword bits of the arc
    int32_t *b_j;       // [team] batch: node index
    int64_t *b_start;   // [team] batch: in-arc start
    int32_t *b_incl;    // [team] batch: inclusive arc count
    uint32_t *b_P;      // [team] batch: keywords to expand
    uint64_t *b_hx;     // [team] batch: M row
    int32_t *b_gx;      // [team] batch: gate - 1
    unsigned long long *sortbuf;  // [acap] (emit only)
    int32_t *scal;      // [SC_N]
    double *dsum;
    int hcap, ncap, acap;
};

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
    return x;
}

// insert (or find) node u; returns its index, -1 on overflow
__device__ __forceinline__ int arena_insert(Arena &S, int32_t u, uint32_t zbu) {
    uint32_t h = hash32((uint32_t)u) & (uint32_t)(S.hcap - 1);
    for (int probe = 0; probe < S.hcap; ++probe) {
        const int32_t k = atomicCAS(S.hkey + h, -1, u);
        if (k == -1) {
            const int idx = atomicAdd(S.scal + SC_NODES, 1);
            if (idx >= S.ncap) { atomicExch(S.scal + SC_OVF, 1); atomicExch(S.hval + h, -2); return -1; }
            S.id[idx] = u;
            S.zb[idx] = zbu;
            __threadfence_block();
            atomicExch(S.hval + h, idx);
            return idx;
        }
        if (k == u) {
            int v;
            while ((v = atomicAdd(S.hval + h, 0)) == -1) { }
            return v >= 0 ? v : -1;
        }
        h = (h + 1) & (uint32_t)(S.hcap - 1);
    }
    atomicExch(S.scal + SC_OVF, 1);
    return -1;
}

__device__ __forceinline__ void fifo_push(Arena &S, int j) {
    const int pos = atomicAdd(S.scal + SC_TAIL, 1);
    S.fifo[pos % S.ncap] = j;
}

// Closure + level-cover + score of the Central Graph at c.  Returns false on arena overflow.
template <class Team>
__device__ bool central_graph(const Team &T, Arena &S, const QueryArgs &a, int32_t c, int depth, double *key) {
    const uint32_t full = (1u << a.q) - 1u;
    const int r = T.rank(), ts = T.size();
    for (int i = r; i < S.hcap; i += ts) { S.hkey[i] = -1; S.hval[i] = -1; }
    for (int i = r; i < S.ncap; i += ts) { S.inmask[i] = 0; S.pending[i] = 0; S.keep[i] = 0; }
    if (r < SC_N) S.scal[r] = 0;
    if (r == 0) *S.dsum = 0.0;
    T.sync();
    if (r == 0) {
        const uint64_t Mc = *reinterpret_cast<const uint64_t *>(a.w.M + (int64_t)c * 8);
        uint32_t zbc = 0;
        for (int i = 0; i < a.q; ++i) if (((Mc >> (8 * i)) & 0xFF) == 0) zbc |= 1u << i;
        const int j = arena_insert(S, c, zbc);  // index 0
        S.inmask[j] = full;
        const uint32_t p = full & ~zbc;
        if (p) { S.pending[j] = p; fifo_push(S, j); }
    }
    T.sync();
    // ---- backward closure, batch by batch (all pending nodes of a round in parallel)
    for (;;) {
        const int head = S.scal[SC_HEAD], tail = S.scal[SC_TAIL];
        if (head == tail || S.scal[SC_OVF]) break;
        T.sync();
        for (int b0 = head; b0 < tail; b0 += ts) {
            int deg = 0;
            if (b0 + r < tail) {
                const int j = S.fifo[(b0 + r) % S.ncap];
                const uint32_t P = atomicExch(S.pending + j, 0u);
                const int32_t x = S.id[j];
                S.b_j[r] = j;
                S.b_P[r] = P;
                const int32_t cid = a.w.pd_cid[x];   // predecessor list from the shared DAG
                int64_t s0 = 0;
                if (P && cid >= 0) { s0 = a.w.pred_ptr[cid]; deg = (int)(a.w.pred_ptr[cid + 1] - s0); }
                S.b_start[r] = s0;
            }
            int tot;
            const int ex = T.scan_excl(deg, &tot);
            S.b_incl[r] = ex + deg;
            T.sync();
            const int nb = min(ts, tail - b0);
            for (int e = r; e < tot; e += ts) {
                int lo = 0, hi = nb - 1;       // owner = first o with incl[o] > e
                while (lo < hi) {
                    const int mid = (lo + hi) >> 1;
                    if (S.b_incl[mid] > e) hi = mid; else lo = mid + 1;
                }
                const int o = lo;
                const int exo = o ? S.b_incl[o - 1] : 0;
                const int64_t pi = S.b_start[o] + (e - exo);
                const int32_t u = a.w.pred_u[pi];
                const uint32_t bz = a.w.pred_b[pi];
                const uint32_t pb = bz & S.b_P[o] & 0xFFu;   // Thm. V.4 arc for the keywords x needs here
                if (!pb) continue;
                const uint32_t zbu = bz >> 8;
                const int j = arena_insert(S, u, zbu);
                if (j < 0) continue;
                const uint32_t old = atomicOr(S.inmask + j, pb);
                const uint32_t nbits = pb & ~old & ~S.zb[j];
                if (nbits) {
                    const uint32_t oldp = atomicOr(S.pending + j, nbits);
                    if (oldp == 0) fifo_push(S, j);
                }
                const int ai = atomicAdd(S.scal + SC_ARCS, 1);
                if (ai >= S.acap) { atomicExch(S.scal + SC_OVF, 1); continue; }
                S.au[ai] = j;
                S.ax[ai] = S.b_j[o];
                S.ab[ai] = pb;
            }
            T.sync();
        }
        if (r == 0) S.scal[SC_HEAD] = tail;
        T.sync();
    }
    T.sync();
    if (S.scal[SC_OVF]) return false;
    const int nn = S.scal[SC_NODES];
    const int na = S.scal[SC_ARCS] < S.acap ? S.scal[SC_ARCS] : S.acap;
    // ---- level-cover
    if (a.level_cover) {
        const uint32_t cov0 = S.zb[0];
        int sstar = a.q + 1;
        if (cov0 != full) {
            if (r == 0) S.scal[SC_COV] = (int)cov0;
            T.sync();
            for (int s = a.q; s >= 1; --s) {
                for (int j = 1 + r; j < nn; j += ts) {
                    const uint32_t con = S.inmask[j] & S.zb[j];
                    if (__popc(con) == s) atomicOr(reinterpret_cast<unsigned *>(S.scal + SC_COV), con);
                }
                T.sync();
                if ((uint32_t)S.scal[SC_COV] == full) { sstar = s; break; }
                T.sync();
            }
        }
        for (int j = r; j < nn; j += ts) {
            const uint32_t con = S.inmask[j] & S.zb[j];
            S.keep[j] = (j == 0 || __popc(con) >= sstar) ? con : 0u;
        }
        T.sync();
        for (;;) {   // forward reachability from the kept sources inside each DAG_i
            if (r == 0) S.scal[SC_CHANGED] = 0;
            T.sync();
            for (int e = r; e < na; e += ts) {
                const uint32_t add = S.keep[S.au[e]] & S.ab[e];
                if (add & ~S.keep[S.ax[e]]) { atomicOr(S.keep + S.ax[e], add); S.scal[SC_CHANGED] = 1; }
            }
            T.sync();
            const int ch = S.scal[SC_CHANGED];
            T.sync();
            if (!ch) break;
        }
        if (r == 0) S.keep[0] = full;
    } else {
        for (int j = r; j < nn; j += ts) S.keep[j] = S.inmask[j];
    }
    T.sync();
    // ---- Eq. 6
    for (int j = r; j < nn; j += ts)
        if (S.keep[j]) atomicAdd(S.dsum, (double)a.g.weight[S.id[j]]);
    T.sync();
    *key = __dmul_rn(a.w.dpow[depth], *S.dsum);
    T.sync();
    return true;
}

// team bitonic sort (ascending) of buf[0..len) padded to a power of two with ~0
template <class Team>
__device__ void team_sort(const Team &T, unsigned long long *buf, int len) {
    int p2 = 1;
    while (p2 < len) p2 <<= 1;
    for (int i = len + T.rank(); i < p2; i += T.size()) buf[i] = ~0ull;
    T.sync();
    for (int k = 2; k <= p2; k <<= 1)
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int i = T.rank(); i < p2; i += T.size()) {
                const int l = i ^ j;
                if (l > i) {
                    const unsigned long long x = buf[i], y = buf[l];
                    const bool up = (i & k) == 0;
                    if ((x > y) == up) { buf[i] = y; buf[l] = x; }
                }
            }
            T.sync();
        }
}

// write the kept nodes / arcs of the arena (after central_graph) sorted and unique
template <class Team>
__device__ bool emit_graph(const Team &T, Arena &S, const QueryArgs &a, int rank_i) {
    const int r = T.rank(), ts = T.size();
    const int nn = S.scal[SC_NODES];
    const int na = S.scal[SC_ARCS];
    // nodes
    if (r == 0) { S.scal[SC_NOUT] = 0; S.scal[SC_AOUT] = 0; }
    T.sync();
    for (int j = r; j < nn; j += ts)
        if (S.keep[j]) S.sortbuf[atomicAdd(S.scal + SC_NOUT, 1)] = (unsigned long long)(uint32_t)S.id[j];
    T.sync();
    const int kn = S.scal[SC_NOUT];
    team_sort(T, S.sortbuf, kn);
    int32_t *hdr = a.w.ans_hdr + 4 * rank_i;
    unsigned long long *arena_ctr = a.w.ctl->arena_used;  // [0] = nodes, [1] = arcs
    __shared__ long long s_off[2];
    long long *off = s_off;  // per-CTA; only one team per CTA emits
    if (r == 0) off[0] = (long long)atomicAdd(arena_ctr + 0, (unsigned long long)kn);
    T.sync();
    const long long no = off[0];
    if (no + kn > (long long)a.w.arena_nodes_cap) {
        if (r == 0) atomicExch(&a.w.ctl->fatal, 1);
        return false;
    }
    for (int i = r; i < kn; i += ts) a.w.arena_nodes[no + i] = (int32_t)S.sortbuf[i];
    T.sync();
    // arcs: union over keywords of kept arcs (keep[u] & bits of the arc)
    if (r == 0) S.scal[SC_AOUT] = 0;
    T.sync();
    for (int e = r; e < na; e += ts)
        if (S.keep[S.au[e]] & S.ab[e])
            S.sortbuf[atomicAdd(S.scal + SC_AOUT, 1)] =
                ((unsigned long long)(uint32_t)S.id[S.au[e]] << 32) | (uint32_t)S.id[S.ax[e]];
    T.sync();
    const int ka = S.scal[SC_AOUT];
    team_sort(T, S.sortbuf, ka);
    // unique (sequential compaction by chunks of the team)
    int kept = 0;
    for (int b0 = 0; b0 < ka; b0 += ts) {
        const int i = b0 + r;
        const int flag = (i < ka && (i == 0 || S.sortbuf[i] != S.sortbuf[i - 1])) ? 1 : 0;
        int tot;
        const int ex = T.scan_excl(flag, &tot);
        T.sync();
        // write into the tail of the buffer region after ka (keys are read-only below i)
        if (flag) S.sortbuf[ka + kept + ex] = S.sortbuf[i];
        kept += tot;
        T.sync();
    }
    if (r == 0) off[1] = (long long)atomicAdd(arena_ctr + 1, (unsigned long long)kept);
    T.sync();
    const long long ao = off[1];
    if (ao + kept > (long long)a.w.arena_arcs_cap) {
        if (r == 0) atomicExch(&a.w.ctl->fatal, 1);
        return false;
    }
    for (int i = r; i < kept; i += ts) {
        const unsigned long long key = S.sortbuf[ka + i];
        a.w.arena_arcs[2 * (ao + i)] = (int32_t)(key >> 32);
        a.w.arena_arcs[2 * (ao + i) + 1] = (int32_t)(key & 0xFFFFFFFFu);
    }
    if (r == 0) {
        hdr[2] = kn;
        hdr[3] = kept;
        a.w.ans_off[2 * rank_i] = no;
        a.w.ans_off[2 * rank_i + 1] = ao;
    }
    T.sync();
    return true;
}

// ------------------------------------------------------------------------------------------ carving
// shared-memory arena of one warp (extract) / one warp + sort buffer (emit)
struct SmemSizes {
    static constexpr int H = kExtHash, N = kExtNodes, A = kExtArcs;
};

__device__ __forceinline__ char *align8(char *p) {
    return reinterpret_cast<char *>((reinterpret_cast<uintptr_t>(p) + 7) & ~uintptr_t(7));
}

__device__ Arena carve(char *&p, int hcap, int ncap, int acap, int team, bool with_sort) {
    Arena S;
    S.hcap = hcap; S.ncap = ncap; S.acap = acap;
    p = align8(p);
    S.b_start = reinterpret_cast<int64_t *>(p); p += sizeof(int64_t) * team;
    S.b_hx = reinterpret_cast<uint64_t *>(p); p += sizeof(uint64_t) * team;
    S.dsum = reinterpret_cast<double *>(p); p += sizeof(double);
    if (with_sort) { S.sortbuf = reinterpret_cast<unsigned long long *>(p); p += sizeof(unsigned long long) * 2 * (size_t)acap; }
    else S.sortbuf = nullptr;
    S.hkey = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * hcap;
    S.hval = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * hcap;
    S.id = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * ncap;
    S.inmask = reinterpret_cast<uint32_t *>(p); p += sizeof(uint32_t) * ncap;
    S.zb = reinterpret_cast<uint32_t *>(p); p += sizeof(uint32_t) * ncap;
    S.pending = reinterpret_cast<uint32_t *>(p); p += sizeof(uint32_t) * ncap;
    S.keep = reinterpret_cast<uint32_t *>(p); p += sizeof(uint32_t) * ncap;
    S.fifo = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * ncap;
    S.au = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * acap;
    S.ax = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * acap;
    S.ab = reinterpret_cast<uint32_t *>(p); p += sizeof(uint32_t) * acap;
    S.b_j = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * team;
    S.b_incl = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * team;
    S.b_P = reinterpret_cast<uint32_t *>(p); p += sizeof(uint32_t) * team;
    S.b_gx = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * team;
    S.scal = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * SC_N;
    p = align8(p);
    return S;
}

__host__ __device__ size_t arena_bytes(int hcap, int ncap, int acap, int team, bool with_sort) {
    size_t b = 8 + sizeof(int64_t) * team + sizeof(uint64_t) * team + sizeof(double);
    if (with_sort) b += sizeof(unsigned long long) * 2 * (size_t)acap;
    b += sizeof(int32_t) * 2 * (size_t)hcap + sizeof(int32_t) * 6 * (size_t)ncap + sizeof(int32_t) * 3 * (size_t)acap;
    b += sizeof(int32_t) * 4 * (size_t)team + sizeof(int32_t) * SC_N + 8;
    return b;
}

// ------------------------------------------------------------------------------------------ extract
__global__ void __launch_bounds__(kExtWarps * 32) k_extract(QueryArgs a) {
    extern __shared__ __align__(16) char smem[];
    const int wid = threadIdx.x >> 5;
    const size_t per = arena_bytes(kExtHash, kExtNodes, kExtArcs, 32, false);
    char *p = smem + per * wid;
    Arena S = carve(p, kExtHash, kExtNodes, kExtArcs, 32, false);
    WarpTeam T;
    Ctl *ctl = a.w.ctl;
    const uint32_t nc = ctl->n_central;
    for (;;) {
        uint32_t idx = 0;
        if (T.rank() == 0) idx = atomicAdd(&ctl->work_ext, 1u);
        idx = __shfl_sync(0xffffffffu, idx, 0);
        if (idx >= nc) break;
        const int32_t c = a.w.centrals[idx];
        double key = 0.0;
        const bool ok = central_graph(T, S, a, c, a.w.cdepth[idx], &key);
        if (T.rank() == 0) {
            if (ok) { a.w.ckey[idx] = key; a.w.cflag[idx] = 0; }
            else { a.w.cflag[idx] = 1; a.w.overflow[atomicAdd(&ctl->n_overflow, 1u)] = (int32_t)idx; }
        }
        __syncwarp();
    }
}

// overflowed candidates: one CTA each over a per-CTA global-memory arena
__global__ void __launch_bounds__(512) k_extract_big(QueryArgs a) {
    __shared__ int scratch[40];
    BlockTeam T{scratch};
    char *p = reinterpret_cast<char *>(a.w.big_ws) + a.w.big_bytes * blockIdx.x;
    Arena S = carve(p, a.w.big_hcap, a.w.big_ncap, a.w.big_acap, blockDim.x, false);
    Ctl *ctl = a.w.ctl;
    const uint32_t no = ctl->n_overflow;
    for (uint32_t t = blockIdx.x; t < no; t += gridDim.x) {
        const int32_t idx = a.w.overflow[t];
        double key = 0.0;
        const bool ok = central_graph(T, S, a, a.w.centrals[idx], a.w.cdepth[idx], &key);
        if (threadIdx.x == 0) {
            if (ok) a.w.ckey[idx] = key;
            else atomicExch(&ctl->fatal, 2);
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------------------------------ select
// Radix select of the k smallest composite keys (fp64 key bits, central id): MSD, 8-bit digits,
// 12 digits, one grid barrier per digit.  Keys are >= 0 so their IEEE bits order like the values.
__device__ __forceinline__ void comp_key(const QueryArgs &a, uint32_t i, uint64_t &hi, uint32_t &lo) {
    hi = (uint64_t)__double_as_longlong(a.w.ckey[i]);
    lo = (uint32_t)a.w.centrals[i];
}
__device__ __forceinline__ uint32_t digit_of(uint64_t hi, uint32_t lo, int d) {
    return d < 8 ? (uint32_t)((hi >> (56 - 8 * d)) & 0xFF) : (lo >> (24 - 8 * (d - 8))) & 0xFF;
}
__device__ __forceinline__ bool prefix_match(uint64_t hi, uint32_t lo, uint64_t phi, uint32_t plo, int d) {
    // digits 0..d-1 equal
    if (d == 0) return true;
    if (d <= 8) {
        const uint64_t m = d == 8 ? ~0ull : (~0ull << (64 - 8 * d));
        return (hi & m) == (phi & m);
    }
    if (hi != phi) return false;
    const uint32_t m = d == 12 ? 0xFFFFFFFFu : (0xFFFFFFFFu << (32 - 8 * (d - 8)));
    return (lo & m) == (plo & m);
}

__global__ void __launch_bounds__(256) k_select(QueryArgs a) {
    cg::grid_group grid = cg::this_grid();
    __shared__ uint32_t sh[256];
    __shared__ uint32_t s_bucket, s_before;
    Ctl *ctl = a.w.ctl;
    const uint32_t nc = ctl->n_central;
    const uint32_t kk = (uint32_t)a.k < nc ? (uint32_t)a.k : nc;
    if (kk == 0) { if (blockIdx.x == 0 && threadIdx.x == 0) ctl->sel_count = 0; return; }
    if (nc <= (uint32_t)KGS_MAX_K) {
        // small candidate set: k_rank sorts all of it in one CTA, no grid-wide passes needed
        if (blockIdx.x == 0) {
            for (uint32_t i = threadIdx.x; i < nc; i += blockDim.x) a.w.sel[i] = (int32_t)i;
            if (threadIdx.x == 0) ctl->sel_count = nc;
        }
        return;
    }
    const int64_t gtid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gsz = (int64_t)gridDim.x * blockDim.x;
    uint64_t phi = 0;
    uint32_t plo = 0;
    uint32_t want = kk;   // rank (1-based) of the threshold inside the current prefix bucket
    if (kk < nc) {
        for (int d = 0; d < 12; ++d) {
            sh[threadIdx.x] = 0;
            __syncthreads();
            for (int64_t i = gtid; i < nc; i += gsz) {
                uint64_t hi; uint32_t lo;
                comp_key(a, (uint32_t)i, hi, lo);
                if (prefix_match(hi, lo, phi, plo, d)) atomicAdd(sh + digit_of(hi, lo, d), 1u);
            }
            __syncthreads();
            if (sh[threadIdx.x]) atomicAdd(&ctl->hist[d][threadIdx.x], sh[threadIdx.x]);
            grid.sync();
            if (threadIdx.x == 0) {
                uint32_t acc = 0, b = 0;
                for (b = 0; b < 256; ++b) {
                    const uint32_t h = __ldcg(&ctl->hist[d][b]);
                    if (acc + h >= want) break;
                    acc += h;
                }
                s_bucket = b; s_before = acc;
            }
            __syncthreads();
            want -= s_before;
            const uint64_t bk = s_bucket;
            if (d < 8) phi |= bk << (56 - 8 * d);
            else plo |= (uint32_t)bk << (24 - 8 * (d - 8));
            __syncthreads();
        }
    } else {
        phi = ~0ull; plo = 0xFFFFFFFFu;
    }
    // collect every candidate <= threshold (exactly kk of them: composites are unique)
    for (int64_t i = gtid; i < nc; i += gsz) {
        uint64_t hi; uint32_t lo;
        comp_key(a, (uint32_t)i, hi, lo);
        if (hi < phi || (hi == phi && lo <= plo)) {
            const uint32_t pos = atomicAdd(&ctl->sel_count, 1u);
            if (pos < (uint32_t)KGS_MAX_K) a.w.sel[pos] = (int32_t)i;
        }
    }
}

// rank the selected winners by composite key (one CTA, bitonic sort in shared memory)
__global__ void __launch_bounds__(1024) k_rank(QueryArgs a) {
    extern __shared__ __align__(16) char smem[];
    unsigned long long *khi = reinterpret_cast<unsigned long long *>(smem);
    uint32_t *klo = reinterpret_cast<uint32_t *>(khi + KGS_MAX_K);
    int32_t *kid = reinterpret_cast<int32_t *>(klo + KGS_MAX_K);
    const uint32_t cnt = a.w.ctl->sel_count;
    int p2 = 1;
    while (p2 < (int)cnt) p2 <<= 1;
    for (int i = threadIdx.x; i < p2; i += blockDim.x) {
        if (i < (int)cnt) {
            const int32_t idx = a.w.sel[i];
            uint64_t hi; uint32_t lo;
            comp_key(a, (uint32_t)idx, hi, lo);
            khi[i] = hi; klo[i] = lo; kid[i] = idx;
        } else { khi[i] = ~0ull; klo[i] = 0xFFFFFFFFu; kid[i] = -1; }
    }
    __syncthreads();
    for (int k = 2; k <= p2; k <<= 1)
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int i = threadIdx.x; i < p2; i += blockDim.x) {
                const int l = i ^ j;
                if (l > i) {
                    const bool gt = khi[i] > khi[l] || (khi[i] == khi[l] && klo[i] > klo[l]);
                    const bool up = (i & k) == 0;
                    if (gt == up) {
                        const unsigned long long th = khi[i]; khi[i] = khi[l]; khi[l] = th;
                        const uint32_t tl = klo[i]; klo[i] = klo[l]; klo[l] = tl;
                        const int32_t ti = kid[i]; kid[i] = kid[l]; kid[l] = ti;
                    }
                }
            }
            __syncthreads();
        }
    const int keep = (int)cnt < a.k ? (int)cnt : a.k;
    for (int i = threadIdx.x; i < keep; i += blockDim.x) a.w.sel[i] = kid[i];
    if (threadIdx.x == 0) a.w.ctl->sel_count = (uint32_t)keep;
}

// ------------------------------------------------------------------------------------------ emit
// One CTA per winner: warp 0 re-runs the shared-memory extractor; winners that overflowed it are
// re-run by the whole CTA over the global arena of this CTA.
__global__ void __launch_bounds__(128) k_emit(QueryArgs a) {
    extern __shared__ __align__(16) char smem[];
    __shared__ int scratch[40];
    Ctl *ctl = a.w.ctl;
    const uint32_t cnt = ctl->sel_count;
    char *p = smem;
    Arena Sw = carve(p, kExtHash, kExtNodes, kExtArcs, 32, true);
    char *pb = reinterpret_cast<char *>(a.w.big_ws) + a.w.big_bytes_emit * blockIdx.x;
    Arena Sb = carve(pb, a.w.big_hcap, a.w.big_ncap, a.w.big_acap, blockDim.x, true);
    BlockTeam BT{scratch};
    WarpTeam WT;
    for (uint32_t rnk = blockIdx.x; rnk < cnt; rnk += gridDim.x) {
        const int32_t idx = a.w.sel[rnk];
        const int32_t c = a.w.centrals[idx];
        const int depth = a.w.cdepth[idx];
        if (threadIdx.x == 0) {
            int32_t *hdr = a.w.ans_hdr + 4 * rnk;
            hdr[0] = c; hdr[1] = depth;
            a.w.ans_key[rnk] = a.w.ckey[idx];
        }
        double key;
        if (!a.w.cflag[idx]) {
            if (threadIdx.x < 32) {
                if (central_graph(WT, Sw, a, c, depth, &key)) emit_graph(WT, Sw, a, (int)rnk);
                else if (threadIdx.x == 0) atomicExch(&ctl->fatal, 3);
            }
        } else {
            if (central_graph(BT, Sb, a, c, depth, &key)) emit_graph(BT, Sb, a, (int)rnk);
            else if (threadIdx.x == 0) atomicExch(&ctl->fatal, 4);
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------------------------------ launchers
static size_t extract_smem() { return arena_bytes(kExtHash, kExtNodes, kExtArcs, 32, false) * kExtWarps; }
static size_t emit_smem() { return arena_bytes(kExtHash, kExtNodes, kExtArcs, 32, true); }

size_t big_arena_bytes(int hcap, int ncap, int acap, bool with_sort) {
    return (arena_bytes(hcap, ncap, acap, 512, with_sort) + 255) & ~size_t(255);
}

cudaError_t launch_extract(const QueryArgs &a, int grid, cudaStream_t s) {
    static bool attr = false;
    const size_t sm = extract_smem();
    if (!attr) {
        cudaFuncSetAttribute(k_extract, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        cudaFuncSetAttribute(k_emit, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)emit_smem());
        attr = true;
    }
    k_extract<<<grid, kExtWarps * 32, sm, s>>>(a);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    k_extract_big<<<a.w.big_ctas, 512, 0, s>>>(a);
    return cudaGetLastError();
}

int select_max_grid(int device) {
    int per_sm = 0, sms = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_select, 256, 0);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    return per_sm * sms;
}

cudaError_t launch_select(const QueryArgs &a, int grid, cudaStream_t s) {
    void *args[] = {(void *)&a};
    cudaError_t e = cudaLaunchCooperativeKernel((const void *)k_select, dim3(grid), dim3(256), args, 0, s);
    if (e != cudaSuccess) return e;
    static bool attr = false;
    const size_t sm = (size_t)KGS_MAX_K * (8 + 4 + 4);
    if (!attr) { cudaFuncSetAttribute(k_rank, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm); attr = true; }
    k_rank<<<1, 1024, sm, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_emit(const QueryArgs &a, int grid, cudaStream_t s) {
    k_emit<<<grid, 128, emit_smem(), s>>>(a);
    return cudaGetLastError();
}

}  // namespace kgs
