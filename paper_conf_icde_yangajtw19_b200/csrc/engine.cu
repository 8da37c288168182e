// engine.cu — the query engine of libkgs on sm_100a (product CUDA path; shares nothing with oracle/).
//
// ONE persistent cooperative kernel answers a batch of queries.  Its CTAs are split into G groups; a
// group pulls the next query index from a device counter and runs the whole hot path for it with
// group-scoped barriers (no host round trip, no further launches):
//
//   search     Alg. 1 ln 1-7 + Alg. 2: reset, initialise M / sources (L254), then per
//              level { enqueue frontiers = compact the level's bitmap, merge new hits, identify central
//              nodes (L256-266, Lemma V.1); termination (Def. 4, Thm. V.3); expansion gated by the
//              activation levels (L210) }.
//   pre-pass   shared predecessor DAG: the Thm. V.4 arcs of the union of all Central Graphs, computed
//              once, round by round, into a CSR keyed by successor.
//   extract    per central node: per-keyword backward closure over the predecessor lists (Def. 2/3,
//              Alg. 3, R11/R12), level-cover (L454, R13), Eq. 6 key (L464, R14/R15).
//   select     top-k by (key, id) (L478, L496): one CTA sorts |C| <= 4096 candidates, else a group-wide
//              radix select over the 96-bit composite key.
//   emit       the winners' graphs as sorted node / unique sorted arc lists.
//
// G = 1 is the single-query latency mode (the whole GPU on one query); G > 1 runs G queries at a time
// (the batch of BASELINE.json configs[3]).
//
// Data layout:
//   st[v]   uint32 status word: byte 0 = hit mask hm (bit i <=> M[v][i] finite, snapshot at the start of
//           the level), byte 1 = K flag (v contains a query keyword: gate 0, else the gate is a_v), byte 2 = nm, the bits
//           newly hit during the current level (atomicOr), byte 3 = a_v.  One 4-byte load per inspected arc
//           gives the target's mask and gate, and the hit that follows is an atomic on the same word
//           (an L2 hit); a frontier node's merge and activation test read one word, not three arrays.
//   M[v*8+i] uint8 hitting level, written once per (v, i) by the thread that set the bit; never reset.
//   fbits   one frontier bitmap per level slot (R = amax+2 slots): "FIdentifier[v] <- 1 for level L" is one
//           bit set on a bitmap word, so pushes never contend on a queue counter.  A node is re-queued
//           exactly at the level where it can make progress again: a_v if it is not yet active (Alg. 2
//           ln 5-7), gate(n)-1 if a neighbour n is still gated (ln 18-19) (reading R22).
//
// Snapshot semantics (reading R10): expansion at level l reads hm as of the start of the level; new hits
// accumulate in nm and are merged when the next level is compacted, so the result equals the sequential
// Alg. 2 (Thm. V.2).  All writes are idempotent (bits OR-ed, level l+1 written once).
#include "kgs_internal.h"

namespace kgs {

// ------------------------------------------------------------------------------------------ groups
__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Barrier over the CTAs of one group (all CTAs are co-resident: cooperative launch).  Thread 0 of each
// CTA adds its arrival to the group's monotonic counter (release) and spins with acquire loads until the
// count reaches this episode's target; the counter is zeroed before every launch (api.cu).  1.4 us per
// barrier over 296 CTAs against 2.0 us for a reset-and-generation barrier (tools/bar_bench.cu).
__device__ __forceinline__ void group_sync(GroupBar *b, int gcount, unsigned &episode) {
    __syncthreads();
    if (threadIdx.x == 0) {
        ++episode;
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&b->arrive) : "memory");
        const unsigned target = episode * (unsigned)gcount;
        while ((int)(ld_acquire(&b->arrive) - target) < 0) { }
    }
    __syncthreads();
}

// The CTA's group (uniform over the CTA: it lives in shared memory, so that neither it nor the running
// query's keywords occupy registers or a stack frame in the whole kernel).
struct Grp {
    int g, grank, gcount;
    int64_t gsz;
    GroupBar *bar;
    mutable unsigned episode;   // barriers passed by this CTA in this launch (thread 0)
    __device__ __forceinline__ int64_t gtid() const { return (int64_t)grank * blockDim.x + threadIdx.x; }
    __device__ __forceinline__ void sync() const { group_sync(bar, gcount, episode); }
};

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

// Append to one list from every active lane: one atomic per warp (ballot + popc).
__device__ __forceinline__ uint32_t warp_slot(uint32_t *counter) {
    const unsigned mask = __activemask();
    const int leader = __ffs(mask) - 1;
    uint32_t base = 0;
    if ((int)lane_id() == leader) base = atomicAdd(counter, (uint32_t)__popc(mask));
    base = __shfl_sync(mask, base, leader);
    return base + __popc(mask & lanemask_lt());
}

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
__device__ __forceinline__ int block_excl_scan(int x, int *total, long long *sh) {
    long long t;
    const long long r = block_excl_scan64((long long)x, &t, sh);
    *total = (int)t;
    return (int)r;
}

__device__ __forceinline__ uint64_t ldrow(const uint8_t *M, int32_t v) {
    return __ldcg(reinterpret_cast<const unsigned long long *>(M) + v);
}

// fields of the status word st[v] (hm | K << 8 | nm << 16 | a << 24; K = 1: v holds a query keyword)
// gate (L210): 0 for a keyword node, else a_v
__device__ __forceinline__ uint32_t st_gate(uint32_t s) { return (s & 0x100u) ? 0u : (s >> 24); }
__device__ __forceinline__ uint32_t st_nm(uint32_t s) { return (s >> 16) & 0xFFu; }
// byte 1 bits 1-7 (rm): keyword i < 7 is reached from a node holding i and another query keyword along
// hitting arcs of keyword i (set at the level-0 merge for such sources, carried by visit_arc's reduction).
// In the exact reading the hitting arcs are the Thm. V.4 predecessor arcs, so rm(c) is exactly the set of
// keywords for which a two-keyword source lies in DAG_i(c) (central_graph's key cut-off validity).
constexpr uint32_t kRmMask = 0x7Fu;
__device__ __forceinline__ uint32_t st_rm(uint32_t s) { return (s >> 9) & kRmMask; }
__device__ __forceinline__ uint32_t st_act(uint32_t s) { return s >> 24; }
// the status word of a node nobody has hit yet: not a keyword node, a
__device__ __forceinline__ uint32_t st_fresh(uint32_t a) { return a << 24; }

struct Q {   // the query a group is answering
    int32_t qi;
    int q;
    uint32_t full;
    int32_t kw[kMaxQ];
};

// phase timestamp of the current query (group leader only)
__device__ __forceinline__ void stamp(const Grp &G, QOut *o, int tag) {
    if (G.gtid() == 0) {
        const int i = o->n_stamp;
        if (i < kMaxStamps) { o->stamp[i] = globaltimer_ns(); o->stamp_tag[i] = tag; o->n_stamp = i + 1; }
    }
}

// Every thread of the CTA passes its x; one global atomic per CTA adds the sum to *dst.
__device__ __forceinline__ void cta_add(unsigned long long x, unsigned long long *dst) {
    __shared__ unsigned long long s_acc;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_down_sync(0xffffffffu, x, o);
    if (threadIdx.x == 0) s_acc = 0ull;
    __syncthreads();
    if ((threadIdx.x & 31) == 0 && x) atomicAdd(&s_acc, x);
    __syncthreads();
    if (threadIdx.x == 0 && s_acc) atomicAdd(dst, s_acc);
}

// ------------------------------------------------------------------------------------------ frontier
// Non-empty flags of the level-slot bitmaps (0..255) and of the pre-pass round bitmaps (kFlagPd + 0/1) are
// kept per CTA in shared memory while a phase pushes, and published to the query's control block by
// publish_flags() before the group barrier that ends the phase (a global check-then-store per push
// stalled every pushing warp on an L2 round trip).
constexpr int kFlagPd = 256;
constexpr int kFlagSlots = kFlagPd + 2;
__device__ __forceinline__ uint32_t *cta_flags() {
    __shared__ uint32_t f[kFlagSlots];
    return f;
}

// Set v's bit in bitmap `bits` and mark CTA flag `fi`.  The bit is set with a reduction (no return
// value, nothing to wait for).
__device__ __forceinline__ void set_bit(uint32_t *bits, int fi, int32_t v) {
    uint32_t *word = bits + (v >> 5);
    const uint32_t bit = 1u << (v & 31);
    asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(word), "r"(bit) : "memory");
    atomicOr(cta_flags() + fi, 1u);   // the CTA's "slot non-empty" flag (shared; every writer sets the same bit)
}

// All threads of the CTA: publish the CTA's flags (then the caller's group barrier makes them visible).
__device__ __forceinline__ void publish_flags(Ctl *ctl) {
    __syncthreads();
    uint32_t *f = cta_flags();
    for (int t = threadIdx.x; t < kFlagSlots; t += blockDim.x)
        if (f[t]) {
            f[t] = 0u;
            if (t < kFlagPd) ctl->slot_flag[t] = 1u; else ctl->pd_flag[t - kFlagPd] = 1u;
        }
}

// append regions of the recorded DAG used by a group: one per CTA, at most kRecStripes
__device__ __forceinline__ int rec_stripes(const Grp &G) { return G.gcount < kRecStripes ? G.gcount : kRecStripes; }

struct Ctx {        // everything a group needs while answering one query
    const EngineArgs &a;
    const DevWork &w;
    Ctl *ctl;
    const Grp &G;
    const Q &qq;
    int rec_ns;         // append regions of the recorded DAG / pre-pass used by the group
    int rec_stripe;     // this CTA's region
    int64_t rec_cap;    // arcs per region
};

// the input id of internal node v (every id leaving the engine, and the ranking tie-break, is an input id)
__device__ __forceinline__ int32_t in_id(const EngineArgs &a, int32_t v) { return a.g.orig ? __ldg(a.g.orig + v) : v; }

// Schedule node v for the joint frontier of level L (FIdentifier[v] <- 1).
__device__ __forceinline__ void push(const Ctx &c, int32_t v, int L) {
    const int s = L < c.a.R ? L : L % c.a.R;   // L < R except for new hits past level R - 1 (no division)
    set_bit(c.w.fbits + (int64_t)s * c.a.W, s, v);
}

constexpr int kWpt = 8;   // bitmap words per thread per compaction step (two 16-byte loads)

// Enqueue frontiers: compact a bitmap (which is cleared) into the light / big queues.
// on_node(v) runs once per set bit and returns whether v goes to the aux list; on_aux(v, pos) runs when
// v is written there.  (A) extracts the node ids of a tile of words with stores only; (B) processes the
// tile's nodes one per thread.  Appends cost one atomic per CTA per tile.  A tile holding more than
// kLocalNodes set bits (dense regions: the hubs of the degree order, relabel.cu) processes that many
// locally and defers the rest to qdef (their queue positions); after the group barrier that follows,
// compact_deferred spreads the deferred nodes over every thread of the group.
constexpr int kLocalNodes = kBlock;

template <class OnNode, class OnAux>
__device__ __forceinline__ void compact_node(int32_t *ql, int64_t pos, const uint8_t *cls, int32_t *qb, uint32_t *nb,
                                             int32_t *aux, uint32_t *naux, OnNode &on_node, OnAux &on_aux) {
    const int32_t v = ql[pos];
    const bool flag = on_node(v);
    if (cls_big(cls[v])) { qb[atomicAdd(nb, 1u)] = v; ql[pos] = -1; }
    if (flag) {
        const uint32_t p = agg_slot(naux, 0x5u);
        aux[p] = v;
        on_aux(v, p);
    }
}

// The deferred nodes of compact(), strided over the group.  Call after a group barrier; returns whether
// there were any (then the caller needs another barrier before reading the queues).
template <class OnNode, class OnAux>
__device__ __forceinline__ bool compact_deferred(const Grp &G, const int32_t *qdef, uint32_t nd, int32_t *ql,
                                                 const uint8_t *cls, int32_t *qb, uint32_t *nb, int32_t *aux,
                                                 uint32_t *naux, OnNode on_node, OnAux on_aux) {
    constexpr int U = 4;   // the queue-position loads of U deferred nodes are in flight together
    for (int64_t j0 = G.gtid(); j0 < nd; j0 += U * G.gsz) {
        int64_t pos[U];
#pragma unroll
        for (int k = 0; k < U; ++k) pos[k] = j0 + k * G.gsz < nd ? (int64_t)__ldcg(qdef + j0 + k * G.gsz) : -1;
#pragma unroll
        for (int k = 0; k < U; ++k)
            if (pos[k] >= 0) compact_node(ql, pos[k], cls, qb, nb, aux, naux, on_node, on_aux);
    }
    return nd != 0;
}

template <class OnNode, class OnAux>
__device__ __forceinline__ void compact(const Grp &G, uint32_t *bits, int64_t W, const uint8_t *cls, int32_t *ql,
                                        uint32_t *nl, int32_t *qb, uint32_t *nb, int32_t *aux, uint32_t *naux,
                                        int32_t *qdef, uint32_t *ndef, long long *sh, uint32_t *tile_ctr, OnNode on_node,
                                        OnAux on_aux) {
    // tiles of blockDim * kWpt words taken from a counter (zero on entry): a CTA whose tiles hold many set
    // bits (the hub regions of the degree order) does not hold the whole group at the next barrier
    const int64_t step = (int64_t)blockDim.x * kWpt;
    for (;;) {
        __syncthreads();
        if (threadIdx.x == 0) sh[37] = (long long)atomicAdd(tile_ctr, 1u);
        __syncthreads();
        const int64_t base = sh[37] * step;
        if (base >= W) break;
        const int64_t w1 = base + step < W ? base + step : W;
        const int64_t wi = base + (int64_t)threadIdx.x * kWpt;
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
        __syncthreads();
        for (long long c0 = 0; c0 < tot; c0 += blockDim.x) {
            if (c0 >= kLocalNodes) {   // dense tile: the rest goes to the group-wide pass
                if (threadIdx.x == 0) sh[36] = (long long)atomicAdd(ndef, (uint32_t)(tot - c0));
                __syncthreads();
                const long long d0 = sh[36];
                for (long long j = c0 + threadIdx.x; j < tot; j += blockDim.x) qdef[d0 + j - c0] = (int32_t)(seg0 + j);
                __syncthreads();
                break;
            }
            const long long j = c0 + threadIdx.x;
            int32_t v = -1;
            int flag = 0;
            if (j < tot) {
                v = ql[seg0 + j];
                flag = on_node(v) ? 1 : 0;
                if (cls_big(cls[v])) { qb[atomicAdd(nb, 1u)] = v; ql[seg0 + j] = -1; }
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

// ------------------------------------------------------------------------------------------ expansion
// w in fixed point 2^-24, rounded down (weights are snapped to that grid at load, so this is exact).
// Saturating, and the path sums wrap modulo 2^32: either way the value never exceeds the true sum, so
// the pruning bound it feeds stays a lower bound.
__device__ __forceinline__ uint32_t weight_fx(float wt) {
    const double x = floor((double)wt * 16777216.0);
    return x <= 0.0 ? 0u : (x >= 4294967295.0 ? 0xFFFFFFFFu : (uint32_t)x);
}

// One inspected arc v -> x of Alg. 2 ln 12-22, for all keywords of v at once (hmv = v's snapshot mask,
// zbv = v's source bits (recorded DAG only) | rm(v) << 8, sx = st[x] gathered by the caller).
__device__ __forceinline__ void visit_arc(const Ctx &c, int l, int32_t v, uint32_t hmv, uint32_t zbv, int32_t x,
                                          uint32_t sx, unsigned &dag) {
    const uint32_t bits = hmv & ~sx & 0xFFu;            // ln 13-15: only instances where x is unhit
    if (!bits) return;
    const uint32_t gate = st_gate(sx);
    if (gate <= (uint32_t)(l + 1)) {                     // ln 16-18: keyword node or a_x <= l+1
        ++dag;                                            // a Thm. V.4 arc (v -> x for these keywords)
        if (c.a.dag_record) {   // recorded predecessor arc
            // one of kRecStripes append regions per CTA: a single counter would serialise millions of
            // atomics per heavy query on one address
            const int stripe = c.rec_stripe;
            const uint32_t ai = warp_slot(&c.ctl->rec_cnt[stripe * kRecStride]);
            const int64_t rcap = c.rec_cap;
            if ((int64_t)ai < rcap) {
                const int64_t r = stripe * rcap + ai;
                c.w.pa_u[r] = v;
                c.w.pa_x[r] = x;
                c.w.pa_b[r] = (uint16_t)(bits | ((zbv & 0xFFu) << 8));
            }
        }
        if (c.a.prune == 2) {   // x is hit at l+1 for these keywords: v is a Thm. V.4 predecessor of (x, i)
            for (uint32_t b = bits; b; b &= b - 1) {
                const int i = __ffs(b) - 1;
                atomicMin(c.w.mw + (int64_t)x * 8 + i, __ldcg(c.w.mw + (int64_t)v * 8 + i));
            }
        }
        // fire and forget (no returned value to wait for): every writer of this level sets the same bits and
        // writes the same level l+1 into entries whose hit bit was clear at the level's start, and the
        // frontier push is a bit set, so repeating them for arcs that lost a race changes nothing (Thm. V.2).
        // The new (node, keyword) pairs are counted when the next merge folds nm into hm.
        // with the new-hit bits, the keywords of these that a two-keyword source reaches v in (rm, byte 1)
        const uint32_t red = (bits << 16) | ((bits & (zbv >> 8) & kRmMask) << 9);
        asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(c.w.st + x), "r"(red) : "memory");
        uint8_t *row = c.w.M + (int64_t)x * 8;
        const uint8_t lv = (uint8_t)(l + 1);
#pragma unroll
        for (int i = 0; i < kMaxQ; ++i)
            if (bits & (1u << i)) row[i] = lv;            // ln 21: m_xi <- l+1
        push(c, x, l + 1);                                // ln 22: FIdentifier[x] <- 1
    } else {
        // ln 19: v must retry when x opens.  A node re-queues once per gated neighbour, often many times
        // at once (the arcs of one node are spread over lanes and warps): the lanes of a warp with the same
        // (node, level) push once, and the push is a fire-and-forget reduction (no read of the word first)
        const uint64_t key = ((uint64_t)(uint32_t)v << 8) | (uint64_t)(gate - 1);
        const unsigned peers = __match_any_sync(__activemask(), key);
        if ((int)lane_id() == __ffs(peers) - 1) push(c, v, (int)gate - 1);
    }
}

// Alg. 2 ln 2-7 for node v at level l: returns its expansion mask (0 = does not expand now).
__device__ __forceinline__ uint32_t prepare(const Ctx &c, int l, int32_t v, bool leader, uint32_t &rm) {
    const uint32_t sv = __ldcg(c.w.st + v);
    rm = st_rm(sv);
    const uint32_t hm = sv & 0xFFu;
    if (c.a.block_central && hm == c.qq.full) return 0;   // ln 2-3: central nodes do not expand
    const int av = (int)st_act(sv);
    if (av > l) {                                          // ln 5-7: not yet active
        if (leader) push(c, v, av);
        return 0;
    }
    return hm;                                             // ln 8-11: every hit instance has m <= l
}

constexpr int kTileMax = kBlock;
constexpr int kBigUnroll = 4;
#ifndef KGS_LIGHT_UNROLL
#define KGS_LIGHT_UNROLL 4
#endif
constexpr int kLightUnroll = KGS_LIGHT_UNROLL;

struct FwdNode {
    int32_t v;
    uint32_t hm;
    uint32_t zb;     // keywords for which v is a source (m = 0), recorded with its arcs
};

struct PullNode {   // a node x pulling at level l: its status word
    int32_t x;
    uint32_t sx;
};

struct PdNode {
    uint32_t P;      // keyword bits to expand backwards
    uint64_t hx;     // M row of the node
    int gx;          // gate - 1
    int32_t cidx;    // compact id
};

struct BigTile {
    long long incl[kTileMax];
    long long start[kTileMax];
    PdNode node[kTileMax];   // FwdNode fits in a PdNode slot
};

// Big frontier nodes (> kBigDeg arcs) in tiles of blockDim entries: every CTA of the group computes the
// same tile prefix of degrees in shared memory; the tile's arcs form one index space that all threads of
// the group stride over (owner found by binary search), kBigUnroll arcs per thread per step with the
// index and status gathers issued before any of them is processed.
template <class NodeT, class Prep, class Visit>
__device__ __forceinline__ void expand_big(const Grp &G, const int32_t *qb, uint32_t cb, const int64_t *ptr,
                                           const int32_t *idx, const uint32_t *st, BigTile &S, long long *sh,
                                           Prep prep, Visit visit, unsigned long long &arcs) {
    NodeT *node = reinterpret_cast<NodeT *>(S.node);
    for (uint32_t t0 = 0; t0 < cb; t0 += blockDim.x) {
        const int nt = (int)min((uint32_t)blockDim.x, cb - t0);
        const int j = threadIdx.x;
        long long deg = 0, s0 = 0;
        if (j < nt) {
            const int32_t v = __ldcg(qb + t0 + j);   // -1: a big node listed in the light queue
            NodeT nd{};
            if (v >= 0 && prep(v, G.grank == 0, nd)) { s0 = ptr[v]; deg = ptr[v + 1] - s0; }
            node[j] = nd;
            S.start[j] = s0;
        }
        long long T;
        const long long ex = block_excl_scan64(deg, &T, sh);
        S.incl[j] = ex + deg;
        __syncthreads();
        if (G.gtid() == 0) arcs += (unsigned long long)T;
        for (long long e = G.gtid(); e < T; e += kBigUnroll * G.gsz) {
            int own[kBigUnroll];
            int32_t x[kBigUnroll];
#pragma unroll
            for (int k = 0; k < kBigUnroll; ++k) {
                const long long ek = e + k * G.gsz;
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
            for (int k = 0; k < kBigUnroll; ++k) sx[k] = own[k] >= 0 ? __ldcg(st + x[k]) : 0u;
#pragma unroll
            for (int k = 0; k < kBigUnroll; ++k)
                if (own[k] >= 0) visit(node[own[k]], x[k], sx[k]);
        }
        __syncthreads();
    }
}

// Light frontier nodes: warp w of the group takes batches w, w + #warps, ... of B nodes each (no shared
// counter); the batch's arcs are balanced over the 32 lanes by a warp scan and a shuffle binary search.
// B = 32 when the frontier is large, fewer (down to 1) when it is small so that every warp gets work.
// Batch bi holds the queue entries bi, bi + nbatch, bi + 2 nbatch, ...: the queue is in node-id order,
// and in the degree order (relabel.cu) neighbouring ids have similar degrees, so strided batches mix
// degrees and cost about the same.  ql = nullptr sweeps the nodes 0..c0-1 in contiguous batches (pull).
// bctr (zero on entry, or null for the static assignment): warps take their batches from this counter, so a
// warp that drew heavy batches does not hold the group at the next barrier.  Used by query groups of at
// most kDynBatchCtas CTAs (batch mode); with the whole grid on one query (latency mode) the thousands of
// warps contending for one counter cost more than the imbalance (p50 0.252 -> 0.278 ms).
constexpr int kDynBatchCtas = 64;
template <class NodeT, class Prep, class Visit>
__device__ __forceinline__ void expand_light(const Grp &G, const int32_t *ql, uint32_t c0, const int64_t *ptr,
                                             const int32_t *idx, const uint32_t *st, Prep prep, Visit visit,
                                             unsigned long long &arcs, uint32_t *bctr = nullptr) {
    const uint32_t warps = (uint32_t)(G.gsz >> 5);
    uint32_t B = (c0 + 2 * warps - 1) / (2 * warps);
    B = B < 1 ? 1u : (B > 32 ? 32u : B);
    const uint32_t nbatch = (c0 + B - 1) / B;
    const unsigned lane = lane_id();
    auto next_batch = [&](uint32_t cur) -> uint32_t {
        if (!bctr) return cur + warps;
        uint32_t b = 0;
        if (lane == 0) b = atomicAdd(bctr, 1u) + warps;   // the first `warps` batches are taken statically
        return __shfl_sync(0xffffffffu, b, 0);
    };
    for (uint32_t bi = (uint32_t)(G.gtid() >> 5); bi < nbatch; bi = next_batch(bi)) {
        const uint32_t i = ql ? bi + lane * nbatch : bi * B + lane;   // no queue: nodes 0..c0-1, contiguous
        NodeT nd{};
        int64_t start = 0;
        int deg = 0;
        if (lane < B && i < c0) {
            const int32_t v = ql ? __ldcg(ql + i) : (int32_t)i;   // -1: a big node, expanded by expand_big
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
            for (int k = 0; k < kLightUnroll; ++k) sx[k] = x[k] >= 0 ? __ldcg(st + x[k]) : 0u;
#pragma unroll
            for (int k = 0; k < kLightUnroll; ++k)
                if (x[k] >= 0) visit(no[k], x[k], sx[k]);
        }
    }
}

// ------------------------------------------------------------------------------------------ pre-pass
// Thm. V.4 test of in-arc u -> x for the keyword bits P of x (hx = M row of x, gx = gate(x) - 1,
// su = st[u] gathered by the caller): m_xi = 1 + max{a_u, m_ui, g_x}, and in exact mode with blocking
// (reading R12) u was not central yet at level m_xi - 1.
__device__ __forceinline__ uint32_t pred_test(const Ctx &c, bool exact_block, uint32_t P, uint64_t hx, int gx,
                                              int32_t u, uint32_t su, uint32_t &zbu) {
    const uint32_t hmu = su & 0xFFu;
    uint32_t cand = P & hmu;
    if (!cand) return 0;
    const int au = (int)st_act(su);
    // m_xi = 1 + max{a_u, m_ui, g_x} needs a_u <= m_xi - 1: a test on the status word alone, before the
    // M row of u is loaded (most in-arcs of the pre-pass are not predecessor arcs)
    {
        const uint32_t rep = (uint32_t)au * 0x01010101u;   // per byte: m_xi > a_u
        const uint32_t g0 = __vcmpgtu4((uint32_t)hx, rep), g1 = __vcmpgtu4((uint32_t)(hx >> 32), rep);
        const uint32_t b0 = ((g0 >> 7) & 1u) | ((g0 >> 14) & 2u) | ((g0 >> 21) & 4u) | ((g0 >> 28) & 8u);
        const uint32_t b1 = ((g1 >> 7) & 1u) | ((g1 >> 14) & 2u) | ((g1 >> 21) & 4u) | ((g1 >> 28) & 8u);
        cand &= b0 | (b1 << 4);
    }
    if (!cand) return 0;
    const uint64_t Mu = ldrow(c.w.M, u);
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
        if ((int)((hx >> (8 * i)) & 0xFF) == need + 1) pb |= 1u << i;
    }
    if (pb && exact_block && hmu == c.qq.full) {
#pragma unroll
        for (int i = 0; i < kMaxQ; ++i)   // u central at depth maxrow: it only expanded at levels < maxrow
            if (((pb >> i) & 1u) && maxrow <= (int)((hx >> (8 * i)) & 0xFF) - 1) pb &= ~(1u << i);
    }
    zbu = zb;
    return pb;
}

__device__ __forceinline__ void pd_visit(const Ctx &c, bool exact_block, const PdNode &nd, int32_t u, uint32_t su,
                                         uint32_t *nbits, int nflag) {
    uint32_t zbu = 0;
    const uint32_t pb = pred_test(c, exact_block, nd.P, nd.hx, nd.gx, u, su, zbu);
    if (!pb) return;
    // the CTA's append region (as the recorded DAG: one counter per CTA, not one per group)
    const int stripe = c.rec_stripe;
    const uint32_t ai = warp_slot(&c.ctl->pd_cnt[stripe * kRecStride]);
    const int64_t rcap = c.rec_cap;
    if ((int64_t)ai < rcap) {   // a list slot only for a stored arc: the CSR never holds unwritten entries
        const uint32_t pos = agg_slot(reinterpret_cast<uint32_t *>(c.w.pcnt + nd.cidx), (unsigned)nd.cidx);
        const int64_t r = stripe * rcap + ai;
        c.w.pa_u[r] = u;
        c.w.pa_x[r] = nd.cidx;
        c.w.pa_b[r] = (uint16_t)(pb | (zbu << 8));
        c.w.pa_slot[r] = (int32_t)pos;
    } else {
        atomicExch(&c.ctl->fatal, 5);
    }
    const uint32_t nb = pb & ~zbu;        // sources (m = 0) have no predecessors
    if (nb) {
        const uint32_t old = atomicOr(c.w.pd_state + u, nb << 8);
        if (((old >> 8) & 0xFFu) == 0) set_bit(nbits, nflag, u);
    }
}

__device__ __forceinline__ bool pd_prepare(const Ctx &c, int32_t x, PdNode &nd) {
    nd.P = __ldcg(c.w.pd_state + x) & 0xFFu;
    nd.hx = ldrow(c.w.M, x);
    nd.gx = (int)st_gate(__ldcg(c.w.st + x)) - 1;
    nd.cidx = __ldcg(c.w.pd_cid + x);
    return nd.P != 0;
}

// every recorded arc index (the kRecStripes append regions of visit_arc), strided over the group
// (the region sizes are staged in shared memory once; a flat index finds its region by binary search)
template <class F>
__device__ __forceinline__ void for_each_record(const Ctx &c, const uint32_t *cnt, F fn) {
    const int ns = c.rec_ns;
    const int64_t rcap = c.rec_cap;
    __shared__ uint32_t s_pre[kRecStripes + 1];
    static_assert(kRecStripes <= kBlock, "one thread per region");
    static_assert(kRecStripes == 4 * kWarp, "four warps scan the region counts");
    __shared__ uint32_t s_wsum[4];
    __syncthreads();
    uint32_t incl = 0;
    if (threadIdx.x < kRecStripes) {   // inclusive scan of the region counts: warp scans + 4 warp totals
        const int64_t k = threadIdx.x < ns ? (int64_t)__ldcg(&cnt[threadIdx.x * kRecStride]) : 0;
        incl = (uint32_t)(k < rcap ? k : rcap);
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
            if ((int)lane_id() >= o) incl += t;
        }
        if (lane_id() == 31) s_wsum[threadIdx.x >> 5] = incl;
    }
    __syncthreads();
    if (threadIdx.x < kRecStripes) {
        for (int w = 0; w < (int)(threadIdx.x >> 5); ++w) incl += s_wsum[w];
        s_pre[threadIdx.x + 1] = incl;
        if (threadIdx.x == 0) s_pre[0] = 0;
    }
    __syncthreads();
    const int64_t T = s_pre[kRecStripes];
    for (int64_t j = c.G.gtid(); j < T; j += c.G.gsz) {
        int lo = 0, hi = kRecStripes - 1;   // region r with s_pre[r] <= j < s_pre[r + 1]
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if ((int64_t)s_pre[mid] <= j) lo = mid; else hi = mid - 1;
        }
        fn(lo * rcap + (j - (int64_t)s_pre[lo]));
    }
}

__device__ void build_pred_csr(const Ctx &c, long long *sh, QOut *qo);

__device__ void pred_dag(const Ctx &c, BigTile &S, long long *sh, QOut *qo, bool round2 = false,
                         int max_rounds = 1 << 30) {
    const Grp &G = c.G;
    Ctl *ctl = c.ctl;
    const bool exact_block = c.a.extract_mode == KGS_EXTRACT_EXACT && c.a.block_central;
    const int64_t W = c.a.W;
    // seeds (the candidates to extract, for every keyword they do not contain) were set by seed_pd: round 0
    // starts from them.  A second call continues the same DAG: done bits persist, the CSR is rebuilt.
    unsigned long long my_arcs = 0, my_arcs_big = 0;   // in-arcs of light / big (> kBigDeg in-arcs) nodes
    int r = 0;
    for (;; ++r) {
        const int slot = r & 1;
        if (!__ldcg(&ctl->pd_flag[slot])) break;
        if (r >= max_rounds) {
            // lazy round 2: the predecessors just found are not expanded further unless a candidate's walk
            // asks for them — drop the next round's frontier and its pending bits (pd_state byte 1)
            uint32_t *bits = c.w.pd_bits + (int64_t)slot * W;
            for (int64_t j = G.gtid(); j < W; j += G.gsz) {
                uint32_t x = __ldcg(bits + j);
                if (!x) continue;
                bits[j] = 0u;
                for (; x; x &= x - 1) {
                    const int32_t v = (int32_t)(j * 32 + __ffs(x) - 1);
                    c.w.pd_state[v] = __ldcg(c.w.pd_state + v) & ~0xFF00u;
                }
            }
            // every CTA has read pd_flag[slot] (and cleared its words) before the flag is reset: a CTA
            // reaching the check above after the reset would skip this barrier and desynchronise the group's
            // barriers (the one-GPU two-process runs hit it as illegal addresses / instructions, r02ag)
            G.sync();
            if (G.gtid() == 0) ctl->pd_flag[slot] = 0u;   // next read: the next call, after build_pred_csr's barriers
            break;
        }
        uint32_t *qn = ctl->pd_qn[slot];
        if (G.gtid() == 0) { ctl->pd_qn[slot ^ 1][0] = 0u; ctl->pd_qn[slot ^ 1][1] = 0u; ctl->pd_ctile[slot ^ 1] = 0u;
                           ctl->pd_xbatch[slot ^ 1] = 0u; }
        auto pd_node = [&](int32_t u) {
            const uint32_t s = __ldcg(c.w.pd_state + u);
            const uint32_t nx = (s >> 8) & 0xFFu, dn = (s >> 16) & 0xFFu;
            const uint32_t bits = nx & ~dn;
            c.w.pd_state[u] = bits | ((dn | bits) << 16);
            return bits != 0 && __ldcg(c.w.pd_cid + u) < 0;
        };
        auto pd_aux = [&](int32_t u, uint32_t pos) { c.w.pd_cid[u] = (int32_t)pos; };
        if (G.gtid() == 0) ctl->pd_ndef[slot ^ 1] = 0u;
        compact(G, c.w.pd_bits + (int64_t)slot * W, W, c.a.g.cls_in, c.w.pd_qlight, &qn[0], c.w.pd_qbig, &qn[1],
                c.w.pd_touched, &ctl->n_cid, c.w.qdef, &ctl->pd_ndef[slot], sh, &ctl->pd_ctile[slot], pd_node, pd_aux);
        G.sync();
        if (compact_deferred(G, c.w.qdef, __ldcg(&ctl->pd_ndef[slot]), c.w.pd_qlight, c.a.g.cls_in, c.w.pd_qbig,
                             &qn[1], c.w.pd_touched, &ctl->n_cid, pd_node, pd_aux))
            G.sync();
        stamp(G, qo, round2 ? TS_PD_MERGE2 : TS_PD_MERGE);
        const uint32_t c0 = __ldcg(&qn[0]), c1 = __ldcg(&qn[1]);
        if (G.gtid() == 0) ctl->pd_flag[slot] = 0u;
        uint32_t *nbits = c.w.pd_bits + (int64_t)(slot ^ 1) * W;
        const int nflag = kFlagPd + (slot ^ 1);
        auto prep = [&](int32_t x, bool, PdNode &nd) { return pd_prepare(c, x, nd); };
        auto visit = [&](const PdNode &nd, int32_t u, uint32_t su) { pd_visit(c, exact_block, nd, u, su, nbits, nflag); };
        expand_big<PdNode>(G, c.w.pd_qbig, c1, c.a.g.in_ptr, c.a.g.in_idx, c.w.st, S, sh, prep, visit, my_arcs_big);
        if (c0 <= (uint32_t)c.a.tile_light)   // small frontier: tiles over the whole group
            expand_big<PdNode>(G, c.w.pd_qlight, c0, c.a.g.in_ptr, c.a.g.in_idx, c.w.st, S, sh, prep, visit, my_arcs);
        else
            expand_light<PdNode>(G, c.w.pd_qlight, c0, c.a.g.in_ptr, c.a.g.in_idx, c.w.st, prep, visit, my_arcs,
                                 G.gcount <= kDynBatchCtas ? &ctl->pd_xbatch[slot] : nullptr);
        publish_flags(ctl);
        G.sync();
        stamp(G, qo, round2 ? TS_PD_EXPAND2 : TS_PD_EXPAND);
    }
    if (my_arcs + my_arcs_big) atomicAdd(&ctl->td_arcs, my_arcs + my_arcs_big);
    if (my_arcs_big) atomicAdd(&ctl->td_arcs_big, my_arcs_big);
    if (G.grank == 0) {   // the append regions' counts, one per thread, then a warp sum (not 128 serial loads)
        __shared__ uint32_t s_np;
        if (threadIdx.x == 0) s_np = 0;
        __syncthreads();
        uint32_t k = threadIdx.x < (unsigned)rec_stripes(G) ? __ldcg(&ctl->pd_cnt[threadIdx.x * kRecStride]) : 0u;
        k = __reduce_add_sync(0xffffffffu, k);
        if ((threadIdx.x & 31) == 0 && k) atomicAdd(&s_np, k);
        __syncthreads();
        if (threadIdx.x == 0) { ctl->pd_rounds = r; ctl->n_parcs = s_np; }
    }
    build_pred_csr(c, sh, qo);
}

// CSR of the predecessor lists: exclusive scan of pcnt over compact ids, then scatter of the arcs
// (pa_u / pa_x = compact id of the successor / pa_b / pa_slot = position in its list).
__device__ void build_pred_csr(const Ctx &c, long long *sh, QOut *qo) {
    const Grp &G = c.G;
    Ctl *ctl = c.ctl;
    const int64_t ncid = (int64_t)__ldcg(&ctl->n_cid);
    const int64_t chunk = (ncid + G.gcount - 1) / G.gcount;
    const int64_t lo = (int64_t)G.grank * chunk, hi = lo + chunk < ncid ? lo + chunk : ncid;
    // pass 1: the CTA's total over its chunk of compact ids
    int part = 0;
    for (int64_t j = lo + threadIdx.x; j < hi; j += blockDim.x) part += __ldcg(c.w.pcnt + j);
    {
        int tot;
        block_excl_scan(part, &tot, sh);
        if (threadIdx.x == 0) c.w.scan_tmp[G.grank] = tot;
    }
    G.sync();
    // pass 2: every CTA sums the totals before it itself (no serial scan on one CTA, no extra barrier),
    // then scans its chunk again writing the offsets
    int off = 0;
    {
        int p = 0;
        for (int b = threadIdx.x; b < G.grank; b += blockDim.x) p += __ldcg(c.w.scan_tmp + b);
        int tot;
        block_excl_scan(p, &tot, sh);
        off = tot;
    }
    int run = off;
    for (int64_t t0 = lo; t0 < lo + chunk; t0 += blockDim.x) {
        const int64_t j = t0 + threadIdx.x;
        const int v = j < hi ? __ldcg(c.w.pcnt + j) : 0;
        int tot;
        const int ex = block_excl_scan(v, &tot, sh);
        if (j < hi) c.w.pred_ptr[j] = run + ex;
        run += tot;
    }
    if (G.grank == G.gcount - 1 && threadIdx.x == 0) c.w.pred_ptr[ncid] = run;
    G.sync();
    auto scatter = [&](int64_t ai) {
        const int64_t pos = (int64_t)__ldcg(c.w.pred_ptr + c.w.pa_x[ai]) + c.w.pa_slot[ai];
        c.w.pred_u[pos] = c.w.pa_u[ai];
        c.w.pred_b[pos] = c.w.pa_b[ai];
    };
    for_each_record(c, ctl->rec_used ? ctl->rec_cnt : ctl->pd_cnt, scatter);
    G.sync();
    stamp(G, qo, TS_PD_CSR);
}

// Which keywords can a source holding two or more query keywords cover for c (the key cut-off's validity,
// central_graph)?  reach(x) = the keywords i such that some node v holding i and at least one other query
// keyword reaches x along predecessor arcs of keyword i (v in DAG_i(x)): over the shared DAG's arcs u -> x
// with keyword bits b, reach(x) |= b & (zb(u) if |zb(u)| >= 2) | b & reach(u), to a fixpoint (a chain is
// at most the search depth long).  Level-cover (R13) can only pick s* >= 2 for c if the keywords of the
// nodes contributing two or more cover Q with zb(c), and each such node v contributes i only if v is a
// source in DAG_i(c) — so s* >= 2 implies reach(c) | zb(c) = Q.  The DAG holds every closure arc of the
// candidates seeded so far (a superset of one candidate's), so reach over-approximates: the test is safe.
// Stored per compact id in lz (free until the lazy passes start; pcnt must keep the list counts, which a
// later lazy pre-pass round extends).
__device__ void mk_reach(const Ctx &c) {
    const Grp &G = c.G;
    Ctl *ctl = c.ctl;
    const uint32_t mk = __ldcg(&ctl->multi_kw) & c.qq.full;
    const int64_t ncid = (int64_t)__ldcg(&ctl->n_cid);
    uint32_t *R = reinterpret_cast<uint32_t *>(c.w.lz);
    for (int64_t j = G.gtid(); j < ncid; j += G.gsz) R[j] = 0u;
    if (G.gtid() == 0) { ctl->mk_changed[0] = 0u; ctl->mk_changed[1] = 0u; }
    G.sync();
    const uint32_t *cnt = ctl->rec_used ? ctl->rec_cnt : ctl->pd_cnt;
    for (int pass = 0;; ++pass) {
        bool changed = false;
        for_each_record(c, cnt, [&](int64_t ai) {
            const uint32_t b = c.w.pa_b[ai];
            const uint32_t pb = b & 0xFFu & mk;
            if (!pb) return;
            // (the records stay as they are: a lazy pre-pass round after this rebuilds the CSR from them)
            const int32_t cu = __ldcg(c.w.pd_cid + __ldcg(c.w.pa_u + ai));
            const uint32_t zbu = b >> 8;
            const uint32_t add = pb & ((__popc(zbu) >= 2 ? zbu : 0u) | (cu >= 0 ? __ldcg(R + cu) : 0u));
            if (!add) return;
            const int32_t xc = c.w.pa_x[ai];
            if (add & ~__ldcg(R + xc)) { atomicOr(R + xc, add); changed = true; }
        });
        if (__syncthreads_or(changed) && threadIdx.x == 0) ctl->mk_changed[pass & 1] = 1u;
        G.sync();
        const bool more = __ldcg(&ctl->mk_changed[pass & 1]) != 0u;
        if (G.gtid() == 0) ctl->mk_changed[(pass + 1) & 1] = 0u;   // read by every CTA before the next barrier
        G.sync();
        if (!more) break;
    }
    if (G.gtid() == 0) ctl->mk_reach = 1u;
    G.sync();
}

// ------------------------------------------------------------------------------------------ search
// The previous query's lightest-path rows (prune mode 2), through its touched list (always complete).
__device__ void reset_mw_prev(const Ctx &c) {
    const DevWork &w = c.w;
    const uint32_t done = __ldcg(w.gstate + 1);
    if (done == 0 || !w.ctl[(done + 1) & 1]->mw_dirty) return;
    const Ctl *pv = w.ctl[(done + 1) & 1];
    const int64_t pt = (int64_t)pv->n_touched;
    const uint4 ones = make_uint4(~0u, ~0u, ~0u, ~0u);
    for (int64_t j = c.G.gtid(); j < 2 * pt; j += c.G.gsz) {
        const int32_t v = w.touched[j >> 1];
        reinterpret_cast<uint4 *>(w.mw + (int64_t)v * 8)[j & 1] = ones;
    }
}

// Top-down only (the state of a vertex-partitioned search, vpart.cu): clear what the previous query
// left in the predecessor pre-pass state, then take |C|, the stop level and reason from the host.
__device__ void td_only_prepare(const Ctx &c, QOut *qo) {
    const DevWork &w = c.w;
    const int64_t gtid = c.G.gtid(), gsz = c.G.gsz, n = c.a.g.n;
    reset_mw_prev(c);
    const uint32_t valid = __ldcg(w.gstate + 2), done = __ldcg(w.gstate + 1);
    if (!valid || done == 0) {
        for (int64_t j = gtid; j < 2 * c.a.W; j += gsz) w.pd_bits[j] = 0u;
        for (int64_t v = gtid; v < n; v += gsz) { w.pd_state[v] = 0u; w.pd_cid[v] = -1; w.pcnt[v] = 0; }
    } else {
        const Ctl *pv = w.ctl[(done + 1) & 1];
        for (int64_t j = gtid; j < (int64_t)pv->n_cid; j += gsz) {
            const int32_t v = w.pd_touched[j];
            w.pd_state[v] = 0u; w.pd_cid[v] = -1; w.pcnt[j] = 0;
        }
    }
    if (gtid == 0) {
        c.ctl->n_central = c.a.td_ncentral;
        c.ctl->levels = c.a.td_levels;
        c.ctl->stop_reason = c.a.td_stop;
        qo->t_search_end = globaltimer_ns();
    }
    c.G.sync();
    stamp(c.G, qo, TS_END);
}

// One pulled level l (kgs_params.direction; called by search()): light candidates by a contiguous sweep of
// all nodes, the ones with more than kBigDeg in-arcs afterwards in group-wide tiles.  (Inlined: out of line, the
// call spilled the push path's level-loop state, p50 0.35 -> 0.43 ms; tools/ab_perf.py.)
__device__ __forceinline__ void pull_expand(const Ctx &c, int l, BigTile &S, long long *sh,
                                         unsigned &my_dag, unsigned long long &my_arcs) {
    const Grp &G = c.G;
    const EngineArgs &a = c.a;
    const DevWork &w = c.w;
    Ctl *ctl = c.ctl;
    const int64_t n = a.g.n;
    const uint32_t full = c.qq.full;
    auto pprep = [&](int32_t x, bool, PullNode &nd) {
        const uint32_t sx = __ldcg(w.st + x);
        nd.x = x;
        nd.sx = sx;
        return (full & ~sx & 0xFFu) != 0u && st_gate(sx) <= (uint32_t)(l + 1);
    };
    auto plight = [&](int32_t x, bool leader, PullNode &nd) {
        if (!pprep(x, leader, nd)) return false;
        if (cls_big(a.g.cls_in[x])) {   // many in-arcs: tiles over the group, after the sweep
            w.pd_qbig[warp_slot(&ctl->pull_nbig[l & 1])] = x;   // (sized for the big-in nodes; idle now)
            return false;
        }
        return true;
    };
    auto pvisit = [&](const PullNode &nd, int32_t u, uint32_t su) {
        const uint32_t hmu = su & 0xFFu;
        if (!(hmu & ~nd.sx & 0xFFu)) return;                 // u has none of the keywords x lacks
        if (a.block_central && hmu == full) return;           // ln 2-3
        if ((int)st_act(su) > l) return;                     // ln 4-7
        uint32_t zb = 0;
        if (a.dag_record) {
            const uint64_t row = ldrow(w.M, u);
            for (uint32_t b = hmu; b; b &= b - 1) {
                const int i = __ffs(b) - 1;
                if (((row >> (8 * i)) & 0xFF) == 0) zb |= 1u << i;
            }
        }
        visit_arc(c, l, u, hmu, zb | (st_rm(su) << 8), nd.x, nd.sx, my_dag);
    };
    expand_light<PullNode>(G, nullptr, (uint32_t)n, a.g.in_ptr, a.g.in_idx, w.st, plight, pvisit, my_arcs);
    G.sync();
    expand_big<PullNode>(G, w.pd_qbig, __ldcg(&ctl->pull_nbig[l & 1]), a.g.in_ptr, a.g.in_idx, w.st, S, sh,
                         pprep, pvisit, my_arcs);
}

// After a pulled level l without hits: would the work list of Alg. 2 (FIdentifier) still hold a node at
// level l + 1?  The pull has no work list, so this recomputes membership: a hit node v (not a blocked
// central) is re-queued at l iff it is inactive (a_v > l, ln 5-7) or it has an out-neighbour x that lacks
// one of v's keywords behind a closed gate (gate(x) > l + 1, ln 17-20).  Both conditions can only turn
// false as l grows unless v gains a keyword, which puts v on the list, so every node satisfying one is
// on the list.  Sets ctl->pull_wait[l & 1]; nodes stop scanning once it is set.  Group-wide, ends with a
// barrier.  Then the stop level of a pulling search is the work-list form's (the oracle's literal Alg. 2).
__device__ __forceinline__ void pull_waiting(const Ctx &c, int l, BigTile &S, long long *sh) {
    const Grp &G = c.G;
    const EngineArgs &a = c.a;
    const DevWork &w = c.w;
    Ctl *ctl = c.ctl;
    const uint32_t full = c.qq.full;
    volatile uint32_t *flag = &ctl->pull_wait[l & 1];
    unsigned long long arcs = 0;
    auto wprep = [&](int32_t v, bool, PullNode &nd) {
        const uint32_t sv = __ldcg(w.st + v);
        const uint32_t hm = sv & 0xFFu;
        if (!hm || (a.block_central && hm == full) || *flag) return false;
        if ((int)st_act(sv) > l) { *flag = 1u; return false; }
        nd.x = v;
        nd.sx = hm;
        return true;
    };
    auto wlight = [&](int32_t v, bool leader, PullNode &nd) {
        if (!wprep(v, leader, nd)) return false;
        if (cls_big(a.g.cls[v])) { w.qbig[warp_slot(&ctl->pull_wbig[l & 1])] = v; return false; }
        return true;
    };
    auto wvisit = [&](const PullNode &nd, int32_t x, uint32_t sx) {
        if ((nd.sx & ~sx & 0xFFu) && st_gate(sx) > (uint32_t)(l + 1) && !*flag) *flag = 1u;
    };
    expand_light<PullNode>(G, nullptr, (uint32_t)a.g.n, a.g.row_ptr, a.g.col_idx, w.st, wlight, wvisit, arcs);
    G.sync();
    expand_big<PullNode>(G, w.qbig, __ldcg(&ctl->pull_wbig[l & 1]), a.g.row_ptr, a.g.col_idx, w.st, S, sh,
                         wprep, wvisit, arcs);
    G.sync();
}

// Every node's status word to "not hit yet" (hm = nm = 0, gate = a, a), 4 nodes per 16-byte store.
__device__ void reset_status_dense(const Ctx &c) {
    const int64_t n = c.a.g.n, n4 = n / 4;
    for (int64_t j = c.G.gtid(); j < n4; j += c.G.gsz) {
        const uint32_t a4 = *reinterpret_cast<const uint32_t *>(c.a.act + j * 4);
        uint4 o;
        o.x = st_fresh(a4 & 0xFFu);
        o.y = st_fresh((a4 >> 8) & 0xFFu);
        o.z = st_fresh((a4 >> 16) & 0xFFu);
        o.w = st_fresh(a4 >> 24);
        reinterpret_cast<uint4 *>(c.w.st)[j] = o;
    }
    for (int64_t v = n4 * 4 + c.G.gtid(); v < n; v += c.G.gsz) c.w.st[v] = st_fresh(c.a.act[v]);
}

__device__ void search(const Ctx &c, BigTile &S, long long *sh, QOut *qo) {
    const Grp &G = c.G;
    const EngineArgs &a = c.a;
    const DevWork &w = c.w;
    Ctl *ctl = c.ctl;
    const int64_t n = a.g.n, W = a.W;
    const int R = a.R, amax = R - 2;
    const uint32_t full = c.qq.full;
    const int64_t gtid = G.gtid(), gsz = G.gsz;

    // ---- reset the state the previous query of this group left behind
    const uint32_t valid = __ldcg(w.gstate + 2), lastR = __ldcg(w.gstate + 3);
    const uint32_t done = __ldcg(w.gstate + 1);
    reset_mw_prev(c);
    if (!valid || (int)lastR != R || done == 0) {
        reset_status_dense(c);
        for (int64_t j = gtid; j < (int64_t)R * W; j += gsz) w.fbits[j] = 0u;
        for (int64_t j = gtid; j < 2 * W; j += gsz) w.pd_bits[j] = 0u;
        for (int64_t v = gtid; v < n; v += gsz) { w.pd_state[v] = 0u; w.pd_cid[v] = -1; w.pcnt[v] = 0; }
    } else {
        const Ctl *pv = w.ctl[(done + 1) & 1];   // the previous query's block
        // Predecessor-list state (pd_cid compact ids, pd_state).  A recorded-DAG query gives compact ids to
        // all of its touched nodes and reads pd_cid / pd_state of no other node (closures and recorded arcs
        // only hold hit nodes), so it resets neither — it only leaves the workspace "dirty" (gstate[2] bit
        // 1).  A pre-pass query reads pd_cid / pd_state of its closure nodes, which may have been touched by
        // any earlier query: after dirty queries it resets both densely (sequential writes), otherwise the
        // previous pre-pass's list.  pcnt is indexed by compact id: its prefix is reset in every case.
        const bool dirty = (valid & 2u) != 0;
        const int64_t pn = (int64_t)pv->n_cid;
        if (a.dag_record) {
            for (int64_t j = gtid; j < pn; j += gsz) w.pcnt[j] = 0;
        } else if (dirty) {
            for (int64_t v = gtid; v < n; v += gsz) { w.pd_state[v] = 0u; w.pd_cid[v] = -1; w.pcnt[v] = 0; }
        } else {
            for (int64_t j = gtid; j < pn; j += gsz) {
                const int32_t v = w.pd_touched[j];
                w.pd_state[v] = 0u; w.pd_cid[v] = -1; w.pcnt[j] = 0;
            }
        }
        const int64_t pt = (int64_t)pv->n_touched;
        if (pt > n / 16) {   // many touched rows: a dense sweep beats scattered 2-byte writes
            reset_status_dense(c);
        } else {
            for (int64_t j = gtid; j < pt; j += gsz) {
                const int32_t v = w.touched[j];
                w.st[v] = st_fresh(st_act(__ldcg(w.st + v)));   // a_v is byte 3 of the word itself
            }
        }
        for (int s = 0; s < R; ++s)   // level slots still pending when the previous query stopped
            if (pv->slot_flag[s])
                for (int64_t j = gtid; j < W; j += gsz) w.fbits[(int64_t)s * W + j] = 0u;
    }
    bool empty = false;
    for (int i = 0; i < c.qq.q; ++i) {
        const int32_t t = c.qq.kw[i];
        if (a.g.kw_ptr[t + 1] == a.g.kw_ptr[t]) empty = true;
    }
    if (gtid == 0) ctl->mw_dirty = a.prune == 2 ? 1u : 0u;
    G.sync();
    stamp(G, qo, TS_RESET);
    // ---- initialisation: M = 0 on T_i, keyword nodes ungated, F_0 = K
    {
        __shared__ int64_t kb[kMaxQ], ko[kMaxQ + 1];   // the keywords' postings, concatenated (shared: no stack)
        if (threadIdx.x == 0) {
            ko[0] = 0;
            for (int i = 0; i < c.qq.q; ++i) {
                const int32_t t = c.qq.kw[i];
                kb[i] = a.g.kw_ptr[t];
                ko[i + 1] = ko[i] + (a.g.kw_ptr[t + 1] - kb[i]);
            }
        }
        __syncthreads();
        for (int64_t j = gtid; j < ko[c.qq.q]; j += gsz) {
            int i = 0;
            while (j >= ko[i + 1]) ++i;
            const int32_t v = a.g.kw_nodes[kb[i] + (j - ko[i])];
            w.M[(int64_t)v * 8 + i] = 0;
            if (a.prune == 2) w.mw[(int64_t)v * 8 + i] = 0u;              // the path {v}: w_v added at merge
            // keyword node (no gate, L210) and hit in B_i at level 0 (new-hit bit i): one atomic
            atomicOr(w.st + v, 0x100u | ((1u << i) << 16));
            push(c, v, 0);
        }
    }
    publish_flags(ctl);
    G.sync();
    stamp(G, qo, TS_SCATTER);

    unsigned long long my_arcs = 0;
    unsigned my_hits = 0, my_dag = 0;
    // push / pull (kgs_params.direction): once a level pulls, every later level pulls too; a pulling
    // search ends by the level rule (no new hit at l >= amax) instead of the empty work-list
    bool pulling = false;
    const bool count_mf = a.direction == KGS_DIR_AUTO;
    // the frontier's arcs are counted (two byte loads per frontier node in the merge, 2-3% of a query)
    // only at levels that follow a frontier of more than n / (4 pull_ratio) nodes: a level cannot reach
    // m / pull_ratio out-arcs from a frontier much smaller than that (the graph's mean degree is m / n),
    // and level 0 (the keyword nodes) is never pulled in the automatic mode
    bool count_lvl = false;
    unsigned long long my_mf = 0;
    for (int l = 0;; ++l) {
        // ---- enqueue frontiers: anything pending at this or a later level?
        int any_pend = 1;
        if (!pulling) {   // the slot flags of levels l..max(l, amax), one per thread (R <= 256 slots)
            const int top = l > amax ? l : amax;
            const int L = l + (int)threadIdx.x;
            const bool pend = L <= top && __ldcg(&ctl->slot_flag[L < R ? L : L % R]) != 0u;
            any_pend = __syncthreads_or(pend);
        }
        if (!any_pend) {
            if (gtid == 0) { ctl->stop_reason = empty ? KGS_STOP_EMPTY_KEYWORD : KGS_STOP_EXHAUSTED; ctl->levels = l; }
            break;
        }
        const int s = l % R;
        uint32_t *qn = ctl->qn[l & 1];
        if (gtid == 0) {
            ctl->qn[(l + 1) & 1][0] = 0u; ctl->qn[(l + 1) & 1][1] = 0u; ctl->ndef[(l + 1) & 1] = 0u;
            ctl->ctile[(l + 1) & 1] = 0u; ctl->xbatch[(l + 1) & 1] = 0u;
            ctl->mf[(l + 1) & 1] = 0ull; ctl->pull_nbig[(l + 1) & 1] = 0u;
        }
        // compact the level's bitmap; merge new hits into hm and identify central nodes (L262-266)
        auto merge_node = [&](int32_t v) {
                    // auto direction: out-arcs of the frontier nodes that can expand (a_v <= l, ln 4-7),
                    // bounded by the power of two of the class byte (no row_ptr load)
                    const uint32_t sv = __ldcg(w.st + v);
                    if (count_lvl && !pulling && (int)st_act(sv) <= l)
                        my_mf += cls_deg_bound(a.g.cls[v]);
                    const uint32_t b = st_nm(sv);
                    if (!b) return false;
                    uint32_t rself = 0;   // a source of two or more query keywords reaches itself (st_rm)
                    if (l == 0 && (b & (b - 1))) { atomicOr(&ctl->multi_kw, b); rself = (b & kRmMask) << 9; }
                    if (l > 0) my_hits += __popc(b);   // new (node, keyword) pairs of level l - 1's expansion
                    const uint32_t old = sv & 0xFFu;
                    const uint32_t nw = old | b;
                    w.st[v] = (sv & 0xFF00FF00u) | nw | rself;   // hm |= nm, nm = 0 (no expansion runs during the merge)
                    if (a.prune == 2) {   // lightest path to v for keyword i = min over predecessors + w_v
                        const uint32_t wv = weight_fx(__ldg(a.g.weight + v));
                        for (uint32_t bb = b; bb; bb &= bb - 1) {
                            uint32_t *p = w.mw + (int64_t)v * 8 + (__ffs(bb) - 1);
                            *p = *p + wv;
                        }
                    }
                    if (nw == full && old != full) {                        // Lemma V.1: depth = l
                        const uint32_t ci = agg_slot(&ctl->n_central, 1u);
                        w.centrals[ci] = v;
                        w.cdepth[ci] = (uint8_t)l;
                    }
                    return old == 0;
                };
        auto merge_aux = [&](int32_t v, uint32_t pos) {   // recorded DAG: compact id = touched position
            if (a.dag_record) { w.pd_touched[pos] = v; w.pd_cid[v] = (int32_t)pos; }
        };
        compact(G, w.fbits + (int64_t)s * W, W, a.g.cls, w.qlight, &qn[0], w.qbig, &qn[1], w.touched,
                &ctl->n_touched, w.qdef, &ctl->ndef[l & 1], sh, &ctl->ctile[l & 1], merge_node, merge_aux);
        if (count_lvl && !pulling) { cta_add(my_mf, &ctl->mf[l & 1]); my_mf = 0; }
        G.sync();
        if (compact_deferred(G, w.qdef, __ldcg(&ctl->ndef[l & 1]), w.qlight, a.g.cls, w.qbig, &qn[1], w.touched,
                             &ctl->n_touched, merge_node, merge_aux)) {
            if (count_lvl && !pulling) { cta_add(my_mf, &ctl->mf[l & 1]); my_mf = 0; }
            G.sync();
        }
        if (gtid == 0) {   // their last readers (level l - 1) passed the barrier above
            ctl->pull_marks[(l + 1) & 1] = 0ull;
            ctl->pull_wait[(l + 1) & 1] = 0u; ctl->pull_wbig[(l + 1) & 1] = 0u;
        }
        stamp(G, qo, TS_MERGE);
        __shared__ uint32_t s_ctl[3];
        if (threadIdx.x == 0) { s_ctl[0] = __ldcg(&qn[0]); s_ctl[1] = __ldcg(&qn[1]); s_ctl[2] = __ldcg(&ctl->n_central); }
        __syncthreads();
        const uint32_t c0 = s_ctl[0], c1 = s_ctl[1], nc = s_ctl[2];
        if (gtid == 0) ctl->frontier_total += (unsigned long long)c0 + c1;
        const bool count_this = count_lvl;
        count_lvl = count_mf && ((unsigned long long)c0 + c1) * 4ull * (unsigned long long)a.pull_ratio > (unsigned long long)n;
        // ---- termination (Def. 4 / Thm. V.3; reading R9: no expansion at d)
        if (empty) {   // some T_i is empty: M holds the initialisation, nothing can be central (R17)
            if (gtid == 0) { ctl->stop_reason = KGS_STOP_EMPTY_KEYWORD; ctl->levels = 0; }
            break;
        }
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
        if (!pulling && (a.direction == KGS_DIR_PULL ||
                         (count_this && __ldcg(&ctl->mf[l & 1]) * (unsigned long long)a.pull_ratio > (unsigned long long)a.g.m &&
                          __ldcg(&ctl->mf[l & 1]) > (unsigned long long)a.pull_min))) {
            pulling = true;
            if (gtid == 0) ctl->pull_at = l + 1;
        }
        if (pulling) {
            // Pull (the level rule): every x that lacks a keyword and whose gate is open
            // (x in K or a_x <= l+1, ln 16-17) scans its in-arcs u -> x; an active u (a_u <= l, not a
            // blocked central, ln 2-7) hits x for the keywords it has and x lacks (ln 12-22).  The same
            // visit_arc as the push, so the hits, the recorded Thm. V.4 arcs and the lightest-path rows
            // are the same; no node is re-queued (ln 19): a pulling search has no work list (a level
            // without hits asks pull_waiting whether the list would still be non-empty).
            const unsigned dag0 = my_dag;   // hitting arcs of this level: some (node, keyword) was marked
            pull_expand(c, l, S, sh, my_dag, my_arcs);
            cta_add((unsigned long long)(my_dag - dag0), &ctl->pull_marks[l & 1]);
            publish_flags(ctl);
            G.sync();
            stamp(G, qo, TS_EXPAND);
            if (__ldcg(&ctl->pull_marks[l & 1]) == 0ull) {
                // no hit at l: the work list at l + 1 holds only re-queued nodes (none once l >= amax)
                bool waiting = false;
                if (l < amax) {
                    pull_waiting(c, l, S, sh);
                    waiting = __ldcg(&ctl->pull_wait[l & 1]) != 0u;
                }
                if (!waiting) {
                    if (gtid == 0) { ctl->stop_reason = KGS_STOP_EXHAUSTED; ctl->levels = l + 1; }
                    break;
                }
            }
            continue;
        }
        auto prep = [&](int32_t v, bool leader, FwdNode &nd) {
            nd.v = v;
            uint32_t rm;
            nd.hm = prepare(c, l, v, leader, rm);
            nd.zb = rm << 8;   // zb (recorded DAG) in bits 0-7, rm in bits 8-14
            if (a.dag_record && nd.hm) {
                const uint64_t row = ldrow(w.M, v);
                for (uint32_t b = nd.hm; b; b &= b - 1) {
                    const int i = __ffs(b) - 1;
                    if (((row >> (8 * i)) & 0xFF) == 0) nd.zb |= 1u << i;
                }
            }
            return nd.hm != 0;
        };
        auto visit = [&](const FwdNode &nd, int32_t x, uint32_t sx) {
            visit_arc(c, l, nd.v, nd.hm, nd.zb, x, sx, my_dag);
        };
        expand_big<FwdNode>(G, w.qbig, c1, a.g.row_ptr, a.g.col_idx, w.st, S, sh, prep, visit, my_arcs);
        if (c0 <= (uint32_t)a.tile_light)   // small frontier: tiles over the whole group
            expand_big<FwdNode>(G, w.qlight, c0, a.g.row_ptr, a.g.col_idx, w.st, S, sh, prep, visit, my_arcs);
        else
            expand_light<FwdNode>(G, w.qlight, c0, a.g.row_ptr, a.g.col_idx, w.st, prep, visit, my_arcs,
                                  G.gcount <= kDynBatchCtas ? &ctl->xbatch[l & 1] : nullptr);
        publish_flags(ctl);
        G.sync();
        stamp(G, qo, TS_EXPAND);
    }
    const unsigned wa = __reduce_add_sync(0xffffffffu, (unsigned)my_arcs);   // per-warp totals fit 32 bits
    const unsigned wh = __reduce_add_sync(0xffffffffu, my_hits);
    const unsigned wd = __reduce_add_sync(0xffffffffu, my_dag);
    __shared__ unsigned long long s_sum[3];
    if (threadIdx.x < 3) s_sum[threadIdx.x] = 0ull;
    __syncthreads();
    if ((threadIdx.x & 31) == 0) {
        if (wa) atomicAdd(&s_sum[0], (unsigned long long)wa);
        if (wh) atomicAdd(&s_sum[1], (unsigned long long)wh);
        if (wd) atomicAdd(&s_sum[2], (unsigned long long)wd);
    }
    __syncthreads();
    if (threadIdx.x == 0) {      // one global atomic per CTA
        if (s_sum[0]) atomicAdd(&ctl->arcs_scanned, s_sum[0]);
        if (s_sum[1]) atomicAdd(&ctl->hits, s_sum[1]);
        if (s_sum[2]) atomicAdd(&ctl->dag_arcs, s_sum[2]);
    }
    G.sync();
    stamp(G, qo, TS_END);
    if (gtid == 0) qo->t_search_end = globaltimer_ns();
}

// ------------------------------------------------------------------------------------------ recorded DAG
// The search recorded every arc v -> x that hit x (Alg. 2 ln 16-21) with its keyword bits: exactly the
// Thm. V.4 predecessor arcs of the exact reading R12 (a blocked central never expands, and every node
// that can expand keyword i into x at level m_xi - 1 is scanned at that level).  Turn them
// into the predecessor CSR keyed by the compact ids the merge gave the touched nodes.  Returns false
// (and leaves the pre-pass state clean) when the record buffer overflowed.
__device__ bool recorded_dag(const Ctx &c, long long *sh, QOut *qo, unsigned long long max_arcs) {
    const Grp &G = c.G;
    Ctl *ctl = c.ctl;
    const DevWork &w = c.w;
    const uint32_t nt = __ldcg(&ctl->n_touched);
    __shared__ unsigned long long s_rec[2];
    if (threadIdx.x == 0) { s_rec[0] = 0ull; s_rec[1] = 0ull; }
    __syncthreads();
    {   // the append regions' counts, one per thread (not 128 serial loads by one thread)
        const int ns = rec_stripes(G);
        const int64_t k = threadIdx.x < (unsigned)ns ? (int64_t)__ldcg(&ctl->rec_cnt[threadIdx.x * kRecStride]) : 0;
        const unsigned long long tot = __reduce_add_sync(0xffffffffu, (unsigned)k);   // < 2^32 per warp (pcap)
        const unsigned over = __any_sync(0xffffffffu, k > w.pcap / ns);
        if ((threadIdx.x & 31) == 0) {
            if (tot) atomicAdd(&s_rec[0], tot);
            if (over) s_rec[1] = 1ull;
        }
    }
    __syncthreads();
    // a region overflowed, or the record is large while pruning will run (the lists of every touched node
    // cost more than the pre-pass's targeted closures and the lazy round 2, r02ai): forget the compact ids,
    // use the pre-pass
    if (s_rec[1] || s_rec[0] > max_arcs) {
        for (int64_t j = G.gtid(); j < nt; j += G.gsz) {   // the pre-pass reads both for its (touched) nodes
            const int32_t v = __ldcg(w.pd_touched + j);
            w.pd_cid[v] = -1;
            w.pd_state[v] = 0u;
        }
        G.sync();
        if (G.gtid() == 0) { ctl->n_parcs = 0; ctl->n_cid = 0; ctl->rec_overflow = 1; }
        G.sync();
        return false;
    }
    for_each_record(c, ctl->rec_cnt, [&](int64_t r) {
        const int32_t cid = __ldcg(w.pd_cid + __ldcg(w.pa_x + r));
        w.pa_x[r] = cid;
        w.pa_slot[r] = atomicAdd(w.pcnt + cid, 1);
    });
    if (G.gtid() == 0) { ctl->n_cid = nt; ctl->rec_used = 1; ctl->n_parcs = (uint32_t)s_rec[0]; }
    G.sync();
    stamp(G, qo, TS_PD_MERGE);
    build_pred_csr(c, sh, qo);
    return true;
}

// ------------------------------------------------------------------------------------------ top-down
struct WarpTeam {
    __device__ __forceinline__ int rank() const { return threadIdx.x & 31; }
    __device__ __forceinline__ int size() const { return 32; }
    __device__ __forceinline__ void sync() const { __syncwarp(); }
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
    long long *sh;   // block scan scratch (>= 40 entries)
    __device__ __forceinline__ int rank() const { return threadIdx.x; }
    __device__ __forceinline__ int size() const { return blockDim.x; }
    __device__ __forceinline__ void sync() const { __syncthreads(); }
    __device__ __forceinline__ int scan_excl(int x, int *total) const { return block_excl_scan(x, total, sh); }
};

enum { SC_NODES = 0, SC_ARCS, SC_HEAD, SC_TAIL, SC_OVF, SC_CHANGED, SC_COV, SC_SSTAR, SC_NOUT, SC_AOUT, SC_CUT, SC_INC, SC_N };

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
    int64_t *b_start;   // [team] batch: predecessor-list start
    int32_t *b_incl;    // [team] batch: inclusive count
    uint32_t *b_P;      // [team] batch: keywords to expand
    unsigned long long *sortbuf;  // [2*acap]
    int32_t *scal;      // [SC_N]
    double *dsum;
    unsigned long long *wsum;     // closure weight so far, 2^-24 fixed point (key cut-off)
    int32_t *hslot;     // [ncap] hash slot of node j (persistent arenas: lazy reset of the next use)
    int32_t *magic;     // kArenaMagic once the arena has been fully reset (persistent arenas)
    int hcap, ncap, acap;
};

// persistent: a global-memory arena that keeps its state between uses (and launches): the next use
// resets only the hash slots and node rows the previous one touched, unless it overflowed.
__host__ __device__ inline size_t arena_bytes(int hcap, int ncap, int acap, int team, bool with_sort,
                                              bool persistent = false) {
    size_t b = 16 + sizeof(int64_t) * team + sizeof(double) + sizeof(unsigned long long);
    if (persistent) b += sizeof(int32_t) * (size_t)ncap + 16;
    if (with_sort) b += sizeof(unsigned long long) * 2 * (size_t)acap;
    b += sizeof(int32_t) * 2 * (size_t)hcap + sizeof(int32_t) * 6 * (size_t)ncap + sizeof(int32_t) * 3 * (size_t)acap;
    b += sizeof(int32_t) * 3 * (size_t)team + sizeof(int32_t) * SC_N + 16;
    return (b + 255) & ~size_t(255);
}
size_t arena_bytes_host(int hcap, int ncap, int acap, int team, bool with_sort) {
    return arena_bytes(hcap, ncap, acap, team, with_sort, true);   // host-allocated arenas are persistent
}

// tier-1 (shared-memory) extraction arena of one warp: most Central Graphs are small
constexpr int kT1Hash = 256, kT1Nodes = 112, kT1Arcs = 160;
constexpr int kSmemArena = 8192;
constexpr int kExtWarps = 8;     // warps per CTA that extract (each owns one tier-1 arena)
// tier-2: one CTA per Central Graph over the whole dynamic shared region
constexpr int kT2Hash = 1024, kT2Nodes = 1024, kT2Arcs = 1536;
static_assert(kSmemArena * kExtWarps <= KGS_MAX_K * 16, "tier-1 arenas must fit the dynamic shared region");

__device__ __forceinline__ char *align8(char *p) {
    return reinterpret_cast<char *>((reinterpret_cast<uintptr_t>(p) + 7) & ~uintptr_t(7));
}

__device__ Arena carve(char *p, int hcap, int ncap, int acap, int team, bool with_sort, bool persistent = false) {
    Arena S;
    S.hcap = hcap; S.ncap = ncap; S.acap = acap;
    p = align8(p);
    if (persistent) {
        S.magic = reinterpret_cast<int32_t *>(p); p += 16;
        S.hslot = reinterpret_cast<int32_t *>(p); p += sizeof(int32_t) * (size_t)ncap;
    } else {
        S.magic = nullptr;
        S.hslot = nullptr;
    }
    S.b_start = reinterpret_cast<int64_t *>(p); p += sizeof(int64_t) * team;
    S.dsum = reinterpret_cast<double *>(p); p += sizeof(double);
    S.wsum = reinterpret_cast<unsigned long long *>(p); p += sizeof(unsigned long long);
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
    S.scal = reinterpret_cast<int32_t *>(p);
    return S;
}

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
    return x;
}

// insert (or find) node u; returns its index, -1 on overflow
__device__ __forceinline__ int arena_insert(Arena &S, int32_t u, uint32_t zbu, bool &fresh) {
    fresh = false;
    uint32_t h = hash32((uint32_t)u) & (uint32_t)(S.hcap - 1);
    for (int probe = 0; probe < S.hcap; ++probe) {
        const int32_t k = atomicCAS(S.hkey + h, -1, u);
        if (k == -1) {
            const int idx = atomicAdd(S.scal + SC_NODES, 1);
            if (idx >= S.ncap) { atomicExch(S.scal + SC_OVF, 1); atomicExch(S.hval + h, -2); return -1; }
            S.id[idx] = u;
            S.zb[idx] = zbu;
            if (S.hslot) S.hslot[idx] = (int32_t)h;
            __threadfence_block();
            atomicExch(S.hval + h, idx);
            fresh = true;
            return idx;
        }
        if (k == u) {
            int v;
            while ((v = atomicAdd(S.hval + h, 0)) == -1) { }
            __threadfence_block();   // acquire: the inserter's id stores precede its publication of hval
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

// Is the closure weight a lower bound of c's key (level-cover keeps every source: s* = 1)?  s* >= 2 needs
// sources holding >= 2 query keywords that cover Q with zb(c): multi is the union of the keyword sets of
// such nodes (graph-wide); per candidate, the keywords i for which one of them lies in DAG_i(c): the
// search's rm bits (exact for keywords 0-6, keyword 7 assumed reached) or mk_reach's fixpoint over the
// shared DAG (per compact id, in lz).  Each is an over-approximation, so is their intersection.
__device__ __forceinline__ bool cut_valid(const Ctx &c, int32_t cn, uint32_t zbc, uint32_t multi) {
    if (!c.a.level_cover) return true;
    uint32_t reach = multi;
    if (c.a.level_cover == 1 && c.a.rm_ok)
        reach &= st_rm(__ldcg(c.w.st + cn)) | (c.qq.q > 7 ? ~kRmMask : 0u);
    if (c.a.level_cover == 1 && c.ctl->mk_reach) {
        const int32_t cid = __ldcg(c.w.pd_cid + cn);
        if (cid >= 0) reach &= (uint32_t)__ldcg(c.w.lz + cid);
    }
    return ((reach | zbc) & c.qq.full) != c.qq.full;
}

// Closure (over the shared predecessor lists) + level-cover + Eq. 6 key of the Central Graph at c.
// Returns CG_OK, CG_OVERFLOW (arena too small: the next tier redoes it) or CG_CUT.
// cut (pruning round 2, exact): the key is known to exceed `cut` (the k-th exact key so far), so c cannot
// rank in the top-k — stop.  Valid when the pruned graph is the whole closure, i.e. when level-cover
// keeps every source (s* = 1): no set of sources holding two or more query keywords can cover Q together
// with c's own keywords (multi = union of the keyword sets of all such nodes of the graph), or
// level_cover = 0.  Then the closure weight so far, times d^lambda, is a lower bound of the key.
// lazy (pruning round 2): the shared DAG may lack the predecessor lists of some closure
// nodes; the walk marks them for the next pre-pass round (pd_state byte 1 + round bitmap 0), goes on over
// what is known (the cut still applies: the nodes found are in the closure) and, if not cut, returns
// CG_INCOMPLETE (no key).
enum { CG_OVERFLOW = 0, CG_OK = 1, CG_CUT = 2, CG_INCOMPLETE = 3 };
constexpr int32_t kArenaMagic = 0x4B475341;   // "KGSA": a persistent arena in a known state
constexpr double kNoCut = __builtin_huge_val();
template <class Team>
__device__ int central_graph(const Team &T, Arena &S, const Ctx &c, int32_t cn, int depth, double *key,
                             double cut = kNoCut, uint32_t multi = 0u, bool lazy = false) {
    const uint32_t full = c.qq.full;
    const int r = T.rank(), ts = T.size();
    // reset: only what the previous use of a persistent arena touched (its node count is still in scal),
    // everything after an overflow (its claimed slots were not recorded) or on first use
    const int prev_nodes = S.magic ? S.scal[SC_NODES] : 0;
    const bool lazy_reset = S.magic && *S.magic == kArenaMagic && S.scal[SC_OVF] == 0 && prev_nodes <= S.ncap;
    T.sync();
    if (lazy_reset) {
        for (int j = r; j < prev_nodes; j += ts) {
            const int h = S.hslot[j];
            S.hkey[h] = -1; S.hval[h] = -1;
            S.inmask[j] = 0; S.pending[j] = 0; S.keep[j] = 0;
        }
    } else {
        for (int i = r; i < S.hcap; i += ts) { S.hkey[i] = -1; S.hval[i] = -1; }
        for (int i = r; i < S.ncap; i += ts) { S.inmask[i] = 0; S.pending[i] = 0; S.keep[i] = 0; }
        if (r == 0 && S.magic) *S.magic = kArenaMagic;
    }
    T.sync();
    if (r < SC_N) S.scal[r] = 0;
    if (r == 0) { *S.dsum = 0.0; *S.wsum = 0ull; }
    T.sync();
    const uint64_t Mc = ldrow(c.w.M, cn);
    uint32_t zbc = 0;
    for (int i = 0; i < c.qq.q; ++i) if (((Mc >> (8 * i)) & 0xFF) == 0) zbc |= 1u << i;
    const bool cut_on = cut < kNoCut && cut_valid(c, cn, zbc, multi);
    auto over_cut = [&]() {   // the closure weight so far, times d^lambda, already exceeds the cut
        return __dmul_rn(c.a.dpow[depth], (double)*reinterpret_cast<volatile unsigned long long *>(S.wsum) *
                                              (1.0 / 16777216.0)) > cut;
    };
    if (r == 0) {
        bool fresh;
        const int j = arena_insert(S, cn, zbc, fresh);  // index 0
        S.inmask[j] = full;
        const uint32_t p = full & ~zbc;
        if (p) { S.pending[j] = p; fifo_push(S, j); }
        if (cut_on) *S.wsum = weight_fx(__ldg(c.a.g.weight + cn));
    }
    T.sync();
    // ---- backward closure, batch by batch (all pending nodes of a round in parallel)
    for (;;) {
        const int head = S.scal[SC_HEAD], tail = S.scal[SC_TAIL];
        if (head == tail || S.scal[SC_OVF] || S.scal[SC_CUT]) break;
        if (cut_on && over_cut()) {
            T.sync();
            return CG_CUT;
        }
        T.sync();
        for (int b0 = head; b0 < tail; b0 += ts) {
            int deg = 0;
            if (b0 + r < tail) {
                const int j = S.fifo[(b0 + r) % S.ncap];
                const uint32_t P = atomicExch(S.pending + j, 0u);
                const int32_t x = S.id[j];
                S.b_j[r] = j;
                S.b_P[r] = P;
                const int32_t cid = __ldcg(c.w.pd_cid + x);   // predecessor list from the shared DAG
                if (lazy && P) {   // keywords whose predecessors the DAG does not hold yet: request them
                    const uint32_t miss = P & ~((__ldcg(c.w.pd_state + x) >> 16) & 0xFFu);
                    if (miss) {
                        const uint32_t old = atomicOr(c.w.pd_state + x, miss << 8);
                        if (((old >> 8) & 0xFFu) == 0) set_bit(c.w.pd_bits, kFlagPd, x);
                        S.scal[SC_INC] = 1;
                    }
                }
                int64_t s0 = 0;
                if (P && cid >= 0) { s0 = __ldcg(c.w.pred_ptr + cid); deg = (int)(__ldcg(c.w.pred_ptr + cid + 1) - s0); }
                S.b_start[r] = s0;
            }
            int tot;
            const int ex = T.scan_excl(deg, &tot);
            S.b_incl[r] = ex + deg;
            T.sync();
            const int nb = min(ts, tail - b0);
            for (int e = r, it = 0; e < tot; e += ts, ++it) {
                // the arena overflowed: the next tier redoes this graph, stop scanning (a hub's list of
                // millions of predecessors kept a tier-1 warp busy for milliseconds, C5)
                if ((it & 31) == 0) {
                    if (*reinterpret_cast<volatile int32_t *>(S.scal + SC_OVF) ||
                        *reinterpret_cast<volatile int32_t *>(S.scal + SC_CUT)) break;
                    // the cut can be decided inside a round (a hub's list of thousands of predecessors)
                    if (cut_on && it && over_cut()) { S.scal[SC_CUT] = 1; break; }
                }
                int lo = 0, hi = nb - 1;       // owner = first o with incl[o] > e
                while (lo < hi) {
                    const int mid = (lo + hi) >> 1;
                    if (S.b_incl[mid] > e) hi = mid; else lo = mid + 1;
                }
                const int o = lo;
                const int exo = o ? S.b_incl[o - 1] : 0;
                const int64_t pi = S.b_start[o] + (e - exo);
                const int32_t u = __ldcg(c.w.pred_u + pi);
                const uint32_t bz = __ldcg(c.w.pred_b + pi);
                const uint32_t pb = bz & S.b_P[o] & 0xFFu;   // Thm. V.4 arc for the keywords x needs here
                if (!pb) continue;
                const uint32_t zbu = bz >> 8;
                bool fresh;
                const int j = arena_insert(S, u, zbu, fresh);
                if (j < 0) continue;
                if (fresh && cut_on) atomicAdd(S.wsum, (unsigned long long)weight_fx(__ldg(c.a.g.weight + u)));
                const uint32_t old = atomicOr(S.inmask + j, pb);
                const uint32_t nbits = pb & ~old & ~zbu;   // zb(u) is a property of u: the inserter stored this value
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
    // an overflowing arena still holds a partial closure: its weight is a lower bound of the key
    if (S.scal[SC_CUT] || ((S.scal[SC_OVF] || S.scal[SC_INC]) && cut_on && over_cut())) { T.sync(); return CG_CUT; }
    if (S.scal[SC_OVF]) return CG_OVERFLOW;
    if (S.scal[SC_INC]) { T.sync(); return CG_INCOMPLETE; }
    const int nn = S.scal[SC_NODES];
    const int na = S.scal[SC_ARCS] < S.acap ? S.scal[SC_ARCS] : S.acap;
    // ---- level-cover: a keyword node's level counts the keywords it contributes (R13: a source
    // of a hitting path in DAG_i(c), inmask & zb) or, with level_cover = 2, the keywords it contains (R13b:
    // zb, its m = 0 keywords)
    if (c.a.level_cover) {
        const uint32_t lmask = c.a.level_cover == 2 ? 0xFFu : 0u;
        const uint32_t cov0 = S.zb[0];
        int sstar = c.qq.q + 1;
        if (cov0 != full) {
            if (r == 0) S.scal[SC_COV] = (int)cov0;
            T.sync();
            for (int s = c.qq.q; s >= 1; --s) {
                for (int j = 1 + r; j < nn; j += ts) {
                    const uint32_t con = (S.inmask[j] | lmask) & S.zb[j];
                    if (__popc(con) == s) atomicOr(reinterpret_cast<unsigned *>(S.scal + SC_COV), con);
                }
                T.sync();
                if ((uint32_t)S.scal[SC_COV] == full) { sstar = s; break; }
                T.sync();
            }
        }
        for (int j = r; j < nn; j += ts) {
            const uint32_t src = S.inmask[j] & S.zb[j];                 // the DAGs j is a kept source of
            const uint32_t lvl = (S.inmask[j] | lmask) & S.zb[j];       // its level-cover level
            S.keep[j] = (j == 0 || __popc(lvl) >= sstar) ? src : 0u;
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
        if (S.keep[j]) atomicAdd(S.dsum, (double)c.a.g.weight[S.id[j]]);
    T.sync();
    *key = __dmul_rn(c.a.dpow[depth], *S.dsum);
    T.sync();
    return CG_OK;
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

// Warp bitonic sort in registers (E elements per lane, element i = e * 32 + lane): the tier-1 emit sorts
// at most 256 nodes or arcs, and sorting them through memory with a warp barrier per step cost a
// single-query launch ~20 us.
template <int E>
__device__ __forceinline__ void warp_sort_regs(unsigned long long *buf, int len) {
    const int lane = (int)(threadIdx.x & 31u);
    unsigned long long x[E];
#pragma unroll
    for (int e = 0; e < E; ++e) x[e] = e * 32 + lane < len ? buf[e * 32 + lane] : ~0ull;
#pragma unroll
    for (int k = 2; k <= 32 * E; k <<= 1)
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            if (j >= 32) {
                const int d = j >> 5;
#pragma unroll
                for (int e = 0; e < E; ++e)
                    if ((e & d) == 0) {
                        const bool up = ((e * 32 + lane) & k) == 0;
                        const unsigned long long a = x[e], b = x[e | d];
                        const unsigned long long lo = a < b ? a : b, hi = a < b ? b : a;
                        x[e] = up ? lo : hi;
                        x[e | d] = up ? hi : lo;
                    }
            } else {
#pragma unroll
                for (int e = 0; e < E; ++e) {
                    const unsigned long long y = __shfl_xor_sync(0xffffffffu, x[e], j);
                    const int i = e * 32 + lane;
                    const bool keep_min = ((i & j) == 0) == ((i & k) == 0);
                    x[e] = keep_min ? (x[e] < y ? x[e] : y) : (x[e] < y ? y : x[e]);
                }
            }
        }
    __syncwarp();
#pragma unroll
    for (int e = 0; e < E; ++e)
        if (e * 32 + lane < len) buf[e * 32 + lane] = x[e];
    __syncwarp();
}
__device__ void team_sort(const WarpTeam &T, unsigned long long *buf, int len) {
    if (len <= 32) warp_sort_regs<1>(buf, len);
    else if (len <= 64) warp_sort_regs<2>(buf, len);
    else if (len <= 128) warp_sort_regs<4>(buf, len);
    else if (len <= 256) warp_sort_regs<8>(buf, len);
    else team_sort<WarpTeam>(T, buf, len);
}

// Reserve cnt entries of an answer arena; -1 if they do not fit, leaving the counter as it was, so later
// (smaller) answers still fit and only the overflowing query is marked (KGS_STOP_CAPACITY).  The common
// case is one atomicAdd (a CAS loop serialised the k concurrent winners of a query on one address: ~15 us
// of a single-query launch); a reservation that lands past cap is undone and retried exactly with CAS (a
// concurrent reservation can then see the counter briefly high and fail too — only when the arena is
// within one answer of full).
__device__ __forceinline__ long long arena_reserve(unsigned long long *ctr, unsigned long long cnt, long long cap) {
    const unsigned long long old = atomicAdd(ctr, cnt);
    if (old + cnt <= (unsigned long long)cap) return (long long)old;
    atomicAdd(ctr, (unsigned long long)(-(long long)cnt));   // undo
    unsigned long long cur = atomicAdd(ctr, 0ull);
    for (;;) {
        if (cur + cnt > (unsigned long long)cap) return -1;
        const unsigned long long prev = atomicCAS(ctr, cur, cur + cnt);
        if (prev == cur) return (long long)cur;
        cur = prev;
    }
}

// write the kept nodes / arcs of the arena (after central_graph) sorted and unique, as answer `rank_i`
template <class Team>
__device__ bool emit_graph(const Team &T, Arena &S, const Ctx &c, int rank_i) {
    const EngineArgs &a = c.a;
    const int r = T.rank(), ts = T.size();
    const int nn = S.scal[SC_NODES];
    const int na = S.scal[SC_ARCS];
    if (r == 0) { S.scal[SC_NOUT] = 0; S.scal[SC_AOUT] = 0; }
    T.sync();
    for (int j = r; j < nn; j += ts)
        if (S.keep[j]) S.sortbuf[atomicAdd(S.scal + SC_NOUT, 1)] = (unsigned long long)(uint32_t)in_id(a, S.id[j]);
    T.sync();
    const int kn = S.scal[SC_NOUT];
    team_sort(T, S.sortbuf, kn);
    const int64_t ans = (int64_t)c.qq.qi * a.k + rank_i;
    if (r == 0) S.b_start[0] = arena_reserve(a.out_used + 0, (unsigned long long)kn, a.out_nodes_cap);   // team broadcast
    T.sync();
    const long long no = S.b_start[0];
    T.sync();
    if (no < 0) {
        if (r == 0) atomicExch(&c.ctl->fatal, 1);
        return false;
    }
    for (int i = r; i < kn; i += ts) a.out_nodes[no + i] = (int32_t)S.sortbuf[i];
    T.sync();
    if (r == 0) S.scal[SC_AOUT] = 0;
    T.sync();
    for (int e = r; e < na; e += ts)
        if (S.keep[S.au[e]] & S.ab[e])
            S.sortbuf[atomicAdd(S.scal + SC_AOUT, 1)] =
                ((unsigned long long)(uint32_t)in_id(a, S.id[S.au[e]]) << 32) | (uint32_t)in_id(a, S.id[S.ax[e]]);
    T.sync();
    const int ka = S.scal[SC_AOUT];
    team_sort(T, S.sortbuf, ka);
    int kept = 0;
    for (int b0 = 0; b0 < ka; b0 += ts) {
        const int i = b0 + r;
        const int flag = (i < ka && (i == 0 || S.sortbuf[i] != S.sortbuf[i - 1])) ? 1 : 0;
        int tot;
        const int ex = T.scan_excl(flag, &tot);
        T.sync();
        if (flag) S.sortbuf[ka + kept + ex] = S.sortbuf[i];
        kept += tot;
        T.sync();
    }
    if (r == 0) S.b_start[0] = arena_reserve(a.out_used + 1, (unsigned long long)kept, a.out_arcs_cap);
    T.sync();
    const long long ao = S.b_start[0];
    T.sync();
    if (ao < 0) {
        if (r == 0) atomicExch(&c.ctl->fatal, 1);
        return false;
    }
    for (int i = r; i < kept; i += ts) {
        const unsigned long long key = S.sortbuf[ka + i];
        a.out_arcs[2 * (ao + i)] = (int32_t)(key >> 32);
        a.out_arcs[2 * (ao + i) + 1] = (int32_t)(key & 0xFFFFFFFFu);
    }
    if (r == 0) {
        a.out_hdr[4 * ans + 2] = kn;
        a.out_hdr[4 * ans + 3] = kept;
        a.out_off[2 * ans] = no;
        a.out_off[2 * ans + 1] = ao;
    }
    T.sync();
    return true;
}

// ------------------------------------------------------------------------------------------ select
__device__ __forceinline__ void comp_key(const Ctx &c, uint32_t i, uint64_t &hi, uint32_t &lo) {
    hi = (uint64_t)__double_as_longlong(__ldcg(c.w.ckey + i));
    lo = (uint32_t)in_id(c.a, __ldcg(c.w.centrals + i));   // ties rank by input id
}
__device__ __forceinline__ uint32_t digit_of(uint64_t hi, uint32_t lo, int d) {
    return d < 8 ? (uint32_t)((hi >> (56 - 8 * d)) & 0xFF) : (lo >> (24 - 8 * (d - 8))) & 0xFF;
}
__device__ __forceinline__ bool prefix_match(uint64_t hi, uint32_t lo, uint64_t phi, uint32_t plo, int d) {
    if (d == 0) return true;
    if (d <= 8) {
        const uint64_t m = d == 8 ? ~0ull : (~0ull << (64 - 8 * d));
        return (hi & m) == (phi & m);
    }
    if (hi != phi) return false;
    const uint32_t m = d == 12 ? 0xFFFFFFFFu : (0xFFFFFFFFu << (32 - 8 * (d - 8)));
    return (lo & m) == (plo & m);
}

// One CTA (group rank 0) ranks cnt <= KGS_MAX_K candidates by (fp64 key asc, central id asc) and keeps
// the first kk in sel[0..kk), ctl->sel_count = kk.  list == nullptr: the candidates are 0..cnt-1.
// Ends with a group barrier.
__device__ void rank_list(const Ctx &c, char *dsmem, const int32_t *list, uint32_t cnt, uint32_t kk) {
    const Grp &G = c.G;
    if (cnt <= 32) {   // one warp sorts in registers: (key bits, input id) with the candidate index riding along
        if (G.grank == 0 && threadIdx.x < 32) {
            const int lane = (int)threadIdx.x;
            uint64_t a = ~0ull, b = ~0ull;   // a = key bits, b = input id << 32 | candidate index
            if (lane < (int)cnt) {
                const int32_t idx = list ? __ldcg(list + lane) : lane;
                uint32_t lo;
                comp_key(c, (uint32_t)idx, a, lo);
                b = ((uint64_t)lo << 32) | (uint32_t)idx;
            }
#pragma unroll
            for (int k = 2; k <= 32; k <<= 1)
#pragma unroll
                for (int j = k >> 1; j > 0; j >>= 1) {
                    const uint64_t oa = __shfl_xor_sync(0xffffffffu, a, j), ob = __shfl_xor_sync(0xffffffffu, b, j);
                    const bool mine_less = a < oa || (a == oa && b < ob);
                    const bool keep_min = ((lane & j) == 0) == ((lane & k) == 0);
                    if (keep_min != mine_less) { a = oa; b = ob; }
                }
            if (lane < (int)kk) c.w.sel[lane] = (int32_t)(uint32_t)b;
            if (lane == 0) c.ctl->sel_count = kk;
        }
        G.sync();
        return;
    }
    if (G.grank == 0) {
        unsigned long long *khi = reinterpret_cast<unsigned long long *>(dsmem);
        uint32_t *klo = reinterpret_cast<uint32_t *>(khi + KGS_MAX_K);
        int32_t *kid = reinterpret_cast<int32_t *>(klo + KGS_MAX_K);
        int p2 = 1;
        while (p2 < (int)cnt) p2 <<= 1;
        for (int i = threadIdx.x; i < p2; i += blockDim.x) {
            if (i < (int)cnt) {
                const int32_t idx = list ? __ldcg(list + i) : i;
                uint64_t hi; uint32_t lo;
                comp_key(c, (uint32_t)idx, hi, lo);
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
        for (int i = threadIdx.x; i < (int)kk; i += blockDim.x) c.w.sel[i] = kid[i];
        if (threadIdx.x == 0) c.ctl->sel_count = kk;
    }
    G.sync();
}

// The kk smallest (key, id) of all |C| centrals, ranked, into sel[0..kk).  |C| <= KGS_MAX_K: one CTA
// sorts every candidate.  Otherwise an MSD radix select over the 96-bit composite (12 digits of 8 bits)
// keeps exactly kk candidates (in elist), which one CTA then sorts: the select runs on one CTA alone up
// to kCtaSelectMax candidates (no group barrier), on the whole group beyond.
constexpr uint32_t kCtaSelectMax = 1u << 18;

__device__ void select_topk(const Ctx &c, long long *sh, char *dsmem, uint32_t kk) {
    const Grp &G = c.G;
    Ctl *ctl = c.ctl;
    const uint32_t nc = __ldcg(&ctl->n_central);
    if (nc <= (uint32_t)KGS_MAX_K) { rank_list(c, dsmem, nullptr, nc, kk); return; }
    __shared__ uint32_t hsh[256];
    __shared__ uint32_t s_bucket, s_before, s_exact;
    const bool group_wide = nc > kCtaSelectMax;
    if (G.gtid() == 0) ctl->sel_count = 0;
    if (group_wide) {
        for (int64_t j = G.gtid(); j < 12 * 256; j += G.gsz) (&ctl->hist[0][0])[j] = 0u;
        G.sync();
    }
    if (group_wide || G.grank == 0) {
        const int64_t t0 = group_wide ? G.gtid() : (int64_t)threadIdx.x;
        const int64_t ts = group_wide ? G.gsz : (int64_t)blockDim.x;
        uint64_t phi = 0;
        uint32_t plo = 0, want = kk;
        for (int d = 0; d < 12; ++d) {
            for (int t = threadIdx.x; t < 256; t += blockDim.x) hsh[t] = 0;
            __syncthreads();
            for (int64_t i = t0; i < nc; i += ts) {
                uint64_t hi; uint32_t lo;
                comp_key(c, (uint32_t)i, hi, lo);
                if (prefix_match(hi, lo, phi, plo, d)) atomicAdd(hsh + digit_of(hi, lo, d), 1u);
            }
            __syncthreads();
            if (group_wide) {
                for (int t = threadIdx.x; t < 256; t += blockDim.x)
                    if (hsh[t]) atomicAdd(&ctl->hist[d][t], hsh[t]);
                G.sync();
                for (int t = threadIdx.x; t < 256; t += blockDim.x) hsh[t] = __ldcg(&ctl->hist[d][t]);
                __syncthreads();
            }
            // the bucket holding the want-th smallest: parallel prefix over the 256 bins
            const uint32_t hv = threadIdx.x < 256 ? hsh[threadIdx.x] : 0u;
            int tot;
            const int ex = block_excl_scan((int)hv, &tot, sh);
            if (threadIdx.x < 256 && (uint32_t)ex < want && want <= (uint32_t)ex + hv) {
                s_bucket = threadIdx.x; s_before = (uint32_t)ex; s_exact = want == (uint32_t)ex + hv;
            }
            __syncthreads();
            want -= s_before;
            const uint64_t bk = s_bucket;
            if (d < 8) phi |= bk << (56 - 8 * d);
            else plo |= (uint32_t)bk << (24 - 8 * (d - 8));
            const bool exact = s_exact;
            __syncthreads();
            if (exact) {   // every candidate of the bucket is selected: the threshold is the bucket's top
                if (d < 8) { phi |= (1ull << (56 - 8 * d)) - 1ull; plo = 0xFFFFFFFFu; }
                else plo |= (1u << (24 - 8 * (d - 8))) - 1u;
                break;
            }
        }
        for (int64_t i = t0; i < nc; i += ts) {   // exactly kk candidates are <= the threshold
            uint64_t hi; uint32_t lo;
            comp_key(c, (uint32_t)i, hi, lo);
            if (hi < phi || (hi == phi && lo <= plo)) {
                const uint32_t pos = atomicAdd(&ctl->sel_count, 1u);
                if (pos < (uint32_t)KGS_MAX_K) c.w.elist[pos] = (int32_t)i;
            }
        }
    }
    G.sync();
    rank_list(c, dsmem, c.w.elist, kk, kk);
}

// ------------------------------------------------------------------------------------------ containment
// NEXT-3, containment removal ("we remove the Central Graph that completely contains smaller ones",
// reading R16): the answers are the k best (key, id) among the candidates whose pruned node set does not
// strictly contain the pruned node set of another Central Graph of C, looked for among the best
// W = min(|C|, KGS_MAX_K).  G(c) can only contain G(c') if it holds c' (c' is always in its own graph), so
// a candidate is checked against the central nodes inside it (st hit mask = all keywords, Lemma V.1).
// One CTA per ranked candidate: its graph in the CTA's large arena (membership by hash lookup), each inner
// central's graph in the CTA's big arena.  Ranked positions are checked a chunk at a time until kk
// survivors are known.  Every key is exact here (the host forces prune = 0).

// index of node u in an arena after central_graph (-1: not in it)
__device__ __forceinline__ int arena_find(const Arena &S, int32_t u) {
    uint32_t h = hash32((uint32_t)u) & (uint32_t)(S.hcap - 1);
    for (int probe = 0; probe < S.hcap; ++probe) {
        const int32_t k = S.hkey[h];
        if (k == u) return S.hval[h];
        if (k == -1) return -1;
        h = (h + 1) & (uint32_t)(S.hcap - 1);
    }
    return -1;
}

// kept nodes of an arena after central_graph (whole CTA)
__device__ __forceinline__ int arena_kept(const Arena &S, long long *sh) {
    const int nn = S.scal[SC_NODES];
    int cnt = 0;
    for (int j = threadIdx.x; j < nn; j += blockDim.x) cnt += S.keep[j] != 0u;
    long long tot;
    block_excl_scan64(cnt, &tot, sh);
    return (int)tot;
}

__device__ void containment_select(const Ctx &c, long long *sh, char *dsmem, uint32_t kk) {
    const Grp &G = c.G;
    const EngineArgs &a = c.a;
    Ctl *ctl = c.ctl;
    const uint32_t nc = __ldcg(&ctl->n_central);
    const uint32_t W = nc < (uint32_t)KGS_MAX_K ? nc : (uint32_t)KGS_MAX_K;
    select_topk(c, sh, dsmem, W);                 // sel[0..W): ranked by (key, id); ends with a barrier
    int32_t *removed = c.w.overflow;              // per ranked position (the extraction lists are done)
    BlockTeam BT{sh};
    Arena SL = carve(a.large_arenas + a.large_arena_bytes * blockIdx.x, a.large_hash, a.large_nodes, a.large_arcs,
                     blockDim.x, false, true);
    Arena S3 = carve(a.cta_arenas + a.cta_arena_bytes * blockIdx.x, a.big_hash, a.big_nodes, a.big_arcs, blockDim.x,
                     true, true);
    __shared__ int s_flag;
    __shared__ uint32_t s_pos;
    const uint32_t chunk = max((uint32_t)G.gcount, 2u * kk);
    for (uint32_t p0 = 0; p0 < W; p0 += chunk) {
        const uint32_t p1 = min(W, p0 + chunk);
        for (uint32_t t = p0 + G.grank; t < p1; t += G.gcount) {
            const int32_t idx = __ldcg(c.w.sel + t);
            const int32_t cn = __ldcg(c.w.centrals + idx);
            double key;
            int rem = 0;
            if (central_graph(BT, SL, c, cn, __ldcg(c.w.cdepth + idx), &key) != CG_OK) {
                if (threadIdx.x == 0) atomicExch(&ctl->fatal, 6);
            } else {
                const int nn = SL.scal[SC_NODES];
                const int nkc = arena_kept(SL, sh);
                for (int j = 0; j < nn && !rem; ++j) {
                    const int32_t x = SL.id[j];
                    if (!SL.keep[j] || x == cn || (__ldcg(c.w.st + x) & 0xFFu) != c.qq.full) continue;
                    if (central_graph(BT, S3, c, x, 0, &key) != CG_OK) {
                        if (threadIdx.x == 0) atomicExch(&ctl->fatal, 6);
                        break;
                    }
                    if (arena_kept(S3, sh) >= nkc) continue;
                    if (threadIdx.x == 0) s_flag = 1;
                    __syncthreads();
                    const int nx = S3.scal[SC_NODES];
                    for (int i = threadIdx.x; i < nx; i += blockDim.x) {
                        if (!S3.keep[i]) continue;
                        const int f = arena_find(SL, S3.id[i]);
                        if (f < 0 || !SL.keep[f]) s_flag = 0;
                    }
                    __syncthreads();
                    rem = s_flag;
                    __syncthreads();
                }
            }
            if (threadIdx.x == 0) removed[t] = rem;
            __syncthreads();
        }
        G.sync();
        if (threadIdx.x == 0) {   // survivors so far (every CTA computes the same count)
            uint32_t kept = 0;
            for (uint32_t t = 0; t < p1; ++t) kept += __ldcg(removed + t) == 0;
            s_pos = kept;
        }
        __syncthreads();
        if (s_pos >= kk) break;
    }
    if (G.grank == 0 && threadIdx.x == 0) {   // the first kk survivors in rank order
        uint32_t kept = 0;
        for (uint32_t t = 0; t < W && kept < kk; ++t)
            if (__ldcg(removed + t) == 0) c.w.sel[kept++] = __ldcg(c.w.sel + t);
        ctl->sel_count = kept;
    }
    G.sync();
}

// ------------------------------------------------------------------------------------------ top-down driver
// Seeds of the predecessor pre-pass: every candidate list[0..cnt) (nullptr: all centrals), for every
// keyword it does not contain itself (those have m = 0 and no predecessors).
__device__ __forceinline__ void pd_round0_reset(const Ctx &c) {   // group leader: round 0 of a pred_dag call
    c.ctl->pd_qn[0][0] = 0u; c.ctl->pd_qn[0][1] = 0u; c.ctl->pd_ndef[0] = 0u; c.ctl->pd_ctile[0] = 0u;
    c.ctl->pd_xbatch[0] = 0u;
}

__device__ void seed_pd(const Ctx &c, const int32_t *list, uint32_t cnt) {
    const Grp &G = c.G;
    if (G.gtid() == 0) pd_round0_reset(c);
    for (int64_t j = G.gtid(); j < cnt; j += G.gsz) {
        const int32_t idx = list ? __ldcg(list + j) : (int32_t)j;
        const int32_t cn = __ldcg(c.w.centrals + idx);
        const uint64_t Mc = ldrow(c.w.M, cn);
        uint32_t zb = 0;
        for (int i = 0; i < c.qq.q; ++i) if (((Mc >> (8 * i)) & 0xFF) == 0) zb |= 1u << i;
        const uint32_t bits = c.qq.full & ~zb;
        if (bits) { atomicOr(c.w.pd_state + cn, bits << 8); set_bit(c.w.pd_bits, kFlagPd, cn); }
    }
    publish_flags(c.ctl);
    G.sync();
}

// Exact Eq. 6 key of every candidate list[0..cnt) (nullptr: all centrals): (A) one warp per candidate
// over a tier-1 arena in shared memory (most Central Graphs are small); (B) the larger ones, a whole CTA
// per candidate over the CTA's shared region; (C) beyond that, the CTA's global-memory arena.
// cflag: 0 = key from tier 1, 1 = from tier 2/3 (emitted by a CTA).
__device__ void extract_list(const Ctx &c, long long *sh, char *dsmem, const int32_t *list, uint32_t cnt, QOut *qo,
                             double cut = kNoCut, bool lazy = false, bool count_eval = true,
                             int32_t *inc_out = nullptr) {
    const Grp &G = c.G;
    const EngineArgs &a = c.a;
    Ctl *ctl = c.ctl;
    const uint32_t multi = __ldcg(&ctl->multi_kw);
    const double kInf = __longlong_as_double(0x7FF0000000000000ll);
    if (G.gtid() == 0) {
        ctl->work_ext = 0; ctl->n_overflow = 0; ctl->work_big = 0; ctl->work_huge = 0; ctl->work_huge2 = 0;
        if (count_eval) ctl->n_eval += cnt;
        ctl->n_inc = 0;
    }
    G.sync();
    if ((threadIdx.x >> 5) < kExtWarps) {
        Arena S1 = carve(dsmem + kSmemArena * (threadIdx.x >> 5), kT1Hash, kT1Nodes, kT1Arcs, 32, false);
        WarpTeam T;
        for (;;) {
            uint32_t t = 0;
            if (T.rank() == 0) t = atomicAdd(&ctl->work_ext, 1u);
            t = __shfl_sync(0xffffffffu, t, 0);
            if (t >= cnt) break;
            const int32_t idx = list ? __ldcg(list + t) : (int32_t)t;
            const int32_t cn = __ldcg(c.w.centrals + idx);
            double key = 0.0;
            const int st = central_graph(T, S1, c, cn, __ldcg(c.w.cdepth + idx), &key, cut, multi, lazy);
            if (T.rank() == 0) {
                if (st == CG_OK) { c.w.ckey[idx] = key; c.w.cflag[idx] = 0; }
                else if (st == CG_CUT) { c.w.ckey[idx] = kInf; c.w.cflag[idx] = 0; atomicAdd(&ctl->n_cut, 1u); }
                else if (st == CG_INCOMPLETE) { c.w.cflag[idx] = 0; inc_out[atomicAdd(&ctl->n_inc, 1u)] = idx; }
                else { c.w.cflag[idx] = 1; c.w.overflow[atomicAdd(&ctl->n_overflow, 1u)] = idx; }
            }
            __syncwarp();
        }
    }
    G.sync();
    stamp(G, qo, cut < kNoCut ? TS_EXTRACT2 : TS_EXTRACT);
    const uint32_t no = __ldcg(&ctl->n_overflow);
    BlockTeam BT{sh};
    if (no) {
        Arena S2 = carve(dsmem, kT2Hash, kT2Nodes, kT2Arcs, kBlock, false);
        for (uint32_t t = G.grank; t < no; t += G.gcount) {
            const int32_t idx = __ldcg(c.w.overflow + t);
            double key = 0.0;
            const int st = central_graph(BT, S2, c, __ldcg(c.w.centrals + idx), __ldcg(c.w.cdepth + idx), &key, cut, multi, lazy);
            if (threadIdx.x == 0) {
                if (st == CG_OK) c.w.ckey[idx] = key;
                else if (st == CG_CUT) { c.w.ckey[idx] = kInf; atomicAdd(&ctl->n_cut, 1u); }
                else if (st == CG_INCOMPLETE) inc_out[atomicAdd(&ctl->n_inc, 1u)] = idx;
                else c.w.overflow[no + atomicAdd(&ctl->work_big, 1u)] = idx;
            }
            __syncthreads();
        }
        G.sync();
        const uint32_t nbig = __ldcg(&ctl->work_big);
        if (nbig) {
            Arena S3 = carve(a.cta_arenas + a.cta_arena_bytes * blockIdx.x, a.big_hash, a.big_nodes, a.big_arcs, blockDim.x, true, true);
            for (uint32_t t = G.grank; t < nbig; t += G.gcount) {
                const int32_t idx = __ldcg(c.w.overflow + no + t);
                double key = 0.0;
                const int st = central_graph(BT, S3, c, __ldcg(c.w.centrals + idx), __ldcg(c.w.cdepth + idx), &key, cut, multi, lazy);
                if (threadIdx.x == 0) {
                    if (st == CG_OK) c.w.ckey[idx] = key;
                    else if (st == CG_CUT) { c.w.ckey[idx] = kInf; atomicAdd(&ctl->n_cut, 1u); }
                    else if (st == CG_INCOMPLETE) inc_out[atomicAdd(&ctl->n_inc, 1u)] = idx;
                    else c.w.overflow[no + nbig + atomicAdd(&ctl->work_huge, 1u)] = idx;
                }
                __syncthreads();
            }
        }
        G.sync();
        const uint32_t nlarge = __ldcg(&ctl->work_huge);
        uint32_t nhuge = 0;
        if (nlarge) {   // tier 3b: every CTA of the group over its large arena
            Arena SL = carve(a.large_arenas + a.large_arena_bytes * blockIdx.x, a.large_hash, a.large_nodes,
                             a.large_arcs, blockDim.x, false, true);
            for (uint32_t t = G.grank; t < nlarge; t += G.gcount) {
                const int32_t idx = __ldcg(c.w.overflow + no + nbig + t);
                double key = 0.0;
                const int st = central_graph(BT, SL, c, __ldcg(c.w.centrals + idx), __ldcg(c.w.cdepth + idx), &key, cut, multi, lazy);
                if (threadIdx.x == 0) {
                    if (st == CG_OK) c.w.ckey[idx] = key;
                    else if (st == CG_CUT) { c.w.ckey[idx] = kInf; atomicAdd(&ctl->n_cut, 1u); }
                    else if (st == CG_INCOMPLETE) inc_out[atomicAdd(&ctl->n_inc, 1u)] = idx;
                    else c.w.overflow[no + nbig + nlarge + atomicAdd(&ctl->work_huge2, 1u)] = idx;
                }
                __syncthreads();
            }
            G.sync();
            nhuge = __ldcg(&ctl->work_huge2);
        }
        if (nhuge) {   // tier 4: the group's huge arena, one CTA
            if (G.grank == 0) {
                Arena S4 = carve(c.w.huge, a.huge_hash, a.huge_nodes, a.huge_arcs, blockDim.x, true, true);
                if (threadIdx.x == 0) ctl->n_tier4 += nhuge;
                for (uint32_t t = 0; t < nhuge; ++t) {
                    const int32_t idx = __ldcg(c.w.overflow + no + nbig + nlarge + t);
                    double key = 0.0;
                    const int st = central_graph(BT, S4, c, __ldcg(c.w.centrals + idx), __ldcg(c.w.cdepth + idx), &key, cut, multi, lazy);
                    if (threadIdx.x == 0) {
                        if (st == CG_OK) c.w.ckey[idx] = key;
                        else if (st == CG_CUT) { c.w.ckey[idx] = kInf; atomicAdd(&ctl->n_cut, 1u); }
                        else if (st == CG_INCOMPLETE) inc_out[atomicAdd(&ctl->n_inc, 1u)] = idx;
                        else atomicExch(&ctl->fatal, 2);
                    }
                    __syncthreads();
                }
            }
            G.sync();
        }
        stamp(G, qo, TS_EXTRACT_BIG);
    }
}

// Emit the ranked winners sel[0..sel_count): one warp per winner (per-warp arena), the winners that
// overflowed tier 1 by a CTA.  work_emit and work_big are zero on entry.
__device__ void emit_answers(const Ctx &c, long long *sh, char *dsmem, QOut *qo) {
    const Grp &G = c.G;
    const EngineArgs &a = c.a;
    Ctl *ctl = c.ctl;
    const uint32_t cnt = __ldcg(&ctl->sel_count);
    BlockTeam BT{sh};
    if ((threadIdx.x >> 5) < kExtWarps) {
        const int gwarp = (int)(blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5));
        Arena S = carve(a.warp_arenas + a.warp_arena_bytes * gwarp, kExtHash, kExtNodes, kExtArcs, 32, true, true);
        Arena S1 = carve(dsmem + kSmemArena * ((threadIdx.x >> 5) % kExtWarps), kT1Hash, kT1Nodes, kT1Arcs, 32, false);
        S1.sortbuf = S.sortbuf;   // tier-1 closure in shared memory, its sort buffer in the global arena
        WarpTeam T;
        for (;;) {
            uint32_t rk = 0;
            if (T.rank() == 0) rk = atomicAdd(&ctl->work_emit, 1u);
            rk = __shfl_sync(0xffffffffu, rk, 0);
            if (rk >= cnt) break;
            const int32_t idx = __ldcg(c.w.sel + rk);
            const int64_t ans = (int64_t)c.qq.qi * a.k + rk;
            if (T.rank() == 0) {
                a.out_hdr[4 * ans + 0] = in_id(a, __ldcg(c.w.centrals + idx));
                a.out_hdr[4 * ans + 1] = __ldcg(c.w.cdepth + idx);
                a.out_key[ans] = __ldcg(c.w.ckey + idx);
            }
            if (__ldcg(c.w.cflag + idx)) {
                if (T.rank() == 0) c.w.overflow[atomicAdd(&ctl->work_big, 1u)] = (int32_t)rk;   // reuse list
                continue;
            }
            double key;
            const int32_t cn = __ldcg(c.w.centrals + idx);
            const int dep = __ldcg(c.w.cdepth + idx);
            if (central_graph(T, S1, c, cn, dep, &key) == CG_OK) emit_graph(T, S1, c, (int)rk);   // tier 1
            else if (central_graph(T, S, c, cn, dep, &key) == CG_OK) emit_graph(T, S, c, (int)rk);
            else if (T.rank() == 0) atomicExch(&ctl->fatal, 3);
        }
    }
    G.sync();
    const uint32_t nbig = __ldcg(&ctl->work_big);
    if (nbig) {
        Arena S = carve(a.cta_arenas + a.cta_arena_bytes * blockIdx.x, a.big_hash, a.big_nodes, a.big_arcs, blockDim.x, true, true);
        Arena S2 = carve(dsmem, kT2Hash, kT2Nodes, kT2Arcs, kBlock, false);
        S2.sortbuf = S.sortbuf;   // tier-2 closure in shared memory, its sort buffer in the CTA's global arena
        for (uint32_t t = G.grank; t < nbig; t += G.gcount) {
            const int rk = __ldcg(c.w.overflow + t);
            const int32_t idx = __ldcg(c.w.sel + rk);
            const int32_t cn = __ldcg(c.w.centrals + idx);
            const int dep = __ldcg(c.w.cdepth + idx);
            double key;
            if (central_graph(BT, S2, c, cn, dep, &key) == CG_OK) emit_graph(BT, S2, c, rk);
            else if (central_graph(BT, S, c, cn, dep, &key) == CG_OK) emit_graph(BT, S, c, rk);
            else if (threadIdx.x == 0) c.w.overflow[nbig + atomicAdd(&ctl->work_huge, 1u)] = rk;
            __syncthreads();
        }
        G.sync();
        const uint32_t nhuge = __ldcg(&ctl->work_huge);
        if (nhuge) {   // tier 4: the group's huge arena, one CTA
            if (G.grank == 0) {
                Arena S4 = carve(c.w.huge, a.huge_hash, a.huge_nodes, a.huge_arcs, blockDim.x, true, true);
                for (uint32_t t = 0; t < nhuge; ++t) {
                    const int rk = __ldcg(c.w.overflow + nbig + t);
                    const int32_t idx = __ldcg(c.w.sel + rk);
                    double key;
                    if (central_graph(BT, S4, c, __ldcg(c.w.centrals + idx), __ldcg(c.w.cdepth + idx), &key) == CG_OK)
                        emit_graph(BT, S4, c, rk);
                    else if (threadIdx.x == 0) atomicExch(&ctl->fatal, 4);
                    __syncthreads();
                }
            }
            G.sync();
        }
    }
    stamp(G, qo, TS_EMIT);
}

// Top-down phase (Alg. 3 + Eq. 6): exact keys, top-k, answer subgraphs.
// Without pruning every central is extracted.  With pruning (kgs_params.prune, DESIGN.md "Top-down
// pruning"): key(c) = d^lambda (x) (sum of kept weights) >= LB(c) = d^lambda (x) w_c exactly in fp64
// (c is always kept, weights are >= 0, rounded addition and multiplication are monotone).  Round 1
// extracts the m smallest (LB, id); T = the k-th smallest exact (key, id) among them.  Every other
// candidate has (LB, id) above the m-th (LB, id) B; if B >= T none of them can rank before T, else
// round 2 extracts every remaining candidate with (LB, id) < T.  The top-k over the extracted
// candidates is then the top-k over all of C.

// Pruning round 2 with the predecessor DAG built lazily (kgs_params.lazy_dag).  The candidates whose key
// cut-off is not valid (cut_valid: level-cover may keep fewer than all of their sources) get their whole
// closures as before.  The others start from their direct predecessors only (one pre-pass round); each
// pass then walks every unfinished candidate over the DAG built so far: the cut stops it as soon as the
// weight of the closure nodes found exceeds the k-th key T (the nodes found are in the closure whatever
// lies beyond, so the bound is exact), a walk that met no missing list gives the exact key, and the others
// request the lists they met missing (central_graph, lazy) — one more pre-pass round over exactly those
// nodes, and the next pass.  A walk that finishes has the same closure as with the whole DAG, so keys and
// answers are unchanged; only the DAG built for candidates that end up cut shrinks.
__device__ void topdown(const Ctx &c, BigTile &S, long long *sh, char *dsmem, QOut *qo) {
    const Grp &G = c.G;
    const EngineArgs &a = c.a;
    Ctl *ctl = c.ctl;
    const uint32_t nc = __ldcg(&ctl->n_central);
    const uint32_t kk = (uint32_t)a.k < nc ? (uint32_t)a.k : nc;
    const uint32_t mcap = min((uint32_t)KGS_MAX_K, max(8u * kk, (uint32_t)a.prune_min));
    // predecessor lists: from the arcs the search recorded, else by the in-arc pre-pass (pred_dag)
    const bool rec = a.dag_record &&
                     recorded_dag(c, sh, qo, a.prune && nc > mcap ? (unsigned long long)a.rec_max : ~0ull);
    if (!a.prune || nc <= mcap) {
        if (!rec) {
            seed_pd(c, nullptr, nc);
            stamp(G, qo, TS_PD_SEED);
            pred_dag(c, S, sh, qo);
        }
        extract_list(c, sh, dsmem, nullptr, nc, qo);
        if (G.gtid() == 0) { ctl->work_big = 0; ctl->work_emit = 0; ctl->work_huge = 0; }   // emit counters (read after the select)
        if (a.containment) containment_select(c, sh, dsmem, kk);
        else select_topk(c, sh, dsmem, kk);
    } else {
        const uint32_t m = mcap;
        for (int64_t i = G.gtid(); i < nc; i += G.gsz) {   // lower bounds; cflag 2 = not extracted
            const int32_t cn = __ldcg(c.w.centrals + i);
            double lb;
            if (a.prune == 2) {   // the kept graph holds a lightest-or-heavier path from T_i to c, every i
                uint32_t mx = 0;
                for (int j = 0; j < c.qq.q; ++j) mx = max(mx, __ldcg(c.w.mw + (int64_t)cn * 8 + j));
                lb = (double)mx * (1.0 / 16777216.0);
            } else {
                lb = (double)__ldg(a.g.weight + cn);
            }
            c.w.ckey[i] = __dmul_rn(a.dpow[__ldcg(c.w.cdepth + i)], lb);
            c.w.cflag[i] = 2;
        }
        G.sync();
        select_topk(c, sh, dsmem, m);                          // sel[0..m): the m smallest (LB, id)
        uint64_t bhi; uint32_t blo;
        comp_key(c, (uint32_t)__ldcg(c.w.sel + m - 1), bhi, blo);
        for (int64_t j = G.gtid(); j < m; j += G.gsz) c.w.elist[j] = __ldcg(c.w.sel + j);
        G.sync();
        if (!rec) {
            seed_pd(c, c.w.elist, m);
            stamp(G, qo, TS_PD_SEED);
            pred_dag(c, S, sh, qo);
        }
        extract_list(c, sh, dsmem, c.w.elist, m, qo);
        rank_list(c, dsmem, c.w.elist, m, kk);                 // T = the kk-th exact (key, id)
        uint64_t thi; uint32_t tlo;
        comp_key(c, (uint32_t)__ldcg(c.w.sel + kk - 1), thi, tlo);
        uint32_t n2 = 0;
        if (bhi < thi || (bhi == thi && blo < tlo)) {
            // round 2: every candidate not extracted yet whose (LB, id) still ranks before T
            for (int64_t i = G.gtid(); i < nc; i += G.gsz) {
                if (__ldcg(c.w.cflag + i) != 2) continue;
                uint64_t hi; uint32_t lo;
                comp_key(c, (uint32_t)i, hi, lo);
                if (hi < thi || (hi == thi && lo < tlo)) c.w.elist[m + agg_slot(&ctl->n_elist2, 7u)] = (int32_t)i;
            }
            G.sync();
            n2 = __ldcg(&ctl->n_elist2);
            // exact cut-off: the k-th key so far (vertex-partitioned top-down has no multi-keyword union)
            const double cut = a.td_only ? kNoCut : __ldcg(c.w.ckey + __ldcg(c.w.sel + kk - 1));
            // lazy DAG (above): partition into qlight, cut valid from the front, the others from the back
            const bool lazy = a.lazy_dag && !rec && !a.td_only && a.level_cover == 1 && a.rm_ok;
            uint32_t nv = 0;
            if (lazy) {
                const uint32_t multi = __ldcg(&ctl->multi_kw);
                if (G.gtid() == 0) { ctl->n_valid = 0u; ctl->n_inc = 0u; }
                G.sync();
                for (int64_t i = G.gtid(); i < n2; i += G.gsz) {
                    const int32_t idx = __ldcg(c.w.elist + m + i);
                    const int32_t cn = __ldcg(c.w.centrals + idx);
                    const uint64_t Mc = ldrow(c.w.M, cn);
                    uint32_t zbc = 0;
                    for (int k = 0; k < c.qq.q; ++k) if (((Mc >> (8 * k)) & 0xFF) == 0) zbc |= 1u << k;
                    if (cut_valid(c, cn, zbc, multi)) c.w.qlight[agg_slot(&ctl->n_valid, 11u)] = idx;
                    else c.w.qlight[n2 - 1 - agg_slot(&ctl->n_inc, 12u)] = idx;
                }
                G.sync();
                nv = __ldcg(&ctl->n_valid);
            }
            // step 0: the candidates whose closures are built whole (all of them without the lazy DAG);
            // steps 1, 2, ...: lazy passes over the others (one call site each for the pre-pass and the
            // extraction: more inlined copies of them spilled the whole kernel)
            int32_t *cur = c.w.qlight, *nxt = c.w.lz;
            for (int step = lazy && nv == n2 ? 1 : 0;; ++step) {
                const bool lz = step > 0;
                const int32_t *L = !lazy ? c.w.elist + m : (lz ? cur : c.w.qlight + nv);
                const uint32_t cnt = !lazy ? n2 : (lz ? (step == 1 ? nv : __ldcg(&ctl->n_inc)) : n2 - nv);
                if (!rec) {
                    if (step <= 1) seed_pd(c, L, cnt);
                    pred_dag(c, S, sh, qo, true, !lz || step >= 16 ? (1 << 30) : 1);
                }
                // where rm cannot decide (no rm, or keyword 7 of a q = 8 query), which of the candidates
                // whose closures are whole can have s* >= 2 is decided from the DAG (mk_reach)
                if (!lz && !a.td_only && a.level_cover == 1 && cnt >= (uint32_t)a.mk_min &&
                    (__ldcg(&ctl->multi_kw) & c.qq.full) && (!a.rm_ok || c.qq.q > 7)) {
                    mk_reach(c);
                    stamp(G, qo, TS_MK);
                }
                extract_list(c, sh, dsmem, L, cnt, qo, cut, lz, step <= 1, nxt);
                if (!lazy || (!lz && nv == 0)) break;
                if (!lz && G.gtid() == 0) ctl->mk_reach = 0u;   // lz becomes a candidate list (next barrier)
                if (lz) {
                    publish_flags(ctl);   // the lists the walks requested (pre-pass round bitmap 0)
                    G.sync();
                    const uint32_t inc = __ldcg(&ctl->n_inc);
                    if (G.gtid() == 0) { ctl->n_lazy_iter = step; pd_round0_reset(c); }
                    if (!inc) break;
                    int32_t *t = cur; cur = nxt; nxt = t;   // the unfinished walks, for the next pass
                }
                G.sync();
            }
        }
        if (G.gtid() == 0) { ctl->work_big = 0; ctl->work_emit = 0; ctl->work_huge = 0; }
        if (m + n2 <= (uint32_t)KGS_MAX_K) {
            rank_list(c, dsmem, c.w.elist, m + n2, kk);
        } else {   // the candidates never extracted rank after every extracted one
            for (int64_t i = G.gtid(); i < nc; i += G.gsz)
                if (__ldcg(c.w.cflag + i) == 2) c.w.ckey[i] = __longlong_as_double(0x7FF0000000000000ll);
            G.sync();
            select_topk(c, sh, dsmem, kk);
        }
    }
    stamp(G, qo, TS_SELECT);
    emit_answers(c, sh, dsmem, qo);
}

// ------------------------------------------------------------------------------------------ engine
#ifndef KGS_MINB
#define KGS_MINB 2   // CTAs per SM the register budget is sized for
#endif
// One query of the batch, end to end, by the CTAs of group G (s_q: the query index and its keywords,
// staged in shared memory by the caller).
__device__ __forceinline__ void run_query(const EngineArgs &a, const Grp &G, const DevWork &w, BigTile &s_big,
                                       long long *sh, char *dsmem, const int32_t *s_q) {
    __shared__ Q s_query;   // written by thread 0 after the previous query's last group barrier
    if (threadIdx.x == 0) {
        s_query.qi = s_q[0];
        s_query.q = s_q[1];
        s_query.full = (1u << s_query.q) - 1u;
        for (int i = 0; i < kMaxQ; ++i) s_query.kw[i] = s_q[2 + i];
    }
    __syncthreads();
    const Q &qq = s_query;
    bool bad = qq.q < 1 || qq.q > kMaxQ;   // device-side validation (kgs_query_batch_device)
    for (int i = 0; !bad && i < qq.q; ++i) {
        if (qq.kw[i] < 0 || qq.kw[i] >= a.g.n_kw) bad = true;
        for (int j = 0; j < i; ++j) if (qq.kw[j] == qq.kw[i]) bad = true;
    }
    if (bad) {
        if (G.gtid() == 0) {
            QOut *qo = a.qout + qq.qi;
            qo->stop_reason = KGS_STOP_INVALID_QUERY; qo->count = 0; qo->levels = 0; qo->fatal = 0;
            qo->n_central = 0; qo->n_stamp = 0; qo->group = G.g; qo->pull_level = -1; qo->n_cut = 0;
        }
        G.sync();
        return;
    }
    const uint32_t done = __ldcg(w.gstate + 1);
    Ctl *ctl = w.ctl[done & 1];
    {   // zero this query's control block
        uint32_t *cw = reinterpret_cast<uint32_t *>(ctl);
        for (int64_t j = G.gtid(); j < (int64_t)(sizeof(Ctl) / 4); j += G.gsz) cw[j] = 0u;
    }
    QOut *qo = a.qout + qq.qi;
    if (G.gtid() == 0) {
        qo->n_stamp = 0; qo->t_start = globaltimer_ns();
        qo->group = a.G > 1 && G.gcount == (int)gridDim.x ? a.G : G.g;   // a.G: the whole grid (deferred)
    }
    G.sync();
    stamp(G, qo, TS_START);
    const int rns = rec_stripes(G);
    const Ctx c{a, w, ctl, G, qq, rns, G.grank % rns, w.pcap / rns};
    if (a.td_only) td_only_prepare(c, qo);
    else search(c, s_big, sh, qo);
    // a query group that finds more than defer_min central nodes leaves the query to the whole grid at the
    // end of the launch (its top-down parallelises over every CTA; on 1/G of the GPU it held the batch)
    const bool defer = a.defer_min > 0 && G.gcount < (int)gridDim.x && !a.search_only &&
                       __ldcg(&ctl->n_central) > (uint32_t)a.defer_min;
    if (defer) {
        if (G.gtid() == 0) a.defer_list[atomicAdd(a.defer_cnt, 1u)] = qq.qi;
    } else if (!a.search_only) {
        topdown(c, s_big, sh, dsmem, qo);   // search_only: workload analysis (no answers)
    }
    if (G.gtid() == 0) {
        if (!defer) {
            qo->levels = ctl->levels;
            qo->stop_reason = ctl->stop_reason;
            qo->count = (int32_t)ctl->sel_count;
            qo->fatal = ctl->fatal;
            qo->n_central = ctl->n_central;
            qo->n_overflow = ctl->n_overflow;
            qo->n_cid = ctl->n_cid;
            qo->n_parcs = ctl->n_parcs;
            qo->n_eval = ctl->n_eval;
            qo->n_tier4 = ctl->n_tier4;
            qo->pull_level = ctl->pull_at - 1;
            qo->n_cut = (int32_t)ctl->n_cut;
            qo->frontier_total = ctl->frontier_total;
            qo->arcs_scanned = ctl->arcs_scanned;
            qo->hits = ctl->hits;
            qo->dag_arcs = ctl->dag_arcs;
            qo->td_arcs = ctl->td_arcs;
            qo->td_arcs_big = ctl->td_arcs_big;
            qo->t_end = globaltimer_ns();
        }
        w.gstate[1] = done + 1;
        // after a top-down-only query the next one resets densely; bit 1: a recorded-DAG query left its
        // compact ids (search() "Predecessor-list state")
        w.gstate[2] = a.td_only ? 0u : (1u | (ctl->rec_used || a.dag_record ? 2u : 0u));
        w.gstate[3] = (uint32_t)a.R;
    }
    G.sync();
}

__device__ __forceinline__ void stage_query(const EngineArgs &a, int32_t *s_q, uint32_t qi) {
    s_q[0] = (int32_t)qi;
    if (qi < (uint32_t)a.nq) {
        s_q[1] = a.qconst > 0 ? a.qconst : a.qlen[qi];
        for (int i = 0; i < kMaxQ; ++i) s_q[2 + i] = a.kw[(int64_t)qi * kMaxQ + i];
    }
}

__global__ void __launch_bounds__(kBlock, KGS_MINB) k_engine(EngineArgs a) {
    // one dynamic shared region, reused phase by phase: expansion tiles (search, pre-pass), the per-warp
    // tier-1 extraction arenas (top-down), the rank sort of the selection
    extern __shared__ __align__(16) char dsmem[];
    BigTile &s_big = *reinterpret_cast<BigTile *>(dsmem);
    __shared__ long long sh[40];
    __shared__ int32_t s_q[2 + kMaxQ];
    // group of this CTA: contiguous ranges, sizes differ by at most one
    __shared__ Grp s_grp;
    if (threadIdx.x == 0) {
        Grp &G = s_grp;
        const int nb = gridDim.x, gsz_b = nb / a.G, extra = nb % a.G;
        const int b = blockIdx.x;
        const int cut = extra * (gsz_b + 1);
        if (b < cut) { G.g = b / (gsz_b + 1); G.grank = b % (gsz_b + 1); G.gcount = gsz_b + 1; }
        else { G.g = extra + (b - cut) / gsz_b; G.grank = (b - cut) % gsz_b; G.gcount = gsz_b; }
        G.gsz = (int64_t)G.gcount * blockDim.x;
        G.bar = a.bars + G.g;
        G.episode = 0;
    }
    __syncthreads();
    for (int t = threadIdx.x; t < kFlagSlots; t += blockDim.x) cta_flags()[t] = 0u;   // (synced below)
    // phase 1: each group takes the batch's queries one by one; phase 2 (query groups only): the deferred
    // queries, every CTA of the grid as one group (group 0's workspace, barrier a.bars[G])
    bool fin = false;
    uint32_t t_def = 0, n_def = 0;
    for (;;) {
        if (!fin) {
            const Grp &G = s_grp;
            const DevWork &w = a.works[G.g];
            if (G.gtid() == 0) w.gstate[0] = atomicAdd(a.next_query, 1u);   // the group leader takes the next query
            G.sync();
            if (threadIdx.x == 0) stage_query(a, s_q, __ldcg(w.gstate));
            __syncthreads();
            if (s_q[0] >= a.nq) {
                if (a.G == 1 || a.defer_min <= 0) break;
                if (threadIdx.x == 0) {
                    Grp &Gf = s_grp;
                    Gf.g = 0; Gf.grank = blockIdx.x; Gf.gcount = gridDim.x;
                    Gf.gsz = (int64_t)Gf.gcount * blockDim.x;
                    Gf.bar = a.bars + a.G;
                    Gf.episode = 0;
                }
                __syncthreads();
                s_grp.sync();   // every group is done: the deferred list is complete
                n_def = __ldcg(a.defer_cnt);
                fin = true;
            }
        }
        if (fin) {
            if (t_def >= n_def) break;
            if (threadIdx.x == 0) stage_query(a, s_q, (uint32_t)__ldcg(a.defer_list + t_def));
            ++t_def;
            __syncthreads();
        }
        run_query(a, s_grp, a.works[s_grp.g], s_big, sh, dsmem, s_q);
    }
}

size_t engine_dyn_smem() { return (size_t)KGS_MAX_K * (8 + 4 + 4); }

int engine_max_grid(int device) {
    // the dynamic shared-memory attribute is per device: set it on every device the engine runs on
    cudaFuncSetAttribute(k_engine, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)engine_dyn_smem());
    int per_sm = 0, sms = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_engine, kBlock, engine_dyn_smem());
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    return per_sm * sms;
}

cudaError_t launch_engine(const EngineArgs &a, int grid, cudaStream_t s) {
    void *args[] = {(void *)&a};
    return cudaLaunchCooperativeKernel((const void *)k_engine, dim3(grid), dim3(kBlock), args, engine_dyn_smem(), s);
}

}  // namespace kgs
