// kgs_internal.h — device data layout and kernel entry points shared by the libkgs translation units.
// Product code (CUDA path).  Shares nothing with oracle/.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/kgs.h"

namespace kgs {

constexpr int kMaxQ = KGS_MAX_Q;
constexpr int kWarp = 32;
constexpr int kBlock = 512;            // threads per CTA of the engine kernel

// Degree classes for the expansion's load balance: light frontier nodes are
// expanded by warp batches, big ones (more than kBigDeg arcs) in tiles spread over the whole group.
constexpr int64_t kBigDeg = 2048;
enum : uint8_t { CLS_LIGHT = 0, CLS_BIG = 1 };
// A class byte is (big flag) | (lg << 1): lg = 0 for no arcs, else 2^(lg-1) >= degree (auto direction).
__host__ __device__ __forceinline__ bool cls_big(uint8_t c) { return (c & 1u) != 0; }
__host__ __device__ __forceinline__ unsigned long long cls_deg_bound(uint8_t c) { return c >> 1 ? 1ull << ((c >> 1) - 1) : 0ull; }

// Per-warp arena of the Central Graph extractor.
constexpr int kExtNodes = 256;
constexpr int kExtArcs = 512;
constexpr int kExtHash = 512;
// Per-CTA arena of the large-graph extractor.
constexpr int kBigNodes = 1 << 16;
constexpr int kBigArcs = 1 << 18;
constexpr int kBigHash = 1 << 17;
// Per-group arena of the huge-graph extractor (tier 4: one CTA of the group, Central Graphs beyond a
// CTA arena — the deepest C4 queries reach them).
constexpr int kHugeNodes = 1 << 22;
constexpr int kHugeArcs = 1 << 24;
constexpr int kHugeHash = 1 << 23;

// Append regions of the recorded DAG (engine.cu visit_arc): one counter per region, 32 bytes apart.
constexpr int kRecStripes = 128;
constexpr int kRecStride = 8;

// Query control block (one per query in flight, zeroed at the start of every query).
struct Ctl {
    uint32_t slot_flag[256];       // level slot s has pending frontier bits
    uint32_t qn[2][2];             // [level parity][light, big] compacted frontier sizes
    uint32_t n_central;
    uint32_t n_touched;
    uint32_t n_overflow;
    uint32_t work_ext;             // extraction work counter
    uint32_t work_emit;            // emit work counter
    int32_t fatal;                 // non-zero: an arena overflowed beyond the large path
    int32_t levels;
    int32_t stop_reason;
    unsigned long long frontier_total;
    unsigned long long arcs_scanned;
    unsigned long long hits;       // new (node, keyword) hits (M entries written)
    uint32_t hist[12][256];        // radix-select histograms (one per digit)
    uint32_t sel_count;
    uint32_t work_big;             // large-graph extraction work counter
    // shared predecessor DAG (top-down pre-pass)
    uint32_t pd_flag[2];
    uint32_t pd_qn[2][2];
    uint32_t n_cid;                // nodes of the union of closures that have predecessor lists
    uint32_t n_parcs;              // predecessor arcs found
    unsigned long long td_arcs;    // in-arcs inspected by the pre-pass
    unsigned long long td_arcs_big;   // ... of them, in-arcs of nodes with more than kBigDeg in-arcs
    int32_t pd_rounds;
    uint32_t n_eval;               // candidates whose exact key was computed (all of C without pruning)
    uint32_t n_elist2;             // second pruning round: candidates whose bound still beats the threshold
    uint32_t mw_dirty;             // this query wrote lightest-path rows (prune mode 2): the next one resets them
    unsigned long long dag_arcs;   // arcs the search traversed that hit their target (the Thm. V.4 arcs)
    uint32_t ndef[2];              // [level parity] compaction: nodes deferred to the group-wide pass
    uint32_t pd_ndef[2];           // [round parity] the same for the predecessor pre-pass
    uint32_t rec_overflow;         // the recorded DAG overflowed pcap: the pre-pass was used
    uint32_t rec_used;             // the predecessor lists came from the recorded DAG (compact ids = touched)
    uint32_t rec_cnt[kRecStripes * kRecStride];   // recorded arcs per append region (stride 32 B)
    uint32_t pd_cnt[kRecStripes * kRecStride];    // pre-pass predecessor arcs per append region
    // push / pull direction (kgs_params.direction)
    unsigned long long mf[2];      // [level parity] out-arcs of the compacted frontier (auto direction)
    unsigned long long pull_marks[2];   // [level parity] new (node, keyword) hits of a pull level
    uint32_t pull_nbig[2];         // [level parity] pull candidates with more than kBigDeg in-arcs
    int32_t pull_at;               // first pulled level + 1 (0: push throughout)
    uint32_t pull_wait[2];         // [level parity] a pulled level without hits: some node is still on Alg. 2's work list
    uint32_t pull_wbig[2];         // [level parity] ... big nodes to check after the sweep
    uint32_t work_huge;            // Central Graphs beyond the CTA arenas (tier 4), this extract / emit pass
    uint32_t multi_kw;             // union of the keyword sets of the nodes holding >= 2 query keywords
    uint32_t n_cut;                // candidates stopped by the exact key cut-off (pruning round 2)
    uint32_t work_huge2;           // ... beyond the per-CTA large arenas too (tier 4, one CTA of the group)
    uint32_t n_tier4;              // Central Graphs this query extracted in the tier-4 arena (all passes)
    uint32_t ctile[2];             // [level parity] compaction: next bitmap tile to take
    uint32_t pd_ctile[2];          // [round parity] the same for the predecessor pre-pass
    uint32_t xbatch[2];            // [level parity] expansion: next warp batch beyond the first round
    uint32_t pd_xbatch[2];         // [round parity] the same for the pre-pass
    uint32_t mk_reach;             // pcnt holds, per compact id, the keywords a multi-keyword source reaches it in
    uint32_t mk_changed[2];        // [pass parity] mk_reach fixpoint
    uint32_t n_inc;                // lazy round 2: candidates whose closure is not complete yet
    uint32_t n_valid;              // lazy round 2: candidates whose key cut-off is valid (partition)
    uint32_t n_lazy_iter;          // lazy round 2: extraction passes
};

// Per-query summary written by the engine (device), read back by the host.
constexpr int kMaxStamps = 48;
struct QOut {
    int32_t levels, stop_reason, count, fatal;
    uint32_t n_central, n_overflow, n_cid, n_parcs, n_eval, n_tier4;
    unsigned long long frontier_total, arcs_scanned, hits, td_arcs, dag_arcs, td_arcs_big;
    unsigned long long t_start, t_search_end, t_end;   // %globaltimer ns
    int32_t group, n_stamp;
    int32_t pull_level, n_cut;     // first pulled level (-1: push throughout); key cut-offs
    unsigned long long stamp[kMaxStamps];
    int32_t stamp_tag[kMaxStamps];
};

__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// tags of the phase stamps
enum { TS_START = 0, TS_RESET, TS_SCATTER, TS_MERGE, TS_EXPAND, TS_PD_SEED, TS_PD_MERGE, TS_PD_EXPAND, TS_PD_CSR,
       TS_END, TS_EXTRACT, TS_EXTRACT_BIG, TS_SELECT, TS_EMIT,
       TS_PD_MERGE2, TS_PD_EXPAND2, TS_EXTRACT2, TS_MK };   // pruning round 2's pre-pass and extraction

struct DevGraph {
    int64_t n, m;
    const int64_t *row_ptr;
    const int32_t *col_idx;
    const int64_t *in_ptr;
    const int32_t *in_idx;
    const float *weight;
    const uint8_t *cls;       // degree class per node (out-arcs)
    const uint8_t *cls_in;    // degree class per node (in-arcs; == cls for a symmetric graph)
    int64_t n_kw;
    const int64_t *kw_ptr;
    const int32_t *kw_nodes;
    const int32_t *orig;      // [n] internal id -> input id (relabel.cu); nullptr: ids are the input ids
};

// Per-group query workspace (all sized for n at load time).  One group answers one query at a time.
struct DevWork {
    uint32_t *st;       // [n] status word: hm | K << 8 | nm << 16 | a << 24 (engine.cu "Data layout")
    uint8_t *M;         // [n*8] hitting levels, node-major, valid where the hm bit is set
    uint32_t *fbits;    // [R][W] frontier bitmaps, slot = level % R (FIdentifier)
    int32_t *qlight;    // [n] compacted frontier of the current level (big nodes replaced by -1)
    int32_t *qbig;      // [n_big] compacted frontier, big nodes
    int32_t *touched;   // [n] nodes whose hm became non-zero (sparse reset of the next query)
    int32_t *qdef;      // [n] compaction: queue positions deferred to the group-wide pass (dense tiles)
    int32_t *centrals;  // [n] central ids in identification order
    uint8_t *cdepth;    // [n] depth per central
    double *ckey;       // [n] Eq. 6 key per central
    int32_t *overflow;  // [n] centrals whose graph exceeds the per-warp extractor
    char *huge;         // tier-4 extraction arena (kHuge*), used by one CTA of the group
    uint8_t *cflag;     // [n] 1 = overflowed the per-warp extractor
    int32_t *sel;       // [KGS_MAX_K] ranked winners (index into centrals)
    int32_t *elist;     // [n] candidates to extract (index into centrals)
    uint32_t *mw;       // [n*8] lightest hitting path per (node, keyword), fixed point 2^-24; all-ones = unset
    Ctl *ctl[2];        // ping-pong: the previous query's block drives the sparse reset
    // shared predecessor DAG over the union of all Central Graphs
    uint32_t *pd_state; // [n] byte0 = bits to expand this round, byte1 = bits for the next round, byte2 = done
    int32_t *pd_cid;    // [n] compact id of a node with a predecessor list, -1 otherwise
    int32_t *pd_touched;// [n] node of each compact id (reset list)
    uint32_t *pd_bits;  // [2][W] round bitmaps
    int32_t *pd_qlight; // [n]
    int32_t *pd_qbig;   // [n_big_in]
    int32_t *pcnt;      // [n] predecessors per compact id
    int32_t *pred_ptr;  // [n+1] CSR offsets per compact id
    int32_t *pred_u;    // [pcap] predecessor node
    uint16_t *pred_b;   // [pcap] low byte: keyword bits of the arc; high byte: zb(pred) (source bits)
    int32_t *pa_u;      // [pcap] arcs in discovery order
    int32_t *pa_x;      // [pcap] compact id of the successor
    uint16_t *pa_b;     // [pcap]
    int32_t *pa_slot;   // [pcap] position inside the successor's list
    int32_t *scan_tmp;  // [4096] block sums of the CSR scan
    int32_t *lz;        // [n] lazy round 2: candidate list (ping-pong with qlight)
    int64_t pcap;
    // group state (device): query counter, validity of the per-node state
    uint32_t *gstate;   // [0] current query index, [1] queries done by this group, [2] state valid, [3] last R
};

struct GroupBar {      // one cache line per group
    unsigned arrive;
    unsigned gen;
    unsigned pad[30];
};

// Batch of queries for one engine launch.
struct EngineArgs {
    DevGraph g;
    const uint8_t *act;         // [n] activation levels at the cached alpha
    int R;                      // level slots = amax + 2
    int64_t W;                  // 32-bit words per bitmap (multiple of 8)
    const double *dpow;         // [256] pow(d, lambda)
    DevWork *works;             // [G] (device array)
    GroupBar *bars;             // [G]
    int G;
    // queries
    int32_t nq;
    const int32_t *kw;          // [nq][KGS_MAX_Q]
    const int32_t *qlen;        // [nq]
    int qconst;                 // > 0: every query has this many keywords (qlen unused)
    uint32_t *next_query;       // global query counter
    int defer_min;              // query groups: a query with more central nodes is left to the whole grid
    uint32_t *defer_cnt;        // deferred queries so far
    int32_t *defer_list;        // [nq] their indices
    // parameters (shared by the batch)
    int k, max_depth, block_central, extract_mode, level_cover;   // level_cover: 0 off, 1 R13, 2 R13b
    int containment;            // NEXT-3 R16: drop Central Graphs that strictly contain another one
    int tile_light;             // light frontiers up to this many nodes are expanded by group-wide tiles
    int td_only;                // 1: skip the search, the state comes from the vertex-partitioned search (vpart.cu)
    int td_levels, td_stop;     //    its stop level / reason
    uint32_t td_ncentral;       //    and |C| (works[0].centrals / cdepth hold the list)
    int prune;                  // top-down pruning: 0 off, 1 bound w_c, 2 bound max_i lightest path_i
    int prune_min;              // round 1 extracts max(8k, prune_min) candidates
    int mk_min;                 // round 2: per-candidate s* >= 2 test (mk_reach) from this many candidates
    int rm_ok;                  // the search's rm bits decide the s* >= 2 test (hitting arcs = Thm. V.4 arcs)
    int lazy_dag;               // pruning round 2 builds the predecessor DAG only as far as the cut needs
    int rec_max;                // with pruning, a recorded DAG of more arcs is dropped for the pre-pass
    int dag_record;             // 1: the search records its Thm. V.4 arcs (predecessor lists without the pre-pass)
    int direction;              // KGS_DIR_AUTO / _PUSH / _PULL
    int pull_ratio;             // auto: pull once the frontier's out-arcs exceed m / pull_ratio
    long long pull_min;         //       and pull_min
    int search_only;            // KGS_SEARCH_ONLY=1 (analysis tool): skip the top-down, no answers
    // outputs
    QOut *qout;                 // [nq]
    int32_t *out_hdr;           // [nq][k][4]: central, depth, n_nodes, n_arcs
    double *out_key;            // [nq][k]
    long long *out_off;         // [nq][k][2]
    int32_t *out_nodes;
    int32_t *out_arcs;          // pairs
    long long out_nodes_cap, out_arcs_cap;
    unsigned long long *out_used;   // [2] arena counters
    // extraction arenas
    char *warp_arenas;          // one per warp of the grid
    size_t warp_arena_bytes;
    char *cta_arenas;           // one per CTA (large-graph path)
    char *large_arenas;         // one per CTA (tier 3b: up to large_nodes / large_arcs, no sort buffer)
    size_t large_arena_bytes;
    int large_hash, large_nodes, large_arcs;
    int big_hash, big_nodes, big_arcs;      // tier 3 (cta_arenas), sized to the graph (at most kBig*)
    int huge_hash, huge_nodes, huge_arcs;   // tier 4 (DevWork::huge), sized to the graph (at most kHuge*)
    size_t cta_arena_bytes;
};

// ---- vertex-partitioned search of one query (vpart.cu) ----
constexpr int64_t kVpBig = 4096;   // owned nodes with more in-arcs are pulled by a whole CTA
struct VpQuery {
    int q;
    uint32_t full;
    int32_t kw[kMaxQ];
};
struct VpBufs {                    // exchange buffers (caller-owned device memory, see kgs_vp_buffers)
    uint8_t *hm;                   // [n_pad] replicated hit masks (all-gather output)
    uint8_t *hm_slice;             // [slice] this rank's hit masks after the level (all-gather input)
    uint8_t *M;                    // [n_pad * 8] node-major hitting levels; rows [lo, hi) are this rank's
    unsigned long long *counts;    // [4] marks, new centrals, waiting work-list nodes, changed nodes (all-reduce sum)
    long long *chg;                // [slice] or null: changed owned nodes of the level, id << 8 | new mask
    int32_t *cent;                 // [slice] this rank's central nodes
    uint8_t *cdep;                 // [slice] their depths
    int32_t *cent_n;               // [1] their count
    int64_t n_pad, lo, hi;
};

// SM count of the current device (cached per device): grids are sized in multiples of it.
int device_sm_count();

// ---- launchers (return cudaError_t) ----
cudaError_t launch_activation(const float *w, int64_t n, double A, double alpha, uint8_t *act, uint32_t *amax,
                              cudaStream_t s);
cudaError_t launch_degree_class(const int64_t *row_ptr, int64_t n, uint8_t *cls, cudaStream_t s);
cudaError_t launch_snap_weights(float *w, int64_t n, cudaStream_t s);
cudaError_t launch_validate(const DevGraph &g, int32_t *err, cudaStream_t s);
cudaError_t launch_levels_out(const uint32_t *st, const uint8_t *M, const int32_t *perm, int64_t n, int q,
                              uint8_t *out, cudaStream_t s);
cudaError_t launch_gather_u8(const uint8_t *src, const int32_t *perm, int64_t n, uint8_t *out, cudaStream_t s);
cudaError_t launch_to_input_ids(const int32_t *ids, const int32_t *orig, int64_t cnt, int32_t *out, cudaStream_t s);
cudaError_t relabel_by_degree(int64_t n, int64_t m, int64_t P, int64_t **row_ptr, int32_t **col_idx, float **weight,
                              int32_t *kw_nodes, int32_t **orig_out, int32_t **perm_out, cudaStream_t s);
int engine_max_grid(int device);
size_t engine_dyn_smem();
size_t arena_bytes_host(int hcap, int ncap, int acap, int team, bool with_sort);
cudaError_t launch_engine(const EngineArgs &a, int grid, cudaStream_t s);
cudaError_t launch_vp_begin(const DevGraph &g, const VpQuery &qd, const uint8_t *act, const VpBufs &b, uint8_t *gate,
                            cudaStream_t s);
cudaError_t launch_vp_biglist(const DevGraph &g, int64_t lo, int64_t hi, int32_t *big, int32_t *nbig, cudaStream_t s);
cudaError_t launch_vp_level(const DevGraph &g, const VpQuery &qd, const uint8_t *act, const VpBufs &b,
                            const uint8_t *gate, uint8_t *X, const int32_t *big, int nbig, int l, int block_central,
                            cudaStream_t s);
cudaError_t launch_vp_waiting(const DevGraph &g, const VpQuery &qd, const uint8_t *act, const VpBufs &b,
                              const uint8_t *gate, int l, int block_central, cudaStream_t s);
cudaError_t launch_vp_apply(const long long *list, int64_t cnt, uint8_t *hm, cudaStream_t s);
cudaError_t launch_vp_pack_st(const uint8_t *hm, const uint8_t *gate, const uint8_t *act, int64_t n, uint32_t *st,
                              cudaStream_t s);

}  // namespace kgs
