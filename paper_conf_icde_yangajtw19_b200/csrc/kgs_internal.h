// kgs_internal.h — device data layout and kernel entry points shared by the libkgs translation units.
// Product code (CUDA path).  Shares nothing with oracle/.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/kgs.h"

namespace kgs {

constexpr int kMaxQ = KGS_MAX_Q;
constexpr int kWarp = 32;

// Degree classes for the expansion's load balance: light frontier nodes are
// expanded by warp batches, big ones (more than kBigDeg arcs) in tiles spread over the whole grid.
constexpr int64_t kBigDeg = 2048;
enum : uint8_t { CLS_LIGHT = 0, CLS_BIG = 1 };

// Per-warp shared-memory capacity of the Central Graph extractor.
constexpr int kExtNodes = 256;
constexpr int kExtArcs = 512;
constexpr int kExtHash = 512;
constexpr int kExtWarps = 4;  // warps per CTA in the extractor
// Per-CTA global-memory arena of the large-graph extractor.
constexpr int kBigNodes = 1 << 16;
constexpr int kBigArcs = 1 << 18;
constexpr int kBigHash = 1 << 17;
constexpr int kBigCtas = 64;

// Device control block, zeroed at the start of every query.
struct Ctl {
    uint32_t slot_flag[256];       // level slot s has pending frontier bits
    uint32_t qn[2][2];             // [level parity][light, big] compacted frontier sizes
    uint32_t n_central;
    uint32_t n_touched;
    uint32_t n_overflow;
    uint32_t work_ext;
    int32_t fatal;                 // non-zero: an arena overflowed beyond the large path
    uint32_t pad0;
    int32_t levels;
    int32_t stop_reason;
    int32_t empty_keyword;
    int32_t pad;
    unsigned long long frontier_total;
    unsigned long long arcs_scanned;
    unsigned long long hits;       // new (node, keyword) hits (M entries written)
    uint32_t hist[12][256];        // radix-select histograms (one per digit)
    uint32_t sel_count;
    uint32_t pad2;
    unsigned long long arena_used[2];  // emitted nodes / arcs
    // shared predecessor DAG (top-down pre-pass)
    uint32_t pd_flag[2];
    uint32_t pd_qn[2][2];
    uint32_t n_cid;                // nodes of the union of closures that have predecessor lists
    uint32_t n_parcs;              // predecessor arcs found
    unsigned long long td_arcs;    // in-arcs inspected by the pre-pass
    int32_t pd_rounds;
    int32_t pad3;
    // phase timestamps (%globaltimer, ns) written by thread 0 of the search kernel
    int32_t n_stamp;
    int32_t pad4;
    unsigned long long stamp[64];
    int32_t stamp_tag[64];
};

__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// tags of the phase stamps
enum { TS_START = 0, TS_RESET, TS_SCATTER, TS_MERGE, TS_EXPAND, TS_PD_SEED, TS_PD_MERGE, TS_PD_EXPAND, TS_PD_CSR, TS_END };

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
};

// Per-query device state (all sized for n at load time).
struct DevWork {
    uint8_t *act;       // [n] activation levels at act_alpha (Eqs. 3-5)
    uint16_t *st;       // [n] low byte: hit mask hm (bit i <=> M[v][i] finite); high byte: gate (0 for K, else a)
    uint32_t *nm;       // [ceil(n/4)] new hits of the current level, one byte per node
    uint8_t *M;         // [n*8] hitting levels, node-major, valid where the hm bit is set
    uint32_t *fbits;    // [R][W] frontier bitmaps, slot = level % R (FIdentifier)
    int64_t W;          // 32-bit words per bitmap
    int R;              // ring of level slots = amax + 2
    int32_t *qlight;    // [n] compacted frontier of the current level, light nodes (ascending ids per CTA)
    int32_t *qbig;      // [n_big] compacted frontier, big nodes
    int32_t *touched;   // [n] nodes whose hm became non-zero (sparse reset of the next query)
    int32_t *centrals;  // [n] central ids in identification order
    uint8_t *cdepth;    // [n] depth per central
    double *ckey;       // [n] Eq. 6 key per central
    int32_t *overflow;  // [n] centrals whose graph exceeds the shared-memory extractor
    uint8_t *cflag;     // [n] 1 = overflowed the shared-memory extractor
    int32_t *sel;       // [KGS_MAX_K] ranked winners (index into centrals)
    int32_t *kw_dev;    // [KGS_MAX_Q] query keyword ids
    double *dpow;       // [256] pow(d, lambda) per depth (host libm)
    Ctl *ctl;
    const Ctl *prev;    // previous query's control block (sparse reset), nullptr -> full reset
    // emitted answers
    int32_t *ans_hdr;   // [KGS_MAX_K][4]: central, depth, n_nodes, n_arcs
    double *ans_key;    // [KGS_MAX_K]
    long long *ans_off; // [KGS_MAX_K][2]: offsets into the node / arc arenas
    int32_t *arena_nodes;
    int32_t *arena_arcs;  // pairs
    long long arena_nodes_cap, arena_arcs_cap;
    // shared predecessor DAG over the union of all Central Graphs
    uint32_t *pd_state;   // [n] byte0 = bits to expand this round, byte1 = bits for the next round, byte2 = done
    int32_t *pd_cid;      // [n] compact id of a node with a predecessor list, -1 otherwise
    int32_t *pd_touched;  // [n] node of each compact id (reset list)
    uint32_t *pd_bits;    // [2][W] round bitmaps
    int32_t *pd_qlight;   // [n]
    int32_t *pd_qbig;     // [n_big_in]
    int32_t *pcnt;        // [n] predecessors per compact id
    int32_t *pred_ptr;    // [n+1] CSR offsets per compact id
    int32_t *pred_u;      // [pcap] predecessor node
    uint16_t *pred_b;     // [pcap] low byte: keyword bits of the arc; high byte: zb(pred) (source bits)
    int32_t *pa_u;        // [pcap] arcs in discovery order
    int32_t *pa_x;        // [pcap] compact id of the successor
    uint16_t *pa_b;       // [pcap]
    int32_t *pa_slot;     // [pcap] position inside the successor's list
    int32_t *scan_tmp;    // [4096] block sums of the CSR scan
    int64_t pcap;
    // large-graph extractor arenas
    void *big_ws;
    size_t big_bytes, big_bytes_emit;
    int big_hcap, big_ncap, big_acap, big_ctas;
};

struct QueryArgs {
    DevGraph g;
    DevWork w;
    int q;
    int k;
    int max_depth;
    int block_central;
    int extract_mode;
    int level_cover;
    int full_reset;     // 1: reset all per-node state; 0: only what the previous query (w.prev) touched
    int prev_R;
};

// ---- launchers (return cudaError_t) ----
cudaError_t launch_activation(const float *w, int64_t n, double A, double alpha, uint8_t *act, uint32_t *amax,
                              cudaStream_t s);
cudaError_t launch_degree_class(const int64_t *row_ptr, int64_t n, uint8_t *cls, cudaStream_t s);
cudaError_t launch_snap_weights(float *w, int64_t n, cudaStream_t s);
cudaError_t launch_search(const QueryArgs &a, int grid, int block, cudaStream_t s);
int search_max_grid(int device, int block);
cudaError_t launch_extract(const QueryArgs &a, int grid, cudaStream_t s);
cudaError_t launch_select(const QueryArgs &a, int grid, cudaStream_t s);
int select_max_grid(int device);
cudaError_t launch_emit(const QueryArgs &a, int grid, cudaStream_t s);
size_t big_arena_bytes(int hcap, int ncap, int acap, bool with_sort);
cudaError_t launch_levels_out(const QueryArgs &a, uint8_t *out, cudaStream_t s);
cudaError_t launch_validate(const DevGraph &g, int32_t *err, cudaStream_t s);

}  // namespace kgs
