// api.cu — the C-ABI of libkgs (include/kgs.h): graph loading, the query engine's buffers, result handles.
// Host code only validates and orchestrates: every step of the query path runs in engine.cu's kernel.
// There is no CPU fallback; without a CUDA device every call fails with KGS_ECUDA.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "kgs_internal.h"

using namespace kgs;

namespace {

thread_local std::string g_err;

kgs_status fail(kgs_status s, const std::string &msg) {
    g_err = msg;
    return s;
}

#define CUDA_TRY(expr)                                                                      \
    do {                                                                                    \
        cudaError_t _e = (expr);                                                            \
        if (_e != cudaSuccess)                                                              \
            return fail(_e == cudaErrorMemoryAllocation ? KGS_ENOMEM : KGS_ECUDA,           \
                        std::string(#expr) + ": " + cudaGetErrorString(_e));                \
    } while (0)

template <class T>
cudaError_t dmalloc(T **p, size_t count) {
    return cudaMalloc((void **)p, sizeof(T) * (count > 0 ? count : 1));
}

template <class T>
cudaError_t grow_pinned(T **p, size_t *cap, size_t need) {
    if (need <= *cap) return cudaSuccess;
    if (*p) cudaFreeHost(*p);
    *p = nullptr;
    const size_t c = std::max(need, 2 * *cap);
    cudaError_t e = cudaMallocHost((void **)p, sizeof(T) * c);
    *cap = e == cudaSuccess ? c : 0;
    return e;
}

template <class T>
cudaError_t grow_dev(T **p, size_t *cap, size_t need) {
    if (need <= *cap) return cudaSuccess;
    if (*p) cudaFree(*p);
    *p = nullptr;
    const size_t c = std::max(need, 2 * *cap);
    cudaError_t e = cudaMalloc((void **)p, sizeof(T) * c);
    *cap = e == cudaSuccess ? c : 0;
    return e;
}

}  // namespace

// ------------------------------------------------------------------------------------------ objects
struct kgs_graph {
    int device = 0;
    int64_t n = 0, m = 0, n_kw = 0;
    double A = 1.0;
    int symmetric = 1;
    // device graph
    int64_t *row_ptr = nullptr, *in_ptr = nullptr, *kw_ptr = nullptr;
    int32_t *col_idx = nullptr, *in_idx = nullptr, *kw_nodes = nullptr;
    float *weight = nullptr;
    uint8_t *cls = nullptr, *cls_in = nullptr;
    int32_t *orig = nullptr, *perm = nullptr;   // internal <-> input ids (relabel.cu); null: identity
    int64_t n_big = 0, n_big_in = 0;   // nodes with more than kBigDeg out- / in-arcs
    int64_t pred_arc_cap = 0;          // kgs_graph_desc.pred_arc_cap (0 = default)
    // per-alpha / per-lambda caches
    uint8_t *act = nullptr;
    uint32_t *amax_dev = nullptr;
    double act_alpha = -1.0;
    int amax = 0, R = 0, R_alloc = 0;
    int64_t W = 0;
    double *dpow = nullptr;
    double dpow_lambda = -1.0;
    // engine groups
    std::vector<DevWork> works;         // host copies of the per-group workspaces
    std::vector<int64_t> pcaps;
    DevWork *works_dev = nullptr;
    int works_dev_n = 0;
    GroupBar *bars = nullptr;
    int grid = 0;
    char *warp_arenas = nullptr, *cta_arenas = nullptr, *large_arenas = nullptr;
    size_t warp_arena_bytes = 0, cta_arena_bytes = 0, large_arena_bytes = 0;
    int large_hash = 0, large_nodes = 0, large_arcs = 0;
    int big_hash = 0, big_nodes = 0, big_arcs = 0, huge_hash = 0, huge_nodes = 0, huge_arcs = 0;
    size_t huge_arena_bytes = 0;
    // batch buffers
    int32_t *d_kw = nullptr, *d_qlen = nullptr;
    size_t d_kw_cap = 0, d_qlen_cap = 0;
    QOut *d_qout = nullptr;
    size_t d_qout_cap = 0;
    int32_t *d_hdr = nullptr;
    size_t d_hdr_cap = 0;
    double *d_key = nullptr;
    size_t d_key_cap = 0;
    long long *d_off = nullptr;
    size_t d_off_cap = 0;
    int32_t *d_nodes = nullptr, *d_arcs = nullptr;
    size_t d_nodes_cap = 0, d_arcs_cap = 0;
    unsigned long long *d_ctr = nullptr;   // [0] next query, [1..2] arena counters, [3] deferred queries
    int32_t *d_defer = nullptr;            // [nq] deferred queries (engine.cu run_query)
    size_t d_defer_cap = 0;
    // pinned host staging
    int32_t *h_kw = nullptr, *h_qlen = nullptr;
    size_t h_kw_cap = 0, h_qlen_cap = 0;
    QOut *h_qout = nullptr;
    size_t h_qout_cap = 0;
    int32_t *h_hdr = nullptr;
    size_t h_hdr_cap = 0;
    double *h_key = nullptr;
    size_t h_key_cap = 0;
    long long *h_off = nullptr;
    size_t h_off_cap = 0;
    int32_t *h_nodes = nullptr, *h_arcs = nullptr;
    size_t h_nodes_cap = 0, h_arcs_cap = 0;
    unsigned long long *h_ctr = nullptr;
    double *h_dpow = nullptr;
    uint32_t *h_amax = nullptr;
    cudaEvent_t ev[2];
    std::mutex mu;
    // vertex-partitioned search of one query (vpart.cu)
    uint8_t *vp_gate = nullptr, *vp_X = nullptr;
    size_t vp_X_cap = 0;
    int32_t *vp_big = nullptr, *vp_nbig_dev = nullptr;
    int vp_nbig = 0;
    int64_t vp_big_lo = -1, vp_big_hi = -1;
    VpBufs vp{};
    VpQuery vq{};
    kgs_params vp_p{};
    int vp_k = 0;
    bool vp_active = false;
    // the last enqueued batch (for the fetch calls)
    int last_nq = 0, last_k = 0, last_G = 1;
    std::vector<int> last_q;
    kgs_params last_p{};
    bool pending = false;
};

struct kgs_result {
    std::vector<kgs_answer> ans;
    std::vector<std::vector<int32_t>> nodes, arcs;
    std::vector<uint8_t> M, act, cdepth;
    std::vector<int32_t> centrals;
    std::vector<double> ckey;
    bool has_levels = false;
    int64_t n = 0;
    int q = 0;
    kgs_stats stats{};
    std::vector<int32_t> ph_tag;
    std::vector<uint64_t> ph_ns;
};

namespace {

void free_work(DevWork &w) {
    void *p[] = {w.st, w.M, w.fbits, w.qlight, w.qbig, w.touched, w.qdef, w.centrals, w.cdepth, w.ckey, w.overflow,
                 w.cflag, w.sel, w.elist, w.mw, w.ctl[0], w.ctl[1], w.pd_state, w.pd_cid, w.pd_touched, w.pd_bits, w.pd_qlight,
                 w.pd_qbig, w.pcnt, w.pred_ptr, w.pred_u, w.pred_b, w.pa_u, w.pa_x, w.pa_b, w.pa_slot, w.scan_tmp, w.lz,
                 w.gstate, w.huge};
    for (void *x : p) if (x) cudaFree(x);
    w = DevWork{};
}

// one group's workspace, sized for the graph (fbits for the largest level ring any group was given:
// every workspace of the graph holds R_alloc slots, so a later alpha with R <= R_alloc fits all of them)
kgs_status alloc_work(kgs_graph *g, DevWork &w, int64_t pcap) {
    const int64_t n = g->n;
    w = DevWork{};
    CUDA_TRY(dmalloc(&w.st, n));
    CUDA_TRY(dmalloc(&w.M, n * 8));
    // M is never reset between queries (a row entry is valid where hm has its bit), but every byte is
    // written once here so that no read of a whole 8-byte row touches uninitialised memory
    CUDA_TRY(cudaMemset(w.M, 0xFF, (size_t)n * 8));
    CUDA_TRY(dmalloc(&w.fbits, (size_t)std::max({g->R_alloc, g->R, 2}) * (size_t)g->W));
    CUDA_TRY(dmalloc(&w.qlight, n));
    CUDA_TRY(dmalloc(&w.qbig, g->n_big));
    CUDA_TRY(dmalloc(&w.touched, n));
    CUDA_TRY(dmalloc(&w.qdef, n));
    CUDA_TRY(dmalloc(&w.centrals, n));
    CUDA_TRY(dmalloc(&w.cdepth, n));
    CUDA_TRY(dmalloc(&w.ckey, n));
    CUDA_TRY(dmalloc(&w.overflow, n));
    CUDA_TRY(cudaMalloc((void **)&w.huge, g->huge_arena_bytes));
    CUDA_TRY(cudaMemset(w.huge, 0, g->huge_arena_bytes));   // persistent arena: not yet in a known state
    CUDA_TRY(dmalloc(&w.cflag, n));
    CUDA_TRY(dmalloc(&w.sel, KGS_MAX_K));
    CUDA_TRY(dmalloc(&w.elist, n));
    CUDA_TRY(dmalloc(&w.mw, n * 8));
    CUDA_TRY(cudaMemset(w.mw, 0xFF, (size_t)n * 8 * sizeof(uint32_t)));
    CUDA_TRY(dmalloc(&w.ctl[0], 1));
    CUDA_TRY(dmalloc(&w.ctl[1], 1));
    CUDA_TRY(cudaMemset(w.ctl[0], 0, sizeof(Ctl)));
    CUDA_TRY(cudaMemset(w.ctl[1], 0, sizeof(Ctl)));
    CUDA_TRY(dmalloc(&w.pd_state, n));
    CUDA_TRY(dmalloc(&w.pd_cid, n));
    CUDA_TRY(dmalloc(&w.pd_touched, n));
    CUDA_TRY(dmalloc(&w.pd_bits, 2 * g->W));
    CUDA_TRY(dmalloc(&w.pd_qlight, n));
    CUDA_TRY(dmalloc(&w.pd_qbig, g->n_big_in));
    CUDA_TRY(dmalloc(&w.pcnt, n));
    CUDA_TRY(dmalloc(&w.pred_ptr, n + 1));
    w.pcap = pcap;
    CUDA_TRY(dmalloc(&w.pred_u, (size_t)pcap));
    CUDA_TRY(dmalloc(&w.pred_b, (size_t)pcap));
    CUDA_TRY(dmalloc(&w.pa_u, (size_t)pcap));
    CUDA_TRY(dmalloc(&w.pa_x, (size_t)pcap));
    CUDA_TRY(dmalloc(&w.pa_b, (size_t)pcap));
    CUDA_TRY(dmalloc(&w.pa_slot, (size_t)pcap));
    CUDA_TRY(dmalloc(&w.scan_tmp, 4096));
    CUDA_TRY(dmalloc(&w.lz, n));
    CUDA_TRY(dmalloc(&w.gstate, 4));
    CUDA_TRY(cudaMemset(w.gstate, 0, 4 * sizeof(uint32_t)));   // not valid: the first query resets densely
    return KGS_OK;
}

}  // namespace

namespace kgs {
kgs_status set_error(kgs_status s, const std::string &msg) { return fail(s, msg); }
int64_t graph_nodes(const kgs_graph *g) { return g->n; }
int graph_device(const kgs_graph *g) { return g->device; }
}  // namespace kgs

extern "C" {

const char *kgs_last_error(void) { return g_err.c_str(); }
const char *kgs_version(void) { return "kgs 0.2 sm_100a engine (" __DATE__ ")"; }

void kgs_params_default(kgs_params *p) {
    if (!p) return;
    std::memset(p, 0, sizeof(*p));
    p->alpha = 0.1;       // Table III
    p->lambda = 0.2;
    p->max_depth = 254;
    p->block_central = 1;
    p->extract_mode = KGS_EXTRACT_EXACT;
    p->level_cover = 1;
    p->want_levels = 0;
    p->prune = 1;
    p->direction = KGS_DIR_AUTO;
    p->pull_ratio = 14;
    p->pull_min = 1ll << 22;
    p->prune_min = 512;
    p->tile_light = 8 * kBlock;
    p->dag_record = -1;
    p->search_only = 0;
    p->mk_min = 4096;
    p->defer_min = 1 << 16;
    p->lazy_dag = 1;
    p->rec_max = 1 << 24;
}

void kgs_free_graph(kgs_graph *g) {
    if (!g) return;
    cudaSetDevice(g->device);
    cudaDeviceSynchronize();
    for (auto &w : g->works) free_work(w);
    void *ptrs[] = {g->row_ptr, g->col_idx, g->kw_ptr, g->kw_nodes, g->weight, g->cls, g->act, g->amax_dev, g->dpow,
                    g->works_dev, g->bars, g->warp_arenas, g->cta_arenas, g->large_arenas, g->d_kw, g->d_qlen, g->d_qout, g->d_hdr,
                    g->d_key, g->d_off, g->d_nodes, g->d_arcs, g->d_ctr, g->d_defer, g->vp_gate, g->vp_X, g->vp_big,
                    g->vp_nbig_dev, g->orig, g->perm};
    for (void *p : ptrs) if (p) cudaFree(p);
    if (!g->symmetric) { cudaFree(g->in_ptr); cudaFree(g->in_idx); cudaFree(g->cls_in); }
    void *hp[] = {g->h_kw, g->h_qlen, g->h_qout, g->h_hdr, g->h_key, g->h_off, g->h_nodes, g->h_arcs, g->h_ctr,
                  g->h_dpow, g->h_amax};
    for (void *p : hp) if (p) cudaFreeHost(p);
    for (auto &e : g->ev) cudaEventDestroy(e);
    delete g;
}

kgs_status kgs_load_graph(const kgs_graph_desc *d, kgs_graph **out) {
    if (!d || !out) return fail(KGS_EINVAL, "null argument");
    *out = nullptr;
    if (d->n_nodes < 0 || d->n_nodes >= (int64_t(1) << 31) || d->n_arcs < 0 || d->n_arcs >= (int64_t(1) << 40) ||
        d->n_keywords < 1 || !(d->avg_dist_A > 0.0) || !std::isfinite(d->avg_dist_A))
        return fail(KGS_EINVAL, "n_nodes / n_arcs / n_keywords / avg_dist_A out of range");
    if (d->n_nodes > 0 && (!d->row_ptr || !d->weight)) return fail(KGS_EINVAL, "missing row_ptr / weight");
    if (d->pred_arc_cap < 0) return fail(KGS_EINVAL, "pred_arc_cap must be >= 0");
    if (d->n_arcs > 0 && !d->col_idx) return fail(KGS_EINVAL, "missing col_idx");
    if (!d->kw_ptr || !d->row_ptr) return fail(KGS_EINVAL, "missing kw_ptr / row_ptr");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
        return fail(KGS_ECUDA, "no CUDA device available (libkgs has no CPU path)");
    if (d->device < 0 || d->device >= ndev) return fail(KGS_EINVAL, "device ordinal out of range");
    CUDA_TRY(cudaSetDevice(d->device));
    const bool on_dev = (d->flags & KGS_INPUT_DEVICE_PTRS) != 0;
    const cudaMemcpyKind kind = on_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    const int64_t n = d->n_nodes, m = d->n_arcs, V = d->n_keywords;

    // host-side structural checks on the offsets (also needed for class counts / the reverse CSR)
    std::vector<int64_t> rp(n + 1), kp(V + 1);
    if (on_dev) CUDA_TRY(cudaMemcpy(rp.data(), d->row_ptr, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToHost));
    else std::memcpy(rp.data(), d->row_ptr, sizeof(int64_t) * (n + 1));
    if (on_dev) CUDA_TRY(cudaMemcpy(kp.data(), d->kw_ptr, sizeof(int64_t) * (V + 1), cudaMemcpyDeviceToHost));
    else std::memcpy(kp.data(), d->kw_ptr, sizeof(int64_t) * (V + 1));
    if (rp[0] != 0 || rp[n] != m) return fail(KGS_EINVAL, "row_ptr[0] must be 0 and row_ptr[n] == n_arcs");
    for (int64_t v = 0; v < n; ++v) {
        if (rp[v + 1] < rp[v]) return fail(KGS_EINVAL, "row_ptr not non-decreasing");
        if (rp[v + 1] - rp[v] >= (int64_t(1) << 31)) return fail(KGS_EINVAL, "a node has 2^31 or more arcs");
    }
    if (kp[0] != 0) return fail(KGS_EINVAL, "kw_ptr[0] must be 0");
    for (int64_t t = 0; t < V; ++t)
        if (kp[t + 1] < kp[t]) return fail(KGS_EINVAL, "kw_ptr not non-decreasing");
    const int64_t P = kp[V];
    if (P > 0 && !d->kw_nodes) return fail(KGS_EINVAL, "missing kw_nodes");

    kgs_graph *g = new kgs_graph();
    g->device = d->device; g->n = n; g->m = m; g->n_kw = V; g->A = d->avg_dist_A;
    g->symmetric = d->symmetric ? 1 : 0;
    g->pred_arc_cap = d->pred_arc_cap;
    auto bail = [&](kgs_status s) { kgs_free_graph(g); return s; };
#define G_TRY(expr)                                                                          \
    do {                                                                                     \
        cudaError_t _e = (expr);                                                             \
        if (_e != cudaSuccess)                                                               \
            return bail(fail(_e == cudaErrorMemoryAllocation ? KGS_ENOMEM : KGS_ECUDA,       \
                             std::string(#expr) + ": " + cudaGetErrorString(_e)));           \
    } while (0)
    for (auto &e : g->ev) G_TRY(cudaEventCreate(&e));
    G_TRY(dmalloc(&g->row_ptr, n + 1));
    G_TRY(dmalloc(&g->col_idx, m));
    G_TRY(dmalloc(&g->weight, n));
    G_TRY(dmalloc(&g->kw_ptr, V + 1));
    G_TRY(dmalloc(&g->kw_nodes, P));
    G_TRY(dmalloc(&g->cls, n));
    G_TRY(cudaMemcpy(g->row_ptr, d->row_ptr, sizeof(int64_t) * (n + 1), kind));
    if (m) G_TRY(cudaMemcpy(g->col_idx, d->col_idx, sizeof(int32_t) * m, kind));
    if (n) G_TRY(cudaMemcpy(g->weight, d->weight, sizeof(float) * n, kind));
    G_TRY(cudaMemcpy(g->kw_ptr, d->kw_ptr, sizeof(int64_t) * (V + 1), kind));
    if (P) G_TRY(cudaMemcpy(g->kw_nodes, d->kw_nodes, sizeof(int32_t) * P, kind));

    DevGraph dg{};
    dg.n = n; dg.m = m; dg.row_ptr = g->row_ptr; dg.col_idx = g->col_idx; dg.weight = g->weight;
    dg.n_kw = V; dg.kw_ptr = g->kw_ptr; dg.kw_nodes = g->kw_nodes;
    int32_t *derr = nullptr;
    G_TRY(dmalloc(&derr, 1));
    G_TRY(cudaMemset(derr, 0, sizeof(int32_t)));
    G_TRY(launch_validate(dg, derr, 0));
    int32_t herr = 0;
    G_TRY(cudaMemcpy(&herr, derr, sizeof(int32_t), cudaMemcpyDeviceToHost));
    cudaFree(derr);
    if (herr) {
        std::string why;
        if (herr & 1) why += " row_ptr decreasing;";
        if (herr & 2) why += " col_idx out of range;";
        if (herr & 4) why += " weight not in [0,1];";
        if (herr & 16) why += " kw_nodes out of range or not strictly increasing;";
        return bail(fail(KGS_EINVAL, "invalid graph:" + why));
    }
    G_TRY(launch_snap_weights(g->weight, n, 0));
    if (!(d->flags & KGS_NO_RELABEL))   // internal order: non-increasing degree (relabel.cu)
        G_TRY(relabel_by_degree(n, m, P, &g->row_ptr, &g->col_idx, &g->weight, g->kw_nodes, &g->orig, &g->perm, 0));
    G_TRY(launch_degree_class(g->row_ptr, n, g->cls, 0));
    for (int64_t v = 0; v < n; ++v)
        if (rp[v + 1] - rp[v] > kBigDeg) ++g->n_big;
    // reverse CSR for extraction along in-arcs (reading R1)
    if (g->symmetric) {
        g->in_ptr = g->row_ptr; g->in_idx = g->col_idx; g->cls_in = g->cls; g->n_big_in = g->n_big;
    } else {
        std::vector<int32_t> ci(m);   // the stored (possibly renumbered) CSR
        if (m) G_TRY(cudaMemcpy(ci.data(), g->col_idx, sizeof(int32_t) * m, cudaMemcpyDeviceToHost));
        G_TRY(cudaMemcpy(rp.data(), g->row_ptr, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToHost));
        std::vector<int64_t> ip(n + 1, 0);
        for (int64_t j = 0; j < m; ++j) ip[ci[j] + 1]++;
        for (int64_t v = 0; v < n; ++v) ip[v + 1] += ip[v];
        std::vector<int64_t> cur(ip.begin(), ip.end() - 1);
        std::vector<int32_t> ii(m);
        for (int64_t u = 0; u < n; ++u)
            for (int64_t j = rp[u]; j < rp[u + 1]; ++j) ii[cur[ci[j]]++] = (int32_t)u;
        G_TRY(dmalloc(&g->in_ptr, n + 1));
        G_TRY(dmalloc(&g->in_idx, m));
        G_TRY(cudaMemcpy(g->in_ptr, ip.data(), sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice));
        if (m) G_TRY(cudaMemcpy(g->in_idx, ii.data(), sizeof(int32_t) * m, cudaMemcpyHostToDevice));
        G_TRY(dmalloc(&g->cls_in, n));
        G_TRY(launch_degree_class(g->in_ptr, n, g->cls_in, 0));
        for (int64_t v = 0; v < n; ++v)
            if (ip[v + 1] - ip[v] > kBigDeg) ++g->n_big_in;
    }
    g->W = ((n + 31) / 32 + 7) / 8 * 8;   // words per bitmap, a multiple of 8 (16-byte vector access)
    G_TRY(dmalloc(&g->act, n));
    G_TRY(dmalloc(&g->amax_dev, 1));
    G_TRY(dmalloc(&g->dpow, 256));
    G_TRY(dmalloc(&g->d_ctr, 4));
    G_TRY(cudaMallocHost(&g->h_ctr, 4 * sizeof(unsigned long long)));
    G_TRY(cudaMallocHost(&g->h_dpow, 256 * sizeof(double)));
    G_TRY(cudaMallocHost(&g->h_amax, sizeof(uint32_t)));
    // the engine: one persistent cooperative grid; extraction arenas per warp and per CTA
    g->grid = engine_max_grid(g->device);
    if (g->grid <= 0) return bail(fail(KGS_ECUDA, "engine occupancy query failed"));
    g->warp_arena_bytes = arena_bytes_host(kExtHash, kExtNodes, kExtArcs, 32, true);
    {   // tiers 3, 3b and 4 sized to the graph (a Central Graph has at most n nodes; its arena arcs are the
        // predecessor entries, at most q per arc): small graphs do not pay for Wikidata-scale arenas
        auto pow2 = [](int64_t x) { int64_t p = 1; while (p < x) p <<= 1; return p; };
        const int64_t pn = pow2(std::max<int64_t>(g->n, 1024)), pm = pow2(std::max<int64_t>(8 * g->m, 4096));
        g->big_nodes = (int)std::min<int64_t>(kBigNodes, pn);
        g->big_arcs = (int)std::min<int64_t>(kBigArcs, pm);
        g->big_hash = 2 * g->big_nodes;
        g->huge_nodes = (int)std::min<int64_t>(kHugeNodes, pn);
        g->huge_arcs = (int)std::min<int64_t>(kHugeArcs, pm);
        g->huge_hash = 2 * g->huge_nodes;
        g->huge_arena_bytes = arena_bytes_host(g->huge_hash, g->huge_nodes, g->huge_arcs, kBlock, true);
    }
    g->cta_arena_bytes = arena_bytes_host(g->big_hash, g->big_nodes, g->big_arcs, kBlock, true);
    G_TRY(cudaMalloc(&g->warp_arenas, g->warp_arena_bytes * (size_t)g->grid * (kBlock / 32)));
    G_TRY(cudaMalloc(&g->cta_arenas, g->cta_arena_bytes * (size_t)g->grid));
    // persistent arenas (engine.cu carve): zero = "not yet reset", the first use resets fully
    G_TRY(cudaMemset(g->warp_arenas, 0, g->warp_arena_bytes * (size_t)g->grid * (kBlock / 32)));
    G_TRY(cudaMemset(g->cta_arenas, 0, g->cta_arena_bytes * (size_t)g->grid));
    {   // tier 3b: per-CTA arenas for Central Graphs beyond 64 K nodes, sized to the graph (at most 1 M nodes /
        // 4 M arcs, 88 MB per CTA at C3 scale)
        auto pow2 = [](int64_t x) { int64_t p = 1; while (p < x) p <<= 1; return p; };
        g->large_nodes = (int)std::min<int64_t>(1 << 20, pow2(std::max<int64_t>(g->n, 1024)));
        g->large_arcs = (int)std::min<int64_t>(1 << 22, pow2(std::max<int64_t>(8 * g->m, 4096)));
        g->large_hash = 2 * g->large_nodes;
        g->large_arena_bytes = arena_bytes_host(g->large_hash, g->large_nodes, g->large_arcs, kBlock, false);
        G_TRY(cudaMalloc(&g->large_arenas, g->large_arena_bytes * (size_t)g->grid));
        G_TRY(cudaMemset(g->large_arenas, 0, g->large_arena_bytes * (size_t)g->grid));
    }
    G_TRY(cudaDeviceSynchronize());
#undef G_TRY
    *out = g;
    return KGS_OK;
}

}  // extern "C"

// ------------------------------------------------------------------------------------------ query engine
namespace {

kgs_status check_params(const kgs_params &p, int32_t k) {
    if (k < 1 || k > KGS_MAX_K) return fail(KGS_EINVAL, "k must be in [1, 4096]");
    if (!(p.alpha > 0.0 && p.alpha < 1.0)) return fail(KGS_EINVAL, "alpha must be in (0, 1)");
    if (!(p.lambda >= 0.0) || !std::isfinite(p.lambda)) return fail(KGS_EINVAL, "lambda must be >= 0");
    if (p.max_depth < 1 || p.max_depth > 254) return fail(KGS_EINVAL, "max_depth must be in [1, 254]");
    if (p.extract_mode != KGS_EXTRACT_EXACT && p.extract_mode != KGS_EXTRACT_LITERAL)
        return fail(KGS_EINVAL, "extract_mode");
    if (p.prune < 0 || p.prune > 2) return fail(KGS_EINVAL, "prune must be 0, 1 or 2");
    if (p.level_cover < 0 || p.level_cover > 2) return fail(KGS_EINVAL, "level_cover must be 0, 1 or 2");
    if (p.containment != 0 && p.containment != 1) return fail(KGS_EINVAL, "containment must be 0 or 1");
    if (p.direction < KGS_DIR_AUTO || p.direction > KGS_DIR_PULL) return fail(KGS_EINVAL, "direction must be 0, 1 or 2");
    if (p.pull_ratio < 1 || p.pull_min < 0 || p.prune_min < 1 || p.tile_light < 0 || p.dag_record < -1 ||
        p.dag_record > 1 || (p.search_only != 0 && p.search_only != 1) || p.mk_min < 0 || p.defer_min < 0 ||
        (p.lazy_dag != 0 && p.lazy_dag != 1) || p.rec_max < 0)
        return fail(KGS_EINVAL, "tuning parameters out of range (pull_ratio >= 1, pull_min >= 0, prune_min >= 1, "
                                "tile_light >= 0, dag_record -1/0/1, search_only 0/1, mk_min >= 0, defer_min >= 0, lazy_dag 0/1, rec_max >= 0)");
    return KGS_OK;
}

kgs_status check_query(const kgs_graph *g, const int32_t *kw, int32_t q) {
    if (q < 1 || q > KGS_MAX_Q) return fail(KGS_EINVAL, "q must be in [1, 8]");
    for (int i = 0; i < q; ++i) {
        if (kw[i] < 0 || kw[i] >= g->n_kw) return fail(KGS_EINVAL, "keyword id out of range");
        for (int j = 0; j < i; ++j)
            if (kw[j] == kw[i]) return fail(KGS_EINVAL, "duplicate keyword id");
    }
    return KGS_OK;
}

// predecessor-arc capacity of a group workspace (kgs_graph_desc.pred_arc_cap; default min(m, 2^28),
// at least 2^20: the level-5 C4 queries record 192 M arcs, their pre-pass 135 M)
int64_t pcap_of(const kgs_graph *g) {
    if (g->pred_arc_cap > 0) return std::max<int64_t>(1024, g->pred_arc_cap);
    return std::max<int64_t>(std::min<int64_t>(g->m, 1ll << 28), 1 << 20);
}

// per-alpha activation cache, level-slot ring, per-lambda depth factors, G group workspaces
kgs_status prepare(kgs_graph *g, const kgs_params &p, int G, cudaStream_t s) {
    bool invalidate = false;
    if (p.alpha != g->act_alpha) {
        // activation cache (Eqs. 3-5) — recomputed only when alpha changes; amax sizes the level ring
        CUDA_TRY(launch_activation(g->weight, g->n, g->A, p.alpha, g->act, g->amax_dev, s));
        CUDA_TRY(cudaMemcpyAsync(g->h_amax, g->amax_dev, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        CUDA_TRY(cudaStreamSynchronize(s));
        g->amax = (int)*g->h_amax;
        g->act_alpha = p.alpha;
        g->R = g->amax + 2;
        invalidate = true;
    }
    if (std::max(g->R, 2) > g->R_alloc) {   // bigger ring: reallocate every group's bitmaps
        CUDA_TRY(cudaStreamSynchronize(s));
        g->R_alloc = std::max(g->R, 2);
        for (auto &w : g->works) {
            cudaFree(w.fbits);
            w.fbits = nullptr;
            CUDA_TRY(dmalloc(&w.fbits, (size_t)g->R_alloc * (size_t)g->W));
        }
        invalidate = true;
    }
    if ((int)g->works.size() < G) {
        CUDA_TRY(cudaStreamSynchronize(s));
        // predecessor-arc capacity per group (recorded search arcs, or pre-pass arcs; 20 B per arc)
        while ((int)g->works.size() < G) {
            const int64_t pcap = pcap_of(g);
            DevWork w;
            kgs_status st = alloc_work(g, w, pcap);
            if (st != KGS_OK) { free_work(w); return st; }
            g->works.push_back(w);
        }
        if (g->works_dev) cudaFree(g->works_dev);
        if (g->bars) cudaFree(g->bars);
        CUDA_TRY(dmalloc(&g->works_dev, g->works.size()));
        CUDA_TRY(dmalloc(&g->bars, g->works.size() + 1));   // + the whole grid's (deferred queries)
        CUDA_TRY(cudaMemset(g->bars, 0, sizeof(GroupBar) * (g->works.size() + 1)));
        g->works_dev_n = 0;
    }
    if (g->works_dev_n != (int)g->works.size() || invalidate) {
        CUDA_TRY(cudaMemcpyAsync(g->works_dev, g->works.data(), sizeof(DevWork) * g->works.size(), cudaMemcpyHostToDevice, s));
        g->works_dev_n = (int)g->works.size();
    }
    if (invalidate)
        for (auto &w : g->works) CUDA_TRY(cudaMemsetAsync(w.gstate, 0, 4 * sizeof(uint32_t), s));
    if (p.lambda != g->dpow_lambda) {
        // Eq. 6 depth factor d^lambda from the host libm (reading R15), one value per depth
        CUDA_TRY(cudaStreamSynchronize(s));
        for (int dd = 0; dd < 256; ++dd) g->h_dpow[dd] = std::pow((double)dd, p.lambda);
        CUDA_TRY(cudaMemcpyAsync(g->dpow, g->h_dpow, sizeof(double) * 256, cudaMemcpyHostToDevice, s));
        CUDA_TRY(cudaStreamSynchronize(s));
        g->dpow_lambda = p.lambda;
    }
    return KGS_OK;
}

// Enqueue one engine launch for nq queries whose padded keyword rows / lengths are in g->d_kw / d_qlen.
struct TdOnly {   // top-down-only launch over the state of a vertex-partitioned search
    int levels, stop;
    uint32_t n_central;
};

kgs_status launch(kgs_graph *g, int nq, int k, const kgs_params &p, int G, cudaStream_t s, int qconst = 0,
                  const TdOnly *td = nullptr) {
    G = std::max(1, std::min({G, nq, g->grid}));
    if ((int)g->works.size() < G) {   // each group needs its own workspace: keep them within free memory
        size_t free_b = 0, total_b = 0;
        cudaMemGetInfo(&free_b, &total_b);
        const size_t per = (size_t)g->n * 109 + (size_t)std::max(g->R, 2) * g->W * 4 + (size_t)(16ll << 20) * 18 +
                           (size_t)pcap_of(g) * 20 +
                           g->huge_arena_bytes;
        const int more = (int)std::min<size_t>((size_t)(G - (int)g->works.size()), (size_t)(0.8 * free_b) / per);
        G = std::max(1, (int)g->works.size() + more);
    }
    kgs_status st = prepare(g, p, G, s);
    if (st != KGS_OK) return st;
    CUDA_TRY(grow_dev(&g->d_qout, &g->d_qout_cap, (size_t)nq));
    CUDA_TRY(grow_dev(&g->d_defer, &g->d_defer_cap, (size_t)nq));
    CUDA_TRY(grow_dev(&g->d_hdr, &g->d_hdr_cap, (size_t)nq * k * 4));
    CUDA_TRY(grow_dev(&g->d_key, &g->d_key_cap, (size_t)nq * k));
    CUDA_TRY(grow_dev(&g->d_off, &g->d_off_cap, (size_t)nq * k * 2));
    // answer arena: 64 nodes per answer on average plus room for a few tier-4 (huge) Central Graphs
    CUDA_TRY(grow_dev(&g->d_nodes, &g->d_nodes_cap, (size_t)nq * k * 64 + (16u << 20)));
    CUDA_TRY(grow_dev(&g->d_arcs, &g->d_arcs_cap, 2 * ((size_t)nq * k * 64 + (32u << 20))));
    CUDA_TRY(cudaMemsetAsync(g->d_ctr, 0, 4 * sizeof(unsigned long long), s));
    // the result headers are copied back whole: clear them so that no byte the engine leaves unwritten
    // (phase stamps beyond n_stamp, answer slots beyond count) is uninitialised memory
    CUDA_TRY(cudaMemsetAsync(g->d_qout, 0, sizeof(QOut) * (size_t)nq, s));
    CUDA_TRY(cudaMemsetAsync(g->d_hdr, 0, sizeof(int32_t) * (size_t)nq * k * 4, s));
    CUDA_TRY(cudaMemsetAsync(g->d_key, 0, sizeof(double) * (size_t)nq * k, s));
    CUDA_TRY(cudaMemsetAsync(g->d_off, 0, sizeof(long long) * (size_t)nq * k * 2, s));
    EngineArgs a{};
    a.g.n = g->n; a.g.m = g->m; a.g.row_ptr = g->row_ptr; a.g.col_idx = g->col_idx; a.g.in_ptr = g->in_ptr;
    a.g.in_idx = g->in_idx; a.g.weight = g->weight; a.g.cls = g->cls; a.g.cls_in = g->cls_in; a.g.n_kw = g->n_kw;
    a.g.kw_ptr = g->kw_ptr; a.g.kw_nodes = g->kw_nodes;
    a.g.orig = g->orig;
    a.act = g->act; a.R = g->R; a.W = g->W; a.dpow = g->dpow;
    a.works = g->works_dev; a.bars = g->bars; a.G = G;
    a.nq = nq; a.kw = g->d_kw; a.qlen = g->d_qlen; a.qconst = qconst;
    a.next_query = reinterpret_cast<uint32_t *>(g->d_ctr);
    a.defer_min = td ? 0 : p.defer_min;
    a.defer_cnt = reinterpret_cast<uint32_t *>(g->d_ctr + 3);
    a.defer_list = g->d_defer;
    a.k = k; a.max_depth = p.max_depth; a.block_central = p.block_central ? 1 : 0; a.extract_mode = p.extract_mode;
    a.level_cover = p.level_cover;
    a.containment = p.containment;
    if (td) { a.td_only = 1; a.td_levels = td->levels; a.td_stop = td->stop; a.td_ncentral = td->n_central; }
    // the parity view wants every central's key.  The path bound needs the Thm. V.4 DAG to be made of
    // arcs the search traversed: exact extraction, or no central blocking.
    a.prune = (p.want_levels || p.containment) ? 0 : p.prune;
    if (a.prune == 2 && !(p.extract_mode == KGS_EXTRACT_EXACT || !p.block_central)) a.prune = 1;
    a.prune_min = p.prune_min;
    a.mk_min = p.mk_min;
    a.lazy_dag = p.lazy_dag;
    a.rec_max = p.rec_max;
    a.rm_ok = !td && (p.extract_mode == KGS_EXTRACT_EXACT || !p.block_central) ? 1 : 0;
    {   // recorded predecessor DAG: valid for the exact reading (R12), and for any mode without central
        // blocking; the literal Thm. V.4 with blocking and the top-down-only launch use the pre-pass.
        // Auto: on for the single-query (latency) launch, where the pre-pass's rounds of group barriers
        // dominate; off for query groups, where the pre-pass's targeted work (closures of the top
        // candidates only) is less total work than building every touched node's list.
        const bool on = p.dag_record < 0 ? G == 1 : p.dag_record != 0;
        a.dag_record = on && !td && (p.extract_mode == KGS_EXTRACT_EXACT || !p.block_central) ? 1 : 0;
    }
    a.direction = p.direction;
    a.search_only = p.search_only;
    a.pull_ratio = p.pull_ratio;
    a.pull_min = p.pull_min;
    a.tile_light = p.tile_light;
    a.qout = g->d_qout; a.out_hdr = g->d_hdr; a.out_key = g->d_key; a.out_off = g->d_off;
    a.out_nodes = g->d_nodes; a.out_arcs = g->d_arcs;
    a.out_nodes_cap = (long long)g->d_nodes_cap; a.out_arcs_cap = (long long)(g->d_arcs_cap / 2);
    a.out_used = g->d_ctr + 1;
    a.warp_arenas = g->warp_arenas; a.warp_arena_bytes = g->warp_arena_bytes;
    a.cta_arenas = g->cta_arenas; a.cta_arena_bytes = g->cta_arena_bytes;
    a.large_arenas = g->large_arenas; a.large_arena_bytes = g->large_arena_bytes;
    a.large_hash = g->large_hash; a.large_nodes = g->large_nodes; a.large_arcs = g->large_arcs;
    a.big_hash = g->big_hash; a.big_nodes = g->big_nodes; a.big_arcs = g->big_arcs;
    a.huge_hash = g->huge_hash; a.huge_nodes = g->huge_nodes; a.huge_arcs = g->huge_arcs;
    CUDA_TRY(cudaMemsetAsync(g->bars, 0, sizeof(GroupBar) * (size_t)(G + 1), s));   // monotonic group barriers
    CUDA_TRY(cudaEventRecord(g->ev[0], s));
    CUDA_TRY(launch_engine(a, g->grid, s));
    CUDA_TRY(cudaEventRecord(g->ev[1], s));
    g->last_nq = nq; g->last_k = k; g->last_G = G; g->last_p = p;
    g->pending = true;
    return KGS_OK;
}

// Copy the last batch's results back (synchronises s) into results[0..nq).
kgs_status fetch(kgs_graph *g, cudaStream_t s, kgs_result **results) {
    if (!g->pending) return fail(KGS_EINVAL, "no query enqueued on this graph");
    const int nq = g->last_nq, k = g->last_k;
    CUDA_TRY(grow_pinned(&g->h_qout, &g->h_qout_cap, (size_t)nq));
    CUDA_TRY(grow_pinned(&g->h_hdr, &g->h_hdr_cap, (size_t)nq * k * 4));
    CUDA_TRY(grow_pinned(&g->h_key, &g->h_key_cap, (size_t)nq * k));
    CUDA_TRY(grow_pinned(&g->h_off, &g->h_off_cap, (size_t)nq * k * 2));
    CUDA_TRY(cudaMemcpyAsync(g->h_qout, g->d_qout, sizeof(QOut) * nq, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaMemcpyAsync(g->h_hdr, g->d_hdr, sizeof(int32_t) * nq * k * 4, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaMemcpyAsync(g->h_key, g->d_key, sizeof(double) * nq * k, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaMemcpyAsync(g->h_off, g->d_off, sizeof(long long) * nq * k * 2, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaMemcpyAsync(g->h_ctr, g->d_ctr, 4 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    g->pending = false;
    // the arena counters never pass their capacity (engine.cu arena_reserve); clamp anyway
    const size_t used_n = std::min<size_t>((size_t)g->h_ctr[1], g->d_nodes_cap);
    const size_t used_a = std::min<size_t>((size_t)g->h_ctr[2], g->d_arcs_cap / 2);
    CUDA_TRY(grow_pinned(&g->h_nodes, &g->h_nodes_cap, std::max<size_t>(used_n, 1)));
    CUDA_TRY(grow_pinned(&g->h_arcs, &g->h_arcs_cap, std::max<size_t>(2 * used_a, 1)));
    if (used_n) CUDA_TRY(cudaMemcpyAsync(g->h_nodes, g->d_nodes, sizeof(int32_t) * used_n, cudaMemcpyDeviceToHost, s));
    if (used_a) CUDA_TRY(cudaMemcpyAsync(g->h_arcs, g->d_arcs, sizeof(int32_t) * 2 * used_a, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    float ms_all = 0.f;
    cudaEventElapsedTime(&ms_all, g->ev[0], g->ev[1]);
    // a capacity overflow fails a single query; in a batch it marks that query (KGS_STOP_CAPACITY, no
    // answers) and leaves the others
    if (nq == 1 && g->h_qout[0].fatal)
        return fail(KGS_EINTERNAL, "a query exceeded an internal capacity (code " +
                                       std::to_string(g->h_qout[0].fatal) + ")");
    for (int j = 0; j < nq; ++j) {
        QOut &o = g->h_qout[j];
        if (o.fatal) { o.stop_reason = KGS_STOP_CAPACITY; o.count = 0; }
        kgs_result *r = new kgs_result();
        r->n = g->n;
        r->q = g->last_q.empty() ? 0 : g->last_q[j];
        const int cnt = std::max(0, std::min(o.count, k));
        r->ans.resize(cnt); r->nodes.resize(cnt); r->arcs.resize(cnt);
        for (int i = 0; i < cnt; ++i) {
            const int64_t ai = (int64_t)j * k + i;
            const int32_t *h = g->h_hdr + 4 * ai;
            const int32_t *pn = g->h_nodes + g->h_off[2 * ai];
            const int32_t *pa = g->h_arcs + 2 * g->h_off[2 * ai + 1];
            r->nodes[i].assign(pn, pn + h[2]);
            r->arcs[i].assign(pa, pa + 2 * (size_t)h[3]);
            kgs_answer &an = r->ans[i];
            an.central = h[0];
            an.depth = h[1];
            an.score_key = g->h_key[ai];
            an.score = (float)an.score_key;
            an.n_nodes = h[2];
            an.nodes = r->nodes[i].data();
            an.n_arcs = h[3];
            an.arcs = r->arcs[i].data();
        }
        kgs_stats &st = r->stats;
        st.levels = o.levels;
        st.stop_reason = o.stop_reason;
        st.n_centrals = o.n_central;
        st.count = cnt;
        st.frontier_total = (int64_t)o.frontier_total;
        st.arcs_scanned = (int64_t)o.arcs_scanned;
        st.overflow = o.n_overflow;
        st.hits = (int64_t)o.hits;
        st.dag_arcs = (int64_t)o.dag_arcs;
        st.td_arcs = (int64_t)o.td_arcs;
        st.td_arcs_big = (int64_t)o.td_arcs_big;
        st.td_pred_arcs = o.n_parcs;
        st.n_evaluated = (int32_t)o.n_eval;
        st.n_tier4 = (int32_t)o.n_tier4;
        st.group = o.group;
        st.pull_level = o.pull_level;
        st.n_cut = o.n_cut;
        if (o.stop_reason != KGS_STOP_INVALID_QUERY && o.t_end >= o.t_start) {
            st.ms_search = (float)((double)(o.t_search_end - o.t_start) * 1e-6);
            st.ms_topdown = (float)((double)(o.t_end - o.t_search_end) * 1e-6);
            st.ms_total = (float)((double)(o.t_end - o.t_start) * 1e-6);
        }
        st.ms_launch = ms_all;
        for (int i = 0; i < std::min(o.n_stamp, kMaxStamps); ++i) {
            r->ph_tag.push_back(o.stamp_tag[i]);
            r->ph_ns.push_back(o.stamp[i]);
        }
        results[j] = r;
    }
    // parity view of a single query (want_levels): M, activation levels and every central of group 0
    if (g->last_p.want_levels && nq == 1 && results[0]) {
        kgs_result *r = results[0];
        const int64_t n = g->n, q = r->q;
        const DevWork &w = g->works[0];
        uint8_t *dM = nullptr;
        const uint32_t nc = g->h_qout[0].n_central;
        CUDA_TRY(dmalloc(&dM, std::max<int64_t>(n * q, (int64_t)nc * 4) + n));
        uint8_t *dA = dM + std::max<int64_t>(n * q, (int64_t)nc * 4);
        CUDA_TRY(launch_levels_out(w.st, w.M, g->perm, n, (int)q, dM, s));   // rows in input order
        CUDA_TRY(launch_gather_u8(g->act, g->perm, n, dA, s));
        r->M.resize(n * q);
        r->act.resize(n);
        CUDA_TRY(cudaMemcpyAsync(r->M.data(), dM, n * q, cudaMemcpyDeviceToHost, s));
        CUDA_TRY(cudaMemcpyAsync(r->act.data(), dA, n, cudaMemcpyDeviceToHost, s));
        std::vector<int32_t> ids(nc);
        std::vector<uint8_t> dep(nc);
        std::vector<double> key(nc);
        if (nc) {
            int32_t *dI = reinterpret_cast<int32_t *>(dM);   // M was copied out above (stream order)
            CUDA_TRY(launch_to_input_ids(w.centrals, g->orig, nc, dI, s));
            CUDA_TRY(cudaMemcpyAsync(ids.data(), dI, sizeof(int32_t) * nc, cudaMemcpyDeviceToHost, s));
            CUDA_TRY(cudaMemcpyAsync(dep.data(), w.cdepth, nc, cudaMemcpyDeviceToHost, s));
            CUDA_TRY(cudaMemcpyAsync(key.data(), w.ckey, sizeof(double) * nc, cudaMemcpyDeviceToHost, s));
        }
        CUDA_TRY(cudaStreamSynchronize(s));
        cudaFree(dM);
        // identification order -> ascending ids (output formatting of the parity view)
        std::vector<uint32_t> ord(nc);
        for (uint32_t i = 0; i < nc; ++i) ord[i] = i;
        std::sort(ord.begin(), ord.end(), [&](uint32_t x, uint32_t y) { return ids[x] < ids[y]; });
        r->centrals.resize(nc); r->cdepth.resize(nc); r->ckey.resize(nc);
        for (uint32_t i = 0; i < nc; ++i) { r->centrals[i] = ids[ord[i]]; r->cdepth[i] = dep[ord[i]]; r->ckey[i] = key[ord[i]]; }
        r->has_levels = true;
    }
    return KGS_OK;
}

// stage host keyword rows into the padded device layout [nq][KGS_MAX_Q]
kgs_status stage_host(kgs_graph *g, int nq, const int32_t *q_ptr, const int32_t *kw_ids, cudaStream_t s) {
    CUDA_TRY(cudaStreamSynchronize(s));   // pinned staging may still be in use by a previous copy
    CUDA_TRY(grow_pinned(&g->h_kw, &g->h_kw_cap, (size_t)nq * KGS_MAX_Q));
    CUDA_TRY(grow_pinned(&g->h_qlen, &g->h_qlen_cap, (size_t)nq));
    CUDA_TRY(grow_dev(&g->d_kw, &g->d_kw_cap, (size_t)nq * KGS_MAX_Q));
    CUDA_TRY(grow_dev(&g->d_qlen, &g->d_qlen_cap, (size_t)nq));
    g->last_q.assign(nq, 0);
    for (int j = 0; j < nq; ++j) {
        const int q = q_ptr[j + 1] - q_ptr[j];
        g->h_qlen[j] = q;
        g->last_q[j] = q;
        for (int i = 0; i < KGS_MAX_Q; ++i) g->h_kw[(int64_t)j * KGS_MAX_Q + i] = i < q ? kw_ids[q_ptr[j] + i] : -1;
    }
    CUDA_TRY(cudaMemcpyAsync(g->d_kw, g->h_kw, sizeof(int32_t) * nq * KGS_MAX_Q, cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaMemcpyAsync(g->d_qlen, g->h_qlen, sizeof(int32_t) * nq, cudaMemcpyHostToDevice, s));
    return KGS_OK;
}

}  // namespace

extern "C" {

kgs_status kgs_query(kgs_graph *g, const int32_t *kw_ids, int32_t q, int32_t k, const kgs_params *pp,
                     void *cuda_stream, kgs_result **out) {
    if (!g || !kw_ids || !out) return fail(KGS_EINVAL, "null argument");
    *out = nullptr;
    kgs_params p;
    if (pp) p = *pp; else kgs_params_default(&p);
    kgs_status st = check_params(p, k);
    if (st != KGS_OK) return st;
    st = check_query(g, kw_ids, q);
    if (st != KGS_OK) return st;
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    const int32_t qp[2] = {0, q};
    st = stage_host(g, 1, qp, kw_ids, s);
    if (st != KGS_OK) return st;
    st = launch(g, 1, k, p, 1, s);
    if (st != KGS_OK) return st;
    return fetch(g, s, out);
}

kgs_status kgs_query_device(kgs_graph *g, const int32_t *kw_ids_dev, int32_t q, int32_t k, const kgs_params *pp,
                            void *cuda_stream) {
    if (!g || !kw_ids_dev) return fail(KGS_EINVAL, "null argument");
    if (q < 1 || q > KGS_MAX_Q) return fail(KGS_EINVAL, "q must be in [1, 8]");
    kgs_params p;
    if (pp) p = *pp; else kgs_params_default(&p);
    kgs_status st = check_params(p, k);
    if (st != KGS_OK) return st;
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    CUDA_TRY(grow_dev(&g->d_kw, &g->d_kw_cap, (size_t)KGS_MAX_Q));
    CUDA_TRY(grow_dev(&g->d_qlen, &g->d_qlen_cap, (size_t)1));
    CUDA_TRY(cudaMemsetAsync(g->d_kw, 0xFF, sizeof(int32_t) * KGS_MAX_Q, s));
    CUDA_TRY(cudaMemcpyAsync(g->d_kw, kw_ids_dev, sizeof(int32_t) * q, cudaMemcpyDeviceToDevice, s));
    g->last_q.assign(1, q);
    return launch(g, 1, k, p, 1, s, q);   // q travels as a kernel argument
}

kgs_status kgs_query_fetch(kgs_graph *g, void *cuda_stream, kgs_result **out) {
    if (!g || !out) return fail(KGS_EINVAL, "null argument");
    std::lock_guard<std::mutex> lk(g->mu);
    CUDA_TRY(cudaSetDevice(g->device));
    if (g->pending && g->last_nq != 1) return fail(KGS_EINVAL, "the pending launch is a batch: use kgs_query_batch_fetch");
    return fetch(g, (cudaStream_t)cuda_stream, out);
}

kgs_status kgs_query_batch(kgs_graph *g, int32_t n_queries, const int32_t *q_ptr, const int32_t *kw_ids, int32_t k,
                           const kgs_params *pp, int32_t n_groups, void *cuda_stream, kgs_result **results) {
    if (!g || !q_ptr || !kw_ids || !results || n_queries < 1) return fail(KGS_EINVAL, "null argument / empty batch");
    kgs_params p;
    if (pp) p = *pp; else kgs_params_default(&p);
    kgs_status st = check_params(p, k);
    if (st != KGS_OK) return st;
    if (q_ptr[0] != 0) return fail(KGS_EINVAL, "q_ptr[0] must be 0");
    for (int j = 0; j < n_queries; ++j) {
        st = check_query(g, kw_ids + q_ptr[j], q_ptr[j + 1] - q_ptr[j]);
        if (st != KGS_OK) return fail(st, "query " + std::to_string(j) + ": " + g_err);
    }
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    st = stage_host(g, n_queries, q_ptr, kw_ids, s);
    if (st != KGS_OK) return st;
    st = launch(g, n_queries, k, p, n_groups > 0 ? n_groups : 8, s);
    if (st != KGS_OK) return st;
    return fetch(g, s, results);
}

kgs_status kgs_query_batch_device(kgs_graph *g, int32_t n_queries, const int32_t *kw_dev, const int32_t *qlen_dev,
                                  int32_t k, const kgs_params *pp, int32_t n_groups, void *cuda_stream) {
    if (!g || !kw_dev || !qlen_dev || n_queries < 1) return fail(KGS_EINVAL, "null argument / empty batch");
    kgs_params p;
    if (pp) p = *pp; else kgs_params_default(&p);
    kgs_status st = check_params(p, k);
    if (st != KGS_OK) return st;
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    CUDA_TRY(grow_dev(&g->d_kw, &g->d_kw_cap, (size_t)n_queries * KGS_MAX_Q));
    CUDA_TRY(grow_dev(&g->d_qlen, &g->d_qlen_cap, (size_t)n_queries));
    CUDA_TRY(cudaMemcpyAsync(g->d_kw, kw_dev, sizeof(int32_t) * n_queries * KGS_MAX_Q, cudaMemcpyDeviceToDevice, s));
    CUDA_TRY(cudaMemcpyAsync(g->d_qlen, qlen_dev, sizeof(int32_t) * n_queries, cudaMemcpyDeviceToDevice, s));
    g->last_q.clear();
    return launch(g, n_queries, k, p, n_groups > 0 ? n_groups : 8, s);
}

kgs_status kgs_query_batch_fetch(kgs_graph *g, void *cuda_stream, kgs_result **results) {
    if (!g || !results) return fail(KGS_EINVAL, "null argument");
    std::lock_guard<std::mutex> lk(g->mu);
    CUDA_TRY(cudaSetDevice(g->device));
    if (g->last_q.empty() && g->pending) {   // device batch: lengths come back from the device
        std::vector<int32_t> ql(g->last_nq);
        CUDA_TRY(cudaMemcpyAsync(ql.data(), g->d_qlen, sizeof(int32_t) * g->last_nq, cudaMemcpyDeviceToHost,
                                 (cudaStream_t)cuda_stream));
        CUDA_TRY(cudaStreamSynchronize((cudaStream_t)cuda_stream));
        g->last_q.assign(ql.begin(), ql.end());
    }
    return fetch(g, (cudaStream_t)cuda_stream, results);
}

// ------------------------------------------------------------------------------------------ vertex partition
int64_t kgs_vp_slice(int64_t n_nodes, int32_t world) {
    if (n_nodes < 0 || world < 1) return 0;
    const int64_t s = (n_nodes + world - 1) / world;
    return (s + 15) / 16 * 16;
}

kgs_status kgs_vp_begin(kgs_graph *g, const int32_t *kw_ids, int32_t q, int32_t k, const kgs_params *pp, int32_t rank,
                        int32_t world, const kgs_vp_buffers *b, void *cuda_stream, int32_t *info) {
    if (!g || !kw_ids || !b || !info) return fail(KGS_EINVAL, "null argument");
    if (world < 1 || rank < 0 || rank >= world) return fail(KGS_EINVAL, "rank / world out of range");
    if (!b->hm || !b->hm_slice || !b->M || !b->counts || !b->cent || !b->cdep || !b->cent_n)
        return fail(KGS_EINVAL, "null exchange buffer");
    kgs_params p;
    if (pp) p = *pp; else kgs_params_default(&p);
    kgs_status st = check_params(p, k);
    if (st != KGS_OK) return st;
    st = check_query(g, kw_ids, q);
    if (st != KGS_OK) return st;
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    st = prepare(g, p, 1, s);   // activation levels at alpha, one workspace for the top-down
    if (st != KGS_OK) return st;
    const int64_t slice = kgs_vp_slice(g->n, world), n_pad = slice * world;
    if (!g->vp_gate) CUDA_TRY(dmalloc(&g->vp_gate, std::max<int64_t>(g->n, 1)));
    CUDA_TRY(grow_dev(&g->vp_X, &g->vp_X_cap, (size_t)n_pad));
    const int64_t lo = std::min<int64_t>((int64_t)rank * slice, g->n), hi = std::min<int64_t>(lo + slice, g->n);
    if (lo != g->vp_big_lo || hi != g->vp_big_hi) {   // owned nodes pulled by a whole CTA
        if (!g->vp_big) {
            CUDA_TRY(dmalloc(&g->vp_big, std::max<int64_t>(g->n_big_in, 1)));
            CUDA_TRY(dmalloc(&g->vp_nbig_dev, 1));
        }
        DevGraph dg{};
        dg.in_ptr = g->in_ptr;
        CUDA_TRY(launch_vp_biglist(dg, lo, hi, g->vp_big, g->vp_nbig_dev, s));
        int32_t nb = 0;
        CUDA_TRY(cudaMemcpyAsync(&nb, g->vp_nbig_dev, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
        CUDA_TRY(cudaStreamSynchronize(s));
        g->vp_nbig = nb;
        g->vp_big_lo = lo; g->vp_big_hi = hi;
    }
    VpQuery qd{};
    qd.q = q;
    qd.full = (1u << q) - 1u;
    for (int i = 0; i < q; ++i) qd.kw[i] = kw_ids[i];
    VpBufs vb{};
    vb.hm = b->hm; vb.hm_slice = b->hm_slice; vb.M = b->M;
    vb.counts = reinterpret_cast<unsigned long long *>(b->counts);
    vb.chg = reinterpret_cast<long long *>(b->chg);
    vb.cent = b->cent; vb.cdep = b->cdep; vb.cent_n = b->cent_n;
    vb.n_pad = n_pad; vb.lo = lo; vb.hi = hi;
    // an empty T_i: nothing can be central (reading R17)
    std::vector<int64_t> kp(2 * q);
    for (int i = 0; i < q; ++i)
        CUDA_TRY(cudaMemcpyAsync(&kp[2 * i], g->kw_ptr + kw_ids[i], 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    bool empty = false;
    for (int i = 0; i < q; ++i) empty |= kp[2 * i + 1] == kp[2 * i];
    DevGraph dg{};
    dg.n = g->n; dg.kw_ptr = g->kw_ptr; dg.kw_nodes = g->kw_nodes;
    CUDA_TRY(launch_vp_begin(dg, qd, g->act, vb, g->vp_gate, s));
    g->vp = vb; g->vq = qd; g->vp_p = p; g->vp_k = k; g->vp_active = true;
    info[0] = g->amax;
    info[1] = empty ? 1 : 0;
    return KGS_OK;
}

kgs_status kgs_vp_level(kgs_graph *g, int32_t level, void *cuda_stream) {
    if (!g) return fail(KGS_EINVAL, "null argument");
    if (!g->vp_active) return fail(KGS_EINVAL, "kgs_vp_begin was not called");
    if (level < 0 || level >= 254) return fail(KGS_EINVAL, "level out of range");
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    DevGraph dg{};
    dg.n = g->n; dg.in_ptr = g->in_ptr; dg.in_idx = g->in_idx;
    CUDA_TRY(launch_vp_level(dg, g->vq, g->act, g->vp, g->vp_gate, g->vp_X, g->vp_big, g->vp_nbig, level,
                             g->vp_p.block_central ? 1 : 0, s));
    return KGS_OK;
}

kgs_status kgs_vp_waiting(kgs_graph *g, int32_t level, void *cuda_stream) {
    if (!g) return fail(KGS_EINVAL, "null argument");
    if (!g->vp_active) return fail(KGS_EINVAL, "kgs_vp_begin was not called");
    if (level < 0 || level >= 254) return fail(KGS_EINVAL, "level out of range");
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    DevGraph dg{};
    dg.n = g->n; dg.row_ptr = g->row_ptr; dg.col_idx = g->col_idx;
    CUDA_TRY(launch_vp_waiting(dg, g->vq, g->act, g->vp, g->vp_gate, level, g->vp_p.block_central ? 1 : 0, s));
    return KGS_OK;
}

kgs_status kgs_vp_topdown(kgs_graph *g, int64_t n_central, const int32_t *centrals_dev, const uint8_t *depth_dev,
                          int32_t levels, int32_t stop_reason, void *cuda_stream, kgs_result **out) {
    if (!g || !out) return fail(KGS_EINVAL, "null argument");
    *out = nullptr;
    if (!g->vp_active) return fail(KGS_EINVAL, "kgs_vp_begin was not called");
    if (n_central < 0 || n_central > g->n || (n_central > 0 && (!centrals_dev || !depth_dev)))
        return fail(KGS_EINVAL, "central list");
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    kgs_params p = g->vp_p;
    if (p.prune == 2) p.prune = 1;   // the lightest-path rows are written by the single-GPU search only
    kgs_status st = prepare(g, p, 1, s);
    if (st != KGS_OK) return st;
    const DevWork &w = g->works[0];
    // the replicated final state in the engine's layout (DevWork::st, M, centrals)
    CUDA_TRY(launch_vp_pack_st(g->vp.hm, g->vp_gate, g->act, g->n, w.st, s));
    CUDA_TRY(cudaMemcpyAsync(w.M, g->vp.M, (size_t)g->n * 8, cudaMemcpyDeviceToDevice, s));
    if (n_central) {
        CUDA_TRY(cudaMemcpyAsync(w.centrals, centrals_dev, sizeof(int32_t) * n_central, cudaMemcpyDeviceToDevice, s));
        CUDA_TRY(cudaMemcpyAsync(w.cdepth, depth_dev, (size_t)n_central, cudaMemcpyDeviceToDevice, s));
    }
    const int32_t qp[2] = {0, g->vq.q};
    st = stage_host(g, 1, qp, g->vq.kw, s);
    if (st != KGS_OK) return st;
    const TdOnly td{levels, stop_reason, (uint32_t)n_central};
    st = launch(g, 1, g->vp_k, p, 1, s, 0, &td);
    if (st != KGS_OK) return st;
    g->vp_active = false;
    return fetch(g, s, out);
}

int32_t kgs_result_count(const kgs_result *r) { return r ? (int32_t)r->ans.size() : 0; }

kgs_status kgs_result_answer(const kgs_result *r, int32_t i, kgs_answer *a) {
    if (!r || !a || i < 0 || i >= (int32_t)r->ans.size()) return fail(KGS_EINVAL, "answer index out of range");
    *a = r->ans[i];
    return KGS_OK;
}

kgs_status kgs_result_levels(const kgs_result *r, uint8_t *M, int64_t cap) {
    if (!r || !M) return fail(KGS_EINVAL, "null argument");
    if (!r->has_levels) return fail(KGS_EINVAL, "query was run without want_levels");
    if (cap < (int64_t)r->M.size()) return fail(KGS_EINVAL, "buffer too small");
    std::memcpy(M, r->M.data(), r->M.size());
    return KGS_OK;
}

kgs_status kgs_result_activation(const kgs_result *r, uint8_t *a, int64_t cap) {
    if (!r || !a) return fail(KGS_EINVAL, "null argument");
    if (!r->has_levels) return fail(KGS_EINVAL, "query was run without want_levels");
    if (cap < (int64_t)r->act.size()) return fail(KGS_EINVAL, "buffer too small");
    std::memcpy(a, r->act.data(), r->act.size());
    return KGS_OK;
}

kgs_status kgs_result_centrals(const kgs_result *r, int32_t *ids, uint8_t *depth, double *score_key, int64_t cap,
                               int64_t *n) {
    if (!r || !n) return fail(KGS_EINVAL, "null argument");
    if (!r->has_levels) return fail(KGS_EINVAL, "query was run without want_levels");
    *n = (int64_t)r->centrals.size();
    if (cap < *n) return fail(KGS_EINVAL, "buffer too small");
    if (ids) std::memcpy(ids, r->centrals.data(), sizeof(int32_t) * r->centrals.size());
    if (depth) std::memcpy(depth, r->cdepth.data(), r->cdepth.size());
    if (score_key) std::memcpy(score_key, r->ckey.data(), sizeof(double) * r->ckey.size());
    return KGS_OK;
}

kgs_status kgs_result_sizes(const kgs_result *r, int32_t *count, int64_t *total_nodes, int64_t *total_arcs) {
    if (!r || !count || !total_nodes || !total_arcs) return fail(KGS_EINVAL, "null argument");
    *count = (int32_t)r->ans.size();
    int64_t tn = 0, ta = 0;
    for (const auto &a : r->ans) { tn += a.n_nodes; ta += a.n_arcs; }
    *total_nodes = tn;
    *total_arcs = ta;
    return KGS_OK;
}

kgs_status kgs_result_export(const kgs_result *r, int32_t *central, int32_t *depth, double *score_key,
                             int64_t *node_off, int32_t *nodes, int64_t *arc_off, int32_t *arcs) {
    if (!r || !central || !depth || !score_key || !node_off || !arc_off) return fail(KGS_EINVAL, "null argument");
    int64_t tn = 0, ta = 0;
    node_off[0] = 0;
    arc_off[0] = 0;
    for (size_t i = 0; i < r->ans.size(); ++i) {
        const kgs_answer &a = r->ans[i];
        central[i] = a.central;
        depth[i] = a.depth;
        score_key[i] = a.score_key;
        if (a.n_nodes) {
            if (!nodes) return fail(KGS_EINVAL, "null nodes buffer");
            std::memcpy(nodes + tn, a.nodes, sizeof(int32_t) * (size_t)a.n_nodes);
        }
        if (a.n_arcs) {
            if (!arcs) return fail(KGS_EINVAL, "null arcs buffer");
            std::memcpy(arcs + 2 * ta, a.arcs, sizeof(int32_t) * 2 * (size_t)a.n_arcs);
        }
        tn += a.n_nodes;
        ta += a.n_arcs;
        node_off[i + 1] = tn;
        arc_off[i + 1] = ta;
    }
    return KGS_OK;
}

kgs_status kgs_result_stats(const kgs_result *r, kgs_stats *s) {
    if (!r || !s) return fail(KGS_EINVAL, "null argument");
    *s = r->stats;
    return KGS_OK;
}

kgs_status kgs_result_phases(const kgs_result *r, int32_t *tags, uint64_t *t_ns, int32_t cap, int32_t *n) {
    if (!r || !n) return fail(KGS_EINVAL, "null argument");
    *n = (int32_t)r->ph_tag.size();
    const int32_t m = std::min<int32_t>(cap, *n);
    for (int32_t i = 0; i < m; ++i) {
        if (tags) tags[i] = r->ph_tag[i];
        if (t_ns) t_ns[i] = r->ph_ns[i];
    }
    return KGS_OK;
}

void kgs_result_free(kgs_result *r) { delete r; }

}  // extern "C"
