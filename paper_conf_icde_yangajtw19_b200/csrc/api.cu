// api.cu — the C-ABI of libkgs (include/kgs.h): graph loading, query orchestration, result handles.
// Host code only orchestrates: every step of the query path runs in the kernels of search.cu and
// topdown.cu.  There is no CPU fallback; without a CUDA device every call fails with KGS_ECUDA.
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

}  // namespace

// ------------------------------------------------------------------------------------------ kernels
namespace kgs {
__global__ void k_validate(DevGraph g, int32_t *err) {
    const int64_t gt = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = gt; v < g.n; v += gs) {
        if (g.row_ptr[v + 1] < g.row_ptr[v]) atomicOr(err, 1);
        const float w = g.weight[v];
        if (!(w >= 0.0f && w <= 1.0f)) atomicOr(err, 4);
    }
    for (int64_t j = gt; j < g.m; j += gs) {
        const int32_t x = g.col_idx[j];
        if (x < 0 || x >= g.n) atomicOr(err, 2);
    }
    for (int64_t t = gt; t < g.n_kw; t += gs) {
        const int64_t b = g.kw_ptr[t], e = g.kw_ptr[t + 1];
        if (e < b) { atomicOr(err, 8); continue; }
        for (int64_t j = b; j < e; ++j) {
            const int32_t v = g.kw_nodes[j];
            if (v < 0 || v >= g.n || (j > b && v <= g.kw_nodes[j - 1])) { atomicOr(err, 16); break; }
        }
    }
}
cudaError_t launch_validate(const DevGraph &g, int32_t *err, cudaStream_t s) {
    k_validate<<<148 * 8, 256, 0, s>>>(g, err);
    return cudaGetLastError();
}

// M for parity output: n*q bytes, 255 where the hit bit is clear
__global__ void k_levels_out(QueryArgs a, uint8_t *out) {
    const int64_t gt = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = gt; v < a.g.n; v += gs) {
        const uint32_t hm = a.w.st[v] & 0xFFu;
        for (int i = 0; i < a.q; ++i)
            out[v * a.q + i] = ((hm >> i) & 1u) ? a.w.M[v * 8 + i] : (uint8_t)KGS_INF_LEVEL;
    }
}
cudaError_t launch_levels_out(const QueryArgs &a, uint8_t *out, cudaStream_t s) {
    k_levels_out<<<148 * 8, 256, 0, s>>>(a, out);
    return cudaGetLastError();
}
}  // namespace kgs

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
    int64_t n_big = 0, n_big_in = 0;   // nodes with more than kBigDeg out- / in-arcs
    // workspace
    DevWork w{};
    uint32_t *amax_dev = nullptr;
    double act_alpha = -1.0;
    int amax = 0;
    int R_alloc = 0;
    double dpow_lambda = -1.0;
    Ctl *ctl_pair[2] = {nullptr, nullptr};
    int query_no = 0;
    bool state_valid = false;  // st/nm/fbits consistent with act and R of the last query
    int last_R = 0;
    int search_grid = 0, search_block = 512, select_grid = 0, extract_grid = 0;
    // pinned host staging
    Ctl *h_ctl = nullptr;
    int32_t *h_kw = nullptr;
    double *h_dpow = nullptr;
    int32_t *h_hdr = nullptr;
    double *h_key = nullptr;
    long long *h_off = nullptr;
    int32_t *h_nodes = nullptr, *h_arcs = nullptr;   // pinned staging of the emitted answer lists
    size_t h_nodes_cap = 0, h_arcs_cap = 0;
    cudaEvent_t ev[4];
    std::mutex mu;
    // last enqueued query (for kgs_query_fetch)
    int last_q = 0, last_k = 0;
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

extern "C" {

const char *kgs_last_error(void) { return g_err.c_str(); }
const char *kgs_version(void) { return "kgs 0.1 sm_100a (" __DATE__ ")"; }

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
}

void kgs_free_graph(kgs_graph *g) {
    if (!g) return;
    cudaSetDevice(g->device);
    cudaDeviceSynchronize();
    void *ptrs[] = {g->row_ptr, g->col_idx, g->kw_ptr, g->kw_nodes, g->weight, g->cls, g->w.act, g->w.st,
                    g->w.nm, g->w.M, g->w.qlight, g->w.qbig, g->w.pd_bits, g->w.fbits, g->w.touched,
                    g->w.centrals, g->w.cdepth, g->w.ckey, g->w.overflow, g->w.cflag, g->w.sel, g->w.kw_dev,
                    g->w.dpow, g->ctl_pair[0], g->ctl_pair[1], g->w.ans_hdr, g->w.ans_key, g->w.ans_off,
                    g->w.arena_nodes, g->w.arena_arcs, g->w.big_ws, g->amax_dev, g->w.pd_state, g->w.pd_cid,
                    g->w.pd_touched, g->w.pd_qlight, g->w.pd_qbig, g->w.pcnt, g->w.pred_ptr,
                    g->w.pred_u, g->w.pred_b, g->w.pa_u, g->w.pa_x, g->w.pa_b, g->w.pa_slot, g->w.scan_tmp};
    for (void *p : ptrs) if (p) cudaFree(p);
    if (!g->symmetric) { cudaFree(g->in_ptr); cudaFree(g->in_idx); cudaFree(g->cls_in); }
    void *hp[] = {g->h_ctl, g->h_kw, g->h_dpow, g->h_hdr, g->h_key, g->h_off, g->h_nodes, g->h_arcs};
    for (void *p : hp) if (p) cudaFreeHost(p);
    for (auto &e : g->ev) cudaEventDestroy(e);
    delete g;
}

kgs_status kgs_load_graph(const kgs_graph_desc *d, kgs_graph **out) {
    if (!d || !out) return fail(KGS_EINVAL, "null argument");
    *out = nullptr;
    if (d->n_nodes < 0 || d->n_nodes >= (int64_t(1) << 31) || d->n_arcs < 0 || d->n_keywords < 1 ||
        !(d->avg_dist_A > 0.0) || !std::isfinite(d->avg_dist_A))
        return fail(KGS_EINVAL, "n_nodes / n_arcs / n_keywords / avg_dist_A out of range");
    if (d->n_nodes > 0 && (!d->row_ptr || !d->weight)) return fail(KGS_EINVAL, "missing row_ptr / weight");
    if (d->n_arcs > 0 && !d->col_idx) return fail(KGS_EINVAL, "missing col_idx");
    if (!d->kw_ptr) return fail(KGS_EINVAL, "missing kw_ptr");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
        return fail(KGS_ECUDA, "no CUDA device available (libkgs has no CPU path)");
    if (d->device < 0 || d->device >= ndev) return fail(KGS_EINVAL, "device ordinal out of range");
    CUDA_TRY(cudaSetDevice(d->device));
    const bool on_dev = (d->flags & KGS_INPUT_DEVICE_PTRS) != 0;
    const cudaMemcpyKind kind = on_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    const int64_t n = d->n_nodes, m = d->n_arcs, V = d->n_keywords;

    // host-side structural checks on the offsets (cheap; also needed for class counts / reverse CSR)
    std::vector<int64_t> rp(n + 1), kp(V + 1);
    if (n >= 0) {
        if (on_dev) CUDA_TRY(cudaMemcpy(rp.data(), d->row_ptr, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToHost));
        else std::memcpy(rp.data(), d->row_ptr, sizeof(int64_t) * (n + 1));
    }
    if (on_dev) CUDA_TRY(cudaMemcpy(kp.data(), d->kw_ptr, sizeof(int64_t) * (V + 1), cudaMemcpyDeviceToHost));
    else std::memcpy(kp.data(), d->kw_ptr, sizeof(int64_t) * (V + 1));
    if (rp[0] != 0 || rp[n] != m) return fail(KGS_EINVAL, "row_ptr[0] must be 0 and row_ptr[n] == n_arcs");
    if (kp[0] != 0 || kp[V] < 0) return fail(KGS_EINVAL, "kw_ptr[0] must be 0");
    for (int64_t t = 0; t < V; ++t)
        if (kp[t + 1] < kp[t]) return fail(KGS_EINVAL, "kw_ptr not non-decreasing");
    const int64_t P = kp[V];
    if (P > 0 && !d->kw_nodes) return fail(KGS_EINVAL, "missing kw_nodes");

    kgs_graph *g = new kgs_graph();
    g->device = d->device; g->n = n; g->m = m; g->n_kw = V; g->A = d->avg_dist_A;
    g->symmetric = d->symmetric ? 1 : 0;
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
    G_TRY(launch_degree_class(g->row_ptr, n, g->cls, 0));
    for (int64_t v = 0; v < n; ++v) {
        const int64_t dg_ = rp[v + 1] - rp[v];
        if (dg_ > kBigDeg) ++g->n_big;
    }
    // reverse CSR for extraction along in-arcs (reading R1)
    if (g->symmetric) {
        g->in_ptr = g->row_ptr; g->in_idx = g->col_idx; g->cls_in = g->cls;
        g->n_big_in = g->n_big;
    } else {
        std::vector<int32_t> ci(m);
        if (on_dev) G_TRY(cudaMemcpy(ci.data(), d->col_idx, sizeof(int32_t) * m, cudaMemcpyDeviceToHost));
        else std::memcpy(ci.data(), d->col_idx, sizeof(int32_t) * m);
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
        for (int64_t v = 0; v < n; ++v) {
            const int64_t dg_ = ip[v + 1] - ip[v];
            if (dg_ > kBigDeg) ++g->n_big_in;
        }
    }
    // per-query workspace sized for n (rings are sized at the first query: they depend on alpha)
    DevWork &w = g->w;
    G_TRY(dmalloc(&w.act, n));
    G_TRY(dmalloc(&w.st, n));
    G_TRY(dmalloc(&w.nm, (n + 3) / 4));
    G_TRY(dmalloc(&w.M, n * 8));
    G_TRY(dmalloc(&w.touched, n));
    G_TRY(dmalloc(&w.centrals, n));
    G_TRY(dmalloc(&w.cdepth, n));
    G_TRY(dmalloc(&w.ckey, n));
    G_TRY(dmalloc(&w.overflow, n));
    G_TRY(dmalloc(&w.cflag, n));
    G_TRY(dmalloc(&w.sel, KGS_MAX_K));
    G_TRY(dmalloc(&w.kw_dev, KGS_MAX_Q));
    G_TRY(dmalloc(&w.dpow, 256));
    G_TRY(dmalloc(&g->ctl_pair[0], 1));
    G_TRY(dmalloc(&g->ctl_pair[1], 1));
    G_TRY(cudaMemset(g->ctl_pair[0], 0, sizeof(Ctl)));
    G_TRY(cudaMemset(g->ctl_pair[1], 0, sizeof(Ctl)));
    G_TRY(dmalloc(&w.ans_hdr, 4 * KGS_MAX_K));
    G_TRY(dmalloc(&w.ans_key, KGS_MAX_K));
    G_TRY(dmalloc(&w.ans_off, 2 * KGS_MAX_K));
    w.arena_nodes_cap = (long long)KGS_MAX_K * kExtNodes + 4 * (long long)kBigNodes;
    w.arena_arcs_cap = (long long)KGS_MAX_K * kExtArcs + 4 * (long long)kBigArcs;
    G_TRY(dmalloc(&w.arena_nodes, (size_t)w.arena_nodes_cap));
    G_TRY(dmalloc(&w.arena_arcs, 2 * (size_t)w.arena_arcs_cap));
    w.big_hcap = kBigHash; w.big_ncap = kBigNodes; w.big_acap = kBigArcs; w.big_ctas = kBigCtas;
    w.big_bytes = big_arena_bytes(kBigHash, kBigNodes, kBigArcs, false);
    w.big_bytes_emit = big_arena_bytes(kBigHash, kBigNodes, kBigArcs, true);
    G_TRY(cudaMalloc(&w.big_ws, w.big_bytes_emit * kBigCtas));
    G_TRY(dmalloc(&g->amax_dev, 1));
    G_TRY(cudaMallocHost(&g->h_ctl, sizeof(Ctl)));
    G_TRY(cudaMallocHost(&g->h_kw, sizeof(int32_t) * KGS_MAX_Q));
    G_TRY(cudaMallocHost(&g->h_dpow, sizeof(double) * 256));
    G_TRY(cudaMallocHost(&g->h_hdr, sizeof(int32_t) * 4 * KGS_MAX_K));
    G_TRY(cudaMallocHost(&g->h_key, sizeof(double) * KGS_MAX_K));
    G_TRY(cudaMallocHost(&g->h_off, sizeof(long long) * 2 * KGS_MAX_K));
    w.W = ((n + 31) / 32 + 7) / 8 * 8;   // words per bitmap, a multiple of 8 (16-byte vector access)
    G_TRY(dmalloc(&w.qlight, n));
    G_TRY(dmalloc(&w.qbig, g->n_big));
    // shared predecessor DAG of the top-down pre-pass
    w.pcap = std::max<int64_t>(std::min<int64_t>(m, int64_t(64) << 20), 1 << 20);
    G_TRY(dmalloc(&w.pd_state, n));
    G_TRY(dmalloc(&w.pd_cid, n));
    G_TRY(dmalloc(&w.pd_touched, n));
    G_TRY(dmalloc(&w.pd_bits, 2 * w.W));
    G_TRY(dmalloc(&w.pd_qlight, n));
    G_TRY(dmalloc(&w.pd_qbig, g->n_big_in));
    G_TRY(dmalloc(&w.pcnt, n));
    G_TRY(dmalloc(&w.pred_ptr, n + 1));
    G_TRY(dmalloc(&w.pred_u, (size_t)w.pcap));
    G_TRY(dmalloc(&w.pred_b, (size_t)w.pcap));
    G_TRY(dmalloc(&w.pa_u, (size_t)w.pcap));
    G_TRY(dmalloc(&w.pa_x, (size_t)w.pcap));
    G_TRY(dmalloc(&w.pa_b, (size_t)w.pcap));
    G_TRY(dmalloc(&w.pa_slot, (size_t)w.pcap));
    G_TRY(dmalloc(&w.scan_tmp, 4096));
    g->search_grid = search_max_grid(g->device, g->search_block);
    g->select_grid = select_max_grid(g->device);
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g->device);
    g->extract_grid = sms * 4;
    if (g->search_grid <= 0 || g->select_grid <= 0) return bail(fail(KGS_ECUDA, "occupancy query failed"));
    G_TRY(cudaDeviceSynchronize());
#undef G_TRY
    *out = g;
    return KGS_OK;
}

}  // extern "C"

// ------------------------------------------------------------------------------------------ query
namespace {

kgs_status check_params(const kgs_graph *g, const kgs_params &p, int32_t q, int32_t k) {
    if (q < 1 || q > KGS_MAX_Q) return fail(KGS_EINVAL, "q must be in [1, 8]");
    if (k < 1 || k > KGS_MAX_K) return fail(KGS_EINVAL, "k must be in [1, 4096]");
    if (!(p.alpha > 0.0 && p.alpha < 1.0)) return fail(KGS_EINVAL, "alpha must be in (0, 1)");
    if (!(p.lambda >= 0.0) || !std::isfinite(p.lambda)) return fail(KGS_EINVAL, "lambda must be >= 0");
    if (p.max_depth < 1 || p.max_depth > 254) return fail(KGS_EINVAL, "max_depth must be in [1, 254]");
    if (p.extract_mode != KGS_EXTRACT_EXACT && p.extract_mode != KGS_EXTRACT_LITERAL)
        return fail(KGS_EINVAL, "extract_mode");
    (void)g;
    return KGS_OK;
}

// Enqueue the whole query on stream s; keyword ids already in g->w.kw_dev.
kgs_status enqueue(kgs_graph *g, int32_t q, int32_t k, const kgs_params &p, cudaStream_t s) {
    DevWork &w = g->w;
    bool full_reset = !g->state_valid;
    if (p.alpha != g->act_alpha) {
        // activation cache (Eqs. 3-5) — recomputed only when alpha changes; amax sizes the rings
        CUDA_TRY(launch_activation(g->weight, g->n, g->A, p.alpha, w.act, g->amax_dev, s));
        uint32_t amax = 0;
        CUDA_TRY(cudaMemcpyAsync(&g->h_ctl->levels, g->amax_dev, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        CUDA_TRY(cudaStreamSynchronize(s));
        std::memcpy(&amax, &g->h_ctl->levels, sizeof(uint32_t));
        g->amax = (int)amax;
        g->act_alpha = p.alpha;
        full_reset = true;
    }
    const int R = g->amax + 2;
    if (R > g->R_alloc) {
        CUDA_TRY(cudaStreamSynchronize(s));
        if (w.fbits) cudaFree(w.fbits);
        CUDA_TRY(dmalloc(&w.fbits, (size_t)R * (size_t)w.W));
        g->R_alloc = R;
        full_reset = true;
    }
    if (R != g->last_R) full_reset = true;
    w.R = R;
    if (p.lambda != g->dpow_lambda) {
        // Eq. 6 depth factor d^lambda from the host libm (reading R15), one value per depth
        CUDA_TRY(cudaStreamSynchronize(s));
        for (int dd = 0; dd < 256; ++dd) g->h_dpow[dd] = std::pow((double)dd, p.lambda);
        CUDA_TRY(cudaMemcpyAsync(w.dpow, g->h_dpow, sizeof(double) * 256, cudaMemcpyHostToDevice, s));
        g->dpow_lambda = p.lambda;
    }
    Ctl *cur = g->ctl_pair[g->query_no & 1];
    Ctl *prev = g->ctl_pair[(g->query_no + 1) & 1];
    CUDA_TRY(cudaMemsetAsync(cur, 0, sizeof(Ctl), s));
    w.ctl = cur;
    w.prev = full_reset ? nullptr : prev;

    QueryArgs a{};
    a.g.n = g->n; a.g.m = g->m; a.g.row_ptr = g->row_ptr; a.g.col_idx = g->col_idx;
    a.g.in_ptr = g->in_ptr; a.g.in_idx = g->in_idx; a.g.weight = g->weight; a.g.cls = g->cls;
    a.g.cls_in = g->cls_in;
    a.g.n_kw = g->n_kw; a.g.kw_ptr = g->kw_ptr; a.g.kw_nodes = g->kw_nodes;
    a.w = w;
    a.q = q; a.k = k; a.max_depth = p.max_depth; a.block_central = p.block_central ? 1 : 0;
    a.extract_mode = p.extract_mode; a.level_cover = p.level_cover ? 1 : 0;
    a.full_reset = full_reset ? 1 : 0;
    a.prev_R = g->last_R;

    CUDA_TRY(cudaEventRecord(g->ev[0], s));
    CUDA_TRY(launch_search(a, g->search_grid, g->search_block, s));
    CUDA_TRY(cudaEventRecord(g->ev[1], s));
    CUDA_TRY(launch_extract(a, g->extract_grid, s));
    CUDA_TRY(launch_select(a, g->select_grid, s));
    CUDA_TRY(launch_emit(a, std::min<int>(k, w.big_ctas), s));
    CUDA_TRY(cudaEventRecord(g->ev[2], s));
    g->query_no++;
    g->state_valid = true;
    g->last_R = R;
    g->last_q = q; g->last_k = k; g->last_p = p;
    g->pending = true;
    return KGS_OK;
}

kgs_status fetch(kgs_graph *g, cudaStream_t s, kgs_result **out) {
    if (!g->pending) return fail(KGS_EINVAL, "no query enqueued on this graph");
    DevWork &w = g->w;
    Ctl *cur = g->ctl_pair[(g->query_no + 1) & 1];  // the last enqueued query's block
    CUDA_TRY(cudaMemcpyAsync(g->h_ctl, cur, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaMemcpyAsync(g->h_hdr, w.ans_hdr, sizeof(int32_t) * 4 * g->last_k, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaMemcpyAsync(g->h_key, w.ans_key, sizeof(double) * g->last_k, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaMemcpyAsync(g->h_off, w.ans_off, sizeof(long long) * 2 * g->last_k, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    g->pending = false;
    const Ctl &c = *g->h_ctl;
    if (c.fatal) return fail(KGS_EINTERNAL, "a Central Graph exceeded the large-graph extractor capacity");
    kgs_result *r = new kgs_result();
    r->n = g->n; r->q = g->last_q;
    const int cnt = (int)std::min<uint32_t>(c.sel_count, (uint32_t)g->last_k);
    r->ans.resize(cnt);
    r->nodes.resize(cnt);
    r->arcs.resize(cnt);
    // the emitted node / arc lists: one pinned copy of each used arena prefix, then split on the host
    const size_t used_n = (size_t)c.arena_used[0], used_a = (size_t)c.arena_used[1];
    if (used_n > g->h_nodes_cap) {
        if (g->h_nodes) cudaFreeHost(g->h_nodes);
        g->h_nodes_cap = std::max<size_t>(used_n, 2 * g->h_nodes_cap);
        CUDA_TRY(cudaMallocHost(&g->h_nodes, sizeof(int32_t) * g->h_nodes_cap));
    }
    if (2 * used_a > g->h_arcs_cap) {
        if (g->h_arcs) cudaFreeHost(g->h_arcs);
        g->h_arcs_cap = std::max<size_t>(2 * used_a, 2 * g->h_arcs_cap);
        CUDA_TRY(cudaMallocHost(&g->h_arcs, sizeof(int32_t) * g->h_arcs_cap));
    }
    if (used_n) CUDA_TRY(cudaMemcpyAsync(g->h_nodes, w.arena_nodes, sizeof(int32_t) * used_n, cudaMemcpyDeviceToHost, s));
    if (used_a) CUDA_TRY(cudaMemcpyAsync(g->h_arcs, w.arena_arcs, sizeof(int32_t) * 2 * used_a, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    for (int i = 0; i < cnt; ++i) {
        const int32_t *h = g->h_hdr + 4 * i;
        const int32_t *pn = g->h_nodes + g->h_off[2 * i];
        const int32_t *pa = g->h_arcs + 2 * g->h_off[2 * i + 1];
        r->nodes[i].assign(pn, pn + h[2]);
        r->arcs[i].assign(pa, pa + 2 * (size_t)h[3]);
    }
    if (g->last_p.want_levels) {
        const int64_t n = g->n, q = g->last_q;
        uint8_t *dM = nullptr;
        CUDA_TRY(dmalloc(&dM, n * q));
        QueryArgs a{};
        a.g.n = n; a.w = w; a.q = (int)q;
        CUDA_TRY(launch_levels_out(a, dM, s));
        r->M.resize(n * q);
        r->act.resize(n);
        CUDA_TRY(cudaMemcpyAsync(r->M.data(), dM, n * q, cudaMemcpyDeviceToHost, s));
        CUDA_TRY(cudaMemcpyAsync(r->act.data(), w.act, n, cudaMemcpyDeviceToHost, s));
        const uint32_t nc = c.n_central;
        std::vector<int32_t> ids(nc);
        std::vector<uint8_t> dep(nc);
        std::vector<double> key(nc);
        if (nc) {
            CUDA_TRY(cudaMemcpyAsync(ids.data(), w.centrals, sizeof(int32_t) * nc, cudaMemcpyDeviceToHost, s));
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
    CUDA_TRY(cudaStreamSynchronize(s));
    for (int i = 0; i < cnt; ++i) {
        const int32_t *h = g->h_hdr + 4 * i;
        kgs_answer &an = r->ans[i];
        an.central = h[0];
        an.depth = h[1];
        an.score_key = g->h_key[i];
        an.score = (float)an.score_key;
        an.n_nodes = h[2];
        an.nodes = r->nodes[i].data();
        an.n_arcs = h[3];
        an.arcs = r->arcs[i].data();
    }
    kgs_stats &st = r->stats;
    st.levels = c.levels;
    st.stop_reason = c.stop_reason;
    st.n_centrals = c.n_central;
    st.count = cnt;
    st.frontier_total = (int64_t)c.frontier_total;
    st.arcs_scanned = (int64_t)c.arcs_scanned;
    st.overflow = c.n_overflow;
    st.hits = (int64_t)c.hits;
    st.td_arcs = (int64_t)c.td_arcs;
    st.td_pred_arcs = (int64_t)c.n_parcs;
    for (int i = 0; i < std::min(c.n_stamp, 64); ++i) {
        r->ph_tag.push_back(c.stamp_tag[i]);
        r->ph_ns.push_back(c.stamp[i]);
    }
    cudaEventElapsedTime(&st.ms_search, g->ev[0], g->ev[1]);
    cudaEventElapsedTime(&st.ms_topdown, g->ev[1], g->ev[2]);
    cudaEventElapsedTime(&st.ms_total, g->ev[0], g->ev[2]);
    *out = r;
    return KGS_OK;
}

}  // namespace

extern "C" {

kgs_status kgs_query_device(kgs_graph *g, const int32_t *kw_ids_dev, int32_t q, int32_t k, const kgs_params *pp,
                            void *cuda_stream) {
    if (!g || !kw_ids_dev) return fail(KGS_EINVAL, "null argument");
    kgs_params p;
    if (pp) p = *pp; else kgs_params_default(&p);
    kgs_status st = check_params(g, p, q, k);
    if (st != KGS_OK) return st;
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    CUDA_TRY(cudaMemcpyAsync(g->w.kw_dev, kw_ids_dev, sizeof(int32_t) * q, cudaMemcpyDeviceToDevice, s));
    return enqueue(g, q, k, p, s);
}

kgs_status kgs_query_fetch(kgs_graph *g, void *cuda_stream, kgs_result **out) {
    if (!g || !out) return fail(KGS_EINVAL, "null argument");
    std::lock_guard<std::mutex> lk(g->mu);
    CUDA_TRY(cudaSetDevice(g->device));
    return fetch(g, (cudaStream_t)cuda_stream, out);
}

kgs_status kgs_query(kgs_graph *g, const int32_t *kw_ids, int32_t q, int32_t k, const kgs_params *pp,
                     void *cuda_stream, kgs_result **out) {
    if (!g || !kw_ids || !out) return fail(KGS_EINVAL, "null argument");
    *out = nullptr;
    kgs_params p;
    if (pp) p = *pp; else kgs_params_default(&p);
    kgs_status st = check_params(g, p, q, k);
    if (st != KGS_OK) return st;
    for (int i = 0; i < q; ++i) {
        if (kw_ids[i] < 0 || kw_ids[i] >= g->n_kw) return fail(KGS_EINVAL, "keyword id out of range");
        for (int j = 0; j < i; ++j)
            if (kw_ids[j] == kw_ids[i]) return fail(KGS_EINVAL, "duplicate keyword id");
    }
    std::lock_guard<std::mutex> lk(g->mu);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CUDA_TRY(cudaSetDevice(g->device));
    std::memcpy(g->h_kw, kw_ids, sizeof(int32_t) * q);
    CUDA_TRY(cudaMemcpyAsync(g->w.kw_dev, g->h_kw, sizeof(int32_t) * q, cudaMemcpyHostToDevice, s));
    st = enqueue(g, q, k, p, s);
    if (st != KGS_OK) return st;
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
