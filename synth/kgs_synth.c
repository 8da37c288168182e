/* kgs_synth.c — seeded synthetic inputs for the Central Graph keyword search hot path.
 *
 * This module generates INPUTS only (graph, node weights, keyword inverted index).  It holds none of
 * the method's query arithmetic: no activation levels (Eqs. 3-5), no BFS, no extraction, no scoring.
 * Both the CPU oracle (oracle/) and the CUDA path (paper_conf_icde_yangajtw19_b200/) consume what it
 * writes; neither shares code with the other.
 *
 * What it builds (recipe in DESIGN.md "Input recipe"):
 *   - R-MAT(a=.57,b=.19,c=.19,d=.05) edge draws, vertex ids permuted, self-loops dropped, deduplicated,
 *     symmetrised -> CSR (row_ptr int64, col_idx int32), rows sorted ascending.  Optional planted hubs.
 *   - per-edge labels (Zipf over R labels; hub edges share one label), node weight by the paper's
 *     "degree of summary" Eq. 2 with min-max normalisation (L178-180), snapped
 *     to the 2^-24 grid (reading R15).  Or uniform random weights on the grid (config C1).
 *   - per-node keywords: 1 + Poisson(2) words drawn from Zipf(s) over the vocabulary, inverted into
 *     kw_ptr (int64) / kw_nodes (int32, ascending per keyword).
 *   - A, the average shortest distance, estimated by sampling pairs.
 *
 * Every random draw is a counter-based hash of (seed, stream, index), so results do not depend on
 * the number of OpenMP threads.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static inline uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
static inline uint64_t rng3(uint64_t seed, uint64_t stream, uint64_t idx) {
    return mix64(mix64(seed ^ (stream * 0xD1B54A32D192ED03ULL)) + idx * 0x9E3779B97F4A7C15ULL);
}
static inline double u01(uint64_t r) { return (double)(r >> 11) * 0x1.0p-53; }

enum { ST_RMAT = 1, ST_PERM = 2, ST_LABEL = 3, ST_WORDS = 4, ST_NWORDS = 5, ST_HUB = 6, ST_WEIGHT = 7, ST_APAIR = 8 };

typedef struct {
    int64_t n, n_arcs;
    int64_t *row_ptr;
    int32_t *col_idx;
    float *weight;
    int64_t n_keywords, n_postings;
    int64_t *kw_ptr;
    int32_t *kw_nodes;
    double A;
    int64_t max_degree, n_isolated;
    /* what the edge labels were drawn from (synth_arc_labels recomputes them) */
    uint64_t seed;
    int64_t n_labels;
    double label_s;
    int32_t hubs[64];
    int n_hubs;
} synth_graph;

static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* in-place sort of a small int32 array: insertion sort for short rows, qsort otherwise */
static void sort_i32(int32_t *p, int64_t len) {
    if (len < 24) {
        for (int64_t i = 1; i < len; ++i) {
            int32_t x = p[i];
            int64_t j = i - 1;
            while (j >= 0 && p[j] > x) { p[j + 1] = p[j]; --j; }
            p[j + 1] = x;
        }
    } else {
        qsort(p, (size_t)len, sizeof(int32_t), cmp_i32);
    }
}

/* Zipf(s) inverse-CDF table over ranks 1..R */
static double *zipf_cdf(int64_t R, double s) {
    double *c = (double *)malloc(sizeof(double) * (size_t)R);
    double acc = 0.0;
    for (int64_t r = 0; r < R; ++r) { acc += pow((double)(r + 1), -s); c[r] = acc; }
    for (int64_t r = 0; r < R; ++r) c[r] /= acc;
    c[R - 1] = 1.0;
    return c;
}
static inline int64_t zipf_draw(const double *cdf, int64_t R, double u) {
    int64_t lo = 0, hi = R - 1;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (cdf[mid] < u) lo = mid + 1; else hi = mid;
    }
    return lo;
}

/* seeded Fisher-Yates permutation of 0..n-1 */
static int32_t *make_perm(int64_t n, uint64_t seed) {
    int32_t *p = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    for (int64_t i = 0; i < n; ++i) p[i] = (int32_t)i;
    for (int64_t i = n - 1; i > 0; --i) {
        int64_t j = (int64_t)(rng3(seed, ST_PERM, (uint64_t)i) % (uint64_t)(i + 1));
        int32_t t = p[i]; p[i] = p[j]; p[j] = t;
    }
    return p;
}

static int is_hub(const int32_t *hubs, int n_hubs, int32_t v) {
    for (int h = 0; h < n_hubs; ++h) if (hubs[h] == v) return 1;
    return 0;
}

/* Build the symmetric deduplicated CSR from R-MAT draws (+ planted hubs). */
static void build_csr(synth_graph *g, int scale, int64_t edge_factor, uint64_t seed, int n_hubs,
                      int64_t hub_arcs, int32_t *hubs_out) {
    const int64_t n = (int64_t)1 << scale;
    const int64_t m_rmat = edge_factor * n;
    const int64_t m_hub = (int64_t)n_hubs * hub_arcs;
    const int64_t m = m_rmat + m_hub;
    const double A_ = 0.57, B_ = 0.19, C_ = 0.19;
    int32_t *perm = make_perm(n, seed);
    for (int h = 0; h < n_hubs; ++h) hubs_out[h] = perm[(int64_t)(rng3(seed, ST_HUB, (uint64_t)h) % (uint64_t)n)];

    int32_t *src = (int32_t *)malloc(sizeof(int32_t) * (size_t)m);
    int32_t *dst = (int32_t *)malloc(sizeof(int32_t) * (size_t)m);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < m; ++e) {
        int64_t s, d;
        if (e < m_rmat) {
            s = 0; d = 0;
            for (int lv = 0; lv < scale; lv += 2) {
                uint64_t r = rng3(seed, ST_RMAT, (uint64_t)e * 16 + (uint64_t)(lv >> 1));
                for (int t = 0; t < 2 && lv + t < scale; ++t) {
                    double u = (double)((r >> (32 * t)) & 0xFFFFFFFFULL) * 0x1.0p-32;
                    int bs = 0, bd = 0;
                    if (u < A_) { } else if (u < A_ + B_) { bd = 1; } else if (u < A_ + B_ + C_) { bs = 1; } else { bs = 1; bd = 1; }
                    s = (s << 1) | bs; d = (d << 1) | bd;
                }
            }
            s = perm[s]; d = perm[d];
        } else {
            int64_t h = (e - m_rmat) / hub_arcs;
            s = hubs_out[h];
            d = (int64_t)(rng3(seed, ST_HUB, 1000 + (uint64_t)e) % (uint64_t)n);
        }
        if (s == d) { src[e] = -1; dst[e] = -1; } else { src[e] = (int32_t)s; dst[e] = (int32_t)d; }
    }
    free(perm);

    int64_t *deg = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < m; ++e) {
        if (src[e] < 0) continue;
#pragma omp atomic
        deg[src[e]]++;
#pragma omp atomic
        deg[dst[e]]++;
    }
    int64_t *off = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
    off[0] = 0;
    for (int64_t v = 0; v < n; ++v) off[v + 1] = off[v] + deg[v];
    int32_t *col = (int32_t *)malloc(sizeof(int32_t) * (size_t)(off[n] > 0 ? off[n] : 1));
    int64_t *cur = deg; /* reuse as cursor */
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; ++v) cur[v] = off[v];
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < m; ++e) {
        if (src[e] < 0) continue;
        int64_t p1, p2;
#pragma omp atomic capture
        p1 = cur[src[e]]++;
#pragma omp atomic capture
        p2 = cur[dst[e]]++;
        col[p1] = dst[e];
        col[p2] = src[e];
    }
    free(src); free(dst);
    /* sort + dedup each row */
    int64_t *nd = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < n; ++v) {
        int32_t *r = col + off[v];
        int64_t len = off[v + 1] - off[v];
        sort_i32(r, len);
        int64_t w = 0;
        for (int64_t i = 0; i < len; ++i) if (w == 0 || r[i] != r[w - 1]) r[w++] = r[i];
        nd[v] = w;
    }
    int64_t *rp = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
    rp[0] = 0;
    for (int64_t v = 0; v < n; ++v) rp[v + 1] = rp[v] + nd[v];
    int32_t *ci = (int32_t *)malloc(sizeof(int32_t) * (size_t)(rp[n] > 0 ? rp[n] : 1));
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < n; ++v) memcpy(ci + rp[v], col + off[v], sizeof(int32_t) * (size_t)nd[v]);
    free(col); free(off); free(nd); free(deg);
    g->n = n; g->n_arcs = rp[n]; g->row_ptr = rp; g->col_idx = ci;
    int64_t mx = 0, iso = 0;
    for (int64_t v = 0; v < n; ++v) {
        int64_t d = rp[v + 1] - rp[v];
        if (d > mx) mx = d;
        if (d == 0) ++iso;
    }
    g->max_degree = mx; g->n_isolated = iso;
}

/* Label of the edge {v, u} (both arcs get the same one): hub edges share label R, the others are a
 * Zipf(label_s) draw keyed by the unordered pair. */
static int32_t edge_label(uint64_t seed, const double *cdf, int64_t R, const int32_t *hubs, int n_hubs, int vh,
                          int32_t v, int32_t u) {
    if (vh || is_hub(hubs, n_hubs, u)) return (int32_t)R;
    uint64_t lo = (uint64_t)(v < u ? v : u), hi = (uint64_t)(v < u ? u : v);
    return (int32_t)zipf_draw(cdf, R, u01(rng3(seed, ST_LABEL, (lo << 32) | hi)));
}

/* Node weights.  mode 0: paper Eq. 2 over Zipf(label_s) edge labels (R labels, hub edges share label R),
 * then min-max normalised over non-isolated nodes (isolated -> 0; max==min -> all 0), snapped to 2^-24.
 * mode 1: uniform random on the 2^-24 grid. */
static void build_weights(synth_graph *g, uint64_t seed, int mode, int64_t R, double label_s,
                          const int32_t *hubs, int n_hubs) {
    const int64_t n = g->n;
    float *w = (float *)malloc(sizeof(float) * (size_t)n);
    g->weight = w;
    if (mode == 1) {
        for (int64_t v = 0; v < n; ++v) {
            uint64_t k = rng3(seed, ST_WEIGHT, (uint64_t)v) & ((1ULL << 24) - 1);
            w[v] = (float)((double)k * 0x1.0p-24);
        }
        return;
    }
    double *raw = (double *)malloc(sizeof(double) * (size_t)n);
    double *cdf = zipf_cdf(R, label_s);
    const int64_t maxd = g->max_degree > 0 ? g->max_degree : 1;
#pragma omp parallel
    {
        int32_t *lab = (int32_t *)malloc(sizeof(int32_t) * (size_t)maxd);
#pragma omp for schedule(dynamic, 1024)
        for (int64_t v = 0; v < n; ++v) {
            int64_t b = g->row_ptr[v], e = g->row_ptr[v + 1], len = e - b;
            if (len == 0) { raw[v] = -1.0; continue; }
            int vh = is_hub(hubs, n_hubs, (int32_t)v);
            for (int64_t j = 0; j < len; ++j)
                lab[j] = edge_label(seed, cdf, R, hubs, n_hubs, vh, (int32_t)v, g->col_idx[b + j]);
            sort_i32(lab, len);
            double num = 0.0, den = 0.0;
            int64_t i = 0;
            while (i < len) {
                int64_t j = i;
                while (j < len && lab[j] == lab[i]) ++j;
                double c = (double)(j - i);
                num += c * log2(1.0 + c);
                den += c;
                i = j;
            }
            raw[v] = num / den;
        }
        free(lab);
    }
    free(cdf);
    double mn = INFINITY, mx = -INFINITY;
    for (int64_t v = 0; v < n; ++v) {
        if (raw[v] < 0) continue;
        if (raw[v] < mn) mn = raw[v];
        if (raw[v] > mx) mx = raw[v];
    }
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; ++v) {
        double x = 0.0;
        if (raw[v] >= 0 && mx > mn) x = (raw[v] - mn) / (mx - mn);
        double q = floor(x * 16777216.0 + 0.5) * 0x1.0p-24;
        w[v] = (float)q;
    }
    free(raw);
}

/* keywords: node v gets 1 + Poisson(mean) distinct words from Zipf(s) over V words */
static void build_keywords(synth_graph *g, uint64_t seed, int64_t V, double word_s, double mean_extra) {
    const int64_t n = g->n;
    double *cdf = zipf_cdf(V, word_s);
    int32_t *cnt = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    const double el = exp(-mean_extra);
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; ++v) {
        /* Poisson by inversion */
        double u = u01(rng3(seed, ST_NWORDS, (uint64_t)v));
        double p = el, F = p;
        int k = 0;
        while (u > F && k < 60) { ++k; p *= mean_extra / k; F += p; }
        /* keywords only on nodes with at least one arc (a KG entity is connected) */
        cnt[v] = (g->row_ptr[v + 1] > g->row_ptr[v]) ? 1 + k : 0;
    }
    int64_t *np_ = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
    np_[0] = 0;
    for (int64_t v = 0; v < n; ++v) np_[v + 1] = np_[v] + cnt[v];
    int32_t *words = (int32_t *)malloc(sizeof(int32_t) * (size_t)(np_[n] > 0 ? np_[n] : 1));
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; ++v) {
        int32_t *r = words + np_[v];
        int len = cnt[v];
        for (int j = 0; j < len; ++j)
            r[j] = (int32_t)zipf_draw(cdf, V, u01(rng3(seed, ST_WORDS, ((uint64_t)v << 7) | (uint64_t)j)));
        sort_i32(r, len);
        int w = 0;
        for (int j = 0; j < len; ++j) if (w == 0 || r[j] != r[w - 1]) r[w++] = r[j];
        cnt[v] = w;
    }
    free(cdf);
    int64_t *kp = (int64_t *)calloc((size_t)V + 1, sizeof(int64_t));
    for (int64_t v = 0; v < n; ++v)
        for (int j = 0; j < cnt[v]; ++j) kp[words[np_[v] + j] + 1]++;
    for (int64_t t = 0; t < V; ++t) kp[t + 1] += kp[t];
    int64_t tot = kp[V];
    int32_t *kn = (int32_t *)malloc(sizeof(int32_t) * (size_t)(tot > 0 ? tot : 1));
    int64_t *cur = (int64_t *)malloc(sizeof(int64_t) * (size_t)V);
    memcpy(cur, kp, sizeof(int64_t) * (size_t)V);
    for (int64_t v = 0; v < n; ++v)
        for (int j = 0; j < cnt[v]; ++j) kn[cur[words[np_[v] + j]]++] = (int32_t)v;
    free(cur); free(words); free(np_); free(cnt);
    g->n_keywords = V; g->n_postings = tot; g->kw_ptr = kp; g->kw_nodes = kn;
}

/* A: mean hop distance over sampled reachable (source, target) pairs.  BFS over the CSR from
 * n_src seeded sources, pairs_per_src seeded targets each (rejecting unreachable ones). */
static double estimate_A(const synth_graph *g, uint64_t seed, int n_src, int pairs_per_src) {
    const int64_t n = g->n;
    double sum = 0.0;
    int64_t cntp = 0;
#pragma omp parallel for schedule(dynamic, 1) reduction(+ : sum, cntp)
    for (int s = 0; s < n_src; ++s) {
        uint8_t *dist = (uint8_t *)malloc((size_t)n);
        int32_t *q = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
        memset(dist, 0xFF, (size_t)n);
        /* pick a non-isolated source */
        int64_t src = -1;
        for (uint64_t t = 0; t < 1000; ++t) {
            int64_t c = (int64_t)(rng3(seed, ST_APAIR, ((uint64_t)s << 20) | t) % (uint64_t)n);
            if (g->row_ptr[c + 1] > g->row_ptr[c]) { src = c; break; }
        }
        if (src >= 0) {
            int64_t qh = 0, qt = 0, reached = 0;
            dist[src] = 0; q[qt++] = (int32_t)src;
            while (qh < qt) {
                int32_t u = q[qh++];
                uint8_t du = dist[u];
                for (int64_t j = g->row_ptr[u]; j < g->row_ptr[u + 1]; ++j) {
                    int32_t x = g->col_idx[j];
                    if (dist[x] == 0xFF) { dist[x] = (uint8_t)(du < 254 ? du + 1 : 254); q[qt++] = x; }
                }
            }
            reached = qt;
            if (reached > 1) {
                for (int p = 0; p < pairs_per_src; ++p) {
                    int32_t t = q[1 + (int64_t)(rng3(seed, ST_APAIR + 100, ((uint64_t)s << 32) | (uint64_t)p) % (uint64_t)(reached - 1))];
                    sum += (double)dist[t];
                    cntp += 1;
                }
            }
        }
        free(dist); free(q);
    }
    return cntp > 0 ? sum / (double)cntp : 1.0;
}

/* ---------------------------------------------------------------- public C entry points (ctypes) */

synth_graph *synth_build(int scale, int64_t edge_factor, uint64_t seed, int n_hubs, int64_t hub_arcs,
                         int weight_mode, int64_t n_labels, double label_s, int64_t vocab, double word_s,
                         double words_mean_extra, int a_sources, int a_pairs_per_source) {
    synth_graph *g = (synth_graph *)calloc(1, sizeof(synth_graph));
    int32_t hubs[64];
    if (n_hubs > 64) n_hubs = 64;
    build_csr(g, scale, edge_factor, seed, n_hubs, hub_arcs, hubs);
    g->seed = seed; g->n_labels = n_labels; g->label_s = label_s; g->n_hubs = n_hubs;
    memcpy(g->hubs, hubs, sizeof(int32_t) * (size_t)n_hubs);
    build_weights(g, seed, weight_mode, n_labels, label_s, hubs, n_hubs);
    build_keywords(g, seed, vocab, word_s, words_mean_extra);
    g->A = estimate_A(g, seed, a_sources, a_pairs_per_source);
    return g;
}

void synth_sizes(const synth_graph *g, int64_t *out /* [6] */) {
    out[0] = g->n; out[1] = g->n_arcs; out[2] = g->n_keywords; out[3] = g->n_postings;
    out[4] = g->max_degree; out[5] = g->n_isolated;
}
double synth_A(const synth_graph *g) { return g->A; }
void synth_copy(const synth_graph *g, int64_t *row_ptr, int32_t *col_idx, float *weight, int64_t *kw_ptr,
                int32_t *kw_nodes) {
    memcpy(row_ptr, g->row_ptr, sizeof(int64_t) * (size_t)(g->n + 1));
    memcpy(col_idx, g->col_idx, sizeof(int32_t) * (size_t)g->n_arcs);
    memcpy(weight, g->weight, sizeof(float) * (size_t)g->n);
    memcpy(kw_ptr, g->kw_ptr, sizeof(int64_t) * (size_t)(g->n_keywords + 1));
    memcpy(kw_nodes, g->kw_nodes, sizeof(int32_t) * (size_t)g->n_postings);
}
/* The edge labels behind the Eq. 2 weights (weight_mode 0), one per CSR arc (in-arcs = out-arcs: the
 * graph is symmetric), so that the load-time preprocessing can be checked against the generator. */
void synth_arc_labels(const synth_graph *g, int32_t *out) {
    double *cdf = zipf_cdf(g->n_labels, g->label_s);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < g->n; ++v) {
        int vh = is_hub(g->hubs, g->n_hubs, (int32_t)v);
        for (int64_t j = g->row_ptr[v]; j < g->row_ptr[v + 1]; ++j)
            out[j] = edge_label(g->seed, cdf, g->n_labels, g->hubs, g->n_hubs, vh, (int32_t)v, g->col_idx[j]);
    }
    free(cdf);
}

void synth_free(synth_graph *g) {
    if (!g) return;
    free(g->row_ptr); free(g->col_idx); free(g->weight); free(g->kw_ptr); free(g->kw_nodes);
    free(g);
}
int synth_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
