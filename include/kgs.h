/* kgs.h — C-ABI of the B200-native Central Graph keyword-search hot path (libkgs.so).
 *
 * The method is Yang, Agrawal, Jagadish, Tung, Wu, "An Efficient Parallel Keyword Search Engine on
 * Knowledge Graphs", ICDE 2019.  "P:Lnnn" cites a line of that paper's text; "R<n>" names a
 * reading of an ambiguous passage listed in DESIGN.md "Readings".
 *
 * Problem (Def. 4): given a knowledge graph G (CSR, node weights, keyword -> nodes
 * inverted index), a query Q of q keyword ids and k, run one BFS instance B_i per keyword from
 * T_i = nodes containing t_i, level-synchronously and gated by minimum activation levels
 * (Eqs. 3-5), until at least k Central Nodes (nodes hit by every B_i) are identified;
 * extract each Central Graph top-down (Thm. V.4, Alg. 3), prune it with level-cover
 * (P:L454), score it by Eq. 6 and return the k best.
 *
 * Conventions for every call:
 *   - Every entry point returns kgs_status (0 = KGS_OK, < 0 = error) except the void/free/count
 *     helpers.  Nothing aborts or throws across the ABI; on error, kgs_last_error() returns a
 *     thread-local message and every output pointer is left NULL/unchanged.
 *   - Host pointers are only read during the call; the caller keeps ownership.  Device pointers are
 *     only accepted where a name or flag says so.
 *   - A kgs_graph is immutable after load and may serve several threads; queries on one graph are
 *     serialised internally (one workspace per graph in this version).
 *   - All work is enqueued on the caller's CUDA stream (NULL = legacy default stream); kgs_query
 *     returns after the results have been copied to host memory (it synchronises that stream).
 */
#ifndef KGS_H
#define KGS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    KGS_OK = 0,
    KGS_EINVAL = -1,    /* malformed argument (see each call) */
    KGS_ENOMEM = -2,    /* device or host allocation failed */
    KGS_ECUDA = -3,     /* a CUDA runtime/launch error (message from kgs_last_error) */
    KGS_ENCCL = -4,     /* reserved for the multi-GPU layer */
    KGS_EINTERNAL = -5  /* an internal invariant failed */
} kgs_status;

#define KGS_MAX_Q 8        /* q <= 8: one 8-byte M row and a uint8 hit mask per node */
#define KGS_MAX_K 4096     /* top-k selection sorts the winners inside one CTA */
#define KGS_INF_LEVEL 255  /* "infinity" in the uint8 node-keyword matrix M */

#define KGS_INPUT_DEVICE_PTRS 1  /* kgs_graph_desc arrays are device pointers (copied, not borrowed) */
#define KGS_NO_RELABEL 2         /* keep the input node order internally (default: renumbered by degree for
                                    L2 locality; every id at the ABI is the input id either way) */

#define KGS_EXTRACT_EXACT 0    /* Thm. V.4 + "predecessor not yet central" (reading R12, default) */
#define KGS_EXTRACT_LITERAL 1  /* Thm. V.4 exactly as printed */

#define KGS_STOP_K 0              /* |C| >= k after identification at level d (Thm. V.3) */
#define KGS_STOP_EXHAUSTED 1      /* the joint frontier became empty (no pending work) */
#define KGS_STOP_MAX_DEPTH 2      /* level reached params.max_depth (truncated) */
#define KGS_STOP_EMPTY_KEYWORD 3  /* some T_i is empty: nothing can be central (reading R17) */
#define KGS_STOP_INVALID_QUERY (-1) /* device batch only: q out of range, keyword id out of range or repeated */
#define KGS_STOP_CAPACITY (-2)    /* batch only: the query exceeded an internal capacity (predecessor arcs,
                                     extraction or answer arena); no answers, the rest of the batch is valid
                                     (a single kgs_query returns KGS_EINTERNAL instead) */

/* Graph description for kgs_load_graph (node-weighted graph stored as CSR).
 *   n_nodes     number of nodes, 0 <= n < 2^31.
 *   n_arcs      number of CSR entries (a bi-directed KG stores every edge as two arcs, reading R21).
 *   row_ptr     [n_nodes + 1], row_ptr[0] = 0, non-decreasing, row_ptr[n] = n_arcs.
 *   col_idx     [n_arcs], 0 <= id < n_nodes.  Out-arcs: B_i expands u -> col_idx (reading R1).
 *   weight      [n_nodes], normalised node weight w' in [0, 1] (Eq. 2 + min-max).
 *               Snapped to the 2^-24 grid on load (reading R15) so Eq. 6 sums are exact.
 *   n_keywords  vocabulary size V >= 1.
 *   kw_ptr      [V + 1] int64 offsets, kw_nodes[kw_ptr[t] .. kw_ptr[t+1]) = T_t, strictly increasing.
 *   avg_dist_A  A, the sampled average shortest distance (Table II), > 0.
 *   symmetric   1: in-arcs == out-arcs (bi-directed KG).  0: the library builds the reverse CSR used
 *               by extraction (reading R1).
 *   device      CUDA device ordinal the graph lives on.
 *   flags       KGS_INPUT_DEVICE_PTRS | KGS_NO_RELABEL, or 0.  The library stores the graph with its
 *               nodes renumbered by non-increasing degree (ties by input id) unless KGS_NO_RELABEL is
 *               set; results are identical (every id returned is the input id, ties rank by input id).
 *   pred_arc_cap  capacity, in arcs, of each query workspace's predecessor-arc buffers (the Thm. V.4 arcs
 *               of the top-down, 20 B each); 0 = min(n_arcs, 2^28), at least 2^20.  A query whose
 *               predecessor DAG exceeds it reports KGS_STOP_CAPACITY (batch) / KGS_EINTERNAL (single). */
typedef struct {
    int64_t n_nodes, n_arcs;
    const int64_t *row_ptr;
    const int32_t *col_idx;
    const float *weight;
    int64_t n_keywords;
    const int64_t *kw_ptr;
    const int32_t *kw_nodes;
    double avg_dist_A;
    int32_t symmetric;
    int32_t device;
    int32_t flags;
    int64_t pred_arc_cap;
} kgs_graph_desc;

typedef struct kgs_graph kgs_graph;   /* opaque: device CSR (+ reverse), weights, index, workspace */
typedef struct kgs_result kgs_result; /* opaque: host copy of the answers (+ optional M / centrals) */

/* Per-query parameters (Table III, Eq. 6).
 *   alpha          in (0, 1), default 0.1 (Eqs. 3-5).
 *   lambda         >= 0, default 0.2 (Eq. 6).
 *   max_depth      1..254, default 254 (255 encodes infinity in M).
 *   block_central  1 (default): a node identified as central no longer expands (Alg. 2 ln 2).
 *   extract_mode   KGS_EXTRACT_EXACT (default) or KGS_EXTRACT_LITERAL.
 *   level_cover    level-cover pruning: 1 (default) a keyword node's level counts the keywords it
 *                  contributes (it is a source of a hitting path of this Central Graph, reading R13);
 *                  2 the keywords it contains (NEXT-3, reading R13b); 0 returns unpruned Central Graphs.
 *   containment    1: drop every Central Graph whose pruned node set strictly contains the pruned node
 *                  set of another Central Graph of C (NEXT-3, reading R16), answers = the k best of
 *                  the rest among the best min(|C|, KGS_MAX_K); forces prune = 0.  0 (default): off.
 *   want_levels    1: also copy M and the central list back (for parity checks); default 0.
 *   prune          exact lower-bound pruning of the top-down phase (Eq. 6 keys are computed only for the
 *                  candidates whose (bound, id) can still beat the k-th exact (key, id); the answers are
 *                  identical, only kgs_result_centrals' keys of skipped candidates are not computed, so
 *                  want_levels = 1 forces prune = 0):
 *                    0  off: every Central Graph is extracted (Alg. 3 as written);
 *                    1  (default) bound d^lambda * w_c (the central node is always kept, weights >= 0);
 *                    2  bound d^lambda * max_i (lightest Thm. V.4 path from T_i to c), computed by the
 *                       search (an atomic min per hitting arc).  Tighter, costs search time.  Needs the
 *                       Thm. V.4 DAG to consist of arcs the search traversed: with extract_mode = LITERAL
 *                       and block_central = 1 it falls back to 1.
 *   direction      expansion direction of Alg. 2 (the north star's push/pull switching):
 *                    KGS_DIR_AUTO (0, default)  push; from the first level whose frontier has more than
 *                                   m / pull_ratio and more than pull_min out-arcs (m = all arcs) on, pull;
 *                    KGS_DIR_PUSH (1)  push only: the frontier nodes scan their out-arcs (Alg. 2 as written);
 *                    KGS_DIR_PULL (2)  pull at every level: every node x that still lacks a keyword and whose
 *                                   gate is open scans its in-arcs for active neighbours (the level rule,
 *                                   SURVEY.md §8(c) O3).
 *                  Results do not depend on it (M, central set, depths, answers, stop level and reason):
 *                  after a pulled level without hits the engine recomputes whether Alg. 2's work list
 *                  would still hold a node (an inactive hit node, or one waiting for a gated neighbour).
 * Engine tuning (results never depend on these; kgs_params_default sets the defaults in brackets):
 *   pull_ratio     >= 1 [14]: the auto direction pulls once the frontier's out-arcs exceed m / pull_ratio
 *   pull_min       >= 0 [2^22]: ... and exceed pull_min
 *   prune_min      >= 1 [512]: pruning round 1 extracts min(4096, max(8k, prune_min)) candidates
 *   tile_light     >= 0 [4096]: light frontiers of at most this many nodes are expanded by group-wide tiles
 *   dag_record     -1 [auto: on for single-query launches] / 0 / 1: the top-down's predecessor lists come
 *                  from the arcs the search recorded (1) or from the in-arc pre-pass (0); the recorded DAG
 *                  is used only where it is exact (extract_mode EXACT, or block_central 0)
 *   search_only    0 [0] / 1: workload analysis — stop after the search (no top-down, no answers)
 *   mk_min         >= 0 [4096]: with level_cover = 1 and at least this many candidates in pruning round 2,
 *                  decide per candidate whether level-cover can keep fewer than all of its sources (a pass
 *                  over the predecessor DAG, engine.cu mk_reach) instead of once per query, so that the
 *                  exact key cut-off applies to more candidates
 *   defer_min      >= 0 [65536]: in a launch of several query groups, a query that identifies more central
 *                  nodes than this is answered at the end of the launch by all CTAs together (its top-down
 *                  parallelises over the whole GPU instead of holding one group); 0 = never
 *   lazy_dag       0 / 1 [1]: pruning round 2 extends the shared predecessor DAG only as far as the
 *                  candidates' walks need before the exact key cut-off stops them (candidates whose cut is
 *                  valid, decided from the search's rm bits); 0 builds every round-2 closure first
 *   rec_max        >= 0 [2^24]: a recorded DAG (dag_record) of more arcs is dropped for the pre-pass when
 *                  pruning runs (more than max(8k, prune_min) central nodes): its lists cover every touched
 *                  node, the pre-pass only the candidates' closures (with the lazy round 2) */
typedef struct {
    double alpha, lambda;
    int32_t max_depth, block_central, extract_mode, level_cover, want_levels, prune;
    int32_t direction;
    int32_t pull_ratio;
    int64_t pull_min;
    int32_t prune_min, tile_light, dag_record, search_only;
    int32_t containment;
    int32_t mk_min;
    int32_t defer_min;
    int32_t lazy_dag;
    int32_t rec_max;
} kgs_params;
enum { KGS_DIR_AUTO = 0, KGS_DIR_PUSH = 1, KGS_DIR_PULL = 2 };

/* One answer (a pruned Central Graph).  Pointers live until kgs_result_free. */
typedef struct {
    int32_t central;     /* the Central Node id */
    int32_t depth;       /* d(C) = max_i h^i_c (Eq. 1, Lemma V.1), before pruning */
    float score;         /* (float)score_key */
    double score_key;    /* Eq. 6 in fp64: pow(d, lambda) * sum of w over the pruned graph; smaller is better (R14) */
    int64_t n_nodes;
    const int32_t *nodes;  /* ascending node ids */
    int64_t n_arcs;
    const int32_t *arcs;   /* [2 * n_arcs] (pred, succ) pairs, lexicographic, unique, union over keywords */
} kgs_answer;

/* Statistics of one query.  Times are CUDA-event milliseconds of the phases (P:L532 profile). */
typedef struct {
    int32_t levels;        /* BFS level at which the search stopped (d when stop_reason == KGS_STOP_K) */
    int32_t stop_reason;   /* KGS_STOP_* */
    int64_t n_centrals;    /* |C|: all Central Nodes identified (candidates for top-down) */
    int64_t count;         /* answers returned = min(k, |C|) */
    int64_t frontier_total;/* sum over levels of the joint frontier size */
    int64_t arcs_scanned;  /* out-arcs inspected by expansion (GTEPS numerator) */
    int64_t overflow;      /* Central Graphs extracted by the large-graph path */
    int64_t hits;          /* (node, keyword) pairs newly hit by expansion (M entries written) */
    int64_t td_arcs;       /* in-arcs inspected by the top-down predecessor pre-pass */
    int64_t td_pred_arcs;  /* predecessor arcs (Thm. V.4) in the union of all Central Graphs */
    float ms_search, ms_topdown, ms_total;   /* this query: bottom-up search, top-down, total (device clock) */
    float ms_launch;       /* the whole engine launch that answered it (all queries of the batch) */
    int32_t group;         /* engine group (set of CTAs) that answered the query; n_groups: the whole grid
                              at the end of the launch (a deferred query, kgs_params.defer_min) */
    int32_t n_evaluated;   /* Central Graphs whose exact key was computed (|C| unless prune skipped some) */
    int64_t dag_arcs;      /* arcs the search traversed that hit their target: the Thm. V.4 arcs of all hit nodes */
    int32_t pull_level;    /* first level expanded by pull (kgs_params.direction), -1: push throughout */
    int32_t n_cut;         /* candidates whose extraction stopped at the exact key cut-off (prune round 2) */
    int32_t n_tier4;       /* Central Graphs extracted in the per-group tier-4 arena (beyond the per-CTA arenas) */
    int64_t td_arcs_big;   /* td_arcs of predecessor-list nodes with more than 2048 in-arcs (the hubs) */
} kgs_stats;

/* Load a graph onto params-independent device state.  Validates the CSR and the index
 * (KGS_EINVAL: n out of range, row_ptr not monotone / wrong ends, col_idx out of range,
 * weight not finite or outside [0, 1], kw_ptr malformed, kw_nodes out of range or not strictly
 * increasing per keyword, A <= 0).  On success *out owns all device memory of the graph. */
kgs_status kgs_load_graph(const kgs_graph_desc *desc, kgs_graph **out);
void kgs_free_graph(kgs_graph *g);

void kgs_params_default(kgs_params *p);

/* Answer one query (Alg. 1).
 *   kw_ids       host array of q distinct keyword ids in [0, n_keywords).
 *   q            1..KGS_MAX_Q.   k  1..KGS_MAX_K.
 *   p            NULL = defaults.
 *   cuda_stream  cudaStream_t to enqueue on (NULL = default stream).
 * Returns KGS_EINVAL for q/k/params out of range or duplicate / out-of-range keyword ids.  An empty
 * T_i is not an error: the result has count 0 and stop_reason KGS_STOP_EMPTY_KEYWORD.
 * On success *out is a new result the caller frees with kgs_result_free. */
kgs_status kgs_query(kgs_graph *g, const int32_t *kw_ids, int32_t q, int32_t k, const kgs_params *p,
                     void *cuda_stream, kgs_result **out);

/* Device-resident variant for pipelines and benchmarks: kw_ids_dev is a DEVICE array of q keyword ids
 * (validated on the device: invalid ids give count 0 and stop_reason -1 in the device header).
 * Enqueues the whole query on the stream and returns without synchronising; the answers stay in the
 * graph's device workspace until the next query on this graph.  kgs_query_fetch (same stream)
 * copies them to a host result, synchronising the stream. */
kgs_status kgs_query_device(kgs_graph *g, const int32_t *kw_ids_dev, int32_t q, int32_t k, const kgs_params *p,
                            void *cuda_stream);
kgs_status kgs_query_fetch(kgs_graph *g, void *cuda_stream, kgs_result **out);

/* Answer a batch of independent queries in ONE launch (BASELINE.json configs[3]).
 *   Query j has the keywords kw_ids[q_ptr[j] .. q_ptr[j+1]) (host arrays, q_ptr[0] = 0).
 *   n_groups  how many queries run at the same time: the engine's CTAs are split into that many groups,
 *             each answering whole queries and taking the next one from a device counter (0 = default 8;
 *             clamped to [1, n_queries]).  Results do not depend on it.
 *   results   [n_queries] receives one kgs_result per query (free each with kgs_result_free).
 * Validation as kgs_query for every query (KGS_EINVAL, nothing enqueued). */
kgs_status kgs_query_batch(kgs_graph *g, int32_t n_queries, const int32_t *q_ptr, const int32_t *kw_ids, int32_t k,
                           const kgs_params *p, int32_t n_groups, void *cuda_stream, kgs_result **results);
/* Device-resident batch: kw_dev [n_queries][KGS_MAX_Q] (unused slots ignored) and qlen_dev [n_queries] in
 * device memory.  Invalid queries are detected on the device and reported with stop_reason
 * KGS_STOP_INVALID_QUERY.  Enqueues without synchronising; kgs_query_batch_fetch (same stream) copies
 * the n_queries results back, synchronising the stream. */
kgs_status kgs_query_batch_device(kgs_graph *g, int32_t n_queries, const int32_t *kw_dev, const int32_t *qlen_dev,
                                  int32_t k, const kgs_params *p, int32_t n_groups, void *cuda_stream);
kgs_status kgs_query_batch_fetch(kgs_graph *g, void *cuda_stream, kgs_result **results);

/* Result accessors.  kgs_result_count = min(k, |C|); answers are ranked by (score_key asc, central asc). */
int32_t kgs_result_count(const kgs_result *r);
kgs_status kgs_result_answer(const kgs_result *r, int32_t i, kgs_answer *a);
/* M (n * q bytes, node-major, 255 = infinity) — only if params.want_levels was 1, else KGS_EINVAL. */
kgs_status kgs_result_levels(const kgs_result *r, uint8_t *M, int64_t cap);
/* Central list ascending with depths (all of C) — only if want_levels was 1.  *n = |C|. */
kgs_status kgs_result_centrals(const kgs_result *r, int32_t *ids, uint8_t *depth, double *score_key, int64_t cap,
                               int64_t *n);
/* Activation levels a (n bytes, Eqs. 3-5 at the query's alpha) — only if want_levels was 1. */
kgs_status kgs_result_activation(const kgs_result *r, uint8_t *a, int64_t cap);
kgs_status kgs_result_stats(const kgs_result *r, kgs_stats *s);
/* Every answer of a result in flat host arrays with one call (kgs_result_answer takes one call per answer):
 * kgs_result_sizes gives count, the total number of answer nodes and of answer arcs; kgs_result_export
 * fills central / depth / score_key [count], node_off / arc_off [count + 1] (answer i's nodes are
 * nodes[node_off[i] .. node_off[i + 1]), its arcs arcs[2 * arc_off[i] .. 2 * arc_off[i + 1])), nodes
 * [total_nodes] and arcs [2 * total_arcs], in rank order.  Caller-owned buffers. */
kgs_status kgs_result_sizes(const kgs_result *r, int32_t *count, int64_t *total_nodes, int64_t *total_arcs);
kgs_status kgs_result_export(const kgs_result *r, int32_t *central, int32_t *depth, double *score_key,
                             int64_t *node_off, int32_t *nodes, int64_t *arc_off, int32_t *arcs);
/* Phase trace of the search kernel (the paper's per-phase profile): *n stamps, each a
 * tag (0 start, 1 reset, 2 sources, 3 merge+identify, 4 expansion, 5..8 top-down pre-pass: seeds,
 * merge, expansion, CSR, 9 end of search) and a %globaltimer time in ns, in execution order. */
kgs_status kgs_result_phases(const kgs_result *r, int32_t *tags, uint64_t *t_ns, int32_t cap, int32_t *n);
void kgs_result_free(kgs_result *r);

/* ---- Vertex-partitioned search of ONE query over P ranks ----
 * Every rank loads the whole graph (kgs_load_graph: the CSR is replicated) and owns the node rows
 * [lo, hi) = [rank * slice, min((rank + 1) * slice, n)), slice = kgs_vp_slice(n, world).  The search is
 * the level rule of Alg. 2 (reading R10) as a pull over the owned rows: at level l an owned x
 * gets keyword i if some in-neighbour u expands i at l (a_u <= l, m_ui <= l, u not a blocked central) and
 * x may be entered (x in K or a_x <= l + 1).  The caller owns the exchange buffers (device memory on the
 * graph's device, n_pad = slice * world) and runs the collectives between the calls:
 *   kgs_vp_begin          sources, owned level-0 centrals               then all_reduce(counts, sum)
 *   kgs_vp_level(l)       one level over the owned rows                  then all_gather(hm <- hm_slice),
 *                                                                             all_reduce(counts, sum)
 *   kgs_vp_waiting(l)     only if the level made no mark, nothing waits for activation and
 *                         l + 1 < amax: hit nodes waiting for a gated neighbour  then all_reduce(counts)
 *   (host: the stop rules of kgs_query — |C| >= k, max_depth, and exhaustion when the work-list of
 *    Alg. 2 is empty: no mark and nothing waiting, which stops at level l + 1)
 *   after the search      all_gather(M <- owned rows), all_gather(central lists)
 *   kgs_vp_topdown        Alg. 3 + level-cover + Eq. 6 + top-k on the replicated state -> kgs_result
 * paper_conf_icde_yangajtw19_b200.dist.vp_query is that driver over torch.distributed.  The result equals
 * kgs_query's.  Calls on one graph must not interleave with other queries between begin and topdown. */
typedef struct {
    uint8_t *hm;        /* [n_pad]     replicated hit masks (bit i = hit by keyword i); all_gather output */
    uint8_t *hm_slice;  /* [slice]     this rank's hit masks after the level; all_gather input */
    uint8_t *M;         /* [n_pad * 8] node-major hitting levels; this rank writes rows [lo, hi) */
    int64_t *counts;    /* [4]         marks, new central nodes, waiting work-list nodes, changed owned nodes
                                       (all_reduce sum) */
    int32_t *cent;      /* [slice]     this rank's central nodes (identification order) */
    uint8_t *cdep;      /* [slice]     their depths */
    int32_t *cent_n;    /* [1]         their count */
    int64_t *chg;       /* [slice] or NULL: the level's changed owned nodes, id << 8 | new hit mask, for a
                                       sparse exchange (kgs_vp_query uses it when few nodes change) */
} kgs_vp_buffers;
/* ceil(n / world) rounded up to a multiple of 16 (0 for bad arguments). */
int64_t kgs_vp_slice(int64_t n_nodes, int32_t world);
/* Validation as kgs_query.  info[0] = amax (max activation level at alpha: the exhaustion rule needs it),
 * info[1] = 1 if some T_i is empty (stop with KGS_STOP_EMPTY_KEYWORD, no level calls). */
kgs_status kgs_vp_begin(kgs_graph *g, const int32_t *kw_ids, int32_t q, int32_t k, const kgs_params *p, int32_t rank,
                        int32_t world, const kgs_vp_buffers *b, void *cuda_stream, int32_t *info);
/* Level l (0 <= l < 254) over the owned rows: reads hm (the state at the start of l), writes hm_slice,
 * the owned M rows, the owned centrals (depth l + 1) and counts. */
kgs_status kgs_vp_level(kgs_graph *g, int32_t level, void *cuda_stream);
/* After a level l without marks (hm = the state after l): counts[2] = owned hit nodes, not blocked, active
 * at l, with an out-neighbour gated at l + 1 that lacks one of their keywords (Alg. 2 ln 17-19). */
kgs_status kgs_vp_waiting(kgs_graph *g, int32_t level, void *cuda_stream);
/* Top-down on the replicated state: b.hm and b.M complete (all ranks' rows), centrals_dev / depth_dev the
 * all-gathered central list (device, n_central entries), levels / stop_reason from the host loop. */
kgs_status kgs_vp_topdown(kgs_graph *g, int64_t n_central, const int32_t *centrals_dev, const uint8_t *depth_dev,
                          int32_t levels, int32_t stop_reason, void *cuda_stream, kgs_result **out);

/* ---- The whole vertex-partitioned query in the library ----
 * kgs_vp_query runs the level loop above on every rank: the level calls, the exchanges (dense all_gather
 * of the owned hit-mask slices, or a sparse all_gather of (id << 8 | mask) change lists when fewer than n/16
 * nodes changed in the level), the counter all_reduces, the stop rules of kgs_query (Def. 4, Thm. V.3,
 * R9, R22), the final gathers of M and of the central lists, and the top-down — and returns the same result
 * as kgs_query on every rank.  The ranks' collectives go through a transport:
 *   all_gather(ctx, send, recv, bytes, stream)   recv[r * bytes ..] = rank r's send (device buffers)
 *   all_reduce_sum_i64(ctx, buf, count, stream)  in place, int64 sum over the ranks (device buffer)
 * each returning 0 on success, enqueued on (or completed with respect to) the given CUDA stream.
 * kgs_vp_nccl_transport gives the library's own NCCL communicator over NVLink / NVSwitch (rank 0 calls
 * kgs_vp_nccl_unique_id and the caller broadcasts the 128 bytes); callers may supply their own (the
 * CPU tests stage through gloo).  Every rank must call kgs_vp_query with the same query and parameters. */
typedef struct {
    void *ctx;
    int32_t (*all_gather)(void *ctx, const void *send, void *recv, int64_t bytes, void *cuda_stream);
    int32_t (*all_reduce_sum_i64)(void *ctx, int64_t *buf, int64_t count, void *cuda_stream);
    int32_t owned;       /* 1: created by kgs_vp_nccl_transport, release with kgs_vp_transport_free */
    int32_t host_staged; /* 1: the callbacks take HOST buffers (the library copies around them) */
} kgs_vp_transport;
kgs_status kgs_vp_nccl_unique_id(uint8_t *id /* [128] */);
kgs_status kgs_vp_nccl_transport(const uint8_t *id /* [128] */, int32_t rank, int32_t world, int32_t device,
                                 kgs_vp_transport *out);
void kgs_vp_transport_free(kgs_vp_transport *t);
kgs_status kgs_vp_query(kgs_graph *g, const int32_t *kw_ids, int32_t q, int32_t k, const kgs_params *p, int32_t rank,
                        int32_t world, const kgs_vp_transport *t, void *cuda_stream, kgs_result **out);

/* ---- Load-time preprocessing: the steps that produce kgs_load_graph's inputs.
 * Both run on the raw CSR before kgs_load_graph, on `device`, on `cuda_stream` (NULL = default),
 * and return when their host outputs are written.  Inputs are host pointers (copied) unless
 * flags & KGS_INPUT_DEVICE_PTRS (borrowed device pointers).  KGS_EINVAL for malformed sizes.     */

/* A, "the average shortest distance (hops) between two nodes ... by sampling" (Table II and
 * 10^4 sampled pairs).  dist[j] = number of arcs of a shortest src[j] -> dst[j] path along
 * out-arcs (0 when src == dst), or -1 when dst is not reached within max_hops (1..254) hops.
 * *mean = the mean of the reachable dist[j] (fp64), or NaN when none is.  row_ptr [n+1] int64,
 * col_idx [n_arcs] int32 (out-arcs), src/dst [n_pairs] int32 in [0, n); dist [n_pairs] host output,
 * mean host output (may be NULL).  Pairs are answered 128 at a time by one bit-parallel BFS.     */
kgs_status kgs_prep_pair_distances(int64_t n_nodes, int64_t n_arcs, const int64_t *row_ptr,
                                   const int32_t *col_idx, int32_t n_pairs, const int32_t *src,
                                   const int32_t *dst, int32_t max_hops, int32_t device, int32_t flags,
                                   void *cuda_stream, int32_t *dist, double *mean);

/* Eq. 2 degree of summary: for node v with in-arc label multiset R_v, where n_r is
 * the number of in-arcs of label r,  w_v = sum_r n_r log2(1 + n_r) / sum_r n_r  (fp64, the terms added
 * in ascending label order), then w'_v = (w_v - min w) / (max w - min w) over the nodes WITH in-arcs
 * (P:L184).  A node without in-arcs summarises nothing: w' = 0, raw w reported as 0, and it takes no
 * part in the min / max (reading R6).  Every w' is 0 when max = min (R26).  w' is produced on the
 * 2^-24 grid: the nearest grid point of the fp64 value, ties up (R27), so kgs_load_graph's snap keeps it.
 * in_row_ptr [n+1] int64, in_label [n_in_arcs] int32 (any order within a row).  w_norm [n] host output
 * (float, the kgs_graph_desc.weight input); w_raw [n] host output (fp64, may be NULL).              */
kgs_status kgs_prep_summary_weights(int64_t n_nodes, int64_t n_in_arcs, const int64_t *in_row_ptr,
                                    const int32_t *in_label, int32_t device, int32_t flags,
                                    void *cuda_stream, float *w_norm, double *w_raw);

/* Thread-local message describing the last non-OK status of this thread. */
const char *kgs_last_error(void);

/* Library build/version string. */
const char *kgs_version(void);

#ifdef __cplusplus
}
#endif
#endif /* KGS_H */
