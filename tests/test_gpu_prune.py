"""Exact lower-bound pruning of the top-down phase (kgs_params.prune).

With pruning the engine computes the exact Eq. 6 key only for the candidates whose lower bound can
still reach the top-k.  The answers must be those of the oracle
(which extracts every Central Graph), and the number of candidates evaluated must be the one the
two-round rule gives when it is replayed here on the oracle's own keys:

  LB(c) = pow(d, lambda) * max_i (lightest Thm. V.4 path from T_i to c)   (exact extraction)

  round 1: the m = min(KGS_MAX_K, max(8k, 512)) smallest (LB, id); T = the k-th smallest exact
           (key, id) among them; B = the m-th (LB, id);
  round 2 (only if B < T): every other candidate with (LB, id) < T.

Graphs have several thousand Central Nodes so that both outcomes (round 2 or not) occur.
"""
import math

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

kgs = pytest.importorskip("paper_conf_icde_yangajtw19_b200")

KGS_MAX_K = 4096


def _gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def medium_graph(seed, n=4000, deg=4, q=3, kw_size=300, wpow=1.0, zero_frac=0.0):
    """Random undirected graph with many Central Nodes; weights on the 2^-24 grid, skewed by wpow."""
    rng = np.random.default_rng(seed)
    m = n * deg // 2
    u = rng.integers(0, n, m)
    v = rng.integers(0, n, m)
    keep = u != v
    edges = list(zip(u[keep].tolist(), v[keep].tolist()))
    w = rng.random(n) ** wpow
    w[rng.random(n) < zero_frac] = 0.0
    w = (np.floor(w * (1 << 24) + 0.5) / (1 << 24)).astype(np.float32)
    kws = [sorted(rng.choice(n, size=kw_size, replace=False).tolist()) for _ in range(q)]
    return synth.from_edges(n, edges, w, kws, 2.0)


def lightest_paths(g, kw, o):
    """Per (node, keyword): the lightest weight (fixed point 2^-24) of a path from T_i to the node along
    Thm. V.4 arcs (m_xi = 1 + max(a_u, m_ui, g_x - 1), u not a blocked central at m_xi - 1), by dynamic
    programming over the oracle's hitting levels, level by level.  numpy, independent of the engine."""
    n = len(g.row_ptr) - 1
    q = len(kw)
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(g.row_ptr))
    dst = np.asarray(g.col_idx, np.int64)
    W = np.floor(np.asarray(g.weight, np.float64) * (1 << 24)).astype(np.int64)
    M = o.M.astype(np.int64)
    a = o.a.astype(np.int64)
    K = np.zeros(n, bool)
    for t in kw:
        K[g.kw_nodes[g.kw_ptr[t]:g.kw_ptr[t + 1]]] = True
    gate = np.where(K, 0, a)
    full = (M < 255).all(1)
    maxrow = np.where(M < 255, M, 0).max(1)
    big = np.int64(1) << 62
    mw = np.full((n, q), big, np.int64)
    for i in range(q):
        lv = M[:, i]
        mw[lv == 0, i] = W[lv == 0]
        mu, mx = lv[src], lv[dst]
        ok = (mu < 255) & (mx < 255) & (mx == 1 + np.maximum(np.maximum(a[src], mu), gate[dst] - 1))
        ok &= ~(full[src] & (maxrow[src] <= mx - 1))
        su, sx = src[ok], dst[ok]
        top = int(lv[lv < 255].max()) if (lv < 255).any() else 0
        for L in range(1, top + 1):
            sel = lv[sx] == L
            cand = np.full(n, big, np.int64)
            np.minimum.at(cand, sx[sel], mw[su[sel], i])
            hit = lv == L
            mw[hit, i] = W[hit] + cand[hit]
    return mw


def expected_evaluated(g, o, k, lam, kw, pmin=512, bound="path"):
    """Replay of the two-round rule on the oracle's exact keys (see the module docstring).  bound="path"
    (exact extraction, the default): LB(c) = pow(d, lambda) * max_i lightest_i(c); bound="weight"
    (literal extraction with central blocking): LB(c) = pow(d, lambda) * w_c."""
    nc = len(o.centrals)
    kk = min(k, nc)
    mcap = min(KGS_MAX_K, max(8 * kk, pmin))
    if nc <= mcap:
        return nc
    C = o.centrals.tolist()
    if bound == "path":
        mw = lightest_paths(g, kw, o)
        lbw = [float(mw[c].max()) / (1 << 24) for c in C]
    else:
        lbw = [float(g.weight[c]) for c in C]
    lb = [math.pow(float(d), lam) * x for x, d in zip(lbw, o.central_depth.tolist())]
    keys = o.central_key.tolist()
    assert all(x <= y for x, y in zip(lb, keys)), "the bound must not exceed the exact key"
    ids = o.centrals.tolist()
    order = sorted(range(nc), key=lambda i: (lb[i], ids[i]))
    first = order[:mcap]
    B = (lb[first[-1]], ids[first[-1]])
    T = sorted((keys[i], ids[i]) for i in first)[kk - 1]
    if not B < T:
        return mcap
    return mcap + sum(1 for i in order[mcap:] if (lb[i], ids[i]) < T)


CASES = [  # seed, graph kwargs, k, lambda, round-1 minimum, extract mode, prune mode
    (1, dict(), 20, 0.2, 512, 0, 1),                                            # |C| 35: no pruning
    (6, dict(q=4, kw_size=250, deg=6), 300, 0.2, 512, 0, 2),                    # 1044 <= 8k: no pruning
    (2, dict(n=20000, deg=16, q=3, kw_size=20, wpow=4.0), 20, 0.2, 512, 0, 1),  # w_c bound, round 2
    (12, dict(n=20000, deg=16, q=3, kw_size=20, wpow=4.0), 5, 0.2, 64, 0, 1),   # w_c bound
    (12, dict(n=20000, deg=16, q=3, kw_size=20, wpow=4.0), 20, 0.2, 512, 0, 2), # path bound: 1078 -> 512
    (10, dict(n=20000, deg=16, q=3, kw_size=20, zero_frac=0.9), 300, 0.0, 512, 0, 2),  # 16574 -> 2400
    (2, dict(n=20000, deg=16, q=3, kw_size=20, wpow=4.0), 20, 0.2, 1, 0, 2),    # 4239 -> 268: round 2
    (12, dict(n=20000, deg=16, q=3, kw_size=20, wpow=4.0), 20, 0.2, 1, 0, 2),   # 1078 -> 160
    (2, dict(n=20000, deg=16, q=3, kw_size=20, wpow=4.0), 20, 0.2, 512, 1, 2),  # literal: falls back to w_c
    (12, dict(n=20000, deg=16, q=3, kw_size=20, wpow=4.0), 5, 0.2, 64, 1, 1),   # literal, w_c bound
]


def _outcome(exp, nc, mcap):
    return "none" if nc <= mcap else ("round1" if exp == mcap else "round2")


def test_pruned_answers_and_evaluated_counts():
    _gpu()
    outcomes = set()
    for seed, kwargs, k, lam, pmin, ext, mode in CASES:
        g = medium_graph(seed, **kwargs)
        G = kgs.kgs_load_graph(g)
        kw = list(range(len(g.kw_ptr) - 1))
        o = oracle.query(g, kw, k, lam=lam, extract_mode=ext)
        ctx = f"seed={seed} k={k} lam={lam} pmin={pmin} ext={ext} mode={mode} |C|={len(o.centrals)}"
        for prune in (mode, 0):
            r = kgs.kgs_query(G, kw, k, kgs.make_params(lam=lam, prune=prune, extract_mode=ext, prune_min=pmin))
            assert r.stats["n_centrals"] == len(o.centrals), ctx
            assert [a.central for a in r.answers] == [a.central for a in o.answers], (ctx, prune)
            for ra, oa in zip(r.answers, o.answers):
                assert ra.score_key == oa.key and ra.depth == oa.depth, (ctx, prune)
                assert ra.nodes.tolist() == oa.nodes.tolist(), (ctx, prune)
                assert ra.arcs.tolist() == oa.arcs.tolist(), (ctx, prune)
            if prune:
                exp = expected_evaluated(g, o, k, lam, kw, pmin, "path" if (ext == 0 and mode == 2) else "weight")
                assert r.stats["n_evaluated"] == exp, (ctx, exp)
                nc = len(o.centrals)
                outcomes.add((mode, _outcome(exp, nc, min(KGS_MAX_K, max(8 * min(k, nc), pmin)))))
            else:
                assert r.stats["n_evaluated"] == len(o.centrals), ctx
        G.close()
    assert {(1, "round2"), (2, "round1"), (2, "round2")} <= outcomes, outcomes


def test_batch_pruned_matches_oracle():
    """The batch engine (several groups) prunes per query with the same result, in both bound modes;
    a mode-2 batch followed by a mode-1 batch checks that the lightest-path rows are reset."""
    _gpu()
    g = medium_graph(10, n=20000, deg=16, q=3, kw_size=20, zero_frac=0.9)
    G = kgs.kgs_load_graph(g)
    rng = np.random.default_rng(3)
    qs = [sorted(rng.choice(3, size=int(rng.integers(2, 4)), replace=False).tolist()) for _ in range(12)]
    for mode in (2, 1, 2):
        for k in (1, 20, 64):
            exp = [oracle.query(g, kw, k) for kw in qs]
            res = kgs.kgs_query_batch(G, qs, k, kgs.make_params(prune=mode), 4)
            for kw, r, o in zip(qs, res, exp):
                assert [a.central for a in r.answers] == [a.central for a in o.answers], (kw, k, mode)
                assert [a.score_key for a in r.answers] == [a.key for a in o.answers], (kw, k, mode)
                bound = "path" if mode == 2 else "weight"
                assert r.stats["n_evaluated"] == expected_evaluated(g, o, k, 0.2, kw, 512, bound), (kw, k, mode)
    G.close()


def test_key_cutoff_in_round_two():
    """Round 2 stops a candidate's extraction once its closure weight times d^lambda exceeds the k-th
    exact key (kgs_stats.n_cut).  Valid when level-cover must keep every source: no node holds two query
    keywords (disjoint keyword sets here), or level_cover = 0.  Answers must be the oracle's."""
    _gpu()
    cuts = 0
    for seed, deg, k in ((0, 16, 5), (0, 16, 20), (1, 16, 5), (1, 16, 20), (0, 8, 50)):
        rng = np.random.default_rng(500 + seed)
        n, q = 6000, 3
        g0 = medium_graph(500 + seed, n=n, deg=deg, q=q, kw_size=10, wpow=3.0)
        perm = rng.permutation(n)
        kws = [sorted(perm[i * 100:(i + 1) * 100].tolist()) for i in range(q)]   # disjoint
        edges = [(u, int(v)) for u in range(n) for v in g0.col_idx[g0.row_ptr[u]:g0.row_ptr[u + 1]] if u < v]
        g = synth.from_edges(n, edges, g0.weight, kws, 2.0)
        G = kgs.kgs_load_graph(g)
        kw = list(range(q))
        for lc in (1, 0):
            o = oracle.query(g, kw, k, level_cover=lc)
            r = kgs.kgs_query(G, kw, k, kgs.make_params(prune=1, level_cover=lc, prune_min=40))
            ctx = f"seed={seed} deg={deg} k={k} lc={lc} |C|={len(o.centrals)}"
            assert [a.central for a in r.answers] == [a.central for a in o.answers], ctx
            for ra, oa in zip(r.answers, o.answers):
                assert ra.score_key == oa.key and ra.nodes.tolist() == oa.nodes.tolist(), ctx
                assert ra.arcs.tolist() == oa.arcs.tolist(), ctx
            cuts += r.stats["n_cut"]
        G.close()
    assert cuts > 0


def test_key_cutoff_per_candidate_multi_keyword_sources():
    """A few nodes hold two query keywords, so graph-wide level-cover could keep only some sources
    (s* >= 2) and the query-wide test switches the cut-off off.  The test is made per candidate — from the
    search's rm bits (keywords 0-6), and from mk_reach's fixpoint over the shared DAG when mk_min allows:
    the keywords for which a two-keyword node reaches c inside DAG_i(c); where they cannot cover Q with
    zb(c), every source is kept and the cut-off applies.  The candidates near the two-keyword nodes (small
    pruned graphs, the likely winners) must still get their exact keys: answers equal the oracle's with
    mk_reach on (mk_min = 0) and off, with the lazy round-2 DAG and without, in latency mode (recorded DAG
    and pre-pass) and in a batch; with literal extraction (no rm) and mk_reach off nothing is cut."""
    _gpu()
    cuts_on = cuts_off = 0
    for seed, deg, k, n_multi in ((0, 16, 5, 3), (1, 16, 20, 10), (2, 8, 20, 30), (3, 16, 50, 6)):
        rng = np.random.default_rng(900 + seed)
        n, q = 6000, 3
        g0 = medium_graph(900 + seed, n=n, deg=deg, q=q, kw_size=10, wpow=3.0)
        perm = rng.permutation(n)
        kws = [perm[i * 100:(i + 1) * 100].tolist() for i in range(q)]
        for j in range(n_multi):   # node holding keywords i and i+1 (every pair, so they cover Q)
            i = j % q
            kws[(i + 1) % q].append(kws[i][j // q])
        kws = [sorted(set(x)) for x in kws]
        edges = [(u, int(v)) for u in range(n) for v in g0.col_idx[g0.row_ptr[u]:g0.row_ptr[u + 1]] if u < v]
        g = synth.from_edges(n, edges, g0.weight, kws, 2.0)
        G = kgs.kgs_load_graph(g)
        kw = list(range(q))
        o = oracle.query(g, kw, k)
        ctx0 = f"seed={seed} deg={deg} k={k} multi={n_multi} |C|={len(o.centrals)}"
        runs = []
        for mk in (0, 1 << 30):
            for lz in (1, 0):
                for rec, rmax in ((1, 1 << 22), (1, 0), (0, 1 << 22)):
                    p = kgs.make_params(prune=1, prune_min=40, mk_min=mk, dag_record=rec, lazy_dag=lz, rec_max=rmax)
                    runs.append((f"mk={mk} lazy={lz} rec={rec} rec_max={rmax}", kgs.kgs_query(G, kw, k, p), mk))
                p = kgs.make_params(prune=1, prune_min=40, mk_min=mk, lazy_dag=lz)
                for j, r in enumerate(kgs.kgs_query_batch(G, [kw, kw[::-1], kw], k, p, 3)):
                    runs.append((f"mk={mk} lazy={lz} batch {j}", r, mk))
        for tag, r, mk in runs:
            ctx = f"{ctx0} {tag}"
            assert [a.central for a in r.answers] == [a.central for a in o.answers], ctx
            for ra, oa in zip(r.answers, o.answers):
                assert ra.score_key == oa.key and ra.nodes.tolist() == oa.nodes.tolist(), ctx
                assert ra.arcs.tolist() == oa.arcs.tolist(), ctx
            if mk == 0:
                cuts_on += r.stats["n_cut"]
        # literal extraction: no rm (its DAG is not the hitting arcs), mk_reach off -> the query-wide test
        ol = oracle.query(g, kw, k, extract_mode=oracle.EXTRACT_LITERAL)
        r = kgs.kgs_query(G, kw, k, kgs.make_params(prune=1, prune_min=40, mk_min=1 << 30,
                                                    extract_mode=kgs.KGS_EXTRACT_LITERAL))
        assert [a.central for a in r.answers] == [a.central for a in ol.answers], ctx0
        cuts_off += r.stats["n_cut"]
        G.close()
    assert cuts_off == 0 and cuts_on > 0, (cuts_on, cuts_off)


def test_deferred_queries_run_on_the_whole_grid():
    """In a launch of query groups, a query with more than defer_min central nodes is left to the end of
    the launch, where every CTA answers it as one group (kgs_stats.group == n_groups).  Answers equal the
    oracle's with deferral on (several deferred queries, mixed with ordinary ones) and off, and a later
    single-query launch on the same workspaces is unaffected."""
    _gpu()
    g = medium_graph(21, n=20000, deg=8, q=4, kw_size=150)
    G = kgs.kgs_load_graph(g)
    rng = np.random.default_rng(21)
    qs = [sorted(rng.choice(4, size=int(rng.integers(2, 5)), replace=False).tolist()) for _ in range(24)]
    exp = {tuple(kw): oracle.query(g, kw, 20) for kw in map(tuple, qs)}
    ncs = sorted(len(o.centrals) for o in exp.values())
    thr = ncs[len(ncs) // 2]   # about half of the queries are deferred
    for dmin, groups in ((thr, 4), (thr, 8), (0, 4), (1, 3)):
        res = kgs.kgs_query_batch(G, qs, 20, kgs.make_params(defer_min=dmin), groups)
        deferred = 0
        for kw, r in zip(qs, res):
            o = exp[tuple(kw)]
            ctx = f"defer_min={dmin} G={groups} kw={kw} |C|={len(o.centrals)}"
            assert [a.central for a in r.answers] == [a.central for a in o.answers], ctx
            for ra, oa in zip(r.answers, o.answers):
                assert ra.score_key == oa.key and ra.nodes.tolist() == oa.nodes.tolist(), ctx
                assert ra.arcs.tolist() == oa.arcs.tolist(), ctx
            assert r.stats["stop_reason"] == o.stop_reason and r.stats["levels"] == o.levels, ctx
            should = dmin > 0 and len(o.centrals) > dmin
            assert (r.stats["group"] == groups) == should, ctx
            deferred += should
        if dmin:
            assert deferred > 0
    r = kgs.kgs_query(G, qs[0], 20)
    assert [a.central for a in r.answers] == [a.central for a in exp[tuple(qs[0])].answers]
    G.close()


@pytest.mark.parametrize("q", [3, 8])
def test_key_cutoff_never_drops_a_two_level_winner(q):
    """Hand-built: the Central Graph that must win keeps only two-keyword sources (s* = 2), while its whole
    closure is heavy.  Keywords 0..q-1, every activation level 0 (A = 0.1).  Candidate c (w 0.5) is joined
    to two-keyword nodes of weight 0 that cover Q (q = 3: m1 holds 0, 1 and m2 holds 1, 2; q = 8: the pairs
    (0, 1), (2, 3), (4, 5), (6, 7) — keyword 7 has no rm bit) and to 20 nodes of each keyword of weight
    0.9: level-cover keeps c and the two-keyword nodes, key 0.5, while the closure weighs 0.5 + 18 q.  60
    filler centrals (w 0.01, one heavy neighbour per keyword, key 0.01 + 0.9 q) fill pruning round 1
    (prune_min 8: the 8k = 40 smallest bounds), so c is extracted in round 2 with the cut at T = the 5th
    key: an invalid cut would drop it.  Answers must be the oracle's (c first), lazy DAG on and off."""
    _gpu()
    n_fill, n_side = 60, 20
    nodes = {}

    def nid(name):
        return nodes.setdefault(name, len(nodes))

    edges, kws, w = [], [[] for _ in range(q)], {}
    c = nid("c")
    w[c] = 0.5
    pairs = [(0, 1), (1, 2)] if q == 3 else [(0, 1), (2, 3), (4, 5), (6, 7)]
    multi = []
    for j, (i1, i2) in enumerate(pairs):
        m = nid(f"m{j}")
        w[m] = 0.0
        kws[i1].append(m)
        kws[i2].append(m)
        edges.append((c, m))
        multi.append(m)
    for i in range(q):
        for j in range(n_side):
            v = nid(f"s{i}_{j}")
            w[v] = 0.9
            kws[i].append(v)
            edges.append((c, v))
    for f in range(n_fill):
        fv = nid(f"f{f}")
        w[fv] = 0.01
        for i in range(q):
            v = nid(f"f{f}_{i}")
            w[v] = 0.9
            kws[i].append(v)
            edges.append((fv, v))
    n = len(nodes)
    wt = np.array([w[i] for i in range(n)], dtype=np.float64)
    wt = (np.floor(wt * (1 << 24) + 0.5) / (1 << 24)).astype(np.float32)
    g = synth.from_edges(n, edges, wt, [sorted(x) for x in kws], 0.1)
    kw = list(range(q))
    o = oracle.query(g, kw, 5)
    assert o.answers[0].central == c and o.answers[0].nodes.tolist() == sorted([c] + multi)
    G = kgs.kgs_load_graph(g)
    runs = []
    for mk in (0, 1 << 30):
        for lz in (1, 0):
            for rec, rmax in ((1, 1 << 22), (1, 0), (0, 1 << 22)):   # rec_max 0: the record is dropped
                runs.append((mk, f"{rec} rec_max={rmax} lazy={lz}", kgs.kgs_query(G, kw, 5, kgs.make_params(
                    prune_min=8, mk_min=mk, dag_record=rec, lazy_dag=lz, rec_max=rmax))))
            for r in kgs.kgs_query_batch(G, [kw, kw[::-1]], 5,
                                         kgs.make_params(prune_min=8, mk_min=mk, lazy_dag=lz), 2):
                runs.append((mk, f"batch lazy={lz}", r))
    for mk, rec, r in runs:
        ctx = f"q={q} mk_min={mk} rec={rec}"
        assert [a.central for a in r.answers] == [a.central for a in o.answers], ctx
        for ra, oa in zip(r.answers, o.answers):
            assert ra.score_key == oa.key and ra.nodes.tolist() == oa.nodes.tolist(), ctx
    G.close()
