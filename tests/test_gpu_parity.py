"""CUDA path (through the C-ABI) vs the oracle, element by element on the same seeded inputs.

Bit-exact: activation levels a, the hitting-level matrix M, the central set with depths, every
central's Eq. 6 key, the ranked top-k ids, the answer subgraphs, stop level / reason.  fp32 scores
must agree within 1e-5 relative (BASELINE.json north_star); they are in fact identical because the
fp64 keys are exact (reading R15), and the test checks both.
"""
import numpy as np
import pytest

import oracle
import refimpl as R
import synth

pytestmark = pytest.mark.gpu

kgs = pytest.importorskip("paper_conf_icde_yangajtw19_b200")


def _gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def compare(G, g, kw, k, *, alpha=0.1, lam=0.2, max_depth=254, block_central=1, extract_mode=0,
            level_cover=1, full=True):
    o = oracle.query(g, kw, k, alpha=alpha, lam=lam, max_depth=max_depth, block_central=block_central,
                     extract_mode=extract_mode, level_cover=level_cover)
    p = kgs.make_params(alpha=alpha, lam=lam, max_depth=max_depth, block_central=block_central,
                        extract_mode=extract_mode, level_cover=level_cover, want_levels=1 if full else 0)
    r = kgs.kgs_query(G, kw, k, p)
    assert o.status == 0
    ctx = f"kw={list(kw)} k={k} alpha={alpha} lam={lam} md={max_depth} blk={block_central} ext={extract_mode} lc={level_cover}"
    if full:
        assert (r.a == o.a).all(), ctx
        bad = np.argwhere(r.M != o.M)
        assert bad.size == 0, f"{ctx}: M differs at {bad[:5].tolist()} gpu={r.M[tuple(bad[0])]} ora={o.M[tuple(bad[0])]}"
        assert r.centrals.tolist() == o.centrals.tolist(), ctx
        assert r.central_depth.tolist() == o.central_depth.tolist(), ctx
        assert r.central_key.tolist() == o.central_key.tolist(), ctx
    assert r.stats["stop_reason"] == o.stop_reason, ctx
    if o.stop_reason != oracle.STOP_EMPTY_KEYWORD:
        assert r.stats["levels"] == o.levels, ctx
    assert r.stats["n_centrals"] == len(o.centrals), ctx
    assert len(r.answers) == len(o.answers), ctx
    for ra, oa in zip(r.answers, o.answers):
        assert ra.central == oa.central and ra.depth == oa.depth, ctx
        assert ra.score_key == oa.key, ctx
        assert ra.score == oa.score and abs(ra.score - oa.score) <= 1e-5 * max(abs(oa.score), 1e-30), ctx
        assert ra.nodes.tolist() == oa.nodes.tolist(), ctx
        assert ra.arcs.tolist() == oa.arcs.tolist(), ctx
    return r, o


def test_golden_examples():
    _gpu()
    d = R.load_golden("fig2_examples_1_3.json")
    g = R.golden_graph(d)
    G = kgs.kgs_load_graph(g)
    for c in d["cases"]:
        for lc in (0, 1):
            r, _ = compare(G, g, d["query"], c["k"], alpha=d["alpha"], block_central=c["block_central"], level_cover=lc)
            assert r.M.tolist() == c["M"]
    for name in ("fig4_example_4.json", "fig5_example_5.json"):
        d = R.load_golden(name)
        g = R.golden_graph(d)
        G = kgs.kgs_load_graph(g)
        r, _ = compare(G, g, d["query"], d["k"], alpha=d["alpha"], lam=d["lambda"])
        assert r.M.tolist() == d["M"]
        assert r.answers[0].nodes.tolist() == d["answer"]["nodes"]
    d = R.load_golden("fig4_example_4.json")
    assert r is not None


def test_random_small_graphs_all_modes():
    _gpu()
    rng = np.random.default_rng(2024)
    for case in range(160):
        n = int(rng.integers(4, 70))
        directed = bool(rng.random() < 0.4)
        q = int(rng.integers(1, 9))
        g = R.random_graph(rng, n, float(rng.uniform(0.03, 0.3)), directed, q, kw_size=(1, 5),
                           wmax=float(rng.choice([0.0, 0.2, 1.0])))
        G = kgs.kgs_load_graph(g, relabel=bool(case % 2))   # internal degree order or input order
        kw = list(range(q))
        for _ in range(3):
            compare(G, g, kw, int(rng.choice([1, 2, 5, 40])), alpha=float(rng.choice([0.05, 0.1, 0.4])),
                    lam=float(rng.choice([0.0, 0.2, 1.0])), max_depth=int(rng.choice([1, 3, 254])),
                    block_central=int(rng.integers(0, 2)), extract_mode=int(rng.integers(0, 2)),
                    level_cover=int(rng.integers(0, 2)))
        G.close()


def test_c1_all_queries():
    """Config C1 (BASELINE.json configs[0]): 100 three-keyword queries, top-5, with the internal degree
    order (default) and with the input order (KGS_NO_RELABEL)."""
    _gpu()
    w = synth.make_workload("C1")
    for relabel in (True, False):
        G = kgs.kgs_load_graph(w.graph, relabel=relabel)
        for kw in w.queries:
            compare(G, w.graph, kw, w.k)
        G.close()


def test_c2_queries_and_state_reuse():
    """Config C2 (1M nodes / 8M edges, 2-4 keywords, top-20): sampled queries; the workspace is reused
    across queries (sparse reset) and alpha changes in between, so stale state would show."""
    _gpu()
    w = synth.make_workload("C2")
    G = kgs.kgs_load_graph(w.graph)
    qs = w.queries[::10]
    for j, kw in enumerate(qs):
        compare(G, w.graph, kw, w.k, alpha=0.4 if j % 7 == 3 else 0.1, full=(j % 3 == 0))
    # determinism (Thm. V.2): same query twice, interleaved with another one
    r1 = kgs.kgs_query(G, qs[0], w.k)
    kgs.kgs_query(G, qs[1], w.k)
    r2 = kgs.kgs_query(G, qs[0], w.k)
    assert [(a.central, a.score_key) for a in r1.answers] == [(a.central, a.score_key) for a in r2.answers]


def test_ragged_and_degenerate():
    """Empty keyword set, q = 1, k > |C|, a node containing all keywords, max_depth truncation,
    isolated nodes and a graph whose size is not a multiple of any tile."""
    _gpu()
    g = synth.from_edges(7, [(0, 1), (1, 2), (2, 3), (4, 5)], [0.5, 0, 0, 0, 0, 0, 0.25],
                         [[0, 2], [2], [], [6], [3, 5]], 2.0)
    G = kgs.kgs_load_graph(g)
    compare(G, g, [0], 5)
    compare(G, g, [0, 1], 1)
    compare(G, g, [0, 2], 3)
    compare(G, g, [0, 3], 3)
    compare(G, g, [1, 4], 100)
    compare(G, g, [0, 4], 100, max_depth=1)
    with pytest.raises(kgs.KgsError):
        kgs.kgs_query(G, [0, 0], 1)
    with pytest.raises(kgs.KgsError):
        kgs.kgs_query(G, [0], 0)
    with pytest.raises(kgs.KgsError):
        kgs.kgs_query(G, [99], 1)


def test_device_resident_path():
    """kgs_query_device (keyword ids already in HBM) + kgs_query_fetch give the same answers."""
    _gpu()
    import torch
    w = synth.make_workload("C1")
    G = kgs.kgs_load_graph(w.graph)
    for kw in w.queries[:10]:
        t = torch.tensor(kw, dtype=torch.int32, device="cuda")
        s = torch.cuda.current_stream().cuda_stream
        kgs.kgs_query_device(G, t.data_ptr(), len(kw), w.k, None, s)
        r = kgs.kgs_query_fetch(G, len(kw), 0, s)
        o = oracle.query(w.graph, kw, w.k)
        assert [a.central for a in r.answers] == [a.central for a in o.answers]
        assert [a.score_key for a in r.answers] == [a.key for a in o.answers]


def test_batch_engine_groups():
    """kgs_query_batch: one engine launch, queries spread over G groups of CTAs; every query's answers
    equal the oracle's whatever G is (C1 all queries, C2 a sample, mixed q)."""
    _gpu()
    for name, count in (("C1", 100), ("C2", 40)):
        w = synth.make_workload(name)
        G = kgs.kgs_load_graph(w.graph)
        qs = w.queries[:count] if name == "C1" else w.queries[::max(1, len(w.queries) // count)][:count]
        exp = [oracle.query(w.graph, kw, w.k) for kw in qs]
        for groups in (1, 3, 8, 64):
            res = kgs.kgs_query_batch(G, qs, w.k, None, groups)
            for kw, r, o in zip(qs, res, exp):
                assert r.stats["stop_reason"] == o.stop_reason and r.stats["levels"] == o.levels, (name, groups, kw)
                assert [a.central for a in r.answers] == [a.central for a in o.answers], (name, groups, kw)
                for ra, oa in zip(r.answers, o.answers):
                    assert ra.score_key == oa.key and ra.nodes.tolist() == oa.nodes.tolist()
                    assert ra.arcs.tolist() == oa.arcs.tolist()
        G.close()


def test_batch_device_invalid_queries():
    """kgs_query_batch_device validates on the device: bad ids / repeated ids / bad q are reported per
    query (KGS_STOP_INVALID_QUERY) and do not disturb the valid queries of the batch."""
    _gpu()
    import torch
    w = synth.make_workload("C1")
    G = kgs.kgs_load_graph(w.graph)
    good = [list(q) for q in w.queries[:6]]
    rows = [good[0], [0, 0, 1], good[1], [w.graph.n_keywords + 5, 1, 2], good[2], [1] * 9]
    ql = [len(r) for r in rows]
    kwp = torch.full((len(rows), 8), -1, dtype=torch.int32)
    for i, r in enumerate(rows):
        kwp[i, :min(8, len(r))] = torch.tensor(r[:8], dtype=torch.int32)
    kwd = kwp.cuda()
    qld = torch.tensor(ql, dtype=torch.int32, device="cuda")
    s = torch.cuda.current_stream().cuda_stream
    kgs.kgs_query_batch_device(G, len(rows), kwd.data_ptr(), qld.data_ptr(), w.k, None, 2, s)
    res = kgs.kgs_query_batch_fetch(G, [min(8, x) for x in ql], s)
    for i in (1, 3, 5):
        assert res[i].stats["stop_reason"] == kgs.KGS_STOP_INVALID_QUERY and res[i].answers == []
    for i, gi in ((0, 0), (2, 1), (4, 2)):
        o = oracle.query(w.graph, good[gi], w.k)
        assert [a.central for a in res[i].answers] == [a.central for a in o.answers]


def test_huge_central_graph_tier4():
    """A Central Graph beyond the per-CTA arena (64 K nodes): a hub c joined to 150 000 nodes holding
    keyword 0 and to one node holding keyword 1 — G(c) has 150 002 nodes, so extraction and emit reach
    the per-group tier-4 arena; latency mode (recorded DAG) and query groups (pre-pass)."""
    _gpu()
    n0 = 150_000
    a, c = n0, n0 + 1
    edges = [(v, c) for v in range(n0)] + [(a, c)]
    g = synth.from_edges(n0 + 2, edges, [0.0] * (n0 + 2), [list(range(n0)), [a]], 2.0)
    G = kgs.kgs_load_graph(g)
    r, o = compare(G, g, [0, 1], 1)
    assert len(r.answers) == 1 and r.answers[0].central == c and len(r.answers[0].nodes) == n0 + 2
    res = kgs.kgs_query_batch(G, [[0, 1], [1, 0], [0, 1]], 1, None, 3)
    for rr in res:
        assert rr.answers[0].central == c and rr.answers[0].nodes.tolist() == o.answers[0].nodes.tolist()
        assert rr.answers[0].arcs.tolist() == o.answers[0].arcs.tolist()
    G.close()


def test_batch_capacity_overflow_is_per_query():
    """A query that exceeds an internal capacity (here the predecessor-arc regions, shrunk to 64 K arcs
    with kgs_graph_desc.pred_arc_cap, against a Central Graph of 150 000 predecessor arcs) is reported per query in a
    batch (KGS_STOP_CAPACITY, no answers); the other queries of the batch keep their exact answers.
    A single kgs_query reports KGS_EINTERNAL."""
    _gpu()
    n0 = 150_000
    a, c = n0, n0 + 1
    g = synth.from_edges(n0 + 2, [(v, c) for v in range(n0)] + [(a, c)], [0.0] * (n0 + 2),
                         [list(range(n0)), [a]], 2.0)
    G = kgs.kgs_load_graph(g, pred_arc_cap=1 << 16)
    qs = [[0, 1], [1], [1, 0], [1]]
    res = kgs.kgs_query_batch(G, qs, 1, None, 2)
    assert [r.stats["stop_reason"] for r in res] == [kgs.KGS_STOP_CAPACITY, kgs.KGS_STOP_K] * 2
    for kw, r in zip(qs, res):
        if kw == [1]:
            o = oracle.query(g, kw, 1)
            assert [(x.central, x.score_key, x.nodes.tolist()) for x in r.answers] == \
                [(x.central, x.key, x.nodes.tolist()) for x in o.answers]
        else:
            assert r.answers == []
    with pytest.raises(kgs.KgsError):
        kgs.kgs_query(G, [0, 1], 1)
    G.close()


def test_level_ring_resizing_across_alpha_and_groups():
    """The level-slot ring has R = amax + 2 slots and amax depends on alpha when the largest weight is
    below 1: a G = 1 query at alpha 0.05 (R = 7), then a G = 8 batch at alpha 0.4 (R = 5, new group
    workspaces), then both again.  Every workspace must hold the largest ring (an undersized one would be
    written out of bounds); every answer must equal the oracle's."""
    _gpu()
    w = synth.make_workload("C1")
    g = w.graph
    g.weight = (np.asarray(g.weight, np.float64) * 0.3).astype(np.float32)
    G = kgs.kgs_load_graph(g)
    qs = w.queries[:24]
    for rnd in range(2):
        for alpha, groups in ((0.05, 1), (0.4, 8), (0.05, 8), (0.4, 1)):
            exp = [oracle.query(g, kw, w.k, alpha=alpha) for kw in qs]
            p = kgs.make_params(alpha=alpha)
            res = kgs.kgs_query_batch(G, qs, w.k, p, groups) if groups > 1 else [kgs.kgs_query(G, kw, w.k, p) for kw in qs]
            for kw, r, o in zip(qs, res, exp):
                ctx = (rnd, alpha, groups, kw)
                assert r.stats["levels"] == o.levels and r.stats["stop_reason"] == o.stop_reason, ctx
                assert [(a.central, a.score_key) for a in r.answers] == [(a.central, a.key) for a in o.answers], ctx
    G.close()


def test_batch_modes_across_launches():
    """The non-default top-down sources in query groups — the recorded DAG (dag_record = 1) and the
    search-only analysis mode — over consecutive launches on the same workspaces: every launch's stop
    level, |C| and (with answers) the answers must equal the oracle's."""
    _gpu()
    w = synth.make_workload("C2")
    G = kgs.kgs_load_graph(w.graph)
    qs = w.queries[::15][:20]
    exp = [oracle.query(w.graph, kw, w.k) for kw in qs]
    for params in (dict(dag_record=1), dict(search_only=1), dict(dag_record=0), dict(dag_record=1, prune=0)):
        p = kgs.make_params(**params)
        for launch in range(3):
            res = kgs.kgs_query_batch(G, qs, w.k, p, 8)
            for kw, r, o in zip(qs, res, exp):
                ctx = (params, launch, kw)
                assert r.stats["levels"] == o.levels and r.stats["stop_reason"] == o.stop_reason, ctx
                assert r.stats["n_centrals"] == len(o.centrals), ctx
                if not params.get("search_only"):
                    assert [(a.central, a.score_key) for a in r.answers] == [(a.central, a.key) for a in o.answers], ctx
                    for ra, oa in zip(r.answers, o.answers):
                        assert ra.nodes.tolist() == oa.nodes.tolist() and ra.arcs.tolist() == oa.arcs.tolist(), ctx
    G.close()
