"""Push / pull direction of the expansion (kgs_params.direction, the north star's "push/pull direction
switching") against the oracle, through the C-ABI.

Pull at every level computes the frontier-free level rule; after a level without
hits it recomputes whether Alg. 2's work list would still be non-empty, so M, the central set, depths,
keys, answers AND the stop level equal the oracle's literal form bit for bit whatever the direction.
The automatic switch (push first, pull from the first level whose active frontier has more than
m / pull_ratio out-arcs, kgs_params) is exercised mid-search with small thresholds.
"""
import os

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


def compare(G, g, kw, k, direction, *, alpha=0.1, lam=0.2, max_depth=254, block_central=1, extract_mode=0,
            level_cover=1, full=True, prune=1, pull_ratio=14, pull_min=1 << 22):
    p = kgs.make_params(alpha=alpha, lam=lam, max_depth=max_depth, block_central=block_central,
                        extract_mode=extract_mode, level_cover=level_cover, want_levels=1 if full else 0,
                        prune=prune, direction=direction, pull_ratio=pull_ratio, pull_min=pull_min)
    r = kgs.kgs_query(G, kw, k, p)
    pulled = r.stats["pull_level"] >= 0
    if direction == kgs.KGS_DIR_PULL:   # -1: stopped at level 0, before any expansion
        assert r.stats["pull_level"] == 0 or (r.stats["pull_level"] == -1 and r.stats["levels"] == 0)
    if direction == kgs.KGS_DIR_PUSH:
        assert not pulled
    o = oracle.query(g, kw, k, alpha=alpha, lam=lam, max_depth=max_depth, block_central=block_central,
                     extract_mode=extract_mode, level_cover=level_cover)
    ctx = f"kw={list(kw)} k={k} dir={direction} pulled_at={r.stats['pull_level']} blk={block_central} ext={extract_mode}"
    if full:
        assert (r.M == o.M).all(), ctx
        assert r.centrals.tolist() == o.centrals.tolist(), ctx
        assert r.central_depth.tolist() == o.central_depth.tolist(), ctx
        assert r.central_key.tolist() == o.central_key.tolist(), ctx
    assert r.stats["stop_reason"] == o.stop_reason, ctx
    if o.stop_reason != oracle.STOP_EMPTY_KEYWORD:
        assert r.stats["levels"] == o.levels, ctx
    assert len(r.answers) == len(o.answers), ctx
    for ra, oa in zip(r.answers, o.answers):
        assert ra.central == oa.central and ra.depth == oa.depth, ctx
        assert ra.score_key == oa.key and ra.score == oa.score, ctx
        assert ra.nodes.tolist() == oa.nodes.tolist(), ctx
        assert ra.arcs.tolist() == oa.arcs.tolist(), ctx
    return r


def test_golden_examples_pull():
    _gpu()
    d = R.load_golden("fig2_examples_1_3.json")
    g = R.golden_graph(d)
    G = kgs.kgs_load_graph(g)
    for c in d["cases"]:
        r = compare(G, g, d["query"], c["k"], kgs.KGS_DIR_PULL, alpha=d["alpha"], block_central=c["block_central"])
        assert r.M.tolist() == c["M"]
    for name in ("fig4_example_4.json", "fig5_example_5.json"):
        d = R.load_golden(name)
        g = R.golden_graph(d)
        G = kgs.kgs_load_graph(g)
        r = compare(G, g, d["query"], d["k"], kgs.KGS_DIR_PULL, alpha=d["alpha"], lam=d["lambda"])
        assert r.M.tolist() == d["M"]
        assert r.answers[0].nodes.tolist() == d["answer"]["nodes"]


def test_random_small_graphs_pull_and_switch():
    """Forced pull, forced push and the automatic switch at several thresholds, on random directed and
    undirected graphs with gates (weights), every extraction / blocking / pruning mode."""
    _gpu()
    rng = np.random.default_rng(77)
    switched = 0
    for case in range(120):
        n = int(rng.integers(4, 70))
        directed = bool(rng.random() < 0.4)
        q = int(rng.integers(1, 9))
        g = R.random_graph(rng, n, float(rng.uniform(0.03, 0.3)), directed, q, kw_size=(1, 5),
                           wmax=float(rng.choice([0.0, 0.2, 1.0])))
        G = kgs.kgs_load_graph(g, relabel=bool(case % 2))
        kw = list(range(q))
        for j in range(3):
            direction = (kgs.KGS_DIR_PULL, kgs.KGS_DIR_PUSH, kgs.KGS_DIR_AUTO)[j]
            ratio = int(rng.choice([1, 2, 4, 14]))
            r = compare(G, g, kw, int(rng.choice([1, 2, 5, 40])), direction, pull_ratio=ratio, pull_min=0,
                        alpha=float(rng.choice([0.05, 0.1, 0.4])), lam=float(rng.choice([0.0, 0.2, 1.0])),
                        max_depth=int(rng.choice([1, 3, 254])), block_central=int(rng.integers(0, 2)),
                        extract_mode=int(rng.integers(0, 2)), level_cover=int(rng.integers(0, 2)),
                        prune=int(rng.integers(0, 3)), full=bool(rng.random() < 0.7))
            switched += direction == kgs.KGS_DIR_AUTO and r.stats["pull_level"] > 0
        G.close()
    assert switched > 0   # some searches switched after at least one push level


def test_c1_c2_pull():
    """C1 (all queries) and a C2 sample with pull at every level; C2 also with the automatic switch."""
    _gpu()
    w = synth.make_workload("C1")
    G = kgs.kgs_load_graph(w.graph)
    for kw in w.queries:
        compare(G, w.graph, kw, w.k, kgs.KGS_DIR_PULL)
    G.close()
    w = synth.make_workload("C2")
    G = kgs.kgs_load_graph(w.graph)
    for j, kw in enumerate(w.queries[::25]):
        compare(G, w.graph, kw, w.k, (kgs.KGS_DIR_PULL, kgs.KGS_DIR_AUTO)[j % 2], full=(j % 3 == 0), pull_ratio=40,
                pull_min=0)
    G.close()


def test_batch_groups_pull():
    """The batch engine (query groups, predecessor pre-pass) with pull at every level."""
    _gpu()
    w = synth.make_workload("C1")
    G = kgs.kgs_load_graph(w.graph)
    qs = w.queries[:60]
    exp = [oracle.query(w.graph, kw, w.k) for kw in qs]
    p = kgs.make_params(direction=kgs.KGS_DIR_PULL)
    for groups in (1, 3, 8):
        res = kgs.kgs_query_batch(G, qs, w.k, p, groups)
        for kw, r, o in zip(qs, res, exp):
            assert r.stats["stop_reason"] == o.stop_reason and r.stats["levels"] == o.levels, (groups, kw)
            assert [a.central for a in r.answers] == [a.central for a in o.answers], (groups, kw)
            for ra, oa in zip(r.answers, o.answers):
                assert ra.score_key == oa.key and ra.nodes.tolist() == oa.nodes.tolist()
                assert ra.arcs.tolist() == oa.arcs.tolist()
    G.close()
