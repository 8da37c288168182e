"""NEXT-3 semantics variants on the GPU against the oracle: the "contains" reading of level-cover
(kgs_params.level_cover = 2, reading R13b) and containment removal (kgs_params.containment = 1, P:L712,
reading R16), single queries and batches, bit-exact answers."""
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


def _same(r, o, ctx):
    assert r.stats["levels"] == o.levels and r.stats["stop_reason"] == o.stop_reason, ctx
    assert [a.central for a in r.answers] == [a.central for a in o.answers], ctx
    for ra, oa in zip(r.answers, o.answers):
        assert ra.score_key == oa.key and ra.depth == oa.depth, ctx
        assert ra.nodes.tolist() == oa.nodes.tolist() and ra.arcs.tolist() == oa.arcs.tolist(), ctx


def test_contains_reading_hand_example():
    _gpu()
    g = synth.from_edges(7, [(0, 3), (1, 2), (2, 0), (5, 6), (6, 0)], [0.1, 0, 0, 0, 0, 0, 0],
                         [[0], [1, 5], [1, 3]], 2.0)
    G = kgs.kgs_load_graph(g)
    r1 = kgs.kgs_query(G, [0, 1, 2], 1, kgs.make_params(level_cover=1))
    r2 = kgs.kgs_query(G, [0, 1, 2], 1, kgs.make_params(level_cover=2))
    assert r1.answers[0].nodes.tolist() == [0, 1, 2, 3, 5, 6]
    assert r2.answers[0].nodes.tolist() == [0, 1, 2] and r2.answers[0].arcs.tolist() == [[1, 2], [2, 0]]
    G.close()


def test_random_graphs_variants():
    _gpu()
    rng = np.random.default_rng(303)
    removed = 0
    for case in range(100):
        n = int(rng.integers(5, 60))
        q = int(rng.integers(2, 5))
        g = R.random_graph(rng, n, float(rng.uniform(0.05, 0.35)), bool(case % 3 == 0), q, kw_size=(1, 4),
                           wmax=float(rng.choice([0.0, 0.2, 1.0])))
        G = kgs.kgs_load_graph(g, relabel=bool(case % 2))
        kw = list(range(q))
        for lc, cont in ((2, 0), (1, 1), (2, 1), (0, 1)):
            k = int(rng.choice([1, 3, 6]))
            o = oracle.query(g, kw, k, level_cover=lc, containment=cont)
            r = kgs.kgs_query(G, kw, k, kgs.make_params(level_cover=lc, containment=cont))
            _same(r, o, (case, lc, cont, k))
            if cont:
                removed += len(oracle.query(g, kw, k, level_cover=lc).answers) != len(o.answers) or \
                    [a.central for a in oracle.query(g, kw, k, level_cover=lc).answers] != [a.central for a in o.answers]
        G.close()
    assert removed > 5


def test_c1_c2_variants_batch_and_single():
    _gpu()
    for name, count in (("C1", 40), ("C2", 12)):
        w = synth.make_workload(name)
        G = kgs.kgs_load_graph(w.graph)
        qs = w.queries[:count] if name == "C1" else w.queries[::25][:count]
        for lc, cont in ((2, 0), (1, 1), (2, 1)):
            p = kgs.make_params(level_cover=lc, containment=cont)
            exp = [oracle.query(w.graph, kw, w.k, level_cover=lc, containment=cont) for kw in qs]
            for groups in (1, 4):
                res = kgs.kgs_query_batch(G, qs, w.k, p, groups)
                for kw, r, o in zip(qs, res, exp):
                    _same(r, o, (name, lc, cont, groups, kw))
            for kw, o in zip(qs[:5], exp[:5]):
                _same(kgs.kgs_query(G, kw, w.k, p), o, (name, lc, cont, "single", kw))
        G.close()
