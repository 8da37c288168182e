"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

C3 (configs[2]: 2^25 nodes, 5.3e8 arcs): the bench's query order (fixed permutation), queries run
through kgs_query_device + kgs_query_fetch exactly as bench.py does, then the whole hitting-level
matrix M (n x q), the central set with depths and Eq. 6 keys, and the ranked answers with their
subgraphs are compared with the oracle element by element.  A sample of queries keeps the oracle
(seconds per query at this size) within a few minutes.
"""
import numpy as np
import pytest

import oracle
import synth

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

kgs = pytest.importorskip("paper_conf_icde_yangajtw19_b200")


@pytest.fixture(scope="module")
def c3():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    w = synth.make_workload("C3")
    G = kgs.kgs_load_graph(w.graph)
    order = np.random.default_rng(12345).permutation(len(w.queries))
    yield w, G, [w.queries[i] for i in order]
    G.close()


def _check(w, r, o, full=True):
    if full:
        assert np.array_equal(r.a, o.a)
        bad = np.argwhere(r.M != o.M)
        assert bad.size == 0, f"M differs at {bad[:5].tolist()}"
        assert r.centrals.tolist() == o.centrals.tolist()
        assert r.central_depth.tolist() == o.central_depth.tolist()
        assert r.central_key.tolist() == o.central_key.tolist()
    assert r.stats["stop_reason"] == o.stop_reason and r.stats["levels"] == o.levels
    assert [a.central for a in r.answers] == [a.central for a in o.answers]
    for ra, oa in zip(r.answers, o.answers):
        assert ra.depth == oa.depth and ra.score_key == oa.key and ra.score == oa.score
        assert ra.nodes.tolist() == oa.nodes.tolist() and ra.arcs.tolist() == oa.arcs.tolist()


def test_c3_bench_launch_configuration(c3):
    """The first timed bench queries, device-resident path (kgs_query_device + fetch)."""
    import torch
    w, G, qs = c3
    s = torch.cuda.current_stream().cuda_stream
    p = kgs.make_params(want_levels=1)
    for kw in qs[5:13]:
        t = torch.tensor(kw, dtype=torch.int32, device="cuda")
        kgs.kgs_query_device(G, t.data_ptr(), len(kw), w.k, p, s)
        r = kgs.kgs_query_fetch(G, len(kw), 1, s)
        _check(w, r, oracle.query(w.graph, kw, w.k))


def test_c3_every_query_size(c3):
    """One query of every size q = 2..8 through the host API (kgs_query)."""
    w, G, _ = c3
    seen = set()
    for kw in w.queries:
        if len(kw) in seen:
            continue
        seen.add(len(kw))
        r = kgs.kgs_query(G, kw, w.k, kgs.make_params(want_levels=1))
        _check(w, r, oracle.query(w.graph, kw, w.k))
    assert seen == set(range(2, 9))


def test_c5_stress_hubs():
    """C5 (configs[4]): C3 + 16 planted hubs of 2^21 arcs, 8 high-frequency keywords, top-100:
    exercises the big-node (grid-wide tile) expansion and the large candidate sets."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    w = synth.make_workload("C5")
    assert w.graph.meta["max_degree"] > (1 << 20)
    G = kgs.kgs_load_graph(w.graph)
    for kw in w.queries[:3]:
        r = kgs.kgs_query(G, kw, w.k, kgs.make_params(want_levels=1))
        _check(w, r, oracle.query(w.graph, kw, w.k))
    G.close()


def test_c3_pull_direction(c3):
    """Pull at every level (kgs_params.direction = KGS_DIR_PULL) at full size: the level-rule search over
    all 2^25 nodes with the hub in-arc tiles, against the oracle."""
    w, G, qs = c3
    for kw in qs[5:7]:
        r = kgs.kgs_query(G, kw, w.k, kgs.make_params(want_levels=1, direction=kgs.KGS_DIR_PULL))
        assert r.stats["pull_level"] == 0
        _check(w, r, oracle.query(w.graph, kw, w.k))
