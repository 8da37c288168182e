"""O2/O3 (bottom-up search) pinned against textbook BFS, gated earliest arrival, the fixpoint I3,
the two search forms (literal Alg. 2 vs level rule) and invariants I1-I6."""
import numpy as np
import pytest

import oracle
import refimpl as R

INF = 255


def _cases(seed, count, n_range=(6, 40)):
    rng = np.random.default_rng(seed)
    for _ in range(count):
        n = int(rng.integers(*n_range))
        directed = bool(rng.random() < 0.4)
        q = int(rng.integers(1, 5))
        p = float(rng.uniform(0.04, 0.25))
        yield R.random_graph(rng, n, p, directed, q, kw_size=(1, 3), wmax=float(rng.choice([0.0, 0.3, 1.0]))), q


def test_zero_activation_no_blocking_is_multisource_bfs():
    """a = 0 everywhere (all w = 0) and no central blocking: M[v][i] is the textbook BFS hop distance
    from T_i (search run to exhaustion with k > n)."""
    for g, q in _cases(11, 60):
        g.weight[:] = 0
        kw = list(range(q))
        r = oracle.query(g, kw, k=10 ** 6, block_central=0)
        assert r.status == 0
        assert (r.a == 0).all()
        adj = R.out_adj(g)
        for i, T in enumerate(R.keyword_sets(g, kw)):
            d = R.bfs_dist(g.n, adj, T)
            assert r.M[:, i].tolist() == d


def test_no_blocking_is_gated_earliest_arrival():
    """No central blocking: M[v][i] is the earliest arrival level under the activation gate
    (non-keyword nodes hit no earlier than a; every node sends no earlier than a)."""
    for g, q in _cases(12, 80):
        kw = list(range(q))
        r = oracle.query(g, kw, k=10 ** 6, block_central=0)
        adj = R.out_adj(g)
        Ts = R.keyword_sets(g, kw)
        K = set().union(*Ts)
        in_K = [v in K for v in range(g.n)]
        for i, T in enumerate(Ts):
            t = R.gated_earliest_arrival(g.n, adj, r.a, in_K, T)
            assert r.M[:, i].tolist() == [x if x <= 254 else INF for x in t]


@pytest.mark.parametrize("block", [0, 1])
def test_literal_equals_level_rule_and_fixpoint(block):
    """Literal Alg. 2 (FIdentifier work list) and the frontier-free level rule give the same M, C
    and depths; M satisfies the fixpoint characterisation I3 and invariants I1, I2, I4, I5, I6."""
    for g, q in _cases(13 + block, 120):
        kw = list(range(q))
        for k in (1, 2, 4, 10 ** 6):
            r1 = oracle.query(g, kw, k=k, block_central=block, bfs_form=oracle.BFS_LITERAL)
            r2 = oracle.query(g, kw, k=k, block_central=block, bfs_form=oracle.BFS_LEVEL_RULE)
            assert (r1.M == r2.M).all()
            assert r1.centrals.tolist() == r2.centrals.tolist()
            assert r1.central_depth.tolist() == r2.central_depth.tolist()
            M = r1.M
            Ts = R.keyword_sets(g, kw)
            K = set().union(*Ts)
            # I1
            for i, T in enumerate(Ts):
                assert set(np.nonzero(M[:, i] == 0)[0].tolist()) == T
            # I2
            for v in range(g.n):
                if v not in K:
                    f = M[v][M[v] != INF]
                    assert (f >= r1.a[v]).all()
            # I5: C = rows all finite, depth = row max (Lemma V.1)
            allf = np.nonzero((M != INF).all(axis=1))[0]
            assert r1.centrals.tolist() == allf.tolist()
            assert r1.central_depth.tolist() == M[allf].max(axis=1).tolist()
            if r1.stop_reason == oracle.STOP_K:
                d = r1.levels
                assert M[M != INF].max() <= d                        # I4
                assert (r1.central_depth < d).sum() < k <= len(r1.centrals)  # I6
                D = d
            else:
                assert len(r1.centrals) < k
                D = 254
            # I3
            assert R.fixpoint_violations(g, kw, r1.a, M, block, D) == []


def test_max_depth_truncation():
    for g, q in _cases(21, 40):
        kw = list(range(q))
        for md in (1, 2, 3):
            r = oracle.query(g, kw, k=10 ** 6, max_depth=md)
            if r.stop_reason == oracle.STOP_MAX_DEPTH:
                assert r.levels == md
                assert (r.M[r.M != INF] <= md).all()


def test_invalid_arguments():
    g, q = next(_cases(5, 1))
    assert oracle.query(g, [0, 0], k=1).status == -1          # duplicate keyword ids
    assert oracle.query(g, [0], k=0).status == -1
    assert oracle.query(g, [0], k=1, alpha=0.0).status == -1
    assert oracle.query(g, [0], k=1, alpha=1.0).status == -1
    assert oracle.query(g, [0], k=1, lam=-1.0).status == -1
    assert oracle.query(g, [0], k=1, max_depth=0).status == -1
    assert oracle.query(g, [0], k=1, max_depth=255).status == -1
    assert oracle.query(g, [g.n_keywords], k=1).status == -1
    assert oracle.query(g, list(range(9)), k=1).status == -1


def test_degenerate_queries():
    """R17: q = 1 -> every T_0 node is central at depth 0; a node containing all keywords is central at
    depth 0 with graph {c} and score 0; an empty T_i yields no answer."""
    import synth
    g = synth.from_edges(4, [(0, 1), (1, 2), (2, 3)], [0.5, 0, 0, 0], [[0, 2], [2], []], 2.0)
    r = oracle.query(g, [0], k=5)
    assert r.centrals.tolist() == [0, 2] and r.central_depth.tolist() == [0, 0]
    r = oracle.query(g, [0, 1], k=1)
    assert r.centrals.tolist() == [2] and r.central_depth.tolist() == [0]
    assert r.answers[0].nodes.tolist() == [2] and r.answers[0].key == 0.0
    r = oracle.query(g, [0, 2], k=1)
    assert r.status == 0 and r.stop_reason == oracle.STOP_EMPTY_KEYWORD and r.answers == []


def test_eval_ids_sampling_is_consistent():
    """oracle.query(eval_ids=...) scores only the listed central nodes: their keys equal the full run's,
    the others are NaN, and the answers are the full ranking restricted to the list."""
    import synth
    w = synth.make_workload("C1")
    for kw in w.queries[:10]:
        full = oracle.query(w.graph, kw, 5)
        if len(full.centrals) < 4:
            continue
        sub = full.centrals[::3]
        part = oracle.query(w.graph, kw, 5, eval_ids=sub)
        assert part.M.tolist() == full.M.tolist() and part.centrals.tolist() == full.centrals.tolist()
        keep = np.isin(full.centrals, sub)
        assert part.central_key[keep].tolist() == full.central_key[keep].tolist()
        assert np.isnan(part.central_key[~keep]).all()
        ranked = sorted(zip(full.central_key[keep].tolist(), full.centrals[keep].tolist()))[:5]
        assert [(a.key, a.central) for a in part.answers] == ranked
