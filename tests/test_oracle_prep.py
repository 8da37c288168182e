"""Pins of the load-time preprocessing oracle (P1 sampled distances, P2 Eq. 2 degree of summary).

P1: hop distances are pinned to closed forms (directed / bi-directed paths, cycles,
grids) and to an all-pairs brute force (Floyd-Warshall min-plus over the adjacency matrix, which
shares nothing with the oracle's BFS).  P2 (Eq. 2; min-max; readings R25/R26)
is pinned to values worked by hand and to the bounds 1 <= w <= log2(1 + deg) (equality on the right
iff every in-edge has the same label; on the left iff all labels differ).
"""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle


def csr(n, arcs):
    arcs = sorted(arcs)
    rp = np.zeros(n + 1, np.int64)
    for u, _ in arcs:
        rp[u + 1] += 1
    rp = np.cumsum(rp)
    ci = np.array([x for _, x in arcs], np.int32)
    return rp, ci


def test_path_distances_closed_form():
    n = 12
    directed = [(i, i + 1) for i in range(n - 1)]
    rp, ci = csr(n, directed)
    src, dst = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    d, mean = oracle.pair_distances(rp, ci, src.ravel(), dst.ravel())
    want = np.where(dst.ravel() >= src.ravel(), dst.ravel() - src.ravel(), -1)
    assert d.tolist() == want.tolist()
    assert mean == pytest.approx(want[want >= 0].mean(), rel=0, abs=1e-15)
    rp, ci = csr(n, directed + [(x, u) for u, x in directed])
    d, _ = oracle.pair_distances(rp, ci, src.ravel(), dst.ravel())
    assert d.tolist() == np.abs(dst.ravel() - src.ravel()).tolist()


def test_cycle_and_grid_closed_forms():
    n = 9
    cyc = [(i, (i + 1) % n) for i in range(n)] + [((i + 1) % n, i) for i in range(n)]
    rp, ci = csr(n, cyc)
    s = np.repeat(np.arange(n), n)
    t = np.tile(np.arange(n), n)
    d, _ = oracle.pair_distances(rp, ci, s, t)
    assert d.tolist() == [min(abs(a - b), n - abs(a - b)) for a, b in zip(s, t)]
    R, C = 4, 5
    arcs = []
    for r in range(R):
        for c in range(C):
            v = r * C + c
            if c + 1 < C:
                arcs += [(v, v + 1), (v + 1, v)]
            if r + 1 < R:
                arcs += [(v, v + C), (v + C, v)]
    rp, ci = csr(R * C, arcs)
    s = np.repeat(np.arange(R * C), R * C)
    t = np.tile(np.arange(R * C), R * C)
    d, _ = oracle.pair_distances(rp, ci, s, t)
    assert d.tolist() == [abs(a // C - b // C) + abs(a % C - b % C) for a, b in zip(s, t)]


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_distances_match_floyd_warshall(seed):
    rng = np.random.default_rng(seed)
    n = 30
    adj = rng.random((n, n)) < 0.06
    np.fill_diagonal(adj, False)
    arcs = [(int(u), int(x)) for u, x in zip(*np.nonzero(adj))]
    rp, ci = csr(n, arcs)
    D = np.where(adj, 1.0, np.inf)
    np.fill_diagonal(D, 0.0)
    for k in range(n):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    s = rng.integers(0, n, 400)
    t = rng.integers(0, n, 400)
    d, mean = oracle.pair_distances(rp, ci, s, t)
    want = np.where(np.isinf(D[s, t]), -1, D[s, t]).astype(np.int64)
    assert d.tolist() == want.tolist()
    d3, _ = oracle.pair_distances(rp, ci, s, t, max_hops=3)
    assert d3.tolist() == np.where(want > 3, -1, want).tolist()


def test_no_reachable_pair_gives_nan_mean():
    rp, ci = csr(3, [])
    d, mean = oracle.pair_distances(rp, ci, [0, 1], [1, 2])
    assert d.tolist() == [-1, -1] and math.isnan(mean)


def test_eq2_worked_values():
    # node 0: labels {7,7,7,9} -> (3 log2 4 + 1 log2 2) / 4 = 7/4
    # node 1: one in-edge -> log2 2 = 1            node 2: {5 x 7} -> log2 8 = 3
    # node 3: no in-edges -> 0 (R25)               node 4: {3 x a, 3 x b} -> (6 + 6) / 6 = 2
    # node 5: {15 x a, 1 x b} -> (15 log2 16 + 1) / 16 = 61/16
    rows = [[9, 7, 7, 7], [4], [5] * 7, [], [1, 2, 1, 2, 2, 1], [3] * 15 + [8]]
    rp = np.cumsum([0] + [len(r) for r in rows]).astype(np.int64)
    lab = np.array([x for r in rows for x in r], np.int32)
    wn, wr = oracle.summary_weights(rp, lab)
    assert wr.tolist() == [1.75, 1.0, 3.0, 0.0, 2.0, 61 / 16]
    # R6: node 3 (no in-edges) is left out of the min / max and gets w' = 0, so min = 1 (node 1), max =
    # 61/16; R27: w' is the grid point nearest (w - 1) / (45/16), ties up -- exact rationals here
    want = []
    for v, x in enumerate(wr.tolist()):
        if v == 3:
            want.append(0.0)
            continue
        t = (Fraction(x) - 1) / (Fraction(61, 16) - 1) * (1 << 24)
        want.append(float(Fraction((t + Fraction(1, 2)).__floor__(), 1 << 24)))
    assert wn.astype(np.float64).tolist() == want
    assert want[1] == 0.0 and want[5] == 1.0 and want[0] == 4473924 / (1 << 24)   # (3/4) / (45/16) = 4/15


def test_eq2_bounds_and_label_order_invariance():
    rng = np.random.default_rng(5)
    deg = rng.integers(1, 40, 200)
    rp = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    lab = rng.integers(0, 6, int(rp[-1])).astype(np.int32)
    wn, wr = oracle.summary_weights(rp, lab)
    assert (wr >= 1.0 - 1e-15).all() and (wr <= np.log2(1.0 + deg) + 1e-12).all()
    lab2 = lab.copy()
    for v in range(200):
        seg = lab2[rp[v]:rp[v + 1]]
        rng.shuffle(seg)
    assert (oracle.summary_weights(rp, lab2)[1] == wr).all()
    single = np.zeros(int(rp[-1]), np.int32)
    assert np.allclose(oracle.summary_weights(rp, single)[1], np.log2(1.0 + deg), rtol=0, atol=1e-13)
    distinct = np.arange(int(rp[-1]), dtype=np.int32)
    assert (oracle.summary_weights(rp, distinct)[1] == 1.0).all()
    assert wn.min() == 0.0 and wn.max() == 1.0


def test_eq2_isolated_nodes_leave_min_max_alone():
    """R6: adding nodes without in-edges changes no other weight (a rule that put their w = 0 into the
    min would rescale every w' to w / max)."""
    rows = [[1, 1, 2], [3], [4, 4, 4, 4], [5, 6]]
    rp = np.cumsum([0] + [len(r) for r in rows]).astype(np.int64)
    lab = np.array([x for r in rows for x in r], np.int32)
    wn, _ = oracle.summary_weights(rp, lab)
    rows2 = [[], rows[0], [], rows[1], rows[2], [], rows[3], []]
    rp2 = np.cumsum([0] + [len(r) for r in rows2]).astype(np.int64)
    wn2, wr2 = oracle.summary_weights(rp2, np.array([x for r in rows2 for x in r], np.int32))
    assert wn2[[1, 3, 4, 6]].tolist() == wn.tolist()
    assert wn2[[0, 2, 5, 7]].tolist() == [0.0] * 4 and wr2[[0, 2, 5, 7]].tolist() == [0.0] * 4
    assert wn.min() == 0.0 and wn.max() == 1.0


def test_eq2_reproduces_the_generator():
    """The Eq. 2 weights the input generator wrote (synth, R-MAT scale 14 with Zipf edge labels and two
    planted hubs; an independent implementation of the dataset recipe) are what P2 computes from the
    generator's labels, bit for bit (same label order, R6, R27)."""
    import synth
    g = synth.rmat_graph(14, 8, 21, n_hubs=2, hub_arcs=3000, n_labels=256, a_sources=1,
                         a_pairs_per_source=1, labels=True)
    lab = g.meta["arc_labels"]
    assert (np.diff(g.row_ptr) == 0).any()                    # isolated nodes exist (R6 matters)
    wn, _ = oracle.summary_weights(g.row_ptr, lab)
    assert np.array_equal(wn, g.weight)


def test_eq2_constant_weights_normalise_to_zero():
    rp = np.array([0, 1, 2, 3], np.int64)
    wn, wr = oracle.summary_weights(rp, np.array([1, 2, 3], np.int32))
    assert wr.tolist() == [1.0, 1.0, 1.0] and wn.tolist() == [0.0, 0.0, 0.0]   # R26
