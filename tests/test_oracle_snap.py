"""O0 (reading R15): the 2^-24 weight grid, and that the oracle's query reads only the snapped weights.

Pins (independent of oracle.c's fp64 arithmetic): exact rational rounding with ``fractions`` (nearest
grid point, ties up), hand values (ties, idempotence, the ends of [0, 1]), and at query level that Eq. 6
keys of off-grid inputs are exact multiples of 2^-24 equal to the rational sum of the snapped weights of
the returned nodes, and that the activation levels are those of the snapped weights.
"""
from fractions import Fraction

import numpy as np

import oracle
import refimpl as R

G24 = 1 << 24


def _exact_snap(w):
    x = Fraction(float(w)) * G24
    r = (x + Fraction(1, 2)).__floor__()          # nearest integer, halves up
    return Fraction(r, G24)


def test_hand_values():
    eps = 2.0 ** -24
    w = np.array([0.0, 1.0, eps, 0.5 * eps, 0.25 * eps, 0.75 * eps, 1.5 * eps, 2.5 * eps, 0.5, 0.1,
                  (7 + 0.5) * eps, (2 ** 20 + 0.5) * eps, 1.0 - eps], np.float32)
    got = oracle.snap_weights(w).astype(np.float64)
    want = [0.0, 1.0, eps, eps, 0.0, eps, 2 * eps, 3 * eps, 0.5, 1677722 * eps, 8 * eps,
            (2 ** 20 + 1) * eps, 1.0 - eps]
    assert got.tolist() == want


def test_exact_rational_and_idempotent():
    rng = np.random.default_rng(11)
    # off-grid float32 values across many binades, plus random ties
    w = np.concatenate([rng.random(3000).astype(np.float32),
                        (rng.random(1000) * 1e-3).astype(np.float32),
                        ((rng.integers(0, 1 << 22, 500) + 0.5) / G24).astype(np.float32)])
    s = oracle.snap_weights(w)
    for wi, si in zip(w, s):
        assert Fraction(float(si)) == _exact_snap(wi), float(wi)
    assert np.array_equal(oracle.snap_weights(s), s)                 # idempotent
    assert (np.abs(s.astype(np.float64) - w.astype(np.float64)) <= 2.0 ** -25).all()   # error bound
    on = (rng.integers(0, G24 + 1, 2000) / G24).astype(np.float32)   # on the grid: unchanged
    assert np.array_equal(oracle.snap_weights(on), on)


def test_query_reads_snapped_weights():
    """Off-grid weights: the oracle's keys are exact sums of snapped weights (lambda = 0: key = sum), and
    its activation levels are those of the snapped weights (exact rationals at half-integer boundaries)."""
    rng = np.random.default_rng(5)
    for case in range(30):
        n = int(rng.integers(6, 40))
        g = R.random_graph(rng, n, 0.2, bool(case % 2), 3, kw_size=(1, 4))
        g.weight = (rng.random(n) * rng.choice([1.0, 1e-4])).astype(np.float32)   # off the grid
        o = oracle.query(g, [0, 1, 2], 5, lam=0.0, alpha=0.1)
        ws = oracle.snap_weights(g.weight)
        assert np.array_equal(o.a, oracle.activation(ws, g.A, 0.1))
        o2 = oracle.query(type(g)(g.row_ptr, g.col_idx, ws, g.kw_ptr, g.kw_nodes, g.A, g.symmetric), [0, 1, 2], 5,
                          lam=0.0, alpha=0.1)
        assert o.M.tolist() == o2.M.tolist() and o.central_key.tolist() == o2.central_key.tolist()
        for an in o.answers:
            exact = sum((_exact_snap(g.weight[v]) for v in an.nodes), Fraction(0))
            assert Fraction(an.key) == exact, (case, an.central)


def test_activation_boundary_uses_snapped_weight():
    """A raw weight just below the Eq. 5 rounding boundary whose grid point lies on it: the level must be
    the snapped weight's (exact rational), which differs from the raw weight's."""
    A, alpha = 3.0, 0.5
    # below alpha: x = A - A (alpha - w) / alpha = 6 w, and x = 2.5 at w* = 5/12 (off the grid:
    # 5/12 * 2^24 = 6990506.67).  raw = 6990506.5 / 2^24 (a float: 13981013 * 2^-25) lies below w* and is
    # a tie that snaps up to the grid point 6990507 / 2^24 above w*.
    raw = np.float32(13981013 * 2.0 ** -25)
    gp = Fraction(6990507, G24)
    assert Fraction(float(oracle.snap_weights(np.array([raw]))[0])) == gp
    x_raw = Fraction(A) - Fraction(A) * (Fraction(alpha) - Fraction(float(raw))) / Fraction(alpha)
    x_q = Fraction(A) - Fraction(A) * (Fraction(alpha) - gp) / Fraction(alpha)
    a_raw = (x_raw + Fraction(1, 2)).__floor__()
    a_q = (x_q + Fraction(1, 2)).__floor__()
    assert (a_raw, a_q) == (2, 3)
    import synth
    g = synth.from_edges(3, [(0, 1), (1, 2)], [0.0, float(raw), 0.0], [[0], [2]], A)
    o = oracle.query(g, [0, 1], 1, alpha=alpha)
    assert int(o.a[1]) == a_q                                                 # the query reads w_q
    assert int(oracle.activation(np.array([raw]), A, alpha)[0]) == a_raw     # O1 alone maps what it gets
