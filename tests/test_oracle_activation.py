"""O1 (Eqs. 3-5) against closed forms and exact rational arithmetic."""
from fractions import Fraction

import numpy as np
import pytest

import oracle


def _exact_a(w, A, alpha):
    """Eq. 5 in exact rational arithmetic, round half up (reading R4), clamp 254."""
    w, A, al = Fraction(float(w)), Fraction(A), Fraction(alpha)
    if w < al:
        x = A - A * (al - w) / al
    elif w == al:
        x = A
    else:
        x = A + A * (w - al) / (1 - al)
    r = int(np.floor(float(x) + 0.5)) if abs(x - Fraction(int(x)) - Fraction(1, 2)) > Fraction(1, 10**9) else None
    return x, r


@pytest.mark.parametrize("A", [1.0, 2.5, 3.68, 3.87, 7.3])
@pytest.mark.parametrize("alpha", [0.05, 0.1, 0.25, 0.4, 0.5])
def test_endpoints(A, alpha):
    w = np.array([0.0, 1.0], np.float32)
    a = oracle.activation(w, A, alpha)
    assert a[0] == 0                                   # full reward: A - A = 0
    assert a[1] == min(254, int(np.floor(2 * A + 0.5)))  # full penalty: A + A = 2A


@pytest.mark.parametrize("A", [1.0, 2.5, 3.68])
def test_w_equals_alpha(A):
    for alpha in (0.25, 0.5, 0.125):                 # exactly representable, so w == alpha holds
        a = oracle.activation(np.array([alpha], np.float32), A, alpha)
        assert a[0] == int(np.floor(A + 0.5))
    # continuity around alpha: both neighbours of alpha on the grid also round to round(A) for A=3.68
    al = 0.25
    eps = 2.0 ** -24
    a = oracle.activation(np.array([al - eps, al + eps], np.float32), 3.68, al)
    assert a.tolist() == [4, 4]


def test_exact_rational_and_monotone():
    rng = np.random.default_rng(7)
    w = np.sort((rng.integers(0, 1 << 24, size=4000) / float(1 << 24)).astype(np.float32))
    for A, alpha in [(3.68, 0.1), (3.87, 0.05), (2.0, 0.4), (5.5, 0.3)]:
        a = oracle.activation(w, A, alpha)
        assert (np.diff(a.astype(int)) >= 0).all()          # non-decreasing in w
        for wi, ai in zip(w[::7], a[::7]):
            x, r = _exact_a(wi, A, alpha)
            if r is not None:
                assert ai == min(254, r), (wi, A, alpha, float(x))


def test_larger_alpha_lowers_levels():
    """Fig. 3 / P:L236-238: larger alpha maps more nodes to a smaller minimum activation level."""
    rng = np.random.default_rng(3)
    w = (rng.integers(0, 1 << 24, size=5000) / float(1 << 24)).astype(np.float32)
    prev = None
    for alpha in (0.05, 0.1, 0.4):
        a = oracle.activation(w, 3.68, alpha).astype(int)
        if prev is not None:
            assert (a <= prev).all()
            assert (a < prev).any()
        prev = a


def test_clamp_and_half_up():
    a = oracle.activation(np.array([1.0], np.float32), 200.0, 0.5)
    assert a[0] == 254                                  # 2A = 400 clamps below the 255 = inf code
    a = oracle.activation(np.array([0.5], np.float32), 2.5, 0.5)
    assert a[0] == 3                                    # x = 2.5 exactly: half rounds up


def test_fig4_weights():
    """the weights map to Ex. 4's activation levels (x = 2.3 -> 2, 3.782 -> 4, 0.575 -> 1)."""
    w = np.array([0, 2 ** -4, 0.125, 2 ** -4, 0, 2 ** -6, 0, 2 ** -6, 0, 2 ** -6], np.float32)
    assert oracle.activation(w, 3.68, 0.1).tolist() == [0, 2, 4, 2, 0, 1, 0, 1, 0, 1]
