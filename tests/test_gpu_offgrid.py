"""Parity on the real input domain: ordinary float32 weights, NOT on the 2^-24 grid.

kgs_load_graph snaps the weights on load (reading R15); the oracle snaps them as its step O0.  With
off-grid inputs both sides must still agree bit for bit: activation levels (a half-integer boundary of
Eq. 5 decided on the snapped weight), M, the central set, every Eq. 6 key, the answers.
"""
import numpy as np
import pytest

import oracle
import refimpl as R
import synth
from test_gpu_parity import compare

pytestmark = pytest.mark.gpu

kgs = pytest.importorskip("paper_conf_icde_yangajtw19_b200")


def _gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _offgrid(rng, w, scale=1.0):
    """float32 weights in [0, 1] that are (almost all) off the grid."""
    x = np.clip(np.asarray(w, np.float64) + rng.uniform(-0.5, 0.5, len(w)) * 2.0 ** -24 * scale, 0.0, 1.0)
    return x.astype(np.float32)


def test_random_graphs_offgrid_weights():
    _gpu()
    rng = np.random.default_rng(77)
    for case in range(80):
        n = int(rng.integers(6, 60))
        q = int(rng.integers(1, 6))
        g = R.random_graph(rng, n, float(rng.uniform(0.05, 0.3)), bool(rng.random() < 0.4), q, kw_size=(1, 5))
        g.weight = (rng.random(n) * rng.choice([1.0, 0.2, 1e-5])).astype(np.float32)
        assert (oracle.snap_weights(g.weight) != g.weight).any()
        G = kgs.kgs_load_graph(g, relabel=bool(case % 2))
        for _ in range(2):
            compare(G, g, list(range(q)), int(rng.choice([1, 3, 20])), alpha=float(rng.choice([0.05, 0.1, 0.4])),
                    lam=float(rng.choice([0.0, 0.2])), block_central=int(rng.integers(0, 2)),
                    level_cover=int(rng.integers(0, 2)))
        G.close()


def test_activation_boundary_tie():
    """The weight 6990506.5 / 2^24 lies below the Eq. 5 boundary 5/12 (A = 3, alpha = 0.5, x = 6w = 2.5) and
    snaps to a grid point above it: level 3 on both sides (the raw weight would give 2)."""
    _gpu()
    raw = float(np.float32(13981013 * 2.0 ** -25))
    g = synth.from_edges(4, [(0, 1), (1, 2), (2, 3)], [0.0, raw, 0.0, 0.0], [[0], [3]], 3.0)
    G = kgs.kgs_load_graph(g)
    r, o = compare(G, g, [0, 1], 1, alpha=0.5)
    assert int(r.a[1]) == 3 and int(o.a[1]) == 3
    G.close()


def test_c2_offgrid_weights():
    """C2 with every weight moved off the grid (by up to half a grid step): sampled queries, full view."""
    _gpu()
    w = synth.make_workload("C2")
    rng = np.random.default_rng(9)
    g = w.graph
    g.weight = _offgrid(rng, g.weight)
    G = kgs.kgs_load_graph(g)
    for j, kw in enumerate(w.queries[::25]):
        compare(G, g, kw, w.k, full=(j % 2 == 0))
    G.close()


def test_prep_weights_fed_to_both_sides():
    """kgs_prep_summary_weights' output (Eq. 2 + min-max) used as the weights of both sides."""
    _gpu()
    w = synth.make_workload("C1")
    g = w.graph
    lab = (g.col_idx % 7).astype(np.int32)
    wn, _ = kgs.kgs_prep_summary_weights(g.row_ptr, lab)
    g.weight = np.asarray(wn, np.float32)
    G = kgs.kgs_load_graph(g)
    for kw in w.queries[:30]:
        compare(G, g, kw, w.k)
    G.close()
