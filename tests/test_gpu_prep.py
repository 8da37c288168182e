"""Load-time preprocessing through the C-ABI vs the oracle.

kgs_prep_pair_distances: bit-exact integer distances (and the mean computed from them) on small
graphs with ragged batches (not a multiple of the 128 pairs one BFS pass carries; bits 0-63 and
64-127 live in different words), unreachable pairs,
src == dst, duplicate pairs, a max_hops cut-off, and a 1M-node R-MAT graph (config C2's) with 150
sampled pairs.  kgs_prep_summary_weights: Eq. 2 in fp64 — the raw w within 1e-13 relative (log2 is
1-ulp on both sides, the run sums are exact integers) and w' within 1e-6 absolute — on random
Zipf-like labels over C2's in-arcs, plus one hub row of 200K in-arcs whose label runs cross many
32-label chunks.
"""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

kgs = pytest.importorskip("paper_conf_icde_yangajtw19_b200")


def _gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _rand_graph(rng, n, p, directed=True):
    adj = rng.random((n, n)) < p
    np.fill_diagonal(adj, False)
    if not directed:
        adj |= adj.T
    rp = np.concatenate([[0], np.cumsum(adj.sum(1))]).astype(np.int64)
    ci = np.nonzero(adj)[1].astype(np.int32)
    return rp, ci


@pytest.mark.parametrize("seed,n,p,pairs", [(0, 50, 0.04, 1), (1, 300, 0.01, 64), (2, 200, 0.02, 65),
                                            (3, 500, 0.005, 201), (4, 400, 0.008, 128), (5, 400, 0.008, 129),
                                            (6, 600, 0.004, 300)])
def test_pair_distances_small(seed, n, p, pairs):
    _gpu()
    rng = np.random.default_rng(seed)
    rp, ci = _rand_graph(rng, n, p)
    s = rng.integers(0, n, pairs).astype(np.int32)
    t = rng.integers(0, n, pairs).astype(np.int32)
    t[::7] = s[::7]                     # src == dst -> 0
    if pairs > 3:
        s[1], t[1] = s[2], t[2]         # a duplicate pair
    want, wmean = oracle.pair_distances(rp, ci, s, t)
    got, gmean = kgs.kgs_prep_pair_distances(rp, ci, s, t)
    assert got.tolist() == want.tolist()
    assert (np.isnan(gmean) and np.isnan(wmean)) or gmean == wmean
    want3, _ = oracle.pair_distances(rp, ci, s, t, max_hops=2)
    got3, _ = kgs.kgs_prep_pair_distances(rp, ci, s, t, max_hops=2)
    assert got3.tolist() == want3.tolist()


def test_pair_distances_empty_and_invalid():
    _gpu()
    rp, ci = np.array([0, 1, 1], np.int64), np.array([1], np.int32)
    d, mean = kgs.kgs_prep_pair_distances(rp, ci, [], [])
    assert d.shape == (0,) and np.isnan(mean)
    with pytest.raises(kgs.KgsError):
        kgs.kgs_prep_pair_distances(rp, ci, [0], [5])
    with pytest.raises(kgs.KgsError):
        kgs.kgs_prep_pair_distances(rp, ci, [0], [1], max_hops=0)
    with pytest.raises(kgs.KgsError):
        kgs.kgs_prep_pair_distances(np.array([0, 2, 1], np.int64), ci, [0], [1])


def test_pair_distances_rmat_c2():
    _gpu()
    g = synth.rmat_graph(20, 8, 11, a_sources=1, a_pairs_per_source=1)
    rng = np.random.default_rng(7)
    nz = np.nonzero(np.diff(g.row_ptr) > 0)[0]
    s = rng.choice(nz, 150).astype(np.int32)
    t = rng.choice(nz, 150).astype(np.int32)
    want, wmean = oracle.pair_distances(g.row_ptr, g.col_idx, s, t)
    got, gmean = kgs.kgs_prep_pair_distances(g.row_ptr, g.col_idx, s, t)
    assert got.tolist() == want.tolist()
    assert gmean == wmean and 1.0 < gmean < 10.0


def _labels(rng, m, n_labels=64):
    return np.minimum(rng.zipf(1.3, m) - 1, n_labels - 1).astype(np.int32)


def test_summary_weights_small_ragged():
    _gpu()
    rng = np.random.default_rng(3)
    deg = rng.integers(0, 100, 777)
    deg[::5] = 0
    rp = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    lab = _labels(rng, int(rp[-1]), 5)
    wn_o, wr_o = oracle.summary_weights(rp, lab)
    wn, wr = kgs.kgs_prep_summary_weights(rp, lab)
    assert np.allclose(wr, wr_o, rtol=1e-13, atol=0)
    assert np.abs(wn - wn_o).max() <= 1e-6
    wn, wr = kgs.kgs_prep_summary_weights(np.array([0, 1, 2], np.int64), np.array([4, 4], np.int32))
    assert wr.tolist() == [1.0, 1.0] and wn.tolist() == [0.0, 0.0]   # R26


def test_summary_weights_c2_and_hub():
    _gpu()
    g = synth.rmat_graph(20, 8, 11, a_sources=1, a_pairs_per_source=1)
    rng = np.random.default_rng(4)
    rp = g.row_ptr.copy()          # symmetric: the in-arcs are the out-arcs
    lab = _labels(rng, int(rp[-1]))
    hub = np.concatenate([np.full(150_000, 3), np.full(30_001, 9), rng.integers(0, 1000, 19_999)]).astype(np.int32)
    rng.shuffle(hub)
    rp = np.concatenate([rp, [rp[-1] + hub.shape[0]]]).astype(np.int64)
    lab = np.concatenate([lab, hub])
    wn_o, wr_o = oracle.summary_weights(rp, lab)
    wn, wr = kgs.kgs_prep_summary_weights(rp, lab)
    assert np.allclose(wr, wr_o, rtol=1e-13, atol=0)
    assert np.abs(wn - wn_o).max() <= 1e-6
    assert wn[-1] == wn_o[-1]


def test_device_pointer_inputs():
    """KGS_INPUT_DEVICE_PTRS: the same answers from borrowed device buffers, on a non-default stream."""
    _gpu()
    import torch
    rng = np.random.default_rng(9)
    rp, ci = _rand_graph(rng, 400, 0.01, directed=False)
    s = rng.integers(0, 400, 150).astype(np.int32)
    t = rng.integers(0, 400, 150).astype(np.int32)
    want, wmean = oracle.pair_distances(rp, ci, s, t)
    dev = [torch.from_numpy(x).cuda() for x in (rp, ci, s, t)]
    st = torch.cuda.Stream()
    got, gmean = kgs.kgs_prep_pair_distances_device(400, ci.shape[0], dev[0].data_ptr(), dev[1].data_ptr(), 150,
                                                    dev[2].data_ptr(), dev[3].data_ptr(), stream=st.cuda_stream)
    assert got.tolist() == want.tolist() and gmean == wmean
    lab = _labels(rng, ci.shape[0], 7)
    wn_o, wr_o = oracle.summary_weights(rp, lab)
    dl = torch.from_numpy(lab).cuda()
    wn, wr = kgs.kgs_prep_summary_weights_device(400, lab.shape[0], dev[0].data_ptr(), dl.data_ptr(),
                                                 stream=st.cuda_stream)
    assert np.allclose(wr, wr_o, rtol=1e-13, atol=0) and np.abs(wn - wn_o).max() <= 1e-6
    assert (dev[1].cpu().numpy() == ci).all()          # borrowed inputs are not modified


def test_summary_weights_reproduce_generator_c2():
    """NEXT-2 against the dataset recipe: kgs_prep_summary_weights on the C2 generator's own edge labels
    (R-MAT scale 20, 1024 Zipf labels) gives the weights the generator wrote, bit for bit (Eq. 2 terms in
    label order, R6 for the 0.5 M nodes without in-arcs, R27 grid), and kgs_load_graph keeps them."""
    _gpu()
    gp = dict(synth.CONFIG_PARAMS["C2"]["graph"])
    g = synth.rmat_graph(**gp, labels=True)
    lab = g.meta["arc_labels"]
    wn, wr = kgs.kgs_prep_summary_weights(g.row_ptr, lab)
    iso = np.diff(g.row_ptr) == 0
    assert iso.sum() > 0 and (wn[iso] == 0).all() and (wr[iso] == 0).all()
    bad = np.flatnonzero(wn != g.weight)
    assert bad.size == 0, f"{bad.size} weights differ, first {bad[:5].tolist()}"
    wn_o, wr_o = oracle.summary_weights(g.row_ptr, lab)
    assert np.array_equal(wn, wn_o) and np.allclose(wr, wr_o, rtol=1e-13, atol=0)
