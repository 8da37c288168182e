"""NEXT-3 semantics variants in the oracle: the "contains" reading of level-cover (R13b) and containment
removal (R16), pinned by a hand-derived example, a reduction to the default reading, and brute force.

* R13b ("nodes contain most keywords"): a keyword node's level counts the query keywords it
  CONTAINS, not only those for which it is a source of a hitting path of this Central Graph (R13).
* R16 ("we remove the Central Graph that completely contains smaller ones"): a Central Graph whose
  pruned node set strictly contains the pruned node set of another Central Graph of C is dropped; the
  answers are the k best (key, id) of the rest.
"""
import numpy as np

import oracle
import refimpl as R
import synth


def test_contains_reading_hand_example():
    """Q = {S, J, U}.  c = 0 holds S and waits (a = 2: w = alpha, A = 2); node 1 holds J and U two hops
    away (1-2-0); node 3 holds U next to c; node 5 holds J two hops away (5-6-0).  c is hit by U at level
    1 (from 3) and by J at level 2 (from 1 and 5), so it is central at depth 2, and node 1's U path
    (level 2) is not a hitting path: 1 lies in DAG_J(c) only.
      R13 (contribute): levels 1 = {1 -> J, 3 -> U, 5 -> J}, c -> S; cover complete at s* = 1: nothing
                        is pruned, G(c) = {0, 1, 2, 3, 5, 6}.
      R13b (contains):  node 1 contains {J, U}: with c's S the cover is complete at s* = 2; the level-1
                        nodes 3 and 5 and their paths are pruned: {0, 1, 2}, arcs 1->2, 2->0."""
    g = synth.from_edges(7, [(0, 3), (1, 2), (2, 0), (5, 6), (6, 0)], [0.1, 0, 0, 0, 0, 0, 0],
                         [[0], [1, 5], [1, 3]], 2.0)
    o1 = oracle.query(g, [0, 1, 2], 1, level_cover=1)
    o2 = oracle.query(g, [0, 1, 2], 1, level_cover=2)
    for o in (o1, o2):
        assert o.a.tolist() == [2, 0, 0, 0, 0, 0, 0]
        assert o.M.tolist() == [[0, 2, 1], [255, 0, 0], [255, 1, 1], [255, 255, 0], [255, 255, 255],
                                [255, 0, 255], [255, 1, 255]]
        assert o.centrals.tolist() == [0] and o.central_depth.tolist() == [2]
    assert o1.answers[0].nodes.tolist() == [0, 1, 2, 3, 5, 6]
    assert o1.answers[0].arcs.tolist() == [[1, 2], [2, 0], [3, 0], [5, 6], [6, 0]]
    assert o2.answers[0].nodes.tolist() == [0, 1, 2]
    assert o2.answers[0].arcs.tolist() == [[1, 2], [2, 0]]


def test_contains_equals_contribute_for_single_keyword_nodes():
    """With pairwise disjoint keyword sets no node holds two keywords, every s* is 1 in both readings and
    every source is kept: the two readings give the same answers."""
    rng = np.random.default_rng(31)
    checked = 0
    for case in range(60):
        n = int(rng.integers(8, 50))
        g = R.random_graph(rng, n, float(rng.uniform(0.05, 0.3)), bool(case % 3 == 0), 1, wmax=0.3)
        q = int(rng.integers(2, 5))
        perm = rng.permutation(n)
        sizes = rng.integers(1, 4, q)
        kws, at = [], 0
        for s in sizes:
            kws.append(sorted(perm[at:at + s].tolist()))
            at += s
        g2 = synth.from_edges(n, [], g.weight, kws, g.A)
        g2.row_ptr, g2.col_idx, g2.symmetric = g.row_ptr, g.col_idx, g.symmetric
        a = oracle.query(g2, list(range(q)), 5, level_cover=1)
        b = oracle.query(g2, list(range(q)), 5, level_cover=2)
        assert [(x.central, x.key, x.nodes.tolist(), x.arcs.tolist()) for x in a.answers] == \
            [(x.central, x.key, x.nodes.tolist(), x.arcs.tolist()) for x in b.answers]
        checked += len(a.answers)
    assert checked > 50


def _all_pruned_sets(g, kw, k, **kw_args):
    """node set and key of every central node's pruned graph, each scored alone (eval_ids = [c])."""
    full = oracle.query(g, kw, k, **kw_args)
    sets = {}
    for c in full.centrals.tolist():
        one = oracle.query(g, kw, k, eval_ids=[c], **kw_args)
        a = one.answers[0]
        sets[c] = (frozenset(a.nodes.tolist()), a.key)
    return full, sets


def test_containment_removal_brute_force():
    """R16 re-derived from the per-central pruned graphs: drop every candidate whose node set strictly
    contains another candidate's, rank the rest by (key, id), keep k; both level-cover readings."""
    rng = np.random.default_rng(8)
    removed_total = 0
    cases = []
    for case in range(40):
        n = int(rng.integers(6, 40))
        q = int(rng.integers(2, 4))
        cases.append((R.random_graph(rng, n, float(rng.uniform(0.08, 0.35)), bool(case % 2), q, kw_size=(1, 4),
                                     wmax=float(rng.choice([0.0, 0.2, 1.0]))), list(range(q))))
    w = synth.make_workload("C1")
    cases += [(w.graph, list(kw)) for kw in w.queries[:6]]
    for g, kw in cases:
        for lc in (1, 2):
            k = 4
            full, sets = _all_pruned_sets(g, kw, k, level_cover=lc)
            keep = [c for c, (nc, _) in sets.items()
                    if not any(c2 != c and n2 < nc for c2, (n2, _) in sets.items())]
            removed_total += len(sets) - len(keep)
            want = sorted((sets[c][1], c) for c in keep)[:k]
            got = oracle.query(g, kw, k, level_cover=lc, containment=1)
            assert [(a.key, a.central) for a in got.answers] == want, (kw, lc)
            for a in got.answers:
                assert frozenset(a.nodes.tolist()) == sets[a.central][0]
            assert got.M.tolist() == full.M.tolist()
    assert removed_total > 20
