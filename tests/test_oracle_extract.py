"""O4-O7 (extraction, level-cover, score, top-k) pinned against recorded hitting paths (I7),
characterising properties of level-cover (I9), Eq. 6 recomputed from the answer (I10) and a
brute-force sort (I11)."""
import numpy as np
import pytest

import oracle
import refimpl as R
import synth


def _random_cases(seed, count):
    rng = np.random.default_rng(seed)
    for _ in range(count):
        n = int(rng.integers(6, 36))
        directed = bool(rng.random() < 0.4)
        q = int(rng.integers(1, 5))
        p = float(rng.uniform(0.05, 0.3))
        yield R.random_graph(rng, n, p, directed, q, kw_size=(1, 4), wmax=float(rng.choice([0.0, 0.2, 1.0]))), q


def _c1_cases(count):
    w = synth.make_workload("C1")
    for kw in w.queries[:count]:
        yield w.graph, list(kw)


def _contrib(c, arcs, Ts, q):
    """contrib(v) = {i : v in T_i and v in DAG_i(c)} from the recorded-path DAGs (reading R13)."""
    con = {}
    for i in range(q):
        nodes, _ = R.closure(c, i, arcs[i])
        for v in nodes:
            if v in Ts[i]:
                con.setdefault(v, set()).add(i)
    return con


@pytest.mark.parametrize("block", [1, 0])
def test_exact_extraction_equals_recorded_paths(block):
    """I7: the Thm. V.4 reconstruction (exact mode, reading R12) returns exactly the union of all
    hitting paths recorded during the search (Def. 2, Def. 3)."""
    cases = list(_random_cases(31 + block, 150)) + list(_c1_cases(25))
    checked = 0
    for g, kw in ((g, list(range(q))) if isinstance(q, int) else (g, q) for g, q in cases):
        for k in (1, 3, 10 ** 6):
            r = oracle.query(g, kw, k=k, block_central=block, level_cover=0)
            rM, depth, arcs = R.recorded_search(g, kw, r.a, k, block_central=block)
            assert (rM == r.M).all()
            assert sorted(depth) == r.centrals.tolist()
            for ans in r.answers:
                nodes, used = R.full_central_graph(ans.central, arcs)
                assert ans.nodes.tolist() == sorted(nodes)
                assert sorted(map(tuple, ans.arcs.tolist())) == sorted(used)
                checked += 1
    assert checked > 100


def test_literal_extraction_is_superset():
    """Literal Thm. V.4 (no not-yet-central test) can only add predecessors (reading R12)."""
    for g, q in _random_cases(41, 120):
        kw = list(range(q))
        ex = oracle.query(g, kw, k=10 ** 6, level_cover=0, extract_mode=oracle.EXTRACT_EXACT)
        li = oracle.query(g, kw, k=10 ** 6, level_cover=0, extract_mode=oracle.EXTRACT_LITERAL)
        ge = {a.central: (set(a.nodes.tolist()), set(map(tuple, a.arcs.tolist()))) for a in ex.answers}
        for a in li.answers:
            n_e, a_e = ge[a.central]
            assert n_e <= set(a.nodes.tolist()) and a_e <= set(map(tuple, a.arcs.tolist()))


def test_level_cover_properties():
    """I9 + the greedy rule of P:L454: keep c; keep keyword-node levels whole from the top down to the
    first level at which the cumulative cover (central node included) equals Q; keep exactly the nodes
    and arcs on hitting paths from kept sources; pruned graph is a subgraph of the unpruned one."""
    cases = [(g, list(range(q))) for g, q in _random_cases(51, 150)] + list(_c1_cases(25))
    for g, kw in cases:
        q = len(kw)
        full = oracle.query(g, kw, k=10 ** 6, level_cover=0)
        pr = oracle.query(g, kw, k=10 ** 6, level_cover=1)
        _, _, arcs = R.recorded_search(g, kw, full.a, 10 ** 6)
        Ts = R.keyword_sets(g, kw)
        Q = set(range(q))
        fmap = {a.central: a for a in full.answers}
        for a in pr.answers:
            c = a.central
            fa = fmap[c]
            kept = set(a.nodes.tolist())
            karcs = set(map(tuple, a.arcs.tolist()))
            assert c in kept
            assert kept <= set(fa.nodes.tolist())
            assert karcs <= set(map(tuple, fa.arcs.tolist()))
            con = _contrib(c, arcs, Ts, q)
            cc = con.get(c, set())
            others = {v: s for v, s in con.items() if v != c}
            if cc == Q:
                assert kept == {c} and not karcs
                continue
            # s* = the largest s whose cumulative cover (c plus every level >= s) equals Q
            def cover(s):
                return set(cc).union(*[others[v] for v in others if len(others[v]) >= s])
            s_star = max(s for s in range(1, q + 1) if cover(s) == Q)
            srcs = {v for v in others if len(others[v]) >= s_star}
            assert srcs <= kept                                                   # whole levels kept
            assert s_star == q or cover(s_star + 1) != Q
            # exactly the hitting paths from kept sources: per keyword, nodes forward-reachable
            exp_nodes, exp_arcs = {c}, set()
            for i in range(q):
                dn, da = R.closure(c, i, arcs[i])
                S_i = {v for v in dn if v in Ts[i] and (v == c or v in srcs)}
                reach, frontier = set(S_i), list(S_i)
                succ = {}
                for u, x in da:
                    succ.setdefault(u, []).append(x)
                while frontier:
                    u = frontier.pop()
                    for x in succ.get(u, []):
                        exp_arcs.add((u, x))
                        if x not in reach:
                            reach.add(x)
                            frontier.append(x)
                exp_nodes |= reach
            assert kept == exp_nodes and karcs == exp_arcs


def test_score_and_topk():
    """I10: key = d^lambda * sum of w over the returned (pruned) nodes, fp32 score = (float)key;
    I11: answers = the first min(k, |C|) centrals by (key asc, id asc)."""
    cases = [(g, list(range(q))) for g, q in _random_cases(61, 100)] + list(_c1_cases(40))
    for g, kw in cases:
        for lam in (0.2, 0.0, 1.0):
            for k in (1, 5):
                r = oracle.query(g, kw, k=k, lam=lam)
                allr = oracle.query(g, kw, k=10 ** 6, lam=lam, max_depth=254)
                order = sorted(zip(r.central_key.tolist(), r.centrals.tolist()))
                assert len(r.answers) == min(k, len(r.centrals))
                assert [a.central for a in r.answers] == [c for _, c in order[:k]]
                for a in r.answers:
                    s = float(np.sum(g.weight[a.nodes].astype(np.float64)))
                    assert a.key == (float(a.depth) ** lam) * s
                    assert a.score == np.float32(a.key)
                del allr
