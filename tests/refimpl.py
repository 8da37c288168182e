"""Independent pins for the oracle — textbook routines and alternative formulations (test-side only).

None of this is the oracle: these are the *other* things the oracle is checked against
(DESIGN.md "Oracle pins"):
  * multi-source textbook BFS distances (special case a = 0, no central blocking);
  * earliest-arrival search with a priority queue under the activation gate (special case: no blocking);
  * the fixpoint characterisation I3 of the hitting-level matrix M ("min over neighbours + 1,
    subject to activation", BASELINE.json north_star);
  * hitting paths recorded during the search (Def. 2, P:L128 — the CPU-Par-d idea) whose
    closure must equal the oracle's Thm. V.4 reconstruction (I7);
  * characterising properties of the level-cover result (I9) and brute-force sorting (I11).
"""
from __future__ import annotations

import heapq
import json
import os
from collections import deque

import numpy as np

INF = 255
GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def golden_graph(d):
    import synth
    if d.get("directed"):
        return synth.from_edges(d["n"], [tuple(e) for e in d["arcs"]], d["weight"], d["keywords"], d["A"],
                                directed=True)
    return synth.from_edges(d["n"], [tuple(e) for e in d["edges"]], d["weight"], d["keywords"], d["A"])


def out_adj(g):
    return [g.col_idx[g.row_ptr[v]:g.row_ptr[v + 1]].tolist() for v in range(g.n)]


def in_adj(g):
    adj = [[] for _ in range(g.n)]
    for u in range(g.n):
        for x in g.col_idx[g.row_ptr[u]:g.row_ptr[u + 1]]:
            adj[int(x)].append(u)
    return adj


def keyword_sets(g, kw_ids):
    return [set(g.kw_nodes[g.kw_ptr[t]:g.kw_ptr[t + 1]].tolist()) for t in kw_ids]


def bfs_dist(n, adj, sources):
    """Textbook multi-source BFS hop distance, INF if unreachable."""
    d = [INF] * n
    dq = deque()
    for s in sources:
        d[s] = 0
        dq.append(s)
    while dq:
        u = dq.popleft()
        for x in adj[u]:
            if d[x] == INF:
                d[x] = d[u] + 1
                dq.append(x)
    return d


def gated_earliest_arrival(n, adj, a, in_K, sources):
    """Earliest level at which each node is reached when a node u can only send from level
    max(t_u, a_u) on and a non-keyword node x can only be reached at a level >= a_x.
    Priority-queue (Dijkstra) search over non-decreasing arrival functions."""
    t = [INF] * n
    pq = []
    for s in sources:
        t[s] = 0
        heapq.heappush(pq, (0, s))
    done = [False] * n
    while pq:
        tu, u = heapq.heappop(pq)
        if done[u] or tu != t[u]:
            continue
        done[u] = True
        depart = max(tu, int(a[u]))
        for x in adj[u]:
            arrive = depart + 1
            if not in_K[x]:
                arrive = max(arrive, int(a[x]))
            if arrive < t[x]:
                t[x] = arrive
                heapq.heappush(pq, (arrive, x))
    return t


def fixpoint_violations(g, kw_ids, a, M, block_central, D):
    """Invariant I3: for n not in T_i, M[n][i] = 1 + min over in-neighbours u (with M[u][i] finite and,
    under blocking, u not yet central when it would send) of max(M[u][i], a_u, g_n), g_n = a_n - 1 for
    n outside K and 0 inside K -- when that value is <= D (the level the search stopped at; 254 if it
    was exhausted); otherwise INF.  Returns the list of (node, keyword) pairs that violate it."""
    n, q = M.shape
    Ts = keyword_sets(g, kw_ids)
    K = set().union(*Ts)
    inn = in_adj(g)
    bad = []
    for x in range(n):
        for i in range(q):
            if x in Ts[i]:
                if M[x, i] != 0:
                    bad.append((x, i))
                continue
            gx = 0 if x in K else int(a[x]) - 1
            best = INF
            for u in inn[x]:
                mu = int(M[u, i])
                if mu == INF:
                    continue
                send = max(mu, int(a[u]), gx)
                if block_central and (M[u] != INF).all() and int(M[u].max()) <= send:
                    continue  # u was central (depth = max row) before level `send`
                best = min(best, send + 1)
            expect = best if best <= D else INF
            if int(M[x, i]) != expect:
                bad.append((x, i))
    return bad


def recorded_search(g, kw_ids, a, k, block_central=1, max_depth=254):
    """Level-synchronous search that RECORDS every expansion arc that hits a node (Def. 2 hitting
    paths; P:L508 CPU-Par-d records paths during the search).  Returns (M, depth dict, arcs) where
    arcs[i] = set of (u, x) such that u hit x in B_i.  Termination: identification then |C| >= k."""
    n = g.n
    q = len(kw_ids)
    Ts = keyword_sets(g, kw_ids)
    K = set().union(*Ts)
    adj = out_adj(g)
    M = np.full((n, q), INF, np.int64)
    for i, T in enumerate(Ts):
        for v in T:
            M[v, i] = 0
    depth = {}
    arcs = [set() for _ in range(q)]
    amax = int(a.max()) if n else 0
    level = 0
    while True:
        for v in range(n):
            if v not in depth and (M[v] != INF).all():
                depth[v] = level
        if len(depth) >= k or level == max_depth:
            break
        new = {}
        for v in range(n):
            if block_central and v in depth:
                continue
            if a[v] > level:
                continue
            for i in range(q):
                if M[v, i] > level:
                    continue
                for x in adj[v]:
                    if M[x, i] != INF:
                        continue
                    if x not in K and a[x] > level + 1:
                        continue
                    new.setdefault((x, i), []).append(v)
        for (x, i), us in new.items():
            M[x, i] = level + 1
            for u in us:
                arcs[i].add((u, x))
        if not new and level >= amax:
            break
        level += 1
    return M, depth, arcs


def closure(c, i, arcs_i):
    """Backward closure from c over recorded arcs of keyword i: the nodes and arcs of all hitting
    paths of c in B_i (Def. 2 / Def. 3)."""
    pred = {}
    for u, x in arcs_i:
        pred.setdefault(x, []).append(u)
    nodes = {c}
    used = set()
    stack = [c]
    while stack:
        x = stack.pop()
        for u in pred.get(x, []):
            used.add((u, x))
            if u not in nodes:
                nodes.add(u)
                stack.append(u)
    return nodes, used


def full_central_graph(c, arcs):
    nodes, used = set(), set()
    for i in range(len(arcs)):
        nd, us = closure(c, i, arcs[i])
        nodes |= nd
        used |= us
    return nodes, used


def random_graph(rng, n, p_edge, directed, q, kw_size=(1, 3), wmax=1.0):
    """Tiny random graph with random weights on the 2^-24 grid and q random keyword sets."""
    import synth
    edges = []
    for u in range(n):
        for v in range(n):
            if u != v and (directed or u < v) and rng.random() < p_edge:
                edges.append((u, v))
    w = (rng.integers(0, 1 << 24, size=n) * wmax / (1 << 24)).astype(np.float32)
    w = (np.floor(w.astype(np.float64) * (1 << 24) + 0.5) / (1 << 24)).astype(np.float32)
    kws = []
    for _ in range(q):
        s = int(rng.integers(kw_size[0], kw_size[1] + 1))
        kws.append(sorted(rng.choice(n, size=s, replace=False).tolist()))
    A = float(rng.choice([1.0, 1.5, 2.0, 2.5, 3.68]))
    return synth.from_edges(n, edges, w, kws, A, directed=directed)
