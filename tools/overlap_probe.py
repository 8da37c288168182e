"""How much adjacency work would B queries share if they traversed the graph together (NEXT-1)?

For B consecutive C3 bench-order queries (latency mode, want_levels = 1: the whole M back), per level l
the set X_l(q) of nodes that expand at l (newly hit and active, or waking up; not a blocked central)
and its out-arcs.  Reports sum over q of arcs(X_l(q)) against arcs(union_q X_l(q)) per level and overall:
the factor by which a joint pass over the union frontier would cut adjacency reads and status gathers.
Usage: overlap_probe.py [B] [groups of B]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

B = int(sys.argv[1]) if len(sys.argv) > 1 else 8
NG = int(sys.argv[2]) if len(sys.argv) > 2 else 4
w = synth.make_workload("C3")
g = w.graph
deg = np.diff(g.row_ptr).astype(np.int64)
order = np.random.default_rng(12345).permutation(len(w.queries))
qs = [w.queries[i] for i in order]
G = kgs.kgs_load_graph(g)
tot_sum = tot_union = 0
for grp in range(NG):
    batch = qs[grp * B:(grp + 1) * B]
    xs = []   # per query: list over levels of boolean masks
    for kw in batch:
        r = kgs.kgs_query(G, kw, w.k, kgs.make_params(want_levels=1))
        M = r.M.astype(np.int32)
        a = r.a.astype(np.int32)
        d = r.stats["levels"]
        fin = M < 255
        full = fin.all(1)
        depth = np.where(full, np.where(fin, M, 0).max(1), 255)
        lv = []
        for l in range(d):
            # the work list (R22): newly hit at l and active, or hit earlier and waking up at l
            # (nodes re-queued for a gated neighbour, Alg. 2 ln 19, are left out)
            new = (M == l).any(1) & (a <= l)
            wake = (fin & (M < l)).any(1) & (a == l)
            lv.append((new | wake) & ~(full & (depth <= l)))
        xs.append(lv)
    L = max(len(x) for x in xs)
    for l in range(L):
        masks = [x[l] for x in xs if l < len(x)]
        s = sum(int(deg[m].sum()) for m in masks)
        u = np.zeros(g.n, bool)
        for m in masks:
            u |= m
        un = int(deg[u].sum())
        tot_sum += s
        tot_union += un
        print(f"group {grp} level {l}: queries {len(masks)}  arcs sum {s:>12,}  union {un:>12,}  share {s / max(un, 1):.2f}x",
              flush=True)
print(f"B={B}: total arcs sum {tot_sum:,} union {tot_union:,} -> joint pass reads {tot_union / max(tot_sum, 1):.3f} of the "
      f"separate passes ({tot_sum / max(tot_union, 1):.2f}x sharing)")
