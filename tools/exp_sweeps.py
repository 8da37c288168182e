"""NEXT-4: synthetic counterparts of the paper's Exp-1/2/3 (Figs. 6-8): query latency on the
C3 graph while sweeping Knum (keywords per query), Topk and alpha around Table III's defaults
(Knum 6, Topk 20, alpha 0.1).  One kgs_query per query (latency mode); per-query time is the library's
device-measured ms_total; the per-phase split is the mean of kgs_result_phases (microseconds).
Trends only: the paper's absolute numbers are Wikidata on a GTX 1080 Ti."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 30
w = synth.make_workload("C3", n_queries=1)
g = w.graph
G = kgs.kgs_load_graph(g, device=0)
BOTTOM_UP = {"reset", "sources", "merge", "expand", "search_end"}
spec = dict(band=(17000, 57000), rare=(300, 600), rare_frac=0.1)


def run(queries, k, alpha):
    p = kgs.make_params(alpha=alpha)
    kgs.kgs_query(G, queries[0], k, p)   # warm
    ms, lev, cen, bu, td = [], [], [], [], []
    for kw in queries:
        r = kgs.kgs_query(G, kw, k, p)
        ph = r.stats.get("phases_us", {})
        bu.append(sum(v for n, v in ph.items() if n in BOTTOM_UP))
        td.append(sum(v for n, v in ph.items() if n not in BOTTOM_UP))
        ms.append(r.stats["ms_total"])
        lev.append(r.stats["levels"])
        cen.append(r.stats["n_centrals"])
    ms = np.array(ms)
    return (f"mean {ms.mean():7.3f} ms  p50 {np.median(ms):7.3f} ms  p95 {np.percentile(ms, 95):7.3f} ms  "
            f"levels {np.mean(lev):4.2f}  centrals {np.mean(cen):9.1f}  "
            f"bottom-up {np.mean(bu):8.1f} us  top-down {np.mean(td):8.1f} us")


print(f"C3 graph: {g.n} nodes, {g.n_arcs} arcs, A = {g.A:.3f}; {N} queries per point")
print("Exp-1 (Knum; Topk 20, alpha 0.1)")
for q in range(2, 9):
    print(f"  Knum {q}: " + run(synth.make_queries(g, 4000 + q, sizes={q: N}, **spec), 20, 0.1))
q6 = synth.make_queries(g, 4006, sizes={6: N}, **spec)
print("Exp-2 (Topk; Knum 6, alpha 0.1)")
for k in (5, 10, 20, 50, 100):
    print(f"  Topk {k:3d}: " + run(q6, k, 0.1))
print("Exp-3 (alpha; Knum 6, Topk 20)")
for a in (0.1, 0.3, 0.5, 0.7, 0.9):
    print(f"  alpha {a}: " + run(q6, 20, a))
G.close()
