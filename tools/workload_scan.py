"""Search-only statistics of every query of a config (kgs_params.search_only = 1: the top-down is skipped,
so no answers): levels, |C|, arcs — to find the queries whose candidate sets make the top-down heavy.
Usage: workload_scan.py [config]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C4"
w = synth.make_workload(name)
G = kgs.kgs_load_graph(w.graph)
res = kgs.kgs_query_batch(G, w.queries, w.k, kgs.make_params(search_only=1), 8)
nc = np.array([r.stats["n_centrals"] for r in res])
lv = np.array([r.stats["levels"] for r in res])
arcs = np.array([r.stats["arcs_scanned"] for r in res])
print(name, len(res), "queries; |C| percentiles 50/90/99/max:", np.percentile(nc, [50, 90, 99]).tolist(), nc.max())
for t in (1000, 10000, 100000):
    print(f"|C| > {t}: {(nc > t).sum()}")
print("levels histogram:", np.bincount(lv).tolist())
for i in np.argsort(-nc)[:15]:
    print(i, w.queries[i], "levels", lv[i], "|C|", nc[i], "arcs", arcs[i])
