"""Per-query push vs pull vs auto on a config's bench-order queries (latency mode, one launch each):
search time and arcs per direction.  Usage: pull_compare.py [config] [n_queries]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C3"
nq = int(sys.argv[2]) if len(sys.argv) > 2 else 20
w = synth.make_workload(name)
order = np.random.default_rng(12345).permutation(len(w.queries))
qs = [w.queries[i] for i in order][:nq]
G = kgs.kgs_load_graph(w.graph)
tot = {}
for d, nm in ((kgs.KGS_DIR_PUSH, "push"), (kgs.KGS_DIR_PULL, "pull"), (kgs.KGS_DIR_AUTO, "auto")):
    p = kgs.make_params(direction=d)
    for kw in qs[:3]:
        kgs.kgs_query(G, kw, w.k, p)
    for j, kw in enumerate(qs):
        r = kgs.kgs_query(G, kw, w.k, p)
        s = r.stats
        tot.setdefault(nm, []).append(s["ms_search"])
        print(f"{nm} q{j} kw={len(kw)} levels={s['levels']} pull_at={s['pull_level']} arcs={s['arcs_scanned']} "
              f"frontier={s['frontier_total']} search_ms={s['ms_search']:.3f} total_ms={s['ms_total']:.3f}", flush=True)
for nm, v in tot.items():
    print(f"{nm}: mean search {np.mean(v):.3f} ms, p50 {np.median(v):.3f} ms")
