"""Where a query's time goes, from the engine's in-kernel phase stamps (%globaltimer at group barriers).

  python tools/phase_summary.py [--config C3] [--queries 80] [--relabel 1] [--groups 1]

Runs the bench's query order one query per launch (latency mode, G groups = 1 by default), then prints
the per-phase time summed over the queries, the mean, and per query class (levels)."""
import argparse
import collections
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3")
ap.add_argument("--queries", type=int, default=80)
ap.add_argument("--relabel", type=int, default=1)
ap.add_argument("--warm", type=int, default=3)
args = ap.parse_args()
w = synth.make_workload(args.config)
order = np.random.default_rng(12345).permutation(len(w.queries))
qs = [w.queries[i] for i in order]
G = kgs.kgs_load_graph(w.graph, relabel=bool(args.relabel))
for i in range(args.warm):
    kgs.kgs_query(G, qs[i], w.k)
tot = collections.Counter()
by_lv = collections.defaultdict(collections.Counter)
n_lv = collections.Counter()
ms = []
for i in range(args.queries):
    r = kgs.kgs_query(G, qs[i % len(qs)], w.k)
    s = r.stats
    ms.append(s["ms_total"])
    tot.update(s["phases_us"])
    by_lv[s["levels"]].update(s["phases_us"])
    n_lv[s["levels"]] += 1
print(f"relabel={args.relabel} queries={args.queries} mean ms_total={np.mean(ms):.3f} p50={np.median(ms):.3f}")
print("phase           total_us   mean_us")
for k, v in tot.most_common():
    print(f"{k:14s} {v:10.0f} {v / args.queries:9.1f}")
for lv in sorted(by_lv):
    c = by_lv[lv]
    print(f"levels={lv} n={n_lv[lv]}: " + " ".join(f"{k}={v / n_lv[lv]:.0f}" for k, v in c.most_common()))
