"""Short driver for ncu captures: load a config's graph, run `--warm` queries, then `--queries` more
(the ones ncu is pointed at with -s / -c).  Uses the same query permutation as bench.py."""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3")
ap.add_argument("--warm", type=int, default=3)
ap.add_argument("--queries", type=int, default=5)
ap.add_argument("--relabel", type=int, default=1)
args = ap.parse_args()
w = synth.make_workload(args.config)
order = np.random.default_rng(12345).permutation(len(w.queries))
qs = [w.queries[i] for i in order]
G = kgs.kgs_load_graph(w.graph, relabel=bool(args.relabel))
for i in range(args.warm + args.queries):
    r = kgs.kgs_query(G, qs[i % len(qs)], w.k)
    print(i, len(qs[i % len(qs)]), r.stats, flush=True)
