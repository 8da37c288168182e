"""Run the same batch launch several times and compare every query's search statistics and answers
(the engine's results must not depend on timing: Thm. V.2 / reading R10).  Usage: determinism_check.py
[config] [reps] [groups]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402
from bench import step_queries  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C4"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
groups = int(sys.argv[3]) if len(sys.argv) > 3 else 8
w = synth.make_workload(name)
qs, _ = step_queries(name, w.queries)
G = kgs.kgs_load_graph(w.graph)
runs = []
for rep in range(reps):
    res = kgs.kgs_query_batch(G, qs, w.k, None, groups)
    runs.append([(r.stats["levels"], r.stats["stop_reason"], r.stats["n_centrals"], r.stats["arcs_scanned"],
                  r.stats["frontier_total"], r.stats["hits"],
                  tuple((a.central, a.score_key, a.n_nodes if hasattr(a, "n_nodes") else len(a.nodes)) for a in r.answers))
                 for r in res])
    print(f"run {rep}: arcs {sum(x[3] for x in runs[-1])}", flush=True)
bad = 0
for i in range(len(qs)):
    vals = [run[i] for run in runs]
    if any(v != vals[0] for v in vals[1:]):
        bad += 1
        if bad <= 10:
            for j, v in enumerate(vals):
                print(f"query {i} run {j}: levels {v[0]} stop {v[1]} |C| {v[2]} arcs {v[3]} frontier {v[4]} hits {v[5]} "
                      f"answers {'same' if v[6] == vals[0][6] else 'DIFFER'}", flush=True)
print(f"{name}: {len(qs)} queries x {reps} launches (G = {groups}): {bad} queries differ", flush=True)
