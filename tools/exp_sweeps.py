"""NEXT-4: synthetic counterparts of the paper's Exp-1/2/3 (Figs. 6-8) on the C3 graph: query
latency while sweeping Knum (keywords per query), Topk and alpha around Table III's defaults (Knum 6,
Topk 20, alpha 0.1), with the per-phase split laid out like the paper's figures:

  init        reset of the previous query's state + initialisation of M / sources
  enq+ident   enqueuing frontiers + identifying central nodes — one fused compaction pass
              here (the paper times them separately; the engine merges new hits, identifies central nodes
              and builds the next queue in the same pass over the level's bitmap)
  expansion   Alg. 2
  top-down    predecessor pre-pass, extraction + level-cover + Eq. 6, top-k, emit

One kgs_query per query (latency mode: the whole GPU on one query); per-phase times from the in-kernel
%globaltimer stamps (kgs_result_phases), per-query totals from the device clock.  Beside every point the
oracle (oracle/, single-threaded, pinned to one core) answers the first --oracle queries of the point with
the same parameters: its time per query is reported and its answers must equal the GPU's (parity at the
sweep's values).  Trends only: the paper's absolute numbers are Wikidata on a GTX 1080 Ti.
Usage: exp_sweeps.py [queries per point] [oracle queries per point]"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 30
NO = int(sys.argv[2]) if len(sys.argv) > 2 else 2
w = synth.make_workload("C3", n_queries=1)
g = w.graph
G = kgs.kgs_load_graph(g, device=0)
PHASE = {"start": "init", "reset": "init", "sources": "init", "merge": "enq+ident", "expand": "expansion",
         "search_end": "expansion"}
spec = dict(band=(17000, 57000), rare=(300, 600), rare_frac=0.1)
mismatch = 0


def run(queries, k, alpha):
    global mismatch
    p = kgs.make_params(alpha=alpha)
    kgs.kgs_query(G, queries[0], k, p)   # warm (activation cache for this alpha)
    ms, lev, cen = [], [], []
    ph = {"init": [], "enq+ident": [], "expansion": [], "top-down": []}
    res = []
    for kw in queries:
        r = kgs.kgs_query(G, kw, k, p)
        res.append(r)
        acc = dict.fromkeys(ph, 0.0)
        for name, us in r.stats.get("phases_us", {}).items():
            acc[PHASE.get(name, "top-down")] += us
        for name in ph:
            ph[name].append(acc[name])
        ms.append(r.stats["ms_total"])
        lev.append(r.stats["levels"])
        cen.append(r.stats["n_centrals"])
    os.sched_setaffinity(0, {min(os.sched_getaffinity(0))})
    t0 = time.perf_counter()
    for kw, r in zip(queries[:NO], res[:NO]):
        o = oracle.query(g, kw, k, alpha=alpha)
        mismatch += [(a.central, a.key, a.nodes.tolist()) for a in o.answers] != \
            [(a.central, a.score_key, a.nodes.tolist()) for a in r.answers]
    ora = (time.perf_counter() - t0) / max(1, min(NO, len(queries))) * 1e3
    os.sched_setaffinity(0, set(range(os.cpu_count())))
    ms = np.array(ms)
    return (f"mean {ms.mean():7.3f} ms  p50 {np.median(ms):6.3f}  p95 {np.percentile(ms, 95):7.3f}  "
            f"levels {np.mean(lev):4.2f}  |C| {np.mean(cen):8.1f}  " +
            "  ".join(f"{n} {np.mean(v):7.1f}" for n, v in ph.items()) + f" us   oracle {ora:8.1f} ms/query")


print(f"C3 graph: {g.n} nodes, {g.n_arcs} arcs, A = {g.A:.3f}; {N} queries per point, oracle on {NO} of them "
      f"(one core); phase columns are mean microseconds per query")
print("Exp-1 (Knum; Topk 20, alpha 0.1)")
for q in range(2, 9):
    print(f"  Knum {q}: " + run(synth.make_queries(g, 4000 + q, sizes={q: N}, **spec), 20, 0.1), flush=True)
q6 = synth.make_queries(g, 4006, sizes={6: N}, **spec)
print("Exp-2 (Topk; Knum 6, alpha 0.1)")
for k in (5, 10, 20, 50, 100):
    print(f"  Topk {k:3d}: " + run(q6, k, 0.1), flush=True)
print("Exp-3 (alpha; Knum 6, Topk 20)")
for a in (0.1, 0.3, 0.5, 0.7, 0.9):
    print(f"  alpha {a}: " + run(q6, 20, a), flush=True)
print(f"oracle parity at every point: {'ok' if mismatch == 0 else f'{mismatch} MISMATCHES'}")
G.close()
