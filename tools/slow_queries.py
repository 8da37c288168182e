"""The slowest latency-mode queries of a NEXT-4 sweep point (C3 graph, Knum 6, Topk 20): per-phase
microseconds and the top-down statistics, with dag_record auto (recorded DAG) and 0 (pre-pass + lazy
round 2).  Usage: slow_queries.py alpha [alpha ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

w = synth.make_workload("C3", n_queries=1)
g = w.graph
G = kgs.kgs_load_graph(g)
q6 = synth.make_queries(g, 4006, sizes={6: 30}, band=(17000, 57000), rare=(300, 600), rare_frac=0.1)
for alpha in (float(x) for x in sys.argv[1:]):
    p = kgs.make_params(alpha=alpha)
    kgs.kgs_query(G, q6[0], 20, p)
    res = [(kgs.kgs_query(G, kw, 20, p).stats, kw) for kw in q6]
    res.sort(key=lambda t: -t[0]["ms_total"])
    for st, kw in res[:3]:
        keys = ("levels", "n_centrals", "n_evaluated", "n_cut", "overflow", "td_pred_arcs", "dag_arcs", "n_tier4")
        print(f"alpha {alpha} rec=auto {st['ms_total']:.2f} ms", {k: st[k] for k in keys},
              {k: round(v) for k, v in st["phases_us"].items()}, flush=True)
        st0 = kgs.kgs_query(G, kw, 20, kgs.make_params(alpha=alpha, dag_record=0)).stats
        print(f"alpha {alpha} rec=0    {st0['ms_total']:.2f} ms", {k: st0[k] for k in keys},
              {k: round(v) for k, v in st0["phases_us"].items()}, flush=True)
