"""Run single C4 queries (by index) in the latency mode with the recorded DAG and with the pre-pass,
printing the search / top-down statistics (capacity debugging).  Usage: c4_one.py idx [idx ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

w = synth.make_workload("C4")
G = kgs.kgs_load_graph(w.graph)
for i in (int(x) for x in sys.argv[1:]):
    kw = w.queries[i]
    for rec in os.environ.get("RECS", "1,0").split(","):
        try:
            r = kgs.kgs_query(G, kw, w.k, kgs.make_params(prune=int(os.environ.get("PRUNE", "1")), dag_record=int(rec)))
            s = r.stats
            print(i, "rec", rec, "q", len(kw), {k: s[k] for k in ("levels", "n_centrals", "arcs_scanned", "td_arcs",
                                                                  "td_pred_arcs", "dag_arcs", "overflow", "ms_search",
                                                                  "ms_topdown", "n_evaluated", "n_cut")}, {k: round(v) for k, v in s["phases_us"].items()}, flush=True)
        except Exception as e:
            print(i, "rec", rec, "failed:", e, flush=True)
