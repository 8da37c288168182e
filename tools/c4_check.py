import os, sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_icde_yangajtw19_b200 as kgs, synth
w = synth.make_workload("C4")
G = kgs.kgs_load_graph(w.graph)
qs = w.queries
mx = []
for b0 in range(0, len(qs), 512):
    sub = qs[b0:b0+512]
    try:
        res = kgs.kgs_query_batch(G, sub, w.k, None, 8)
    except Exception as e:
        print("batch", b0, "failed", e, flush=True); break
    st = [r.stats for r in res]
    j = int(np.argmax([s["td_pred_arcs"] for s in st]))
    print("batch", b0, "max td_pred_arcs", st[j]["td_pred_arcs"], "td_arcs", st[j]["td_arcs"], "centrals", st[j]["n_centrals"], "q", sub[j], flush=True)
