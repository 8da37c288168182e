"""Workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck) over the engine:
C1 (every query, single launches and one batch of query groups) and a C2 sample (single + batch), each
answer compared with the oracle so a sanitizer run is also a parity run.
Usage: compute-sanitizer --tool <tool> python tools/sanitize_run.py [n_c1] [n_c2]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

# SAN_PARAMS="mk_min=0 prune_min=40 defer_min=20": kgs_params overrides for both launch kinds (drives the
# per-candidate cut-off test and the deferred whole-grid queries on the small configs)
P = os.environ.get("SAN_PARAMS", "")
params = kgs.make_params(**{k: int(v) for k, v in (x.split("=") for x in P.split())}) if P else None
n1 = int(sys.argv[1]) if len(sys.argv) > 1 else 100
n2 = int(sys.argv[2]) if len(sys.argv) > 2 else 3
bad = 0
for name, cnt in (("C1", n1), ("C2", n2)):
    if cnt <= 0:
        continue
    w = synth.make_workload(name)
    qs = w.queries[:cnt] if name == "C1" else w.queries[::97][:cnt]
    exp = [oracle.query(w.graph, kw, w.k) for kw in qs]
    G = kgs.kgs_load_graph(w.graph)
    single = [kgs.kgs_query(G, kw, w.k, params) for kw in qs]
    batch = kgs.kgs_query_batch(G, qs, w.k, params, 4)
    for kw, o, r1, r2 in zip(qs, exp, single, batch):
        want = [(a.central, a.key, a.nodes.tolist(), a.arcs.tolist()) for a in o.answers]
        for r in (r1, r2):
            got = [(a.central, a.score_key, a.nodes.tolist(), a.arcs.tolist()) for a in r.answers]
            bad += got != want
    G.close()
    print(f"{name}: {len(qs)} queries x (single, batch G=4) checked against the oracle", flush=True)
print("mismatches:", bad)
sys.exit(1 if bad else 0)
