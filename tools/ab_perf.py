"""A/B timing of a libkgs build (KGS_LIB): C3 latency mode (one launch per query, bench order) and batch
mode (one launch, G groups).  Usage: KGS_LIB=... ab_perf.py [n_latency] [batch] [G]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

nl = int(sys.argv[1]) if len(sys.argv) > 1 else 150
batch = int(sys.argv[2]) if len(sys.argv) > 2 else 1400
groups = int(sys.argv[3]) if len(sys.argv) > 3 else 8
w = synth.make_workload("C3")
order = np.random.default_rng(12345).permutation(len(w.queries))
qs = [w.queries[i] for i in order]
G = kgs.kgs_load_graph(w.graph)
s = torch.cuda.current_stream()
for kw in qs[:5]:
    kgs.kgs_query(G, kw, w.k)
lat = []
for kw in qs[:nl]:
    t = torch.tensor(kw, dtype=torch.int32, device="cuda")
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    kgs.kgs_query_device(G, t.data_ptr(), len(kw), w.k, None, s.cuda_stream)
    e1.record(s)
    kgs.kgs_query_fetch(G, len(kw), 0, s.cuda_stream)
    lat.append(e0.elapsed_time(e1))
bq = (qs * ((batch + len(qs) - 1) // len(qs)))[:batch]
kwp = torch.full((len(bq), 8), -1, dtype=torch.int32)
for i, q in enumerate(bq):
    kwp[i, :len(q)] = torch.tensor(q, dtype=torch.int32)
kwd = kwp.cuda()
qld = torch.tensor([len(q) for q in bq], dtype=torch.int32, device="cuda")
best = 1e9
for rep in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    kgs.kgs_query_batch_device(G, len(bq), kwd.data_ptr(), qld.data_ptr(), w.k, None, groups, s.cuda_stream)
    e1.record(s)
    kgs.kgs_query_batch_fetch(G, [len(q) for q in bq], s.cuda_stream)
    best = min(best, e0.elapsed_time(e1))
print(f"{os.environ.get('KGS_LIB', 'default')}: latency p50 {np.median(lat):.4f} ms mean {np.mean(lat):.4f} ms "
      f"p95 {np.percentile(lat, 95):.4f} ms | batch {len(bq) / best * 1e3:.1f} q/s (G={groups})", flush=True)
