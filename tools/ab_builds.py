"""A/B of engine builds on the same box: each build's package directory (binding + libkgs.so) is put first
on sys.path.  C3 latency mode (one launch per query, bench order: p50 / mean), two C4 level-5 queries in
latency mode (search / top-down ms) and the C3 bench batch (350 queries, G = 8).
Usage: ab_builds.py PKG_PARENT_DIR   (the directory that holds paper_conf_icde_yangajtw19_b200/)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.abspath(sys.argv[1]))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

print("package", kgs.__file__, flush=True)
w = synth.make_workload("C3")
order = np.random.default_rng(12345).permutation(len(w.queries))
qs = [w.queries[i] for i in order]
G = kgs.kgs_load_graph(w.graph)
s = torch.cuda.current_stream()
for kw in qs[:5]:
    kgs.kgs_query(G, kw, w.k)
for rep in range(2):
    lat = []
    for kw in qs[:200]:
        t = torch.tensor(kw, dtype=torch.int32, device="cuda")
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        kgs.kgs_query_device(G, t.data_ptr(), len(kw), w.k, None, s.cuda_stream)
        e1.record(s)
        kgs.kgs_query_fetch(G, len(kw), 0, s.cuda_stream)
        lat.append(e0.elapsed_time(e1))
    print(f"latency 200 C3 queries: p50 {np.median(lat):.3f} ms mean {np.mean(lat):.3f} ms", flush=True)
c4 = synth.config_queries("C4", w.graph)
for i in (2683, 11):
    r = kgs.kgs_query(G, c4[i], w.k)
    st = r.stats
    print(f"C4 {i}: search {st['ms_search']:.2f} ms top-down {st['ms_topdown']:.2f} ms "
          f"expand {st['phases_us'].get('expand', 0):.0f} us merge {st['phases_us'].get('merge', 0):.0f} us", flush=True)
kwp = torch.full((350, 8), -1, dtype=torch.int32)
for i, q in enumerate(qs[:350]):
    kwp[i, :len(q)] = torch.tensor(q, dtype=torch.int32)
kwd = kwp.cuda()
qld = torch.tensor([len(q) for q in qs[:350]], dtype=torch.int32, device="cuda")
for rep in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    kgs.kgs_query_batch_device(G, 350, kwd.data_ptr(), qld.data_ptr(), w.k, None, 8, s.cuda_stream)
    e1.record(s)
    kgs.kgs_query_batch_fetch(G, [len(q) for q in qs[:350]], s.cuda_stream)
    print(f"batch 350 C3 G=8: {e0.elapsed_time(e1):.2f} ms", flush=True)
