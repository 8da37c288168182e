"""Throughput of the query engine on a config's query set for several group counts G (one launch per
batch, device-resident keyword ids, CUDA-event timing).  Usage: batch_sweep.py [config] [G,...] [batch]"""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C3"
groups = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "1,2,4,8,16").split(",")]
batch = int(sys.argv[3]) if len(sys.argv) > 3 else 0
w = synth.make_workload(name)
order = np.random.default_rng(12345).permutation(len(w.queries))
qs = [w.queries[i] for i in order]
if batch:
    qs = (qs * ((batch + len(qs) - 1) // len(qs)))[:batch]
G = kgs.kgs_load_graph(w.graph, relabel=os.environ.get("KGS_RELABEL", "1") != "0")
kwp = torch.full((len(qs), 8), -1, dtype=torch.int32)
for i, q in enumerate(qs):
    kwp[i, :len(q)] = torch.tensor(q, dtype=torch.int32)
kwd = kwp.cuda()
qld = torch.tensor([len(q) for q in qs], dtype=torch.int32, device="cuda")
s = torch.cuda.current_stream()
# PARAMS="defer_min=0 mk_min=4096": kgs_params overrides
params = kgs.make_params(**{k: int(v) for k, v in (x.split("=") for x in os.environ.get("PARAMS", "").split())})
for g in groups:
    for rep in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(s)
        kgs.kgs_query_batch_device(G, len(qs), kwd.data_ptr(), qld.data_ptr(), w.k, params, g, s.cuda_stream)
        e1.record(s)
        res = kgs.kgs_query_batch_fetch(G, [len(q) for q in qs], s.cuda_stream)
        ms = e0.elapsed_time(e1)
        lat = sorted(r.stats["ms_total"] for r in res)
    print(f"{name} G={g:3d} batch={len(qs)} launch {ms:8.2f} ms  {len(qs) / ms * 1e3:9.1f} q/s  "
          f"query latency p50 {lat[len(lat) // 2]:.3f} ms p95 {lat[int(len(lat) * .95)]:.3f} ms "
          f"deferred {sum(r.stats['group'] == g for r in res) if g > 1 else 0} "
          f"max {lat[-1]:.1f} ms  {os.environ.get('PARAMS', '')}", flush=True)
    ph = {}
    for r in res:
        for k, v in r.stats["phases_us"].items():
            ph[k] = ph.get(k, 0.0) + v
    tot = sum(ph.values()) or 1.0
    print("   group-time share: " + " ".join(f"{k}={v / tot:.1%}" for k, v in sorted(ph.items(), key=lambda x: -x[1])),
          flush=True)
    # the same split by query class: |C| <= 512 (no pruning: every central extracted) and > 512
    for lo, hi in ((0, 512), (513, 10 ** 5), (10 ** 5 + 1, 10 ** 9)):
        sub = [r for r in res if lo <= r.stats["n_centrals"] <= hi]
        if not sub:
            continue
        ph = {}
        for r in sub:
            for k, v in r.stats["phases_us"].items():
                ph[k] = ph.get(k, 0.0) + v
        print(f"   |C| in [{lo}, {hi}]: {len(sub)} queries, group time {sum(ph.values()) / tot:.1%} of all: " +
              " ".join(f"{k}={v / tot:.1%}" for k, v in sorted(ph.items(), key=lambda x: -x[1])[:12]), flush=True)
