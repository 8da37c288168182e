"""Driver for an ncu capture of ONE batch launch of the engine (the bench's launch shape): load a
config's graph, run a warm batch (launch 1), then the captured batch (launch 2, `-s 1 -c 1`).
Usage: profile_batch.py [config] [batch] [groups] [param=value ...]   (kgs_params fields, e.g. search_only=1)"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
import synth  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C3"
batch = int(sys.argv[2]) if len(sys.argv) > 2 else 128
groups = int(sys.argv[3]) if len(sys.argv) > 3 else 8
over = dict(a.split("=") for a in sys.argv[4:])
params = kgs.make_params(**{k: int(v) for k, v in over.items()})
w = synth.make_workload(name)
from bench import step_queries  # noqa: E402  (the bench's query order: C3 permuted, C4 as generated)
qs, _ = step_queries(name, w.queries)
G = kgs.kgs_load_graph(w.graph)
if os.environ.get("L2GRAN"):   # experiment: cudaLimitMaxL2FetchGranularity (0x05) on the primary context
    import ctypes
    torch.cuda.init()
    rt = ctypes.CDLL("libcudart.so.12")
    rc = rt.cudaDeviceSetLimit(0x05, ctypes.c_size_t(int(os.environ["L2GRAN"]))) if os.environ["L2GRAN"] != "0" else -1
    got = ctypes.c_size_t(0)
    rt.cudaDeviceGetLimit(ctypes.byref(got), 0x05)
    print("L2 fetch granularity", os.environ["L2GRAN"], "rc", rc, "now", got.value, flush=True)
s = torch.cuda.current_stream()
for rep in range(2):
    sub = [qs[(rep * batch + j) % len(qs)] for j in range(batch)]
    kwp = torch.full((batch, 8), -1, dtype=torch.int32)
    for i, q in enumerate(sub):
        kwp[i, :len(q)] = torch.tensor(q, dtype=torch.int32)
    kwd = kwp.cuda()
    qld = torch.tensor([len(q) for q in sub], dtype=torch.int32, device="cuda")
    kgs.kgs_query_batch_device(G, batch, kwd.data_ptr(), qld.data_ptr(), w.k, params, groups, s.cuda_stream)
    res = kgs.kgs_query_batch_fetch(G, [len(q) for q in sub], s.cuda_stream)
    st = [r.stats for r in res]
    print(f"launch {rep}: {batch} queries, G={groups}, ms_launch {st[0]['ms_launch']:.2f}, "
          f"arcs {sum(x['arcs_scanned'] for x in st)}, td_arcs {sum(x['td_arcs'] for x in st)}, "
          f"centrals {sum(x['n_centrals'] for x in st)}, dag_arcs {sum(x['dag_arcs'] for x in st)}, "
          f"hits {sum(x['hits'] for x in st)}, frontier {sum(x['frontier_total'] for x in st)}, "
          f"pred_arcs {sum(x['td_pred_arcs'] for x in st)}, td_arcs_big {sum(x['td_arcs_big'] for x in st)}",
          flush=True)
