"""Find small graphs on which the exact key cut-off of pruning round 2 fires (tests/test_gpu_prune.py)."""
import os
import sys

sys.path.insert(0, '.')
sys.path.insert(0, 'tests')
os.environ["KGS_PRUNE_MIN"] = "40"
import numpy as np  # noqa: E402
import synth  # noqa: E402
import paper_conf_icde_yangajtw19_b200 as kgs  # noqa: E402
from test_gpu_prune import medium_graph  # noqa: E402

for seed in range(2):
    for deg in (8, 16):
        for ksz in (100, 250):
            rng = np.random.default_rng(500 + seed)
            n, q = 6000, 3
            g0 = medium_graph(500 + seed, n=n, deg=deg, q=q, kw_size=10, wpow=3.0)
            perm = rng.permutation(n)
            kws = [sorted(perm[i * ksz:(i + 1) * ksz].tolist()) for i in range(q)]
            edges = [(u, int(v)) for u in range(n) for v in g0.col_idx[g0.row_ptr[u]:g0.row_ptr[u + 1]] if u < v]
            g = synth.from_edges(n, edges, g0.weight, kws, 2.0)
            G = kgs.kgs_load_graph(g)
            for k in (5, 20, 50):
                r = kgs.kgs_query(G, [0, 1, 2], k, kgs.make_params(prune=1))
                s = r.stats
                print(seed, deg, ksz, k, {x: s[x] for x in ("levels", "n_centrals", "n_evaluated", "n_cut")}, flush=True)
            G.close()
