import os, sys
sys.path.insert(0, '/root/repo'); sys.path.insert(0, '/root/repo/tests')
import numpy as np, oracle, refimpl as R, paper_conf_icde_yangajtw19_b200 as kgs
rng = np.random.default_rng(2024)
for case in range(160):
    n = int(rng.integers(4, 70)); directed = bool(rng.random() < 0.4); q = int(rng.integers(1, 9))
    g = R.random_graph(rng, n, float(rng.uniform(0.03, 0.3)), directed, q, kw_size=(1, 5), wmax=float(rng.choice([0.0, 0.2, 1.0])))
    G = kgs.kgs_load_graph(g); kw = list(range(q))
    for _ in range(3):
        kk=int(rng.choice([1, 2, 5, 40])); al=float(rng.choice([0.05, 0.1, 0.4])); lam=float(rng.choice([0.0, 0.2, 1.0])); md=int(rng.choice([1, 3, 254])); bc=int(rng.integers(0, 2)); em=int(rng.integers(0, 2)); lc=int(rng.integers(0, 2))
        o = oracle.query(g, kw, kk, alpha=al, lam=lam, max_depth=md, block_central=bc, extract_mode=em, level_cover=lc)
        r = kgs.kgs_query(G, kw, kk, kgs.make_params(alpha=al, lam=lam, max_depth=md, block_central=bc, extract_mode=em, level_cover=lc, want_levels=1))
        if not (r.M == o.M).all():
            bad = np.argwhere(r.M != o.M)
            print("case", case, "n", n, "directed", directed, "q", q, "k", kk, "alpha", al, "md", md, "blk", bc, "bad", bad[:4].tolist(), "levels", r.stats['levels'], o.levels)
            print(" a", o.a.tolist()); print(" M_o", o.M.tolist()); print(" M_g", r.M.tolist())
            print(" edges", [(u, int(x)) for u in range(n) for x in g.col_idx[g.row_ptr[u]:g.row_ptr[u+1]]])
            print(" kw", [g.kw_nodes[g.kw_ptr[t]:g.kw_ptr[t+1]].tolist() for t in range(q)])
            sys.exit(0)
    G.close()
print("all ok")
