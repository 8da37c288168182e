"""Time the NEXT-2 preprocessing on the C3 graph: A from 10^4 sampled pairs and Eq. 2 weights
over random in-arc labels.  Wall clock around each C-ABI call (host inputs, so the copies are included)."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_icde_yangajtw19_b200 as kgs
import synth

P = int(sys.argv[1]) if len(sys.argv) > 1 else 10_000
g = synth.rmat_graph(25, 8, 1, a_sources=1, a_pairs_per_source=1)
rng = np.random.default_rng(0)
nz = np.nonzero(np.diff(g.row_ptr) > 0)[0]
s = rng.choice(nz, P).astype(np.int32)
t = rng.choice(nz, P).astype(np.int32)
kgs.kgs_prep_pair_distances(g.row_ptr, g.col_idx, s[:64], t[:64])
t0 = time.perf_counter()
d, mean = kgs.kgs_prep_pair_distances(g.row_ptr, g.col_idx, s, t)
t1 = time.perf_counter()
print(f"pair distances: n={g.n} arcs={g.n_arcs} pairs={P} A={mean:.4f} unreachable={(d < 0).sum()} "
      f"max={d.max()} time={t1 - t0:.3f} s")
lab = np.minimum(rng.zipf(1.3, g.n_arcs) - 1, 1023).astype(np.int32)
kgs.kgs_prep_summary_weights(g.row_ptr, lab)
t0 = time.perf_counter()
wn, wr = kgs.kgs_prep_summary_weights(g.row_ptr, lab)
t1 = time.perf_counter()
print(f"summary weights: arcs={g.n_arcs} time={t1 - t0:.3f} s  (host->device copy of {g.n_arcs * 4 / 1e9:.2f} GB "
      f"labels included) w range [{wr.min():.3f}, {wr.max():.3f}]")
