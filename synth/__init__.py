"""Seeded synthetic inputs for the Central Graph keyword-search hot path.

Input generation only: this module holds none of the method's query arithmetic (no activation map,
no BFS, no extraction, no score).  The oracle (``oracle/``) and the CUDA path
(``paper_conf_icde_yangajtw19_b200``) both consume what it returns and share nothing else.

Configs follow BASELINE.json ``configs`` / SURVEY.md §8(d) (C1..C5); the recipe is restated in
DESIGN.md "Input recipe".  Graph seed = config number, query seed = 1000 + config number.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libkgs_synth.so")
_lib = None


def build_lib(force: bool = False) -> str:
    src = os.path.join(_HERE, "kgs_synth.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-ffp-contract=off",
                               "-o", _LIB_PATH, src, "-lm"])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build_lib()
        lib = ctypes.CDLL(_LIB_PATH)
        lib.synth_build.restype = ctypes.c_void_p
        lib.synth_build.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_uint64, ctypes.c_int, ctypes.c_int64,
                                    ctypes.c_int, ctypes.c_int64, ctypes.c_double, ctypes.c_int64, ctypes.c_double,
                                    ctypes.c_double, ctypes.c_int, ctypes.c_int]
        lib.synth_sizes.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
        lib.synth_A.restype = ctypes.c_double
        lib.synth_A.argtypes = [ctypes.c_void_p]
        lib.synth_copy.argtypes = [ctypes.c_void_p] + [ctypes.c_void_p] * 5
        lib.synth_free.argtypes = [ctypes.c_void_p]
        lib.synth_arc_labels.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
        lib.synth_num_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


@dataclass
class Graph:
    """A synthetic knowledge graph: symmetric CSR + normalised node weights + keyword inverted index."""
    row_ptr: np.ndarray      # int64 [n+1]
    col_idx: np.ndarray      # int32 [arcs]
    weight: np.ndarray       # float32 [n], on the 2^-24 grid, in [0, 1]
    kw_ptr: np.ndarray       # int64 [V+1]
    kw_nodes: np.ndarray     # int32 [postings], ascending per keyword
    A: float                 # average shortest distance (sampled)
    symmetric: bool = True
    meta: dict = field(default_factory=dict)

    @property
    def n(self) -> int:
        return int(self.row_ptr.shape[0] - 1)

    @property
    def n_arcs(self) -> int:
        return int(self.col_idx.shape[0])

    @property
    def n_keywords(self) -> int:
        return int(self.kw_ptr.shape[0] - 1)

    def kw_size(self, t: int) -> int:
        return int(self.kw_ptr[t + 1] - self.kw_ptr[t])


def rmat_graph(scale: int, edge_factor: int, seed: int, *, n_hubs: int = 0, hub_arcs: int = 0,
               weight_mode: int = 0, n_labels: int = 1024, label_s: float = 1.2, vocab: int = 1 << 17,
               word_s: float = 1.0, words_mean_extra: float = 2.0, a_sources: int = 16,
               a_pairs_per_source: int = 625, labels: bool = False) -> Graph:
    """R-MAT(.57,.19,.19,.05) symmetric CSR with Eq.2 (weight_mode=0) or uniform (1) weights.
    labels=True also returns the per-arc edge labels the Eq. 2 weights were computed from, in
    ``meta["arc_labels"]`` (int32 [arcs])."""
    lib = _load()
    h = lib.synth_build(scale, edge_factor, seed, n_hubs, hub_arcs, weight_mode, n_labels, label_s, vocab,
                        word_s, words_mean_extra, a_sources, a_pairs_per_source)
    try:
        sz = np.zeros(6, dtype=np.int64)
        lib.synth_sizes(h, sz.ctypes.data)
        n, arcs, V, post, maxd, iso = (int(x) for x in sz)
        rp = np.empty(n + 1, np.int64)
        ci = np.empty(arcs, np.int32)
        w = np.empty(n, np.float32)
        kp = np.empty(V + 1, np.int64)
        kn = np.empty(post, np.int32)
        lib.synth_copy(h, rp.ctypes.data, ci.ctypes.data, w.ctypes.data, kp.ctypes.data, kn.ctypes.data)
        A = float(lib.synth_A(h))
        lab = None
        if labels:
            lab = np.empty(arcs, np.int32)
            lib.synth_arc_labels(h, lab.ctypes.data)
    finally:
        lib.synth_free(h)
    meta = dict(scale=scale, edge_factor=edge_factor, seed=seed, n_hubs=n_hubs, hub_arcs=hub_arcs,
                weight_mode=weight_mode, n_labels=n_labels, vocab=vocab, max_degree=maxd, isolated=iso,
                gen_threads=int(lib.synth_num_threads()))
    if lab is not None:
        meta["arc_labels"] = lab
    return Graph(rp, ci, w, kp, kn, A, True, meta)


def from_edges(n: int, edges, weight, keywords, A: float, *, directed: bool = False) -> Graph:
    """Small hand-written graphs (paper figures).  ``edges`` = list of (u, v); undirected edges are
    stored as two arcs unless ``directed``.  ``keywords`` = list of node lists (keyword id = index)."""
    adj = [set() for _ in range(n)]
    for u, v in edges:
        adj[u].add(v)
        if not directed:
            adj[v].add(u)
    rp = np.zeros(n + 1, np.int64)
    for v in range(n):
        rp[v + 1] = rp[v] + len(adj[v])
    ci = np.array([x for v in range(n) for x in sorted(adj[v])], dtype=np.int32)
    kp = np.zeros(len(keywords) + 1, np.int64)
    for t, lst in enumerate(keywords):
        kp[t + 1] = kp[t] + len(lst)
    kn = np.array([x for lst in keywords for x in sorted(lst)], dtype=np.int32)
    return Graph(rp, ci, np.asarray(weight, np.float32), kp, kn, float(A), not directed,
                 dict(hand_written=True))


# --------------------------------------------------------------------------- configs (BASELINE.json)

@dataclass
class Workload:
    name: str
    graph: Graph
    queries: list          # list of tuples of keyword ids
    k: int
    alpha: float = 0.1
    lam: float = 0.2


CONFIG_PARAMS = {
    # C1: tiny toy KG, ~1k nodes / ~4k edges, uniform random weights, 3-keyword queries, top-5
    "C1": dict(graph=dict(scale=10, edge_factor=4, seed=1, weight_mode=1, n_labels=64, vocab=64),
               qspec=dict(sizes={3: 100}, band=(8, 64), rare=None), k=5),
    # C2: 1M nodes / 8M edges power-law, 2-4 keyword queries, top-20
    "C2": dict(graph=dict(scale=20, edge_factor=8, seed=2, n_labels=1024, vocab=1 << 17),
               qspec=dict(sizes={2: 100, 3: 100, 4: 100}, band=(550, 1900), rare=None), k=20),
    # C3: Wikidata-scale, 2^25 nodes / 2^28 edges, 2-8 keyword queries, top-20
    "C3": dict(graph=dict(scale=25, edge_factor=8, seed=3, n_labels=4096, vocab=1 << 22),
               qspec=dict(sizes={q: 50 for q in range(2, 9)}, band=(17000, 57000), rare=(300, 600),
                          rare_frac=0.1), k=20),
    # C4: the C3 graph, 4096 queries with q ~ U{2..8}
    "C4": dict(graph=dict(scale=25, edge_factor=8, seed=3, n_labels=4096, vocab=1 << 22),
               qspec=dict(uniform_q=(2, 8), count=4096, band=(17000, 57000), rare=(300, 600),
                          rare_frac=0.1), k=20, qseed=1004),
    # C5: stress, C3 + 16 hubs of 2^21 arcs, 8 high-frequency keywords (>100k nodes each), top-100
    "C5": dict(graph=dict(scale=25, edge_factor=8, seed=5, n_labels=4096, vocab=1 << 22, n_hubs=16,
                          hub_arcs=1 << 21),
               qspec=dict(sizes={8: 10}, band=(100000, 1 << 62), rare=None), k=100),
}


def make_queries(g: Graph, seed: int, *, sizes=None, uniform_q=None, count=0, band=(1, 1 << 62), rare=None,
                 rare_frac=0.0) -> list:
    """Draw queries: each keyword from the frequency ``band`` (|T_i| in [lo, hi]), or with probability
    ``rare_frac`` from the ``rare`` band (Table V's Q11-like rare keyword).  Keywords distinct in a query."""
    rng = np.random.default_rng(seed)
    size = np.diff(g.kw_ptr)
    pool = np.nonzero((size >= band[0]) & (size <= band[1]))[0]
    rpool = np.nonzero((size >= rare[0]) & (size <= rare[1]))[0] if rare else np.zeros(0, np.int64)
    if pool.size == 0:
        raise ValueError(f"no keyword with |T| in {band}")
    qs = []
    plan = []
    if sizes:
        for q, c in sizes.items():
            plan += [q] * c
    else:
        lo, hi = uniform_q
        plan = list(rng.integers(lo, hi + 1, size=count))
    for q in plan:
        chosen = []
        while len(chosen) < q:
            src = rpool if (rpool.size and rng.random() < rare_frac) else pool
            t = int(src[rng.integers(0, src.size)])
            if t not in chosen:
                chosen.append(t)
        qs.append(tuple(chosen))
    return qs


def config_queries(name: str, g: Graph) -> list:
    """The query set of config ``name`` drawn from an already generated graph ``g`` of the same recipe
    (C4 shares the C3 graph: bench.py generates it once)."""
    p = CONFIG_PARAMS[name]
    qs = dict(p["qspec"])
    band = qs.pop("band")
    return make_queries(g, p.get("qseed", 1000 + int(name[1:])), band=band, **qs)


def make_workload(name: str, *, scale_override: int | None = None, n_queries: int | None = None) -> Workload:
    """Build one BASELINE.json config.  ``scale_override`` shrinks the graph for tests (same recipe)."""
    p = CONFIG_PARAMS[name]
    gp = dict(p["graph"])
    if scale_override is not None:
        gp["scale"] = scale_override
    g = rmat_graph(**gp)
    cfg_no = int(name[1:])
    qs = dict(p["qspec"])
    band = qs.pop("band")
    if scale_override is not None and scale_override != p["graph"]["scale"]:
        f = 2.0 ** (scale_override - p["graph"]["scale"])
        band = (max(2, int(band[0] * f)), max(3, int(band[1] * f)))
        if qs.get("rare"):
            qs["rare"] = (max(1, int(qs["rare"][0] * f)), max(2, int(qs["rare"][1] * f)))
    queries = make_queries(g, p.get("qseed", 1000 + cfg_no), band=band, **qs)
    if n_queries is not None:
        queries = queries[:n_queries]
    g.meta["config"] = name
    return Workload(name, g, queries, p["k"])
