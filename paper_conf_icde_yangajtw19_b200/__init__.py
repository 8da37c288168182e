"""B200-native Central Graph keyword search (Yang et al., ICDE 2019) — Python binding of libkgs.so.

Argument marshalling only: every step of the query path runs in the CUDA kernels behind the C-ABI
declared in ``include/kgs.h``.  There is no CPU fallback: if ``libkgs.so`` is missing or no CUDA
device is present, the calls raise.

The names mirror the C-ABI (``kgs_load_graph``, ``kgs_query``, ``kgs_query_device``, ...); the
``Graph`` / ``Result`` classes are thin owners of the opaque handles.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("KGS_LIB", os.path.join(_HERE, "libkgs.so"))   # KGS_LIB: ablation builds

KGS_OK, KGS_EINVAL, KGS_ENOMEM, KGS_ECUDA, KGS_ENCCL, KGS_EINTERNAL = 0, -1, -2, -3, -4, -5
KGS_MAX_Q, KGS_MAX_K = 8, 4096
KGS_INPUT_DEVICE_PTRS = 1
KGS_NO_RELABEL = 2
KGS_EXTRACT_EXACT, KGS_EXTRACT_LITERAL = 0, 1
KGS_DIR_AUTO, KGS_DIR_PUSH, KGS_DIR_PULL = 0, 1, 2
KGS_STOP_K, KGS_STOP_EXHAUSTED, KGS_STOP_MAX_DEPTH, KGS_STOP_EMPTY_KEYWORD = 0, 1, 2, 3


class KgsError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"kgs status {status}: {msg}")
        self.status = status


class kgs_graph_desc(ctypes.Structure):
    _fields_ = [("n_nodes", ctypes.c_int64), ("n_arcs", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p), ("weight", ctypes.c_void_p),
                ("n_keywords", ctypes.c_int64), ("kw_ptr", ctypes.c_void_p), ("kw_nodes", ctypes.c_void_p),
                ("avg_dist_A", ctypes.c_double), ("symmetric", ctypes.c_int32), ("device", ctypes.c_int32),
                ("flags", ctypes.c_int32), ("pred_arc_cap", ctypes.c_int64)]


class kgs_params(ctypes.Structure):
    _fields_ = [("alpha", ctypes.c_double), ("lambda_", ctypes.c_double), ("max_depth", ctypes.c_int32),
                ("block_central", ctypes.c_int32), ("extract_mode", ctypes.c_int32),
                ("level_cover", ctypes.c_int32), ("want_levels", ctypes.c_int32), ("prune", ctypes.c_int32),
                ("direction", ctypes.c_int32), ("pull_ratio", ctypes.c_int32), ("pull_min", ctypes.c_int64),
                ("prune_min", ctypes.c_int32), ("tile_light", ctypes.c_int32), ("dag_record", ctypes.c_int32),
                ("search_only", ctypes.c_int32), ("containment", ctypes.c_int32), ("mk_min", ctypes.c_int32),
                ("defer_min", ctypes.c_int32), ("lazy_dag", ctypes.c_int32),
                ("rec_max", ctypes.c_int32)]


class kgs_answer(ctypes.Structure):
    _fields_ = [("central", ctypes.c_int32), ("depth", ctypes.c_int32), ("score", ctypes.c_float),
                ("score_key", ctypes.c_double), ("n_nodes", ctypes.c_int64),
                ("nodes", ctypes.POINTER(ctypes.c_int32)), ("n_arcs", ctypes.c_int64),
                ("arcs", ctypes.POINTER(ctypes.c_int32))]


class kgs_stats(ctypes.Structure):
    _fields_ = [("levels", ctypes.c_int32), ("stop_reason", ctypes.c_int32), ("n_centrals", ctypes.c_int64),
                ("count", ctypes.c_int64), ("frontier_total", ctypes.c_int64), ("arcs_scanned", ctypes.c_int64),
                ("overflow", ctypes.c_int64), ("hits", ctypes.c_int64), ("td_arcs", ctypes.c_int64),
                ("td_pred_arcs", ctypes.c_int64), ("ms_search", ctypes.c_float), ("ms_topdown", ctypes.c_float),
                ("ms_total", ctypes.c_float), ("ms_launch", ctypes.c_float), ("group", ctypes.c_int32),
                ("n_evaluated", ctypes.c_int32), ("dag_arcs", ctypes.c_int64), ("pull_level", ctypes.c_int32),
                ("n_cut", ctypes.c_int32), ("n_tier4", ctypes.c_int32), ("td_arcs_big", ctypes.c_int64)]


class kgs_vp_buffers(ctypes.Structure):
    _fields_ = [("hm", ctypes.c_void_p), ("hm_slice", ctypes.c_void_p), ("M", ctypes.c_void_p),
                ("counts", ctypes.c_void_p), ("cent", ctypes.c_void_p), ("cdep", ctypes.c_void_p),
                ("cent_n", ctypes.c_void_p), ("chg", ctypes.c_void_p)]


# collectives of the vertex partition's transport (kgs_vp_transport): all_gather(ctx, send, recv, bytes,
# stream) and all_reduce_sum_i64(ctx, buf, count, stream), 0 = success
VP_ALL_GATHER = ctypes.CFUNCTYPE(ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64,
                                 ctypes.c_void_p)
VP_ALL_REDUCE = ctypes.CFUNCTYPE(ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p)


class kgs_vp_transport(ctypes.Structure):
    _fields_ = [("ctx", ctypes.c_void_p), ("all_gather", VP_ALL_GATHER), ("all_reduce_sum_i64", VP_ALL_REDUCE),
                ("owned", ctypes.c_int32), ("host_staged", ctypes.c_int32)]


EXPORTED = ["kgs_load_graph", "kgs_free_graph", "kgs_params_default", "kgs_query", "kgs_query_device",
            "kgs_query_fetch", "kgs_result_count", "kgs_result_answer", "kgs_result_levels",
            "kgs_result_centrals", "kgs_result_activation", "kgs_result_stats", "kgs_result_phases",
            "kgs_result_free", "kgs_last_error", "kgs_version", "kgs_query_batch", "kgs_query_batch_device",
            "kgs_query_batch_fetch", "kgs_vp_slice", "kgs_vp_begin", "kgs_vp_level", "kgs_vp_waiting",
            "kgs_vp_topdown", "kgs_prep_pair_distances", "kgs_prep_summary_weights", "kgs_vp_nccl_unique_id",
            "kgs_vp_nccl_transport", "kgs_vp_transport_free", "kgs_vp_query", "kgs_result_sizes",
            "kgs_result_export"]

PHASE_NAMES = ["start", "reset", "sources", "merge", "expand", "pd_seed", "pd_merge", "pd_expand", "pd_csr",
               "search_end", "extract", "extract_big", "select", "emit", "pd_merge2", "pd_expand2", "extract2",
               "mk_reach"]
KGS_STOP_INVALID_QUERY = -1
KGS_STOP_CAPACITY = -2

_lib = None


def lib():
    """Load libkgs.so (raises if it was not built: the product has no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built; run `make` (or __graft_entry__.build())")
        L = ctypes.CDLL(LIB_PATH)
        vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        L.kgs_load_graph.argtypes = [ctypes.POINTER(kgs_graph_desc), ctypes.POINTER(vp)]
        L.kgs_load_graph.restype = i32
        L.kgs_free_graph.argtypes = [vp]
        L.kgs_free_graph.restype = None
        L.kgs_params_default.argtypes = [ctypes.POINTER(kgs_params)]
        L.kgs_params_default.restype = None
        L.kgs_query.argtypes = [vp, vp, i32, i32, ctypes.POINTER(kgs_params), vp, ctypes.POINTER(vp)]
        L.kgs_query.restype = i32
        L.kgs_query_device.argtypes = [vp, vp, i32, i32, ctypes.POINTER(kgs_params), vp]
        L.kgs_query_device.restype = i32
        L.kgs_query_fetch.argtypes = [vp, vp, ctypes.POINTER(vp)]
        L.kgs_query_fetch.restype = i32
        L.kgs_result_count.argtypes = [vp]
        L.kgs_result_count.restype = i32
        L.kgs_result_answer.argtypes = [vp, i32, ctypes.POINTER(kgs_answer)]
        L.kgs_result_answer.restype = i32
        L.kgs_result_levels.argtypes = [vp, vp, i64]
        L.kgs_result_levels.restype = i32
        L.kgs_result_activation.argtypes = [vp, vp, i64]
        L.kgs_result_activation.restype = i32
        L.kgs_result_centrals.argtypes = [vp, vp, vp, vp, i64, ctypes.POINTER(i64)]
        L.kgs_result_centrals.restype = i32
        L.kgs_result_stats.argtypes = [vp, ctypes.POINTER(kgs_stats)]
        L.kgs_result_stats.restype = i32
        L.kgs_result_sizes.argtypes = [vp, vp, vp, vp]
        L.kgs_result_sizes.restype = i32
        L.kgs_result_export.argtypes = [vp] * 8
        L.kgs_result_export.restype = i32
        L.kgs_query_batch.argtypes = [vp, i32, vp, vp, i32, ctypes.POINTER(kgs_params), i32, vp, vp]
        L.kgs_query_batch.restype = i32
        L.kgs_query_batch_device.argtypes = [vp, i32, vp, vp, i32, ctypes.POINTER(kgs_params), i32, vp]
        L.kgs_query_batch_device.restype = i32
        L.kgs_query_batch_fetch.argtypes = [vp, vp, vp]
        L.kgs_query_batch_fetch.restype = i32
        L.kgs_result_phases.argtypes = [vp, vp, vp, i32, ctypes.POINTER(i32)]
        L.kgs_result_phases.restype = i32
        L.kgs_result_free.argtypes = [vp]
        L.kgs_result_free.restype = None
        L.kgs_last_error.argtypes = []
        L.kgs_last_error.restype = ctypes.c_char_p
        L.kgs_vp_slice.argtypes = [i64, i32]
        L.kgs_vp_slice.restype = i64
        L.kgs_vp_begin.argtypes = [vp, vp, i32, i32, ctypes.POINTER(kgs_params), i32, i32,
                                   ctypes.POINTER(kgs_vp_buffers), vp, vp]
        L.kgs_vp_begin.restype = i32
        L.kgs_vp_level.argtypes = [vp, i32, vp]
        L.kgs_vp_level.restype = i32
        L.kgs_vp_waiting.argtypes = [vp, i32, vp]
        L.kgs_vp_waiting.restype = i32
        L.kgs_vp_topdown.argtypes = [vp, i64, vp, vp, i32, i32, vp, ctypes.POINTER(vp)]
        L.kgs_vp_topdown.restype = i32
        L.kgs_vp_nccl_unique_id.argtypes = [vp]
        L.kgs_vp_nccl_unique_id.restype = i32
        L.kgs_vp_nccl_transport.argtypes = [vp, i32, i32, i32, ctypes.POINTER(kgs_vp_transport)]
        L.kgs_vp_nccl_transport.restype = i32
        L.kgs_vp_transport_free.argtypes = [ctypes.POINTER(kgs_vp_transport)]
        L.kgs_vp_transport_free.restype = None
        L.kgs_vp_query.argtypes = [vp, vp, i32, i32, ctypes.POINTER(kgs_params), i32, i32,
                                   ctypes.POINTER(kgs_vp_transport), vp, ctypes.POINTER(vp)]
        L.kgs_vp_query.restype = i32
        L.kgs_prep_pair_distances.argtypes = [i64, i64, vp, vp, i32, vp, vp, i32, i32, i32, vp, vp, vp]
        L.kgs_prep_pair_distances.restype = i32
        L.kgs_prep_summary_weights.argtypes = [i64, i64, vp, vp, i32, i32, vp, vp, vp]
        L.kgs_prep_summary_weights.restype = i32
        L.kgs_version.argtypes = []
        L.kgs_version.restype = ctypes.c_char_p
        _lib = L
    return _lib


def _check(st: int):
    if st != KGS_OK:
        raise KgsError(st, lib().kgs_last_error().decode())


def kgs_params_default() -> kgs_params:
    p = kgs_params()
    lib().kgs_params_default(ctypes.byref(p))
    return p


def make_params(alpha=0.1, lam=0.2, max_depth=254, block_central=1, extract_mode=KGS_EXTRACT_EXACT,
                level_cover=1, want_levels=0, prune=1, direction=0, **tuning) -> kgs_params:
    """kgs_params from the defaults; ``tuning`` sets other fields by name (containment, pull_ratio,
    pull_min, prune_min, tile_light, dag_record, search_only, mk_min, defer_min, lazy_dag, rec_max)."""
    p = kgs_params_default()
    p.alpha, p.lambda_, p.max_depth = float(alpha), float(lam), int(max_depth)
    p.block_central, p.extract_mode = int(block_central), int(extract_mode)
    p.level_cover, p.want_levels, p.prune = int(level_cover), int(want_levels), int(prune)
    p.direction = int(direction)
    names = {f for f, _ in kgs_params._fields_}
    for k, v in tuning.items():
        if k not in names:
            raise TypeError(f"unknown kgs_params field {k}")
        setattr(p, k, int(v))
    return p


class Graph:
    """Owner of a kgs_graph handle (device CSR, weights, keyword index, query workspace)."""

    def __init__(self, handle, n, n_keywords):
        self.handle = handle
        self.n = n
        self.n_keywords = n_keywords

    def close(self):
        if self.handle:
            lib().kgs_free_graph(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def kgs_load_graph(g, device: int = 0, relabel: bool = True, pred_arc_cap: int = 0) -> Graph:
    """Load a graph given as host numpy arrays (attributes row_ptr, col_idx, weight, kw_ptr, kw_nodes,
    A, symmetric — e.g. a synth.Graph).  relabel=False sets KGS_NO_RELABEL (keep the input node order
    internally; results are identical either way)."""
    rp = np.ascontiguousarray(g.row_ptr, np.int64)
    ci = np.ascontiguousarray(g.col_idx, np.int32)
    w = np.ascontiguousarray(g.weight, np.float32)
    kp = np.ascontiguousarray(g.kw_ptr, np.int64)
    kn = np.ascontiguousarray(g.kw_nodes, np.int32)
    d = kgs_graph_desc(rp.shape[0] - 1, ci.shape[0], rp.ctypes.data, ci.ctypes.data, w.ctypes.data,
                       kp.shape[0] - 1, kp.ctypes.data, kn.ctypes.data if kn.size else None, float(g.A),
                       1 if getattr(g, "symmetric", True) else 0, int(device), 0 if relabel else KGS_NO_RELABEL,
                       int(pred_arc_cap))
    h = ctypes.c_void_p()
    _check(lib().kgs_load_graph(ctypes.byref(d), ctypes.byref(h)))
    return Graph(h, rp.shape[0] - 1, kp.shape[0] - 1)


def kgs_load_graph_device(n, n_arcs, row_ptr_ptr, col_idx_ptr, weight_ptr, n_keywords, kw_ptr_ptr, kw_nodes_ptr,
                          A: float, symmetric: bool = True, device: int = 0, relabel: bool = True,
                          pred_arc_cap: int = 0) -> Graph:
    """Load a graph whose arrays already live in device memory (KGS_INPUT_DEVICE_PTRS): raw device
    pointers (e.g. torch CUDA tensors' data_ptr()), int64 row_ptr / kw_ptr, int32 col_idx / kw_nodes,
    float32 weight.  The library copies them; the caller keeps ownership."""
    d = kgs_graph_desc(int(n), int(n_arcs), row_ptr_ptr, col_idx_ptr, weight_ptr, int(n_keywords), kw_ptr_ptr,
                       kw_nodes_ptr, float(A), 1 if symmetric else 0, int(device),
                       KGS_INPUT_DEVICE_PTRS | (0 if relabel else KGS_NO_RELABEL), int(pred_arc_cap))
    h = ctypes.c_void_p()
    _check(lib().kgs_load_graph(ctypes.byref(d), ctypes.byref(h)))
    return Graph(h, int(n), int(n_keywords))


@dataclass
class Answer:
    central: int
    depth: int
    score: float
    score_key: float
    nodes: np.ndarray
    arcs: np.ndarray   # [n_arcs, 2]


class Result:
    """One query's answers (kgs_result_*), plus its statistics.  The statistics dict (with the per-phase
    times) is built on first access from the raw copies taken before the handle was freed: a batch of
    thousands of results does not pay for it unless it is read."""

    def __init__(self, answers, raw_stats, tags, tns, nph):
        self.answers = answers
        self._raw = (raw_stats, tags, tns, nph)
        self._stats = None
        self.M = self.a = self.centrals = self.central_depth = self.central_key = None

    @property
    def stats(self) -> dict:
        if self._stats is None:
            st, tags, tns, m = self._raw
            stats = {f: getattr(st, f) for f, _ in kgs_stats._fields_}
            # per-phase durations (us): time from the previous stamp to this one, summed by phase name
            ph = {}
            if m > 1:
                dur = np.diff(tns[:m].astype(np.int64)) / 1e3
                sums = np.bincount(tags[1:m], weights=dur)
                for t in np.flatnonzero(np.bincount(tags[1:m])):
                    ph[PHASE_NAMES[t] if t < len(PHASE_NAMES) else str(t)] = float(sums[t])
            stats["phases_us"] = ph
            self._stats = stats
        return self._stats


def _read_result(h, n, q, want_levels) -> Result:
    L = lib()
    try:
        # every answer in flat arrays with one call (kgs_result_export); answers hold views into them
        cnt, tn, ta = ctypes.c_int32(), ctypes.c_int64(), ctypes.c_int64()
        _check(L.kgs_result_sizes(h, ctypes.byref(cnt), ctypes.byref(tn), ctypes.byref(ta)))
        cnt = cnt.value
        cen = np.empty(cnt, np.int32)
        dep = np.empty(cnt, np.int32)
        key = np.empty(cnt, np.float64)
        noff = np.empty(cnt + 1, np.int64)
        aoff = np.empty(cnt + 1, np.int64)
        nodes = np.empty(max(tn.value, 1), np.int32)
        arcs = np.empty(max(2 * ta.value, 2), np.int32)
        _check(L.kgs_result_export(h, cen.ctypes.data, dep.ctypes.data, key.ctypes.data, noff.ctypes.data,
                                   nodes.ctypes.data, aoff.ctypes.data, arcs.ctypes.data))
        arcs2 = arcs.reshape(-1, 2)
        # Python scalars in one conversion per array (indexing numpy element by element is the slow part)
        cl, dl, kl = cen.tolist(), dep.tolist(), key.tolist()
        sl = key.astype(np.float32).tolist()
        nl, al = noff.tolist(), aoff.tolist()
        answers = [Answer(cl[i], dl[i], sl[i], kl[i], nodes[nl[i]:nl[i + 1]], arcs2[al[i]:al[i + 1]])
                   for i in range(cnt)]
        st = kgs_stats()
        _check(L.kgs_result_stats(h, ctypes.byref(st)))
        tags = np.zeros(64, np.int32)
        tns = np.zeros(64, np.uint64)
        nph = ctypes.c_int32()
        _check(L.kgs_result_phases(h, tags.ctypes.data, tns.ctypes.data, 64, ctypes.byref(nph)))
        res = Result(answers, st, tags, tns, min(nph.value, 64))
        if want_levels:
            M = np.empty(n * q, np.uint8)
            _check(L.kgs_result_levels(h, M.ctypes.data, M.size))
            act = np.empty(n, np.uint8)
            _check(L.kgs_result_activation(h, act.ctypes.data, act.size))
            nc = ctypes.c_int64()
            cap = n
            ids = np.empty(cap, np.int32)
            dep = np.empty(cap, np.uint8)
            key = np.empty(cap, np.float64)
            _check(L.kgs_result_centrals(h, ids.ctypes.data, dep.ctypes.data, key.ctypes.data, cap, ctypes.byref(nc)))
            k = nc.value
            res.M, res.a = M.reshape(n, q), act
            res.centrals, res.central_depth, res.central_key = ids[:k].copy(), dep[:k].copy(), key[:k].copy()
        return res
    finally:
        L.kgs_result_free(h)


def kgs_query(graph: Graph, kw_ids, k: int, params: kgs_params | None = None, stream: int = 0) -> Result:
    """One query with host keyword ids; answers copied back to the host (kgs_query)."""
    kw = np.ascontiguousarray(np.asarray(kw_ids, dtype=np.int32))
    p = params if params is not None else kgs_params_default()
    h = ctypes.c_void_p()
    _check(lib().kgs_query(graph.handle, kw.ctypes.data, int(kw.shape[0]), int(k), ctypes.byref(p),
                           ctypes.c_void_p(stream), ctypes.byref(h)))
    return _read_result(h, graph.n, int(kw.shape[0]), p.want_levels)


def kgs_query_device(graph: Graph, kw_ids_dev_ptr: int, q: int, k: int, params: kgs_params | None = None,
                     stream: int = 0) -> None:
    """Enqueue a query whose keyword ids are already in device memory; no synchronisation."""
    p = params if params is not None else kgs_params_default()
    _check(lib().kgs_query_device(graph.handle, ctypes.c_void_p(kw_ids_dev_ptr), int(q), int(k), ctypes.byref(p),
                                  ctypes.c_void_p(stream)))


def kgs_query_fetch(graph: Graph, q: int, want_levels: int = 0, stream: int = 0) -> Result:
    h = ctypes.c_void_p()
    _check(lib().kgs_query_fetch(graph.handle, ctypes.c_void_p(stream), ctypes.byref(h)))
    return _read_result(h, graph.n, q, want_levels)


def kgs_query_batch(graph: Graph, queries, k: int, params: kgs_params | None = None, n_groups: int = 0,
                    stream: int = 0) -> list:
    """A batch of queries in one engine launch (host keyword ids in, host results out)."""
    p = params if params is not None else kgs_params_default()
    qp = np.zeros(len(queries) + 1, np.int32)
    for j, kw in enumerate(queries):
        qp[j + 1] = qp[j] + len(kw)
    kw = np.ascontiguousarray(np.concatenate([np.asarray(q, np.int32) for q in queries]), np.int32)
    hs = (ctypes.c_void_p * len(queries))()
    _check(lib().kgs_query_batch(graph.handle, len(queries), qp.ctypes.data, kw.ctypes.data, int(k), ctypes.byref(p),
                                 int(n_groups), ctypes.c_void_p(stream), hs))
    return [_read_result(ctypes.c_void_p(hs[j]), graph.n, len(queries[j]), 0) for j in range(len(queries))]


def kgs_query_batch_device(graph: Graph, n_queries: int, kw_dev_ptr: int, qlen_dev_ptr: int, k: int,
                           params: kgs_params | None = None, n_groups: int = 0, stream: int = 0) -> None:
    """Enqueue a batch whose padded keyword rows [n][8] and lengths [n] are in device memory."""
    p = params if params is not None else kgs_params_default()
    _check(lib().kgs_query_batch_device(graph.handle, int(n_queries), ctypes.c_void_p(kw_dev_ptr),
                                        ctypes.c_void_p(qlen_dev_ptr), int(k), ctypes.byref(p), int(n_groups),
                                        ctypes.c_void_p(stream)))


def kgs_query_batch_fetch(graph: Graph, qlens, stream: int = 0) -> list:
    hs = (ctypes.c_void_p * len(qlens))()
    _check(lib().kgs_query_batch_fetch(graph.handle, ctypes.c_void_p(stream), hs))
    return [_read_result(ctypes.c_void_p(hs[j]), graph.n, int(qlens[j]), 0) for j in range(len(qlens))]


def kgs_version() -> str:
    return lib().kgs_version().decode()


# ---- vertex-partitioned search of one query (driver: dist.vp_query) ----
def kgs_vp_slice(n_nodes: int, world: int) -> int:
    return int(lib().kgs_vp_slice(int(n_nodes), int(world)))


def kgs_vp_begin(graph: Graph, kw_ids, k: int, params: kgs_params | None, rank: int, world: int,
                 bufs: kgs_vp_buffers, stream: int = 0) -> tuple:
    """Returns (amax, empty)."""
    kw = np.ascontiguousarray(np.asarray(kw_ids, dtype=np.int32))
    p = params if params is not None else kgs_params_default()
    info = np.zeros(2, np.int32)
    _check(lib().kgs_vp_begin(graph.handle, kw.ctypes.data, int(kw.shape[0]), int(k), ctypes.byref(p), int(rank),
                              int(world), ctypes.byref(bufs), ctypes.c_void_p(stream), info.ctypes.data))
    return int(info[0]), bool(info[1])


def kgs_vp_level(graph: Graph, level: int, stream: int = 0) -> None:
    _check(lib().kgs_vp_level(graph.handle, int(level), ctypes.c_void_p(stream)))


def kgs_vp_waiting(graph: Graph, level: int, stream: int = 0) -> None:
    _check(lib().kgs_vp_waiting(graph.handle, int(level), ctypes.c_void_p(stream)))


def kgs_vp_topdown(graph: Graph, n_central: int, cent_ptr: int, dep_ptr: int, levels: int, stop_reason: int, q: int,
                   want_levels: int = 0, stream: int = 0) -> Result:
    h = ctypes.c_void_p()
    _check(lib().kgs_vp_topdown(graph.handle, int(n_central), ctypes.c_void_p(cent_ptr), ctypes.c_void_p(dep_ptr),
                                int(levels), int(stop_reason), ctypes.c_void_p(stream), ctypes.byref(h)))
    return _read_result(h, graph.n, int(q), want_levels)


def kgs_vp_nccl_unique_id() -> bytes:
    """128-byte NCCL unique id (rank 0; broadcast it to the other ranks)."""
    buf = (ctypes.c_uint8 * 128)()
    _check(lib().kgs_vp_nccl_unique_id(buf))
    return bytes(buf)


def kgs_vp_nccl_transport(uid: bytes, rank: int, world: int, device: int) -> kgs_vp_transport:
    """The library's own NCCL communicator for kgs_vp_query (free with kgs_vp_transport_free)."""
    t = kgs_vp_transport()
    buf = (ctypes.c_uint8 * 128).from_buffer_copy(uid)
    _check(lib().kgs_vp_nccl_transport(buf, int(rank), int(world), int(device), ctypes.byref(t)))
    return t


def kgs_vp_transport_free(t: kgs_vp_transport) -> None:
    lib().kgs_vp_transport_free(ctypes.byref(t))


def kgs_vp_query(graph: Graph, kw_ids, k: int, params: kgs_params | None, rank: int, world: int,
                 transport: kgs_vp_transport, stream: int = 0) -> Result:
    """The whole vertex-partitioned query in the library (level loop, exchanges, stop rules, top-down)."""
    kw = np.ascontiguousarray(np.asarray(kw_ids, dtype=np.int32))
    p = params if params is not None else kgs_params_default()
    h = ctypes.c_void_p()
    _check(lib().kgs_vp_query(graph.handle, kw.ctypes.data, int(kw.shape[0]), int(k), ctypes.byref(p), int(rank),
                              int(world), ctypes.byref(transport), ctypes.c_void_p(stream), ctypes.byref(h)))
    return _read_result(h, graph.n, int(kw.shape[0]), p.want_levels)


# ---- load-time preprocessing: the inputs kgs_load_graph takes ----
def kgs_prep_pair_distances(row_ptr, col_idx, src, dst, max_hops: int = 254, device: int = 0,
                            stream: int = 0) -> tuple:
    """Hop distances of sampled (src, dst) pairs along out-arcs, and their mean over the reachable
    pairs: A of P:L184 / P:L524.  Returns (dist int32 [n_pairs], -1 = unreachable; mean)."""
    rp = np.ascontiguousarray(np.asarray(row_ptr, dtype=np.int64))
    ci = np.ascontiguousarray(np.asarray(col_idx, dtype=np.int32))
    s = np.ascontiguousarray(np.asarray(src, dtype=np.int32))
    d = np.ascontiguousarray(np.asarray(dst, dtype=np.int32))
    if s.shape != d.shape:
        raise ValueError("src and dst differ in length")
    out = np.empty(s.shape[0], np.int32)
    mean = ctypes.c_double(0.0)
    _check(lib().kgs_prep_pair_distances(int(rp.shape[0] - 1), int(ci.shape[0]), rp.ctypes.data, ci.ctypes.data,
                                         int(s.shape[0]), s.ctypes.data, d.ctypes.data, int(max_hops), int(device),
                                         0, ctypes.c_void_p(stream), out.ctypes.data, ctypes.byref(mean)))
    return out, float(mean.value)


def kgs_prep_summary_weights(in_row_ptr, in_label, device: int = 0, stream: int = 0) -> tuple:
    """Eq. 2 degree of summary from the in-arc labels, min-max normalised.
    Returns (w_norm float32 [n], w_raw float64 [n])."""
    rp = np.ascontiguousarray(np.asarray(in_row_ptr, dtype=np.int64))
    lab = np.ascontiguousarray(np.asarray(in_label, dtype=np.int32))
    n = int(rp.shape[0] - 1)
    wn = np.empty(n, np.float32)
    wr = np.empty(n, np.float64)
    _check(lib().kgs_prep_summary_weights(n, int(lab.shape[0]), rp.ctypes.data, lab.ctypes.data, int(device), 0,
                                          ctypes.c_void_p(stream), wn.ctypes.data, wr.ctypes.data))
    return wn, wr


def kgs_prep_pair_distances_device(n_nodes: int, n_arcs: int, row_ptr_ptr: int, col_idx_ptr: int, n_pairs: int,
                                   src_ptr: int, dst_ptr: int, max_hops: int = 254, device: int = 0,
                                   stream: int = 0) -> tuple:
    """kgs_prep_pair_distances with borrowed device inputs (KGS_INPUT_DEVICE_PTRS)."""
    out = np.empty(int(n_pairs), np.int32)
    mean = ctypes.c_double(0.0)
    _check(lib().kgs_prep_pair_distances(int(n_nodes), int(n_arcs), ctypes.c_void_p(row_ptr_ptr),
                                         ctypes.c_void_p(col_idx_ptr), int(n_pairs), ctypes.c_void_p(src_ptr),
                                         ctypes.c_void_p(dst_ptr), int(max_hops), int(device), KGS_INPUT_DEVICE_PTRS,
                                         ctypes.c_void_p(stream), out.ctypes.data, ctypes.byref(mean)))
    return out, float(mean.value)


def kgs_prep_summary_weights_device(n_nodes: int, n_in_arcs: int, in_row_ptr_ptr: int, in_label_ptr: int,
                                    device: int = 0, stream: int = 0) -> tuple:
    """kgs_prep_summary_weights with borrowed device inputs (KGS_INPUT_DEVICE_PTRS)."""
    wn = np.empty(int(n_nodes), np.float32)
    wr = np.empty(int(n_nodes), np.float64)
    _check(lib().kgs_prep_summary_weights(int(n_nodes), int(n_in_arcs), ctypes.c_void_p(in_row_ptr_ptr),
                                          ctypes.c_void_p(in_label_ptr), int(device), KGS_INPUT_DEVICE_PTRS,
                                          ctypes.c_void_p(stream), wn.ctypes.data, wr.ctypes.data))
    return wn, wr
