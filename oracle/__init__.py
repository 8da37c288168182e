"""CPU oracle for the Central Graph keyword-search hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl reference``
legs may import this module.  The product path (``paper_conf_icde_yangajtw19_b200``) never imports it
and shares no code with it.  The arithmetic lives in ``oracle.c`` (plain single-threaded C following
PAPER.md step by step); this file only marshals arguments through ctypes.

Pins: see DESIGN.md "Oracle pins" and tests/test_oracle_*.py.  Every function is pinned; the score
*direction* (reading R14) is a reading, not a value the paper prints.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

STOP_K, STOP_EXHAUSTED, STOP_MAX_DEPTH, STOP_EMPTY_KEYWORD = 0, 1, 2, 3
EXTRACT_EXACT, EXTRACT_LITERAL = 0, 1
BFS_LITERAL, BFS_LEVEL_RULE = 0, 1


def build_lib(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        # -ffp-contract=off: Eqs. 3-5 are evaluated one rounded operation at a time (reading R4)
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-ffp-contract=off", "-fno-fast-math",
                               "-o", _LIB_PATH, src, "-lm"])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build_lib()
        L = ctypes.CDLL(_LIB_PATH)
        vp, i64, i32, dbl = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_double
        L.oracle_query.restype = vp
        L.oracle_query.argtypes = [i64, vp, vp, vp, i64, vp, vp, dbl, i32, vp, i32, i64, dbl, dbl, i32, i32, i32, i32, i32,
                                   vp, i64, i32]
        L.oracle_activation.argtypes = [i64, vp, dbl, dbl, vp]
        L.oracle_snap_weights.argtypes = [i64, vp, vp]
        for f in ("oracle_a", "oracle_M", "oracle_centrals", "oracle_central_depth", "oracle_central_key"):
            getattr(L, f).restype = vp
            getattr(L, f).argtypes = [vp]
        L.oracle_status.restype = i32
        L.oracle_status.argtypes = [vp]
        L.oracle_n_centrals.restype = i64
        L.oracle_n_centrals.argtypes = [vp]
        L.oracle_count.restype = i64
        L.oracle_count.argtypes = [vp]
        L.oracle_stats.argtypes = [vp, vp]
        L.oracle_answer.argtypes = [vp, i64] + [vp] * 8
        L.oracle_free.argtypes = [vp]
        L.oracle_pair_distances.argtypes = [i64, vp, vp, i64, vp, vp, i32, vp, vp]
        L.oracle_summary_weights.argtypes = [i64, vp, vp, vp, vp]
        _lib = L
    return _lib


def snap_weights(weight: np.ndarray) -> np.ndarray:
    """O0 (reading R15): every weight to the nearest point of the 2^-24 grid, ties up.  ``query`` applies
    it before the activation map and the score."""
    L = _load()
    w = np.ascontiguousarray(weight, np.float32)
    out = np.empty(w.shape[0], np.float32)
    L.oracle_snap_weights(w.shape[0], w.ctypes.data, out.ctypes.data)
    return out


def activation(weight: np.ndarray, A: float, alpha: float) -> np.ndarray:
    """O1: Eqs. 3-5 for every node."""
    L = _load()
    w = np.ascontiguousarray(weight, np.float32)
    out = np.empty(w.shape[0], np.uint8)
    L.oracle_activation(w.shape[0], w.ctypes.data, float(A), float(alpha), out.ctypes.data)
    return out


@dataclass
class Answer:
    central: int
    depth: int
    key: float
    score: float
    nodes: np.ndarray   # int32 ascending
    arcs: np.ndarray    # int32 [n_arcs, 2] (pred, succ) lexicographic


@dataclass
class Result:
    status: int
    a: np.ndarray | None = None
    M: np.ndarray | None = None            # uint8 [n, q], 255 = inf
    centrals: np.ndarray | None = None     # int32 ascending
    central_depth: np.ndarray | None = None
    central_key: np.ndarray | None = None  # float64, per central
    levels: int = 0
    stop_reason: int = 0
    answers: list | None = None


def query(g, kw_ids, k: int, *, alpha: float = 0.1, lam: float = 0.2, max_depth: int = 254,
          block_central: int = 1, extract_mode: int = EXTRACT_EXACT, bfs_form: int = BFS_LITERAL,
          level_cover: int = 1, eval_ids=None, containment: int = 0) -> Result:
    """One query through the oracle.  ``g`` is a synth.Graph-like object (row_ptr, col_idx, weight,
    kw_ptr, kw_nodes, A, symmetric).  ``eval_ids`` (test sampling at sizes where scoring every central
    node is out of reach): only these central nodes are extracted and scored (the others' keys are NaN)
    and the answers rank them alone.  ``level_cover``: 0 off, 1 the "contribute" reading (R13, default), 2
    the "contains" reading (R13b, NEXT-3).  ``containment`` = 1: drop every Central Graph that strictly
    contains another one's node set (R16, NEXT-3)."""
    L = _load()
    kw = np.ascontiguousarray(np.asarray(kw_ids, dtype=np.int32))
    q = int(kw.shape[0])
    rp = np.ascontiguousarray(g.row_ptr, np.int64)
    ci = np.ascontiguousarray(g.col_idx, np.int32)
    w = np.ascontiguousarray(g.weight, np.float32)
    kp = np.ascontiguousarray(g.kw_ptr, np.int64)
    kn = np.ascontiguousarray(g.kw_nodes, np.int32)
    n = rp.shape[0] - 1
    ev = None if eval_ids is None else np.ascontiguousarray(np.asarray(eval_ids, dtype=np.int32))
    h = L.oracle_query(n, rp.ctypes.data, ci.ctypes.data, w.ctypes.data, kp.shape[0] - 1, kp.ctypes.data,
                       kn.ctypes.data, float(g.A), 1 if g.symmetric else 0, kw.ctypes.data, q, int(k),
                       float(alpha), float(lam), int(max_depth), int(block_central), int(extract_mode),
                       int(bfs_form), int(level_cover), None if ev is None else ev.ctypes.data,
                       0 if ev is None else int(ev.shape[0]), int(containment))
    try:
        st = L.oracle_status(h)
        if st != 0:
            return Result(status=st)

        def arr(ptr, count, dt):
            if count == 0:
                return np.zeros(0, dt)
            return np.ctypeslib.as_array(ctypes.cast(ptr, ctypes.POINTER(np.ctypeslib.as_ctypes_type(dt))),
                                         shape=(count,)).copy()
        nc = int(L.oracle_n_centrals(h))
        stats = np.zeros(4, np.int64)
        L.oracle_stats(h, stats.ctypes.data)
        res = Result(status=0,
                     a=arr(L.oracle_a(h), n, np.uint8),
                     M=arr(L.oracle_M(h), n * q, np.uint8).reshape(n, q),
                     centrals=arr(L.oracle_centrals(h), nc, np.int32),
                     central_depth=arr(L.oracle_central_depth(h), nc, np.uint8),
                     central_key=arr(L.oracle_central_key(h), nc, np.float64),
                     levels=int(stats[0]), stop_reason=int(stats[1]), answers=[])
        cnt = int(L.oracle_count(h))
        c32, d32 = ctypes.c_int32(), ctypes.c_int32()
        key, sc = ctypes.c_double(), ctypes.c_float()
        nn, na = ctypes.c_int64(), ctypes.c_int64()
        pn, pa = ctypes.c_void_p(), ctypes.c_void_p()
        for i in range(cnt):
            L.oracle_answer(h, i, ctypes.byref(c32), ctypes.byref(d32), ctypes.byref(key), ctypes.byref(sc),
                            ctypes.byref(nn), ctypes.byref(pn), ctypes.byref(na), ctypes.byref(pa))
            res.answers.append(Answer(int(c32.value), int(d32.value), float(key.value), float(sc.value),
                                      arr(pn.value, nn.value, np.int32),
                                      arr(pa.value, 2 * na.value, np.int32).reshape(-1, 2)))
        return res
    finally:
        L.oracle_free(h)


def pair_distances(row_ptr, col_idx, src, dst, max_hops: int = 254):
    """P1: hop distance of each sampled pair by a plain BFS; (dist, mean)."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(col_idx, dtype=np.int32)
    s = np.ascontiguousarray(src, dtype=np.int32)
    d = np.ascontiguousarray(dst, dtype=np.int32)
    out = np.empty(s.shape[0], np.int32)
    mean = ctypes.c_double(0.0)
    _load().oracle_pair_distances(int(rp.shape[0] - 1), rp.ctypes.data, ci.ctypes.data, int(s.shape[0]),
                                  s.ctypes.data, d.ctypes.data, int(max_hops), out.ctypes.data, ctypes.byref(mean))
    return out, float(mean.value)


def summary_weights(in_row_ptr, in_label):
    """P2, Eq. 2 + min-max normalisation; (w_norm float32, w_raw float64)."""
    rp = np.ascontiguousarray(in_row_ptr, dtype=np.int64)
    lab = np.ascontiguousarray(in_label, dtype=np.int32)
    n = int(rp.shape[0] - 1)
    wn = np.empty(n, np.float32)
    wr = np.empty(n, np.float64)
    _load().oracle_summary_weights(n, rp.ctypes.data, lab.ctypes.data, wn.ctypes.data, wr.ctypes.data)
    return wn, wr
