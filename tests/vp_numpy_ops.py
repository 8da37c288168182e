"""Test-only model of the vertex-partitioned query (libkgs kgs_vp_query, csrc/vpquery.cu) for CPU runs with
gloo: numpy stand-ins of the level kernels (kgs_vp_begin / kgs_vp_level / kgs_vp_waiting) and the same host
protocol in Python (vp_search: the exchanges — dense, or sparse change lists when fewer than n/16 nodes
changed — and the stop rules), checked against the oracle.  The product runs the protocol in C++
(tests/test_gpu_vp.py checks that one on the GPU).  Same contract as the kernels: this rank writes only its
rows [lo, hi) of M / hm_slice / the central list.  Level rule of Alg. 2
in pull form: x gets keyword i at level l iff m_xi = inf, (x in K or a_x <= l + 1) and some in-neighbour
u with a_u <= l, m_ui <= l, and (u not central or blocking off)."""
import numpy as np
import torch
import torch.distributed as dist

import oracle

STOP_K, STOP_EXHAUSTED, STOP_MAX_DEPTH, STOP_EMPTY_KEYWORD = 0, 1, 2, 3


def vp_alloc(n, slice_, world):
    n_pad = slice_ * world
    return dict(hm=torch.zeros(n_pad, dtype=torch.uint8), hm_slice=torch.zeros(slice_, dtype=torch.uint8),
                M=torch.full((n_pad * 8,), 255, dtype=torch.uint8), counts=torch.zeros(4, dtype=torch.int64),
                cent=torch.zeros(max(slice_, 1), dtype=torch.int32), cdep=torch.zeros(max(slice_, 1), dtype=torch.uint8),
                cent_n=torch.zeros(1, dtype=torch.int32), chg=[])


def _all_gather(t):
    parts = [torch.empty_like(t) for _ in range(dist.get_world_size())]
    dist.all_gather(parts, t)
    return torch.cat(parts)


def vp_search(ops, kw, k, max_depth, rank, world):
    """kgs_vp_query's host protocol (vpquery.cu) over gloo: level, all_reduce(counts), dense or sparse
    exchange, stop rules; then the all_gathers of M and of the central lists."""
    b = ops.bufs
    slice_ = b["hm_slice"].shape[0]
    n = ops.n
    amax, empty = ops.begin(kw, k, rank, world)
    if empty:
        return dict(levels=0, stop=STOP_EMPTY_KEYWORD, n_central=0, cent=b["cent"][:0], cdep=b["cdep"][:0], sparse=0)
    dist.all_reduce(b["counts"])
    n_central = int(b["counts"][1])
    level, sparse = 0, 0
    while True:
        if n_central >= k:
            stop = STOP_K
            break
        if level == max_depth:
            stop = STOP_MAX_DEPTH
            break
        ops.level(level)
        mine = int(b["counts"][3])
        dist.all_reduce(b["counts"])
        marks, new_c, waiting, changed = (int(x) for x in b["counts"].tolist())
        if changed * 16 < n:   # sparse: per-rank change counts, then the padded (id << 8 | mask) lists
            sparse += 1
            per = _all_gather(torch.tensor([mine], dtype=torch.int64)).tolist()
            width = max(1, max(per))
            pad = torch.full((width,), -1, dtype=torch.int64)
            pad[:mine] = torch.tensor(b["chg"][:mine], dtype=torch.int64)
            for e in _all_gather(pad).tolist():
                if e >= 0:
                    b["hm"][e >> 8] = e & 0xFF
        else:
            b["hm"].copy_(_all_gather(b["hm_slice"]))
        n_central += new_c
        if marks == 0 and waiting == 0 and level + 1 < amax:
            ops.waiting(level)
            dist.all_reduce(b["counts"])
            waiting = int(b["counts"][2])
        level += 1
        if marks == 0 and waiting == 0:
            stop = STOP_EXHAUSTED
            break
    mine_M = b["M"][rank * slice_ * 8:(rank + 1) * slice_ * 8].clone()
    b["M"].copy_(_all_gather(mine_M))
    cnt = int(b["cent_n"][0])
    counts = _all_gather(torch.tensor([cnt], dtype=torch.int64)).tolist()
    width = max(max(counts), 1)
    cpad = torch.full((width,), -1, dtype=torch.int32)
    dpad = torch.zeros(width, dtype=torch.uint8)
    cpad[:cnt] = b["cent"][:cnt]
    dpad[:cnt] = b["cdep"][:cnt]
    call, dall = _all_gather(cpad), _all_gather(dpad)
    keep = torch.cat([torch.arange(r * width, r * width + counts[r]) for r in range(world)])
    assert keep.shape[0] == n_central
    return dict(levels=level, stop=stop, n_central=n_central, cent=call[keep], cdep=dall[keep], sparse=sparse)


def slice_size(n, world):
    s = (n + world - 1) // world
    return (s + 15) // 16 * 16


class NumpyVpOps:
    def __init__(self, g, alpha=0.1, block_central=1):
        self.g = g
        self.n = g.n
        self.a = oracle.activation(g.weight, g.A, alpha).astype(np.int64)
        self.block = block_central
        src = np.repeat(np.arange(self.n, dtype=np.int64), np.diff(g.row_ptr))
        dst = np.asarray(g.col_idx, np.int64)
        order = np.argsort(dst, kind="stable")          # in-arcs u -> x grouped by x
        self.in_src = src[order]
        self.in_ptr = np.zeros(self.n + 1, np.int64)
        np.add.at(self.in_ptr, dst + 1, 1)
        self.in_ptr = np.cumsum(self.in_ptr)
        self.bufs = None

    def alloc(self, world):
        self.slice = slice_size(self.n, world)
        self.bufs = vp_alloc(self.n, self.slice, world)

    def begin(self, kw, k, rank, world):
        g, b = self.g, self.bufs
        self.q = len(kw)
        self.full = (1 << self.q) - 1
        self.lo = min(rank * self.slice, self.n)
        self.hi = min(self.lo + self.slice, self.n)
        hm = np.zeros(b["hm"].shape[0], np.uint8)
        M = b["M"].numpy().reshape(-1, 8)
        self.isk = np.zeros(self.n, bool)
        empty = False
        for i, t in enumerate(kw):
            v = np.asarray(g.kw_nodes[g.kw_ptr[t]:g.kw_ptr[t + 1]], np.int64)
            empty |= v.size == 0
            hm[v] |= np.uint8(1 << i)
            M[v, i] = 0
            self.isk[v] = True
        b["hm"].copy_(torch.from_numpy(hm))
        self.ncent = 0
        b["counts"].zero_()
        b["chg"] = []
        b["cent_n"].zero_()
        own = np.arange(self.lo, self.hi)
        for x in own[hm[own] == self.full]:
            self._central(int(x), 0)
        return int(self.a.max()) if self.n else 0, bool(empty)

    def _central(self, x, depth):
        b = self.bufs
        b["cent"][self.ncent] = x
        b["cdep"][self.ncent] = depth
        self.ncent += 1
        b["cent_n"][0] = self.ncent
        b["counts"][1] += 1

    def level(self, l):
        b = self.bufs
        b["counts"].zero_()
        b["chg"] = []
        hm = b["hm"].numpy()[:self.n].astype(np.int64)
        M = b["M"].numpy().reshape(-1, 8)
        X = np.where((self.a <= l) & ~((self.block != 0) & (hm == self.full)), hm, 0)
        marks = wait = 0
        out = b["hm_slice"].numpy()
        for x in range(self.lo, self.hi):
            h = int(hm[x])
            if h and not (self.block and h == self.full) and self.a[x] > l:
                wait += 1                      # not active yet: stays on the work-list (Alg. 2 ln 4-7)
            gate_ok = self.isk[x] or self.a[x] <= l + 1
            need = (self.full & ~h) if gate_ok else 0
            acc = 0
            if need:
                us = self.in_src[self.in_ptr[x]:self.in_ptr[x + 1]]
                if us.size:
                    acc = int(np.bitwise_or.reduce(X[us]))
            nb = acc & need
            out[x - self.lo] = h | nb
            if nb:
                b["chg"].append((x << 8) | (h | nb))
            for i in range(self.q):
                if (nb >> i) & 1:
                    M[x, i] = l + 1
            marks += bin(nb).count("1")
            if nb and (h | nb) == self.full:
                self._central(x, l + 1)
        b["counts"][0] = marks
        b["counts"][2] = wait
        b["counts"][3] = len(b["chg"])

    def waiting(self, l):
        """Active hit nodes with a gated out-neighbour lacking one of their keywords (Alg. 2 ln 17-19)."""
        b, g = self.bufs, self.g
        b["counts"].zero_()
        hm = b["hm"].numpy()[:self.n].astype(np.int64)
        wait = 0
        for f in range(self.lo, self.hi):
            h = int(hm[f])
            if not h or (self.block and h == self.full) or self.a[f] > l:
                continue
            vn = np.asarray(g.col_idx[g.row_ptr[f]:g.row_ptr[f + 1]], np.int64)
            gated = ~self.isk[vn] & (self.a[vn] > l + 1)
            if np.any(gated & ((h & ~hm[vn]) != 0)):
                wait += 1
        b["counts"][2] = wait
