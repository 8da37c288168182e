"""Test-only numpy stand-in for libkgs's vertex-partition level kernels (kgs_vp_begin / kgs_vp_level), so
the host protocol of paper_conf_icde_yangajtw19_b200.dist.vp_search (exchanges over torch.distributed,
stop rules) can be checked against the oracle on CPU with gloo.  Same contract as dist.LibVpOps: this
rank writes only its rows [lo, hi) of M / hm_slice / the central list.  Level rule of Alg. 2
in pull form: x gets keyword i at level l iff m_xi = inf, (x in K or a_x <= l + 1) and some in-neighbour
u with a_u <= l, m_ui <= l, and (u not central or blocking off)."""
import numpy as np
import torch

import oracle
from paper_conf_icde_yangajtw19_b200 import dist as kd


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
        self.bufs = kd.vp_alloc(self.n, self.slice, world, "cpu")

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
            for i in range(self.q):
                if (nb >> i) & 1:
                    M[x, i] = l + 1
            marks += bin(nb).count("1")
            if nb and (h | nb) == self.full:
                self._central(x, l + 1)
        b["counts"][0] = marks
        b["counts"][2] = wait

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
