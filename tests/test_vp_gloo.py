"""Vertex-partitioned search of one query over gloo on CPU, world sizes 2 and 3: the
protocol of kgs_vp_query (csrc/vpquery.cu) — per-level exchanges (dense all-gather of the hit masks, or
sparse change lists), all-reduce of the counters, the stop rules, the final all-gathers of M and of the
central lists — as the test-side model vp_numpy_ops.vp_search over numpy stand-ins of the level kernels, so
this runs without a GPU; the state every rank ends with must equal the oracle's search.  The transport the
product uses with gloo (dist.GroupTransport, host-staged callbacks) is checked on its own, and the C-ABI
slice rule against the library (a host-only call)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _cases():
    import refimpl as R
    import synth
    out = []
    w = synth.make_workload("C1")
    for kw in w.queries[:6]:
        out.append((w.graph, list(kw), w.k, dict()))
    rng = np.random.default_rng(77)
    for case in range(8):
        n = int(rng.integers(5, 60))
        q = int(rng.integers(1, 5))
        g = R.random_graph(rng, n, float(rng.uniform(0.05, 0.3)), bool(rng.random() < 0.5), q, kw_size=(1, 4),
                           wmax=float(rng.choice([0.0, 0.2, 1.0])))
        out.append((g, list(range(q)), int(rng.choice([1, 3, 50])),
                    dict(alpha=float(rng.choice([0.05, 0.1, 0.4])), max_depth=int(rng.choice([2, 254])),
                         block_central=int(rng.integers(0, 2)))))
    g = synth.from_edges(7, [(0, 1), (1, 2), (2, 3), (4, 5)], [0.5, 0, 0, 0, 0, 0, 0.25],
                         [[0, 2], [2], [], [6], [3, 5]], 2.0)
    out += [(g, [0, 2], 3, dict()), (g, [1, 4], 100, dict()), (g, [0, 1], 1, dict())]   # empty T_i, etc.
    return out


def _worker(rank, world, port, out_q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    sys.path.insert(0, os.path.join(root, "tests"))
    import torch.distributed as dist

    from vp_numpy_ops import NumpyVpOps, vp_search

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    res = []
    for g, kw, k, par in _cases():
        ops = NumpyVpOps(g, alpha=par.get("alpha", 0.1), block_central=par.get("block_central", 1))
        ops.alloc(world)
        s = vp_search(ops, kw, k, par.get("max_depth", 254), rank, world)
        M = ops.bufs["M"].numpy().reshape(-1, 8)[:g.n, :len(kw)].copy()
        order = np.argsort(s["cent"].numpy(), kind="stable")
        res.append(dict(levels=s["levels"], stop=s["stop"], n_central=s["n_central"], M=M, sparse=s["sparse"],
                        cent=s["cent"].numpy()[order].tolist(), cdep=s["cdep"].numpy()[order].tolist()))
    out_q.put((rank, res))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_vp_search_equals_oracle(world):
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for ci, (g, kw, k, par) in enumerate(_cases()):
        o = oracle.query(g, kw, k, alpha=par.get("alpha", 0.1), max_depth=par.get("max_depth", 254),
                         block_central=par.get("block_central", 1))
        for r in range(world):
            s = got[r][ci]
            ctx_ = (ci, r, kw, k, par)
            assert s["stop"] == o.stop_reason, ctx_
            assert s["levels"] == o.levels or o.stop_reason == oracle.STOP_EMPTY_KEYWORD, ctx_
            assert s["cent"] == o.centrals.tolist() and s["cdep"] == o.central_depth.tolist(), ctx_
            assert (s["M"] == o.M).all(), ctx_
    assert any(got[0][ci]["sparse"] for ci in range(len(_cases())))   # the sparse exchange was exercised


def test_vp_slice_rule_matches_library():
    kgs = pytest.importorskip("paper_conf_icde_yangajtw19_b200")
    from vp_numpy_ops import slice_size
    for n, w in [(0, 1), (1, 1), (7, 2), (1024, 3), (33554432, 8), (1000003, 5)]:
        s = kgs.kgs_vp_slice(n, w)
        assert s == slice_size(n, w) and s % 16 == 0 and s * w >= n
    assert kgs.kgs_vp_slice(5, 0) == 0


def _transport_worker(rank, world, port, out_q):
    import ctypes
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import torch
    import torch.distributed as dist

    from paper_conf_icde_yangajtw19_b200 import dist as kd
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    gt = kd.GroupTransport()
    send = (ctypes.c_uint8 * 5)(*[rank * 10 + i for i in range(5)])
    recv = (ctypes.c_uint8 * (5 * world))()
    rc1 = gt.t.all_gather(None, ctypes.addressof(send), ctypes.addressof(recv), 5, None)
    buf = (ctypes.c_int64 * 4)(rank, 1, -rank, 1 << 40)
    rc2 = gt.t.all_reduce_sum_i64(None, ctypes.addressof(buf), 4, None)
    out_q.put((rank, rc1, rc2, list(recv), list(buf), gt.t.host_staged))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_group_transport_callbacks(world):
    """dist.GroupTransport (the gloo transport of kgs_vp_query): all_gather / all_reduce callbacks on host
    buffers give every rank the concatenation / the sum."""
    pytest.importorskip("paper_conf_icde_yangajtw19_b200")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_transport_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, rc1, rc2, recv, buf, staged in got:
        assert rc1 == 0 and rc2 == 0 and staged == 1
        assert recv == [r * 10 + i for r in range(world) for i in range(5)]
        assert buf == [sum(range(world)), world, -sum(range(world)), world << 40]
