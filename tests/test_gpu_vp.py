"""Vertex-partitioned search of one query on the GPU (kgs_vp_* kernels + dist.vp_query): world sizes 1, 2
and 3 as processes sharing cuda:0 over gloo (the box has one GPU; NCCL refuses two ranks on one
device, so the collectives are staged through host memory — the kernels and the protocol are the same).
Every rank's answers must equal the oracle's (central ids, depths, Eq. 6 keys, subgraphs), and with
want_levels the replicated M and central list too."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


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
    for kw in w.queries[:12]:
        out.append((("C1",), list(kw), w.k, dict()))
    w2 = synth.make_workload("C2")
    for kw in w2.queries[::25]:
        out.append((("C2",), list(kw), w2.k, dict()))
    rng = np.random.default_rng(91)
    for case in range(10):
        out.append((("rand", case), list(range(int(rng.integers(1, 5)))), int(rng.choice([1, 3, 40])),
                    dict(alpha=float(rng.choice([0.05, 0.1, 0.4])), max_depth=int(rng.choice([2, 254])),
                         block_central=int(rng.integers(0, 2)), extract_mode=int(rng.integers(0, 2)),
                         want_levels=int(rng.integers(0, 2)))))
    out += [(("tiny",), [0, 2], 3, dict(want_levels=1)), (("tiny",), [1, 4], 100, dict()),
            (("tiny",), [0, 1], 1, dict())]
    return out


def _graph(key, cache):
    import refimpl as R
    import synth
    if key in cache:
        return cache[key]
    if key[0] in ("C1", "C2"):
        g = synth.make_workload(key[0]).graph
    elif key[0] == "rand":
        rng = np.random.default_rng(1000 + key[1])
        n = int(rng.integers(5, 80))
        g = R.random_graph(rng, n, float(rng.uniform(0.05, 0.3)), bool(rng.random() < 0.5), 4, kw_size=(1, 5),
                           wmax=float(rng.choice([0.0, 0.2, 1.0])))
    else:
        g = synth.from_edges(7, [(0, 1), (1, 2), (2, 3), (4, 5)], [0.5, 0, 0, 0, 0, 0, 0.25],
                             [[0, 2], [2], [], [6], [3, 5]], 2.0)
    cache[key] = g
    return g


def _worker(rank, world, port, out_q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    sys.path.insert(0, os.path.join(root, "tests"))
    import torch
    import torch.distributed as dist

    import paper_conf_icde_yangajtw19_b200 as kgs
    from paper_conf_icde_yangajtw19_b200 import dist as kd

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    cache, loaded, res = {}, {}, []
    for key, kw, k, par in _cases():
        g = _graph(key, cache)
        if key not in loaded:
            loaded[key] = kgs.kgs_load_graph(g)
        p = kgs.make_params(**par)
        r = kd.vp_query(loaded[key], kw, k, p)
        item = dict(answers=[(a.central, a.depth, a.score_key, a.nodes.tolist(), a.arcs.tolist()) for a in r.answers],
                    stop=r.stats["stop_reason"], levels=r.stats["levels"], n_centrals=r.stats["n_centrals"])
        if par.get("want_levels"):
            item.update(M=r.M, cent=r.centrals.tolist(), cdep=r.central_depth.tolist())
        res.append(item)
    out_q.put((rank, res))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [1, 2, 3])
def test_vp_query_equals_oracle(world):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=900) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    cache = {}
    for ci, (key, kw, k, par) in enumerate(_cases()):
        g = _graph(key, cache)
        o = oracle.query(g, kw, k, alpha=par.get("alpha", 0.1), max_depth=par.get("max_depth", 254),
                         block_central=par.get("block_central", 1), extract_mode=par.get("extract_mode", 0))
        exp = [(a.central, a.depth, a.key, a.nodes.tolist(), a.arcs.tolist()) for a in o.answers]
        for r in range(world):
            s = got[r][ci]
            ctx_ = (ci, key, r, kw, k, par)
            assert s["stop"] == o.stop_reason, ctx_
            if o.stop_reason != oracle.STOP_EMPTY_KEYWORD:
                assert s["levels"] == o.levels, ctx_
            assert s["n_centrals"] == len(o.centrals), ctx_
            assert s["answers"] == exp, ctx_
            if par.get("want_levels"):
                assert (s["M"] == o.M).all(), ctx_
                assert s["cent"] == o.centrals.tolist() and s["cdep"] == o.central_depth.tolist(), ctx_
