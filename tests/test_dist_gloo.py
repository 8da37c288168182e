"""World-size-2 gloo test (CPU) of the multi-GPU host logic: round-robin sharding, header packing,
the all-gather and the merge by query id, and the variable-size gather of the answer subgraphs.  The per-query answers come from the oracle (test
infrastructure), standing in for libkgs which needs a GPU."""
import os
import socket

import pytest
import torch
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import torch.distributed as dist

    import oracle
    import synth
    from paper_conf_icde_yangajtw19_b200 import dist as kd

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    w = synth.make_workload("C1")
    qs = w.queries[:13]                       # ragged: 13 queries over 2 ranks
    mine = kd.shard(len(qs), rank, world)
    local = []
    for qi in mine:
        r = oracle.query(w.graph, qs[qi], w.k)
        local.append([(a.central, a.depth, a.key) for a in r.answers])
    hdr = kd.pack_headers(mine.tolist(), local, w.k)
    merged = kd.merge_headers(kd.gather_headers(hdr, len(qs), world), w.k)
    # the answer subgraphs: sizes first, then a padded all-gather (variable payloads)
    subs = [[(a.nodes, a.arcs) for a in oracle.query(w.graph, qs[qi], w.k).answers] for qi in mine]
    index, data = kd.pack_payloads(mine.tolist(), subs)
    payloads = kd.gather_payloads(index, data)
    if rank == 0:
        out_q.put((merged, {q: [(n.tolist(), a.tolist()) for n, a in v] for q, v in payloads.items()}))
    dist.barrier()
    dist.destroy_process_group()


def test_sharded_gather_equals_single_process():
    import oracle
    import synth
    from paper_conf_icde_yangajtw19_b200 import dist as kd

    assert kd.shard(13, 0, 2).tolist() == list(range(0, 13, 2))
    assert kd.shard(13, 1, 2).tolist() == list(range(1, 13, 2))
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    merged, payloads = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    w = synth.make_workload("C1")
    qs = w.queries[:13]
    assert sorted(merged) == list(range(13))
    for qi, kw in enumerate(qs):
        r = oracle.query(w.graph, kw, w.k)
        assert merged[qi] == [(a.central, a.depth, a.key) for a in r.answers]
        got = payloads.get(qi, [])
        assert [n for n, _ in got] == [a.nodes.tolist() for a in r.answers]
        assert [x for _, x in got] == [a.arcs.reshape(-1, 2).tolist() for a in r.answers]
