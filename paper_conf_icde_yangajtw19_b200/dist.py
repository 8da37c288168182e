"""Multi-GPU query sharding for the Central Graph search (BASELINE.json configs[3]).

Queries are independent and the graph fits every GPU, so the path shards with no data-path
collective: every rank holds a replica of the graph (kgs_load_graph), answers the queries dealt to it
round-robin, and one all-gather of fixed-size top-k headers (central id, depth, Eq. 6 key) over the
process group (NCCL on GPUs, gloo on CPU for tests) gives every rank the merged answers.

torch.distributed is plumbing only; the query path is libkgs.
"""
from __future__ import annotations

import numpy as np
import torch

HDR_FIELDS = 3   # central id, depth, score key (float64)


def shard(n_items: int, rank: int, world: int) -> np.ndarray:
    """Round-robin deal of item indices to ranks (rank r gets r, r+world, ...)."""
    return np.arange(rank, n_items, world, dtype=np.int64)


def pack_headers(query_ids, answers_per_query, k: int) -> torch.Tensor:
    """[n_local, 1 + k*3] float64 rows: query id, then (central, depth, key) for up to k answers,
    padded with central = -1."""
    n = len(query_ids)
    out = torch.full((n, 1 + k * HDR_FIELDS), -1.0, dtype=torch.float64)
    for r, (qid, answers) in enumerate(zip(query_ids, answers_per_query)):
        out[r, 0] = float(qid)
        for j, a in enumerate(answers[:k]):
            out[r, 1 + HDR_FIELDS * j + 0] = float(a[0])
            out[r, 1 + HDR_FIELDS * j + 1] = float(a[1])
            out[r, 1 + HDR_FIELDS * j + 2] = float(a[2])
    return out


def gather_headers(local: torch.Tensor, n_total: int, world: int, group=None) -> torch.Tensor:
    """All-gather the per-rank header blocks.  Ranks hold ceil/floor(n_total / world) rows; blocks are
    padded to the same row count (query id -1) so one all_gather suffices."""
    import torch.distributed as dist
    rows = (n_total + world - 1) // world
    if not _is_nccl(group):   # gloo: collectives on host tensors
        local = local.cpu()
    pad = torch.full((rows, local.shape[1]), -1.0, dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    outs = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(outs, pad, group=group)
    return torch.cat(outs, dim=0)


def merge_headers(gathered: torch.Tensor, k: int) -> dict:
    """query id -> list of (central, depth, key) in rank order of the answering rank."""
    res = {}
    g = gathered.cpu().numpy()
    for row in g:
        qid = int(row[0])
        if qid < 0:
            continue
        ans = []
        for j in range(k):
            c = int(row[1 + HDR_FIELDS * j])
            if c < 0:
                break
            ans.append((c, int(row[2 + HDR_FIELDS * j]), float(row[3 + HDR_FIELDS * j])))
        res[qid] = ans
    return res


def pack_payloads(query_ids, answers_per_query) -> tuple:
    """The answer subgraphs of this rank's queries as two flat int32 tensors: `index` rows (query id,
    answer rank, #nodes, #arcs) and `data` = for each answer its nodes then its (pred, succ) arc pairs."""
    idx, parts = [], []
    for qid, answers in zip(query_ids, answers_per_query):
        for j, (nodes, arcs) in enumerate(answers):
            nodes = np.asarray(nodes, np.int32).reshape(-1)
            arcs = np.asarray(arcs, np.int32).reshape(-1)
            idx.append((int(qid), j, nodes.size, arcs.size // 2))
            parts += [nodes, arcs]
    index = torch.tensor(np.asarray(idx, np.int32).reshape(-1, 4))
    data = torch.from_numpy(np.concatenate(parts) if parts else np.zeros(0, np.int32))
    return index, data


def gather_payloads(index: torch.Tensor, data: torch.Tensor, group=None) -> dict:
    """Variable-size all-gather of every rank's packed subgraphs (sizes first, then one padded
    all-gather of each tensor), unpacked to {query id: [(nodes, arcs), ...] in answer order}."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    if not _is_nccl(group):   # gloo: collectives on host tensors
        index, data = index.cpu(), data.cpu()
    dev = index.device
    sizes = torch.tensor([index.shape[0], data.shape[0]], dtype=torch.int64, device=dev)
    all_sizes = [torch.empty_like(sizes) for _ in range(world)]
    dist.all_gather(all_sizes, sizes, group=group)
    all_sizes = [tuple(int(x) for x in t.tolist()) for t in all_sizes]
    mi, md = max(max(a for a, _ in all_sizes), 1), max(max(b for _, b in all_sizes), 1)
    ipad = torch.zeros((mi, 4), dtype=torch.int32, device=dev)
    dpad = torch.zeros(md, dtype=torch.int32, device=dev)
    ipad[: index.shape[0]] = index
    dpad[: data.shape[0]] = data
    iout = [torch.empty_like(ipad) for _ in range(world)]
    dout = [torch.empty_like(dpad) for _ in range(world)]
    dist.all_gather(iout, ipad, group=group)
    dist.all_gather(dout, dpad, group=group)
    res = {}
    for (ni, _), it, dt in zip(all_sizes, iout, dout):
        it, dt = it.cpu().numpy(), dt.cpu().numpy()
        off = 0
        for qid, j, nn, na in it[:ni]:
            nodes = dt[off: off + nn]
            arcs = dt[off + nn: off + nn + 2 * na].reshape(-1, 2)
            off += nn + 2 * na
            res.setdefault(int(qid), []).append((int(j), nodes, arcs))
    return {q: [(n, a) for _, n, a in sorted(v, key=lambda t: t[0])] for q, v in res.items()}


def run_sharded(graph, queries, k: int, rank: int, world: int, params=None, group=None, device="cuda"):
    """Answer this rank's share of `queries` with libkgs and all-gather every rank's top-k headers.
    Returns (merged dict query id -> answers, local results)."""
    import paper_conf_icde_yangajtw19_b200 as kgs
    mine = shard(len(queries), rank, world)
    local = []
    for qi in mine:
        r = kgs.kgs_query(graph, list(queries[qi]), k, params)
        local.append([(a.central, a.depth, a.score_key) for a in r.answers])
    hdr = pack_headers(mine.tolist(), local, k).to(device)
    gathered = gather_headers(hdr, len(queries), world, group)
    return merge_headers(gathered, k), local


# --------------------------------------------------------------------------- vertex partition (one query)
# SURVEY §8(e) "a single query": 1-D vertex partition, CSR replicated, one exchange per level.  The level
# loop, the exchanges (dense or sparse) and the stop rules run in the library (kgs_vp_query, vpquery.cu);
# this module only provides the transport: the library's own NCCL communicator when the group is NCCL, or
# host-staged callbacks over the group's collectives (gloo, the CPU / one-GPU tests).


def _is_nccl(group=None) -> bool:
    import torch.distributed as dist
    return dist.get_backend(group) == "nccl"


class GroupTransport:
    """kgs_vp_transport whose callbacks run torch.distributed collectives of `group` on HOST buffers (the
    library copies its device buffers around them: host_staged = 1).  For gloo groups."""

    def __init__(self, group=None):
        import ctypes

        import torch.distributed as dist

        from . import VP_ALL_GATHER, VP_ALL_REDUCE, kgs_vp_transport
        self.dist, self.ctypes, self.group = dist, ctypes, group
        self.world = dist.get_world_size(group)
        self._ag = VP_ALL_GATHER(self._all_gather)
        self._ar = VP_ALL_REDUCE(self._all_reduce)
        self.t = kgs_vp_transport(None, self._ag, self._ar, 0, 1)

    def _all_gather(self, ctx, send, recv, nbytes, stream):
        try:
            c = self.ctypes
            x = torch.frombuffer(bytearray(c.string_at(send, nbytes)), dtype=torch.uint8) if nbytes else \
                torch.zeros(0, dtype=torch.uint8)
            parts = [torch.empty(nbytes, dtype=torch.uint8) for _ in range(self.world)]
            self.dist.all_gather(parts, x, group=self.group)
            out = torch.cat(parts).contiguous()
            if out.numel():
                c.memmove(recv, out.data_ptr(), out.numel())
            return 0
        except Exception:   # noqa: BLE001 — reported to the library as a failed collective
            return -1

    def _all_reduce(self, ctx, buf, count, stream):
        try:
            c = self.ctypes
            x = torch.frombuffer(bytearray(c.string_at(buf, 8 * count)), dtype=torch.int64)
            self.dist.all_reduce(x, group=self.group)
            c.memmove(buf, x.data_ptr(), 8 * count)
            return 0
        except Exception:   # noqa: BLE001
            return -1


_nccl_transports = {}


def nccl_transport(group=None):
    """The library's NCCL communicator for `group` (rank 0 makes the id, the group broadcasts it), cached."""
    import torch.distributed as dist

    import paper_conf_icde_yangajtw19_b200 as kgs
    key = id(group)
    if key not in _nccl_transports:
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        dev = torch.cuda.current_device()
        uid = torch.zeros(128, dtype=torch.uint8, device=f"cuda:{dev}")
        if rank == 0:
            uid.copy_(torch.frombuffer(bytearray(kgs.kgs_vp_nccl_unique_id()), dtype=torch.uint8))
        dist.broadcast(uid, 0, group=group)
        _nccl_transports[key] = kgs.kgs_vp_nccl_transport(bytes(uid.cpu().numpy()), rank, world, dev)
    return _nccl_transports[key]


def vp_query(graph, kw, k: int, params=None, group=None):
    """One query answered by all ranks of `group` with the vertex-partitioned search (every rank holds the
    graph): kgs_vp_query over the group's transport.  Every rank returns the same Result (= kgs_query's)."""
    import torch.distributed as dist

    import paper_conf_icde_yangajtw19_b200 as kgs
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    p = params if params is not None else kgs.kgs_params_default()
    stream = torch.cuda.current_stream().cuda_stream
    if _is_nccl(group):
        t = nccl_transport(group)
        return kgs.kgs_vp_query(graph, kw, k, p, rank, world, t, stream)
    gt = GroupTransport(group)
    return kgs.kgs_vp_query(graph, kw, k, p, rank, world, gt.t, stream)
