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
# SURVEY §8(e) "a single query": 1-D vertex partition, CSR replicated, one exchange per level.  The
# level kernels are libkgs's (kgs_vp_*); this driver only moves their buffers between ranks and applies
# the stop rules of Def. 4 / Thm. V.3 to the reduced counters.  NCCL collectives run on the device
# buffers directly; with gloo (tests) they are staged through host memory.

STOP_K, STOP_EXHAUSTED, STOP_MAX_DEPTH, STOP_EMPTY_KEYWORD = 0, 1, 2, 3


def _is_nccl(group=None) -> bool:
    import torch.distributed as dist
    return dist.get_backend(group) == "nccl"


def all_gather_into(out: torch.Tensor, inp: torch.Tensor, group=None) -> None:
    """out = concat over ranks of inp (equal sizes)."""
    import torch.distributed as dist
    if _is_nccl(group):
        dist.all_gather_into_tensor(out, inp, group=group)
        return
    world = dist.get_world_size(group)
    parts = [torch.empty(inp.shape, dtype=inp.dtype) for _ in range(world)]
    dist.all_gather(parts, inp.cpu(), group=group)
    out.copy_(torch.cat(parts).to(out.device))


def all_reduce_sum(t: torch.Tensor, group=None) -> None:
    import torch.distributed as dist
    if _is_nccl(group):
        dist.all_reduce(t, group=group)
        return
    h = t.cpu()
    dist.all_reduce(h, group=group)
    t.copy_(h.to(t.device))


def vp_alloc(n: int, slice_: int, world: int, device) -> dict:
    """The exchange buffers of kgs_vp_buffers (torch owns the device memory)."""
    n_pad = slice_ * world
    return dict(hm=torch.zeros(n_pad, dtype=torch.uint8, device=device),
                hm_slice=torch.zeros(slice_, dtype=torch.uint8, device=device),
                M=torch.full((n_pad * 8,), 255, dtype=torch.uint8, device=device),
                counts=torch.zeros(3, dtype=torch.int64, device=device),
                cent=torch.zeros(max(slice_, 1), dtype=torch.int32, device=device),
                cdep=torch.zeros(max(slice_, 1), dtype=torch.uint8, device=device),
                cent_n=torch.zeros(1, dtype=torch.int32, device=device))


def vp_search(ops, kw, k: int, max_depth: int, rank: int, world: int, group=None) -> dict:
    """The level loop over `ops` (begin / level on this rank's rows; see LibVpOps).  Returns the stop
    level and reason, |C| and the all-gathered state (hm, M, central list)."""
    b = ops.bufs
    slice_ = b["hm_slice"].shape[0]
    amax, empty = ops.begin(kw, k, rank, world)
    if empty:   # reading R17: some T_i is empty, nothing can be central
        return dict(levels=0, stop=STOP_EMPTY_KEYWORD, n_central=0, cent=b["cent"][:0], cdep=b["cdep"][:0])
    all_reduce_sum(b["counts"], group)
    n_central = int(b["counts"][1].item())
    level = 0
    while True:
        if n_central >= k:
            stop = STOP_K
            break
        if level == max_depth:
            stop = STOP_MAX_DEPTH
            break
        ops.level(level)
        all_gather_into(b["hm"], b["hm_slice"], group)
        all_reduce_sum(b["counts"], group)
        marks, new_c, waiting = (int(x) for x in b["counts"].tolist())
        n_central += new_c
        if marks == 0 and waiting == 0 and level + 1 < amax:   # gated neighbours are possible
            ops.waiting(level)
            all_reduce_sum(b["counts"], group)
            waiting = int(b["counts"][2].item())
        if marks == 0 and waiting == 0:   # the work-list of Alg. 2 is empty at level + 1
            level += 1
            stop = STOP_EXHAUSTED
            break
        level += 1
    # owned M rows and central lists to every rank
    mine = b["M"][rank * slice_ * 8:(rank + 1) * slice_ * 8].clone()
    all_gather_into(b["M"], mine, group)
    cnt = b["cent_n"].to(torch.int64)
    counts = torch.zeros(world, dtype=torch.int64, device=cnt.device)
    all_gather_into(counts, cnt, group)
    counts = counts.tolist()
    width = max(max(counts), 1)
    cpad = torch.full((width,), -1, dtype=torch.int32, device=b["cent"].device)
    dpad = torch.zeros(width, dtype=torch.uint8, device=b["cent"].device)
    cpad[:counts[rank]] = b["cent"][:counts[rank]]
    dpad[:counts[rank]] = b["cdep"][:counts[rank]]
    call = torch.empty(width * world, dtype=torch.int32, device=cpad.device)
    dall = torch.empty(width * world, dtype=torch.uint8, device=cpad.device)
    all_gather_into(call, cpad, group)
    all_gather_into(dall, dpad, group)
    keep = torch.cat([torch.arange(r * width, r * width + counts[r], device=cpad.device) for r in range(world)])
    cent, cdep = call[keep].contiguous(), dall[keep].contiguous()
    assert cent.shape[0] == n_central, (cent.shape[0], n_central)
    return dict(levels=level, stop=stop, n_central=n_central, cent=cent, cdep=cdep)


class LibVpOps:
    """The level kernels of libkgs (kgs_vp_begin / kgs_vp_level / kgs_vp_topdown) over torch buffers."""

    def __init__(self, graph, params=None, device=None):
        import paper_conf_icde_yangajtw19_b200 as kgs
        self.kgs = kgs
        self.graph = graph
        self.params = params if params is not None else kgs.kgs_params_default()
        self.device = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.stream = torch.cuda.current_stream(self.device).cuda_stream
        self.bufs = None
        self.k = 0

    def alloc(self, world: int):
        slice_ = self.kgs.kgs_vp_slice(self.graph.n, world)
        self.bufs = vp_alloc(self.graph.n, slice_, world, self.device)
        b = self.bufs
        self.cbufs = self.kgs.kgs_vp_buffers(b["hm"].data_ptr(), b["hm_slice"].data_ptr(), b["M"].data_ptr(),
                                             b["counts"].data_ptr(), b["cent"].data_ptr(), b["cdep"].data_ptr(),
                                             b["cent_n"].data_ptr())

    def begin(self, kw, k, rank, world):
        self.kw, self.k = list(kw), int(k)
        return self.kgs.kgs_vp_begin(self.graph, kw, k, self.params, rank, world, self.cbufs, self.stream)

    def level(self, level):
        self.kgs.kgs_vp_level(self.graph, level, self.stream)

    def waiting(self, level):
        self.kgs.kgs_vp_waiting(self.graph, level, self.stream)

    def topdown(self, s):
        return self.kgs.kgs_vp_topdown(self.graph, s["n_central"], s["cent"].data_ptr(), s["cdep"].data_ptr(),
                                       s["levels"], s["stop"], len(self.kw), self.params.want_levels, self.stream)


def vp_query(graph, kw, k: int, params=None, group=None):
    """One query answered by all ranks of `group` with the vertex-partitioned search (every rank holds
    the graph).  Every rank returns the same Result (= kgs_query's)."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    ops = LibVpOps(graph, params)
    ops.alloc(world)
    s = vp_search(ops, kw, k, ops.params.max_depth, rank, world, group)
    return ops.topdown(s)
