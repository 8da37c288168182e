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
