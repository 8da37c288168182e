#!/usr/bin/env python
"""Benchmark of the Central Graph keyword-search hot path (BASELINE.json metric: p50 query latency,
queries/s and GTEPS on the Wikidata-scale synthetic graph).

  python bench.py [--gpus N --steps K --warmup W]          CUDA path (libkgs), one rank per GPU
  python bench.py --impl reference [...]                   the CPU oracle on this box's host cores

Workload (--workload): C4 (BASELINE.json configs[3], the default: the Wikidata-scale graph, 2^25 nodes /
2^28 edges, a batch of 4096 queries with q ~ U{2..8}, top-20) or C3 (configs[2]: the same graph shape,
350 queries with q = 2..8).  A step = the
workload's whole batch through the whole hot path (activation gate, search, central detection, extraction
+ level-cover + Eq. 6 of the candidate central graphs, top-k, answer emit) in ONE engine launch per rank.
N > 1 (torchrun): every rank holds a replica of the graph (rank 0 generates it and broadcasts it over
NCCL), the step's batch is dealt round-robin over the ranks (dist.shard: total work fixed, strong
scaling), and the top-k headers and answer subgraphs are all-gathered over NCCL inside the timed region.

`value` = queries/s of device time over K steps (CUDA events on the launching stream, L2 flushed with a
512 MiB write between steps, outside the events; max over ranks).  The single-query latency mode (one
launch per query, the whole GPU on it) gives `p50_ms` / `p95_ms` and the expansion-phase roofline.
`e2e` = the same batches through kgs_query_batch from host keyword ids to host answers (wall clock,
H2D + D2H inside).  `cpu_baseline` = the oracle on ~15 s of the step's queries, pinned to one core.
"""
from __future__ import annotations

import argparse
import glob
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "p50 query latency (ms) & queries/s, Wikidata-scale graph; GTEPS"
WORKLOAD = "C4"      # the step's batch: C4's 4096 queries (configs[3]) or C3's 350 (configs[2], --workload C3)
# Queries the CPU oracle cannot finish in a bench run: C4's seven level-5 queries, ~10^6 central nodes
# each (profiles/r02b_c4_scan.txt), whose every Central Graph the oracle extracts (hours per query; the
# GPU parity tests check them on a seeded sample, tests/test_gpu_fullsize.py).  The oracle's bounded
# sample (cpu_baseline, --impl reference) skips them and says so.
ORACLE_SKIP = {"C4": (11, 1422, 1619, 2557, 2683, 2906, 3629)}
GROUPS = 8           # engine groups in batch mode (queries answered at the same time)
# DRAM bytes/s a stream of independent random 4-byte gathers moves on this B200 (37.7 G gathers/s, 124 B of
# DRAM read per gather: tools/rand_gather_bench.cu, profiles/r02d_random_access.txt)
RANDOM_GATHER_DRAM_GBS = 37.7 * 124
RELABEL = os.environ.get("KGS_RELABEL", "1") != "0"   # ablation: 0 keeps the input node order internally


def _env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.rows = []
        self.proc = None
        self.th = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-i", str(self.index), "-lms", "50"], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
            return
        self.th = threading.Thread(target=self._read, daemon=True)
        self.th.start()

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        if self.th:
            self.th.join(timeout=2)
        sm = [float(r[1]) for r in self.rows if len(r) >= 9 and r[1].replace(".", "").isdigit()]
        smax = [float(r[2]) for r in self.rows if len(r) >= 9 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            if len(r) >= 9:
                for nm, v in zip(names, r[5:9]):
                    if v.lower() == "active":
                        reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


ENGINE_SOURCES = ("paper_conf_icde_yangajtw19_b200/csrc/*.cu", "paper_conf_icde_yangajtw19_b200/csrc/*.h",
                  "include/kgs.h")


def source_hash() -> str:
    """sha256 over the engine's sources (csrc/*.cu, *.h, include/kgs.h): identifies the build an ncu
    capture was taken of (tools/make_batch_profile.py stores it next to the DRAM bytes)."""
    import hashlib
    h = hashlib.sha256()
    for pat in ENGINE_SOURCES:
        for f in sorted(glob.glob(os.path.join(ROOT, pat))):
            h.update(os.path.basename(f).encode())
            with open(f, "rb") as fh:
                h.update(fh.read())
    return h.hexdigest()


def load_traffic(workload: str):
    """DRAM bytes per query of the engine from the newest committed ncu capture of the bench's own launch
    shape (profiles/r*_batch_traffic.json for this workload), with the git sha / source hash it was
    taken at.  Returns (bytes per query or None, info dict)."""
    # a capture of the running sources first (src_sha256), then the newest capture (captured_unix; older
    # files without it by name)
    cands = []
    here = source_hash()
    for f in glob.glob(os.path.join(ROOT, "profiles", "r*_batch_traffic.json")):
        with open(f) as fh:
            d = json.load(fh)
        if d.get("workload", "C3") != workload:
            continue
        cands.append((d.get("src_sha256") == here, d.get("captured_unix", 0), os.path.basename(f), d))
    if not cands:
        return None, {"traffic_source": None}
    match, _, name, d = max(cands, key=lambda t: (t[0], t[1], t[2]))
    return d["dram_bytes_per_query"], {"traffic_source": name, "traffic_sha": d.get("git_sha"),
                                       "traffic_matches_source": match, "traffic_l2_hit_pct": d.get("l2_hit_pct"),
                                       "traffic_same_work": d.get("same_work")}


def cpu_info() -> dict:
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count()}


class pinned_core:
    """Run the oracle on ONE host core (the `taskset -c <cpu>` of the CPU-baseline protocol)."""

    def __enter__(self):
        self.old = os.sched_getaffinity(0)
        self.cpu = min(self.old)
        os.sched_setaffinity(0, {self.cpu})
        return self

    def __exit__(self, *exc):
        os.sched_setaffinity(0, self.old)
        return False


def expansion_bytes(st: dict) -> float:
    """SURVEY.md §8(d) B_bfs: the bytes the expansion must move for one query — per frontier entry 16 B
    row_ptr + 2 B own status + 1 B activation + 4 B queue slot, per inspected out-arc 4 B col_idx + 2 B
    neighbour status, per new (node, keyword) hit 1 B M + 1 B new-hit mask + 4 B next frontier."""
    return st["frontier_total"] * 23.0 + st["arcs_scanned"] * 6.0 + st.get("hits", 0) * 6.0


def algorithmic_bytes(st: dict) -> float:
    """SURVEY.md §8(d) / DESIGN.md §7: bytes the hot path must move for one query.
    search: per frontier entry 16 B row_ptr + 2 B own status + 1 B activation + 4 B queue slot; per
    inspected out-arc 4 B col_idx + 2 B neighbour status; per new (node, keyword) hit 1 B M write +
    1 B new-hit mask + 4 B next frontier (amortised).  top-down pre-pass: per inspected in-arc 4 B in_idx
    + 2 B status; per predecessor arc 4 B node + 2 B bits written and read back."""
    return (st["frontier_total"] * 23.0 + st["arcs_scanned"] * 6.0 + st.get("hits", 0) * 6.0 +
            st.get("td_arcs", 0) * 6.0 + st.get("td_pred_arcs", 0) * 12.0)


# ------------------------------------------------------------------------------------------ workloads
def build_workload(name: str):
    """C3 (configs[2]) or C4 (configs[3]: the C3 graph with its own 4096-query set)."""
    import synth
    t0 = time.time()
    if name == "C4":
        w = synth.make_workload("C3")
        w = synth.Workload("C4", w.graph, synth.config_queries("C4", w.graph), synth.CONFIG_PARAMS["C4"]["k"])
    else:
        w = synth.make_workload(name)
    return w, time.time() - t0


def step_queries(name: str, queries):
    """The queries of one step in their order: C3's 350 in the bench permutation, C4's 4096 as generated."""
    if name == "C3":
        order = np.random.default_rng(12345).permutation(len(queries))
        return [queries[i] for i in order], [int(i) for i in order]
    return list(queries), list(range(len(queries)))


class _RemoteGraph:
    def __init__(self, n, n_arcs):
        self.n, self.n_arcs = n, n_arcs


def load_replicated(name, rank, world, dev, kgs):
    """Rank 0 generates the workload once; every rank receives the arrays over NCCL (device to device)
    and loads its replica from device pointers (KGS_INPUT_DEVICE_PTRS)."""
    import torch
    import torch.distributed as dist
    from types import SimpleNamespace
    t0 = time.time()
    cuda = f"cuda:{dev}"
    if rank == 0:
        w, _ = build_workload(name)
        g = w.graph
        qmax = max(len(q) for q in w.queries)
        meta = torch.tensor([g.n, g.n_arcs, g.n_keywords, g.kw_nodes.shape[0], len(w.queries), qmax, w.k],
                            dtype=torch.int64, device=cuda)
        A = torch.tensor([g.A], dtype=torch.float64, device=cuda)
    else:
        meta = torch.zeros(7, dtype=torch.int64, device=cuda)
        A = torch.zeros(1, dtype=torch.float64, device=cuda)
    dist.broadcast(meta, 0)
    dist.broadcast(A, 0)
    n, m, V, P, nq, qmax, k = (int(x) for x in meta.tolist())
    if rank == 0:
        t = [torch.from_numpy(g.row_ptr).to(cuda), torch.from_numpy(g.col_idx).to(cuda),
             torch.from_numpy(g.weight).to(cuda), torch.from_numpy(g.kw_ptr).to(cuda),
             torch.from_numpy(g.kw_nodes).to(cuda)]
        qt = torch.full((nq, qmax), -1, dtype=torch.int32)
        for i, q in enumerate(w.queries):
            qt[i, :len(q)] = torch.tensor(q, dtype=torch.int32)
        qt = qt.to(cuda)
    else:
        t = [torch.empty(n + 1, dtype=torch.int64, device=cuda), torch.empty(m, dtype=torch.int32, device=cuda),
             torch.empty(n, dtype=torch.float32, device=cuda), torch.empty(V + 1, dtype=torch.int64, device=cuda),
             torch.empty(P, dtype=torch.int32, device=cuda)]
        qt = torch.empty((nq, qmax), dtype=torch.int32, device=cuda)
    for x in t:
        dist.broadcast(x, 0)
    dist.broadcast(qt, 0)
    gen_s = time.time() - t0
    t1 = time.time()
    G = kgs.kgs_load_graph_device(n, m, t[0].data_ptr(), t[1].data_ptr(), t[2].data_ptr(), V, t[3].data_ptr(),
                                  t[4].data_ptr(), float(A.item()), True, dev, relabel=RELABEL)
    torch.cuda.synchronize(dev)
    load_s = time.time() - t1
    del t
    qh = qt.cpu().numpy()
    queries = [tuple(int(x) for x in row if x >= 0) for row in qh]
    return SimpleNamespace(queries=queries, k=k), _RemoteGraph(n, m), G, gen_s, load_s


def graph_desc(name, g):
    return f"R-MAT scale 25, edge factor 8: {g.n} nodes, {g.n_arcs} arcs" + (" (the C3 graph)" if name == "C4" else "")


def run_reference(args):
    """The oracle, as it stands, on ONE pinned host core (bench.py --impl reference): rank 0 only.  A step
    is one query of the workload (the oracle is single-threaded); K steps after W warm-up queries."""
    rank, world = _env_int("RANK", 0), _env_int("WORLD_SIZE", 1)
    if rank != 0:
        return 0
    import oracle
    name = args.workload
    w, gen_s = build_workload(name)
    qs, ids = step_queries(name, w.queries)
    skip = set(ORACLE_SKIP.get(name, ()))
    qs = [q for q, i in zip(qs, ids) if i not in skip]
    lat = []
    with pinned_core() as pc:
        for i in range(args.warmup):
            oracle.query(w.graph, qs[i % len(qs)], w.k)
        t_all = time.perf_counter()
        for i in range(args.steps):
            kw = qs[(args.warmup + i) % len(qs)]
            t0 = time.perf_counter()
            oracle.query(w.graph, kw, w.k)
            lat.append((time.perf_counter() - t0) * 1e3)
        tot = time.perf_counter() - t_all
    qps = args.steps / tot
    line = {"impl": "reference", "metric": METRIC, "value": qps, "unit": "queries/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot * 1e3 / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": {"workload": name, "graph": graph_desc(name, w.graph), "k": w.k, "queries": len(qs),
                       "step": "one query (the oracle is single-threaded; a step of the GPU arm is a batch)"},
            "p50_ms": statistics.median(lat),
            "cpu_baseline": {"value": qps, "unit": "queries/s", "cores": 1, "kind": "oracle", "pinned_cpu": pc.cpu,
                             **cpu_info(),
                             "sample": f"{args.steps} consecutive {name} queries after {args.warmup} warm-up"
                                       + (f" (skipping the {len(skip)} level-5 queries {sorted(skip)}, hours each "
                                          f"for the oracle)" if skip else "")},
            "e2e": {"value": qps, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="kgs", choices=["kgs", "reference"])
    ap.add_argument("--workload", default=WORKLOAD, choices=["C3", "C4"])
    ap.add_argument("--groups", type=int, default=GROUPS)
    ap.add_argument("--latency-steps", type=int, default=200)
    ap.add_argument("--cpu-sample-s", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        return run_reference(args)

    import torch
    rank, world, local = _env_int("RANK", 0), _env_int("WORLD_SIZE", 1), _env_int("LOCAL_RANK", 0)
    dist = None
    if world > 1:
        import torch.distributed as dist
        # KGS_BENCH_ONE_GPU=1 (test of the multi-rank path on a one-GPU box): every rank on cuda:0 over
        # gloo (NCCL refuses two ranks on one device); the collectives of dist.py stage through the host
        if os.environ.get("KGS_BENCH_ONE_GPU") == "1":
            local = 0
            args.groups = max(1, args.groups // world)   # the ranks share one GPU's memory
            torch.cuda.set_device(0)
            dist.init_process_group("gloo")
        else:
            torch.cuda.set_device(local)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = local
    torch.cuda.set_device(dev)
    cuda = f"cuda:{dev}"
    import paper_conf_icde_yangajtw19_b200 as kgs
    from paper_conf_icde_yangajtw19_b200 import dist as kd

    name = args.workload
    if world == 1:
        w, gen_s = build_workload(name)
        g = w.graph
        t0 = time.time()
        G = kgs.kgs_load_graph(g, device=dev, relabel=RELABEL)
        load_s = time.time() - t0
    else:
        w, g, G, gen_s, load_s = load_replicated(name, rank, world, dev, kgs)
    allq, qids_all = step_queries(name, w.queries)
    # one step = the workload's whole batch, dealt round-robin over the ranks (dist.shard): strong scaling
    mine = kd.shard(len(allq), rank, world).tolist()
    queries = [allq[i] for i in mine]
    qids = [qids_all[i] for i in mine]
    B = len(queries)
    stream = torch.cuda.current_stream(dev)
    sh = stream.cuda_stream
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=cuda)
    kwp = torch.full((B, 8), -1, dtype=torch.int32)
    for r, q in enumerate(queries):
        kwp[r, :len(q)] = torch.tensor(q, dtype=torch.int32)
    kwd = kwp.to(cuda)
    qld = torch.tensor([len(q) for q in queries], dtype=torch.int32, device=cuda)
    qlens = [len(q) for q in queries]
    p = kgs.kgs_params_default()

    # ---- batch mode (value): one engine launch per step
    for s_ in range(args.warmup):
        kgs.kgs_query_batch_device(G, B, kwd.data_ptr(), qld.data_ptr(), w.k, p, args.groups, sh)
        kgs.kgs_query_batch_fetch(G, qlens, sh)
    torch.cuda.synchronize(dev)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    stats, answers, subgraphs = [], [], []
    clk = ClockSampler(dev)
    clk.start()
    if dist:
        dist.barrier()
    torch.cuda.synchronize(dev)
    for i in range(args.steps):
        flush.fill_(i & 0xFF)                       # L2 flush between timed steps (outside the events)
        ev[i][0].record(stream)
        kgs.kgs_query_batch_device(G, B, kwd.data_ptr(), qld.data_ptr(), w.k, p, args.groups, sh)
        ev[i][1].record(stream)
        res = kgs.kgs_query_batch_fetch(G, qlens, sh)   # after the end event: not timed
        stats += [r.stats for r in res]
        if i == args.steps - 1:
            answers = [(qids[j], [(a.central, a.depth, a.score_key) for a in r.answers]) for j, r in enumerate(res)]
            subgraphs = [(qids[j], [(a.nodes, a.arcs) for a in r.answers]) for j, r in enumerate(res)]
    gather_ms = 0.0
    if dist:
        # NCCL all-gather of every rank's top-k headers (central, depth, key) and answer subgraphs
        # (sizes, then a padded gather of the variable payloads) of the last step
        hdr = kd.pack_headers([q for q, _ in answers], [a for _, a in answers], w.k).to(cuda)
        pidx, pdat = kd.pack_payloads([q for q, _ in subgraphs], [s_ for _, s_ in subgraphs])
        pidx, pdat = pidx.to(cuda), pdat.to(cuda)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        kd.gather_headers(hdr, len(allq), world)
        kd.gather_payloads(pidx, pdat)
        e1.record(stream)
    torch.cuda.synchronize(dev)
    if dist:
        dist.barrier()
        gather_ms = e0.elapsed_time(e1)
    clocks = clk.stop()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    dev_ms = sum(step_ms) + gather_ms
    if dist:
        t = torch.tensor([dev_ms], dtype=torch.float64, device=cuda)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dev_ms = float(t.item())
    total_queries = args.steps * len(allq)
    value = total_queries / (dev_ms / 1e3)
    arcs = sum(s_["arcs_scanned"] for s_ in stats)   # GTEPS: arcs the search expanded
    alg = sum(algorithmic_bytes(s_) for s_ in stats)
    exp_b = sum(expansion_bytes(s_) for s_ in stats)
    exp_us = sum(s_["phases_us"].get("expand", 0.0) for s_ in stats)   # group time, G groups at once
    n_groups = max(1, min(args.groups, B))

    # ---- single-query latency mode: the whole GPU on one query, one launch per query
    lat, lat_stats = [], []
    if rank == 0:
        nlat = min(args.latency_steps, len(queries))
        qdev = [torch.tensor(list(q), dtype=torch.int32, device=cuda) for q in queries[:nlat + args.warmup]]
        for i in range(args.warmup):
            kgs.kgs_query_device(G, qdev[i].data_ptr(), len(queries[i]), w.k, p, sh)
            kgs.kgs_query_fetch(G, len(queries[i]), 0, sh)
        for i in range(nlat):
            j = args.warmup + i
            flush.fill_(i & 0xFF)
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            kgs.kgs_query_device(G, qdev[j].data_ptr(), len(queries[j]), w.k, p, sh)
            a1.record(stream)
            r = kgs.kgs_query_fetch(G, len(queries[j]), 0, sh)
            lat.append(a0.elapsed_time(a1))
            lat_stats.append(r.stats)

    # ---- e2e: host keyword ids -> kgs_query_batch -> answers on the host (wall clock)
    e2e_ms, d2h = [], 0
    for i in range(min(args.steps, 3)):
        torch.cuda.synchronize(dev)
        if dist:
            dist.barrier()
        t0 = time.perf_counter()
        res = kgs.kgs_query_batch(G, queries, w.k, p, args.groups, sh)
        el = (time.perf_counter() - t0) * 1e3
        if dist:
            t = torch.tensor([el], dtype=torch.float64, device=cuda)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            el = float(t.item())
        e2e_ms.append(el)
        d2h += sum(32 + a.nodes.nbytes + a.arcs.nbytes + 24 for r in res for a in r.answers)
    e2e_qps = len(e2e_ms) * len(allq) / (sum(e2e_ms) / 1e3)
    h2d = B * (4 * 8 + 4)

    if rank != 0:
        if dist:
            dist.destroy_process_group()
        return 0
    peak, peak_kind = load_peaks()
    tr, tr_info = load_traffic(name)
    achieved = alg / (sum(step_ms) / 1e3) / 1e9
    lat_alg = sum(algorithmic_bytes(s_) for s_ in lat_stats)
    lat_exp_b = sum(expansion_bytes(s_) for s_ in lat_stats)
    lat_exp_us = sum(s_["phases_us"].get("expand", 0.0) for s_ in lat_stats)
    exp_lat = lat_exp_b / (lat_exp_us * 1e-6) / 1e9 if lat_exp_us else None
    exp_bat = exp_b / (exp_us * 1e-6 / n_groups) / 1e9 if exp_us else None
    line = {
        "metric": METRIC, "value": value, "unit": "queries/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": dev_ms / args.steps, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": name, "graph": graph_desc(name, g), "k": w.k, "queries_per_step": len(allq),
                   "queries_per_rank": B, "engine_groups": args.groups, "alpha": 0.1, "lambda": 0.2,
                   "l2": "flushed between timed steps (512 MiB write)", "gen_s": round(gen_s, 1),
                   "load_s": round(load_s, 1), "node_order": "degree (internal relabel)" if RELABEL else "input",
                   "parallelism": f"query-sharded x{world} (dist.shard, replicated graph)" if world > 1 else "single GPU"},
        "p50_ms": statistics.median(lat) if lat else None,
        "p95_ms": float(np.percentile(lat, 95)) if lat else None,
        "latency_mode": {"queries": len(lat), "qps": len(lat) / (sum(lat) / 1e3) if lat else None,
                         "note": "one engine launch per query (G = 1), CUDA events per query"},
        "gteps": arcs / (dev_ms / 1e3) / 1e9 * world,
        "roofline": {"kernel": "k_engine", "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "peak_kind": peak_kind,
                     "traffic": (tr * len(allq)) if tr else None, **tr_info,
                     "algorithmic_bytes_per_launch": alg / args.steps,
                     "latency_mode_achieved": (lat_alg / (sum(lat) / 1e3) / 1e9) if lat else None,
                     # the BFS expansion phase alone (north_star's target): B_bfs / expansion time from the
                     # in-kernel %globaltimer stamps; latency mode = the whole GPU on one query's levels,
                     # batch = summed group expansion time / G (groups expand concurrently)
                     "expansion_achieved": exp_lat, "expansion_frac": (exp_lat / peak) if exp_lat else None,
                     "expansion_frac_batch_est": (exp_bat / peak) if exp_bat else None,
                     "expansion_bytes_per_query": (lat_exp_b / len(lat_stats)) if lat_stats else None,
                     # what the DRAM actually moved (the ncu capture's bytes per query x queries / the step
                     # time) against what a pure random 4-byte gather stream moves on this part (37.7 G
                     # gathers/s x 124 B of DRAM each, profiles/r02d_random_access.txt): the engine's
                     # accesses are random lines, so this, not the algorithmic bytes, is how close the
                     # launch runs to its memory system's ceiling for this access pattern
                     "dram_achieved": (tr * len(allq) / (dev_ms / args.steps / 1e3) / 1e9) if tr else None,
                     "dram_frac": (tr * len(allq) / (dev_ms / args.steps / 1e3) / 1e9 / peak) if tr else None,
                     "random_gather_dram_ceiling": RANDOM_GATHER_DRAM_GBS,
                     "random_gather_frac": (tr * len(allq) / (dev_ms / args.steps / 1e3) / 1e9 /
                                            RANDOM_GATHER_DRAM_GBS) if tr else None},
        "e2e": {"value": e2e_qps, "unit": "queries/s", "ms_per_step": statistics.median(e2e_ms),
                "h2d_bytes_per_step": h2d * world, "d2h_bytes_per_step": d2h * world / len(e2e_ms)},
        "gpu_launches": args.steps,   # one k_engine launch per step (per rank)
        "clocks": clocks,
        "stats_mean": {k: float(np.mean([s_[k] for s_ in stats])) for k in
                       ("levels", "n_centrals", "frontier_total", "arcs_scanned", "td_arcs", "overflow")},
    }
    if not args.no_cpu_baseline and world == 1:
        import oracle
        skip = set(ORACLE_SKIP.get(name, ()))
        sample = [q for q, i in zip(queries, qids) if i not in skip]
        done = 0
        with pinned_core() as pc:
            t0 = time.perf_counter()
            while time.perf_counter() - t0 < args.cpu_sample_s and done < len(sample):
                oracle.query(g, sample[done], w.k)
                done += 1
            el = time.perf_counter() - t0
        line["cpu_baseline"] = {"value": done / el, "unit": "queries/s", "cores": 1, "kind": "oracle",
                                "pinned_cpu": pc.cpu, **cpu_info(),
                                "sample": f"the first {done} {name} queries of a step ({el:.1f} s, single-threaded "
                                          f"oracle pinned to one core"
                                          + (f"; the level-5 queries {sorted(skip)} skipped: hours each for the "
                                             f"oracle)" if skip else ")")}
    print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
