"""Build profiles/<tag>_summary.md and profiles/<tag>_engine_traffic.json from ncu captures of the
query engine (one k_engine launch per query in tools/profile_run.py).

Inputs (produced on the GPU box):
  <dram.csv>      ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,
                  lts__t_sector_hit_rate.pct,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed
                  -k regex:k_engine over `profile_run.py --warm W --queries N`
  <queries.log>   the profile_run.py output of that run (per-query stats, same order)
Usage: make_profile_summary.py tag dram.csv queries.log [skip queries] [skip launches]
"""
import ast
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag, f_dram, f_q = sys.argv[1:4]
skip = int(sys.argv[4]) if len(sys.argv) > 4 else 3
lskip = int(sys.argv[5]) if len(sys.argv) > 5 else skip   # launches already skipped by ncu -s: 0
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "ms": 1e6, "%": 1}


def read_metrics(path):
    rows = list(csv.reader(open(path)))
    hdr, per = None, collections.OrderedDict()
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if "k_engine" not in d["Kernel Name"]:
                continue
            per.setdefault(int(d["ID"]), {})[d["Metric Name"]] = float(d["Metric Value"].replace(",", "")) * SCALE.get(
                d["Metric Unit"], 1)
    return collections.OrderedDict(sorted(per.items()))   # by launch id (numeric)


def alg_bytes(s):   # bench.py algorithmic_bytes
    return (s["frontier_total"] * 23 + s["arcs_scanned"] * 6 + s["hits"] * 6 + s.get("td_arcs", 0) * 6 +
            s.get("td_pred_arcs", 0) * 12)


per = read_metrics(f_dram)
qs = []
for line in open(f_q):
    try:
        _, _, d = line.split(" ", 2)
        qs.append(ast.literal_eval(d))
    except (ValueError, SyntaxError):
        pass
launches = list(per.values())[lskip:]
qs = qs[skip:skip + len(launches)]
n = min(len(launches), len(qs))
traffic = [m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"] for m in launches[:n]]
times = [m["gpu__time_duration.sum"] for m in launches[:n]]
alg = [alg_bytes(s) for s in qs[:n]]
hit = [m.get("lts__t_sector_hit_rate.pct", 0) for m in launches[:n]]
dpct = [m.get("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", 0) for m in launches[:n]]
res = {"kernel": "k_engine", "launches": n, "queries": f"C3 bench order, queries {skip}..{skip + n - 1}, one per launch",
       "mean_dram_bytes_per_query": sum(traffic) / n, "mean_algorithmic_bytes_per_query": sum(alg) / n,
       "traffic_over_algorithmic": sum(traffic) / max(1, sum(alg)), "mean_ncu_time_us": sum(times) / n / 1e3,
       "mean_l2_hit_pct": sum(hit) / n, "mean_dram_throughput_pct": sum(dpct) / n}
json.dump(res, open(os.path.join(ROOT, "profiles", f"{tag}_engine_traffic.json"), "w"), indent=1)
lines = [f"# Profile summary {tag} — k_engine (the whole query path in one kernel)", "",
         f"{n} launches of `tools/profile_run.py` ({res['queries']}), ncu `--clock-control none` "
         "(cold cache, serialised: compare shares and ratios, not absolute times).", "",
         f"* mean DRAM traffic per query: {res['mean_dram_bytes_per_query'] / 1e6:.1f} MB",
         f"* mean algorithmic bytes per query: {res['mean_algorithmic_bytes_per_query'] / 1e6:.1f} MB "
         f"(traffic / algorithmic = {res['traffic_over_algorithmic']:.1f})",
         f"* mean L2 hit rate {res['mean_l2_hit_pct']:.1f}%, mean DRAM throughput {res['mean_dram_throughput_pct']:.1f}% "
         f"of peak, mean ncu time {res['mean_ncu_time_us']:.0f} us", "",
         "| query | q | levels | centrals | out-arcs | in-arcs (pre-pass) | alg. MB | DRAM MB | ncu us |",
         "|---|---|---|---|---|---|---|---|---|"]
for i in range(n):
    s = qs[i]
    lines.append(f"| {skip + i} | - | {s['levels']} | {s['n_centrals']} | {s['arcs_scanned']} | {s.get('td_arcs', 0)} | "
                 f"{alg[i] / 1e6:.1f} | {traffic[i] / 1e6:.1f} | {times[i] / 1e3:.0f} |")
open(os.path.join(ROOT, "profiles", f"{tag}_summary.md"), "w").write("\n".join(lines) + "\n")
print("\n".join(lines[:10]))
