"""Build profiles/<tag>_summary.md and profiles/<tag>_k_search_traffic.json from ncu captures.

Inputs (produced on the GPU box, see DESIGN.md §9 "Profiling"):
  <launches.csv>   ncu --metrics gpu__time_duration.sum launch list of tools/profile_run.py
  <dram.csv>       ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,
                   lts__t_sector_hit_rate.pct -k regex:k_search over the same queries
  <queries.log>    tools/profile_run.py output of the dram run (per-query stats, same order)
Usage: make_profile_summary.py tag launches.csv dram.csv queries.log [skip]
"""
import ast
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag, f_launch, f_dram, f_q = sys.argv[1:5]
skip = int(sys.argv[5]) if len(sys.argv) > 5 else 5
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "ms": 1e6, "%": 1}


def read_metrics(path):
    rows = list(csv.reader(open(path)))
    hdr, per, names = None, collections.OrderedDict(), {}
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            per.setdefault(d["ID"], {})[d["Metric Name"]] = float(d["Metric Value"].replace(",", "")) * SCALE.get(
                d["Metric Unit"], 1)
            names[d["ID"]] = d["Kernel Name"].split("(")[0].replace("kgs::", "")
    return per, names


per, names = read_metrics(f_launch)
agg = collections.defaultdict(list)
for i, m in per.items():
    if names[i] in ("k_validate", "k_snap", "k_degree_class"):
        continue
    agg[names[i]].append(m["gpu__time_duration.sum"])
tot = sum(sum(v) for v in agg.values())
lines = [f"# Profile summary {tag}", "", "Cold-cache, serialised ncu launch list of `tools/profile_run.py` on C3 "
         "(bench query order); absolute times are inflated by ncu, compare shares.", "",
         "| kernel | launches | mean us | share |", "|---|---|---|---|"]
for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
    lines.append(f"| {k} | {len(v)} | {sum(v) / len(v) / 1e3:.1f} | {sum(v) / tot * 100:.1f}% |")

dper, _ = read_metrics(f_dram)
qs = []
for line in open(f_q):
    try:
        _, _, d = line.split(" ", 2)
        qs.append(ast.literal_eval(d))
    except (ValueError, SyntaxError):
        pass
qs = qs[skip:skip + len(dper)]


def alg_bytes(s):
    return s["frontier_total"] * 23 + s["arcs_scanned"] * 6 + s["hits"] * 6


traffic = [m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"] for m in dper.values()]
times = [m["gpu__time_duration.sum"] for m in dper.values()]
hit = [m.get("lts__t_sector_hit_rate.pct", 0) for m in dper.values()]
alg = [alg_bytes(s) for s in qs]
n = min(len(traffic), len(alg))
res = {"kernel": "k_search", "launches": n, "queries": f"C3 bench order, queries {skip}..{skip + n - 1}",
       "mean_dram_bytes_per_launch": sum(traffic[:n]) / n, "mean_algorithmic_bytes_per_launch": sum(alg[:n]) / n,
       "traffic_over_algorithmic": sum(traffic[:n]) / max(1, sum(alg[:n])),
       "mean_ncu_time_us": sum(times[:n]) / n / 1e3, "mean_l2_hit_pct": sum(hit[:n]) / n}
json.dump(res, open(os.path.join(ROOT, "profiles", f"{tag}_k_search_traffic.json"), "w"), indent=1)
lines += ["", "## k_search DRAM traffic vs algorithmic bytes", "",
          f"{n} launches ({res['queries']}): mean DRAM traffic {res['mean_dram_bytes_per_launch'] / 1e6:.1f} MB per "
          f"launch vs {res['mean_algorithmic_bytes_per_launch'] / 1e6:.1f} MB algorithmic "
          f"(x{res['traffic_over_algorithmic']:.1f}); L2 hit rate {res['mean_l2_hit_pct']:.1f}%; "
          f"mean ncu time {res['mean_ncu_time_us']:.0f} us.", ""]
open(os.path.join(ROOT, "profiles", f"{tag}_summary.md"), "w").write("\n".join(lines) + "\n")
print("\n".join(lines))
