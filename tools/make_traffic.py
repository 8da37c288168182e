"""profiles/<tag>_batch_traffic.json (bench.py roofline.traffic) from a SINGLE-PASS ncu capture of one
batch launch: `ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,
lts__t_sector_hit_rate.pct --clock-control none -k regex:k_engine -s 1 -c 1 python tools/profile_batch.py ...`.
A `--set full` capture replays the kernel ~40 times from saved memory, and its last pass did only part of
the launch's work (r02w: 884 M of 1327 M arcs), so its DRAM bytes do not describe the bench's launch; four
metrics fit one pass, no replay.  profile_batch.py prints the work of the uncaptured launch 0 and the
captured launch 1 (same queries): both are recorded, and they must agree.
Usage: make_traffic.py tag metrics.csv profile_batch.log queries git_sha [workload]"""
import csv
import json
import os
import re
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag, f_csv, f_log, nq, sha = sys.argv[1:6]
workload = sys.argv[6] if len(sys.argv) > 6 else "C3"
nq = int(nq)
sys.path.insert(0, ROOT)
from bench import source_hash  # noqa: E402
lines = [ln for ln in open(f_csv) if ln.startswith('"')]
rows = list(csv.DictReader(lines))
SC = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-9, "us": 1e-6, "ms": 1e-3,
      "usecond": 1e-6, "msecond": 1e-3, "nsecond": 1e-9, "%": 1}
m = {}
for r in rows:
    if "k_engine" in r["Kernel Name"]:
        m[r["Metric Name"]] = float(r["Metric Value"].replace(",", "")) * SC.get(r["Metric Unit"], 1)
arcs = {}
for ln in open(f_log):
    g = re.match(r"launch (\d+): .* arcs (\d+),", ln)
    if g:
        arcs[int(g.group(1))] = int(g.group(2))
rd, wr = m["dram__bytes_read.sum"], m["dram__bytes_write.sum"]
res = {"kernel": "k_engine", "launch": f"{nq} {workload} queries, G = 8 (bench shape), one launch",
       "capture": "single pass (--metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,"
                  "lts__t_sector_hit_rate.pct), no kernel replay",
       "workload": workload, "git_sha": sha, "src_sha256": source_hash(), "captured_unix": int(time.time()),
       "duration_s_under_ncu": m.get("gpu__time_duration.sum"),
       "arcs_captured_launch": arcs.get(1), "arcs_uncaptured_launch": arcs.get(0),
       "same_work": arcs.get(0) is not None and arcs.get(0) == arcs.get(1),
       "dram_bytes_read": rd, "dram_bytes_write": wr, "dram_bytes_per_launch": rd + wr,
       "dram_bytes_per_query": (rd + wr) / nq, "l2_hit_pct": m.get("lts__t_sector_hit_rate.pct")}
json.dump(res, open(os.path.join(ROOT, "profiles", f"{tag}_batch_traffic.json"), "w"), indent=1)
print(json.dumps(res, indent=1))
