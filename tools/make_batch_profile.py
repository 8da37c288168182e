"""profiles/<tag>_batch_ncu.md + <tag>_batch_traffic.json from one `ncu --set full` capture of a batch
launch of the engine (tools/profile_batch.py: the bench's 350 C3 queries, G = 8, one launch).
Usage: make_batch_profile.py tag details.csv raw.csv hot_lines.txt [queries] [git_sha] [workload]
The traffic json records the git sha the capture was taken at and the sha256 of the engine sources
(bench.source_hash) so that bench.py can tell whether its roofline.traffic describes the running build."""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag, f_det, f_raw, f_hot = sys.argv[1:5]
nq = int(sys.argv[5]) if len(sys.argv) > 5 else 350
git_sha = sys.argv[6] if len(sys.argv) > 6 else None
workload = sys.argv[7] if len(sys.argv) > 7 else "C3"
sys.path.insert(0, ROOT)
from bench import source_hash  # noqa: E402
rows = list(csv.reader(open(f_det)))
hdr = rows[0]
want = {"GPU Speed Of Light Throughput": None, "Memory Workload Analysis": None, "Scheduler Statistics": None,
        "Warp State Statistics": None, "Occupancy": None}
items = []
vals = {}
for r in rows[1:]:
    d = dict(zip(hdr, r))
    if "k_engine" not in d.get("Kernel Name", ""):
        continue
    sec = d.get("Section Name")
    if sec in want and d.get("Metric Name"):
        items.append((sec, d["Metric Name"], d["Metric Unit"], d["Metric Value"]))
        vals[d["Metric Name"]] = (d["Metric Value"], d["Metric Unit"])


def num(name, scale=None):
    v, u = vals[name]
    x = float(v.replace(",", ""))
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ms": 1e-3, "us": 1e-6,
            "ns": 1e-9, "Tbyte/s": 1e12, "Gbyte/s": 1e9}.get(u, 1)
    return x * mult


dur = num("Duration")
bw = num("Memory Throughput") if vals.get("Memory Throughput", ("", ""))[1].endswith("/s") else None
res = {"kernel": "k_engine", "launch": f"{nq} {workload} queries, G = 8 (bench shape), one launch",
       "workload": workload, "git_sha": git_sha, "src_sha256": source_hash(), "duration_s_under_ncu": dur}
# DRAM bytes of the launch: dram__bytes_read.sum + dram__bytes_write.sum from the raw page
raw = list(csv.reader(open(f_raw)))
rh, ru = raw[0], raw[1]
SC = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
for r in raw[2:]:
    d = dict(zip(rh, r))
    if "k_engine" not in d.get("Kernel Name", ""):
        continue
    rd = float(d["dram__bytes_read.sum"].replace(",", "")) * SC[ru[rh.index("dram__bytes_read.sum")]]
    wr = float(d["dram__bytes_write.sum"].replace(",", "")) * SC[ru[rh.index("dram__bytes_write.sum")]]
    res["dram_bytes_read"], res["dram_bytes_write"] = rd, wr
    res["dram_bytes_per_launch"] = rd + wr
    res["dram_bytes_per_query"] = (rd + wr) / nq
    res["l2_hit_pct"] = float(d["lts__t_sector_hit_rate.pct"])
# (kernel replay: the DRAM bytes of the last pass; bench.py's roofline.traffic comes from the single-pass
# capture of tools/make_traffic.py instead)
json.dump(res, open(os.path.join(ROOT, "profiles", f"{tag}_batch_fullset.json"), "w"), indent=1)
out = [f"# Batch-launch profile {tag} — k_engine, {res['launch']}", "",
       "`ncu --set full --import-source on --clock-control none` of one launch (tools/experiments/gpu_ncu_batch.sh).  "
       "Times under ncu are not bench values.  Kernel replay restores memory before each of ~40 passes; the "
       "work of the pass whose counters are shown can differ from the bench launch's (see the launch lines of "
       "profile_batch.py) — the DRAM bytes per launch behind bench.py's roofline.traffic come from a "
       "single-pass capture (tools/make_traffic.py, <tag>_batch_traffic.json).", ""]
if "dram_bytes_per_launch" in res:
    out.append(f"* DRAM traffic per launch: {res['dram_bytes_per_launch'] / 1e9:.1f} GB "
               f"({res['dram_bytes_per_query'] / 1e6:.0f} MB per query)")
out += ["", "| section | metric | unit | value |", "|---|---|---|---|"]
out += [f"| {a} | {b} | {c} | {d} |" for a, b, c, d in items]
out += ["", "## Warp-stall samples and L2 sectors per source line (tools/ncu_hot.py)", "", "```"]
out += open(f_hot).read().splitlines()[:45]
out += ["```", ""]
open(os.path.join(ROOT, "profiles", f"{tag}_batch_ncu.md"), "w").write("\n".join(out))
print("\n".join(out[:12]))
