"""Aggregate ncu --page source --print-source=cuda,sass CSV by CUDA source line: warp-stall samples
(total + top stall reasons) and L2 sectors.  Usage: ncu_hot.py report.ncu-rep [kernel-regex] [top] [samples|l2sec]"""
import csv
import collections
import io
import re
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
cmd = ["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"]
if len(sys.argv) > 2 and sys.argv[2]:
    cmd += ["-k", "regex:" + sys.argv[2]]
out = subprocess.run(cmd, capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
cur_file, cur_line, cur_src = None, None, None
hdr = None
agg = collections.defaultdict(lambda: collections.Counter())
src = {}
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        cur_file = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < len(hdr):
        continue
    if r[0]:
        cur_line, cur_src = r[0], r[1]
        src[(cur_file, cur_line)] = cur_src.strip()
        continue
    key = (cur_file, cur_line)
    d = dict(zip(hdr[2:], r[2:]))
    try:
        agg[key]["samples"] += int(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
        agg[key]["l2sec"] += int(d.get("L2 Theoretical Sectors Global", "0") or 0)
        for k, v in d.items():
            if k.startswith("stall_") and "Not Issued" not in k and v not in ("", "0", "-"):
                agg[key][k] += int(v)
    except ValueError:
        pass
tot = sum(c["samples"] for c in agg.values()) or 1
tot_l2 = sum(c["l2sec"] for c in agg.values()) or 1
order = sys.argv[4] if len(sys.argv) > 4 else "samples"   # or "l2sec"
print(f"total samples {tot}, total L2 sectors {tot_l2}")
for key, c in sorted(agg.items(), key=lambda x: -x[1][order])[:top]:
    stalls = sorted(((k, v) for k, v in c.items() if k.startswith("stall_")), key=lambda x: -x[1])[:3]
    s = ", ".join(f"{k[6:]}={v}" for k, v in stalls)
    print(f"{c['samples']/tot*100:5.1f}% {key[0]}:{key[1]:>4s} l2sec={c['l2sec']:>9d} ({c['l2sec']/tot_l2*100:4.1f}%) "
          f"[{s}] {src.get(key, '')[:80]}")
