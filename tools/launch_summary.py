"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV): per-kernel count, total, mean, share."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = None
agg = collections.defaultdict(list)
skip = set(sys.argv[2].split(",")) if len(sys.argv) > 2 else set()
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d["Metric Name"] == "gpu__time_duration.sum":
            k = d["Kernel Name"].split("(")[0].replace("kgs::", "")
            if k not in skip:
                agg[k].append(float(d["Metric Value"].replace(",", "")))
tot = sum(sum(v) for v in agg.values())
print(f"{'kernel':28s} {'launches':>8s} {'total ms':>10s} {'mean us':>10s} {'share':>7s}")
for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
    print(f"{k:28s} {len(v):8d} {sum(v)/1e6:10.3f} {sum(v)/len(v)/1e3:10.1f} {sum(v)/tot*100:6.1f}%")
