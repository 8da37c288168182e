"""Pretty-print tools/profile_run.py output: one line per query with the per-phase times (us)."""
import ast
import sys

for line in open(sys.argv[1]):
    try:
        i, q, d = line.split(" ", 2)
        d = ast.literal_eval(d)
    except (ValueError, SyntaxError):
        continue
    ph = {k: round(v) for k, v in d["phases_us"].items()}
    print(i, "q=" + q, "C", d["n_centrals"], "lv", d["levels"], "arcs", d["arcs_scanned"], "dag", d.get("dag_arcs"), "td", d["td_arcs"],
          "search %.3f td %.3f" % (d["ms_search"], d["ms_topdown"]), ph)
