"""Per-kernel totals of an ncu launch list (--metrics gpu__time_duration.sum --csv) and the bench line's breakdown."""
import collections
import csv
import json
import sys

if len(sys.argv) > 2:
    d = json.loads(open(sys.argv[2]).read().strip().splitlines()[-1])
    print(d["value"], d["ms_per_step"], d["e2e"]["value"])
    for q, v in d["per_query"].items():
        print(q, round(v["ms_match"], 2), {k: round(x, 2) for k, x in v["breakdown_ms"].items()},
              round(v["hit_rate"], 3), v["host_copied_gb"])
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
t, n = collections.Counter(), collections.Counter()
for r in rows[1:]:
    try:
        v = float(r[vi].replace(",", ""))
    except ValueError:
        continue
    name = r[ki].split("(")[0][-40:]
    t[name] += v
    n[name] += 1
tot = sum(t.values())
for k, v in t.most_common(12):
    print(f"{k:40s} {n[k]:4d} {v / 1e6:9.3f} ms {100 * v / tot:5.1f}%")
