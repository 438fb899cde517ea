"""Print the headline and per-query breakdown of a bench JSON line (dev aid)."""
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value %.0f  ms/step %.2f" % (d["value"], d["ms_per_step"]))
for q, v in d.get("per_query", {}).items():
    print(q, "batch %.2f match %.2f ext %.2f l2 %.2f hit %.3f copied %.3f GB" % (v["ms_per_batch"], v["ms_match"], v["ms_extend"], v["ms_level2"], v["hit_rate"], v["host_copied_gb"]), {k: round(x, 2) for k, x in v["breakdown_ms"].items()})
