"""Matching-order probe on a scaled C4-shaped graph (planted 8-cliques, 1% budget): per-order match time, host
bytes and counts (which must agree). usage: python scripts/order_probe.py <query> <order>|id ..."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gcsm_inputs as gi
from paper_conf_ipps_wei024_b200 import Gcsm

t = time.time()
cfg = os.environ.get("CFG", "C4")
if cfg == "C4":
    w = gi.make_workload("C4", scale=int(os.environ.get("SCALE", 24)),
                         n_edges=int(os.environ.get("EDGES", 250_000_000)), n_batches=3)
else:  # full size
    w = gi.make_workload(cfg, n_batches=3)
print(json.dumps({"gen_s": time.time() - t, "adj_gb": w.adj_bytes / 1e9}), flush=True)
q = sys.argv[1]
k, qe, ql = gi.query(q)
for o in sys.argv[2:]:
    order = None if o == "id" else [int(x) for x in o.split(",")]
    g = Gcsm(w.n, w.row_ptr, w.col, w.labels, device=0)
    g.set_query(k, qe, ql, order)
    g.set_cache_budget(int(w.adj_bytes * float(os.environ.get("BUDGET", 0.01))))
    res = []
    for b, (ins, dele) in enumerate(w.batches):
        a, r = g.apply_batch(ins, dele)
        st = g.stats()
        res.append({"added": a, "removed": r, "ms_match": round(st["ms_match"], 2), "ms_copy": round(st["ms_copy"], 2),
                    "copied_gb": round(st["host_copied_bytes"] / 1e9, 3), "frontier": st["frontier"]})
    g.close()
    print(json.dumps({"q": q, "order": o, "batches": res}), flush=True)
