"""Quick per-step breakdown on C2 (dev probe, not the bench)."""
import sys, time, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import gcsm_inputs as gi
from paper_conf_ipps_wei024_b200 import Gcsm
t = time.time()
w = gi.make_workload("C2")
print("gen", time.time() - t, "n", w.n, "adj", w.adj_bytes, flush=True)
for q in sys.argv[1:] or ["k4", "c4"]:
    k, qe, ql = gi.query(q)
    for frac in (0.1, 0.0, 1.0):
        g = Gcsm(w.n, w.row_ptr, w.col, device=0)
        g.set_query(k, qe, ql)
        g.set_cache_budget(int(w.adj_bytes * frac))
        for b in range(4):
            t = time.time()
            a, r = g.apply_batch(*w.batches[b])
            wall = time.time() - t
            st = g.stats()
            keep = {x: (round(v, 2) if isinstance(v, float) else v) for x, v in st.items()}
            print(q, frac, b, "wall %.1f ms" % (wall * 1e3), json.dumps(keep), flush=True)
        g.close()
