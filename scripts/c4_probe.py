"""C4 (1.8B-edge FR-shaped graph in pinned host memory): generation cost, star closed form, 6-vertex queries."""
import json, os, resource, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import gcsm_inputs as gi
import oracle
from paper_conf_ipps_wei024_b200 import Gcsm

t = time.time()
w = gi.make_workload("C4", n_batches=3)
gen = time.time() - t
deg = np.diff(w.row_ptr)
print(json.dumps({"gen_s": gen, "n": w.n, "adj_gb": w.adj_bytes / 1e9, "max_deg": int(deg.max()),
                  "nonisolated": int((deg > 0).sum()), "maxrss_gb": resource.getrusage(resource.RUSAGE_SELF).ru_maxrss / 1e6}),
      flush=True)
budget = int(w.adj_bytes * 0.01)
for q in sys.argv[1:] or ["star3", "prism6", "k4tri6", "k6"]:
    if q == "star3":
        k, qe, ql = 4, np.array([(0, 1), (0, 2), (0, 3)], np.int32), None
    else:
        k, qe, ql = gi.query(q)
    t = time.time()
    g = Gcsm(w.n, w.row_ptr, w.col, device=0)
    g.set_query(k, qe, ql)
    g.set_cache_budget(budget)
    create_s = time.time() - t
    rp, col = w.row_ptr, w.col
    for b, (ins, dele) in enumerate(w.batches):
        t = time.time()
        a, r = g.apply_batch(ins, dele)
        dt = time.time() - t
        st = g.stats()
        rec = {"q": q, "batch": b, "create_s": create_s, "added": a, "removed": r, "wall_ms": dt * 1e3,
               **{x: round(st[x], 3) for x in ("ms_match", "ms_extend", "ms_estimate", "ms_pack", "ms_merge", "ms_normalize")},
               "cache_mb": st["cache_bytes"] / 2**20, "frontier": st["frontier"], "miss_gb": st["miss_bytes"] / 1e9,
               "copied_gb": st["host_copied_bytes"] / 1e9, "hit_rate": (st["hit_bytes"] + st["delta_bytes"]) /
               max(1, st["hit_bytes"] + st["delta_bytes"] + st["miss_bytes"])}
        if q == "star3":  # degree closed form at full size
            I, D, _ = oracle.normalize_batch(w.n, rp, col, ins, dele)
            U = np.unique(np.concatenate([I.ravel(), D.ravel()]))
            d = np.diff(rp)[U].astype(object)
            di = np.array([int(np.count_nonzero(I == u)) for u in U], dtype=object)
            dd = np.array([int(np.count_nonzero(D == u)) for u in U], dtype=object)
            s, d1 = d - dd, d - dd + di
            P = lambda x: x * (x - 1) * (x - 2)
            rec["closed_form_ok"] = (a, r) == (int((P(d1) - P(s)).sum()), int((P(d) - P(s)).sum()))
            rp, col = oracle.apply_batch(w.n, rp, col, I, D)
        print(json.dumps(rec), flush=True)
    g.close()
