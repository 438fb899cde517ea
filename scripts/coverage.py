"""Fig. 15 of the paper on our workloads: (a) the share of list accesses made to the top-p% most
frequently accessed vertices, from the oracle's exact access counts C_v (R17); (b) the coverage |S ∩ T| / |S| of
the top-p% set S by the GPU's cached set T after one batch (10 % budget). The batch's updated vertices travel to
HBM with the batch (R32), so T = cached ∪ U. usage: python scripts/coverage.py [config] [queries...]"""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import gcsm_inputs as gi
import oracle
from paper_conf_ipps_wei024_b200 import Gcsm

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
w = gi.make_workload(cfg, n_batches=1)
queries = sys.argv[2:] or w.queries
ins, dele = w.batches[0]
I, D, _ = oracle.normalize_batch(w.n, w.row_ptr, w.col, ins, dele)
U = np.unique(np.concatenate([I.ravel(), D.ravel()]))
for q in queries:
    k, qe, ql = gi.query(q)
    t = time.time()
    acc = np.asarray(oracle.access_counts(w.n, w.row_ptr, w.col, w.labels, k, qe, ql, ins, dele), dtype=np.float64)
    t_or = time.time() - t
    g = Gcsm(w.n, w.row_ptr, w.col, w.labels, device=0)
    g.set_query(k, qe, ql, gi.order(q))
    g.set_cache_budget(int(w.adj_bytes * w.budget_frac))
    g.apply_batch(ins, dele)
    T = set(g.cached().tolist()) | set(U.tolist())
    g.close()
    nz = np.nonzero(acc)[0]
    order = nz[np.lexsort((nz, -acc[nz]))]  # most accessed first
    tot = acc.sum()
    rec = {"config": cfg, "query": q, "accessed_vertices": int(len(nz)), "oracle_s": round(t_or, 1), "share": {},
           "coverage": {}}
    for p in (1, 2, 3, 4, 5):
        top = order[: max(1, len(order) * p // 100)]
        rec["share"][f"top{p}%"] = round(float(acc[top].sum() / tot), 4)
        rec["coverage"][f"top{p}%"] = round(sum(1 for v in top.tolist() if v in T) / len(top), 4)
    print(json.dumps(rec), flush=True)
