"""One C4 context (prism6 + k4tri6 + k6, budget 1%), NB batches: the target of an ncu capture of prism6's
k_extend (batch 1 = the 4th k_extend launch: --launch-skip 3 --launch-count 1)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gcsm_inputs as gi
from paper_conf_ipps_wei024_b200 import Gcsm

nb = int(os.environ.get("NB", "2"))
w = gi.make_workload(os.environ.get("CFG", "C4"), n_batches=nb)
queries = os.environ.get("QUERIES", ",".join(w.queries)).split(",")
g = Gcsm(w.n, w.row_ptr, w.col, device=0)
for qi, q in enumerate(queries):
    k, qe, ql = gi.query(q)
    (g.set_query if qi == 0 else g.add_query)(k, qe, ql, gi.order(q))
g.set_cache_budget(int(w.adj_bytes * w.budget_frac))
for ins, dele in w.batches:
    t = time.time()
    g.apply_batch(ins, dele)
    print("batch", round(time.time() - t, 3), [g.query_counts(i) for i in range(len(queries))],
          round(g.query_stats(0)["ms_extend"], 1), flush=True)
g.close()
