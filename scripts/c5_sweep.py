"""C5 (BASELINE configs[4]) on one B200: batch-size sweep 1K..64K updated edges on the C4 graph (FR-shaped, 1.8 B
edges, planted 8-cliques, 14.4 GB pinned host graph), cache budget 1 %, prism6 + K4+2tri6 in one context.
The stream is the P:331 protocol with max(12 x 8192, 3 x 64K) edges; consecutive 1K batches are concatenated into
the larger batches (a batch of B is B consecutive stream updates). One context processes, in stream order, a 1K
warm-up batch and then one batch of each size. Prints one JSON line per batch size."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import gcsm_inputs as gi
from paper_conf_ipps_wei024_b200 import Gcsm

t = time.time()
w = gi.make_workload("C4", batch=1024, n_stream=3 * 65536)
print(json.dumps({"gen_s": round(time.time() - t, 1), "adj_gb": w.adj_bytes / 1e9, "small_batches": len(w.batches)}),
      flush=True)
queries = sys.argv[1:] or ["prism6", "k4tri6"]
g = Gcsm(w.n, w.row_ptr, w.col, w.labels, device=0)
for i, q in enumerate(queries):
    k, qe, ql = gi.query(q)
    (g.set_query if i == 0 else g.add_query)(k, qe, ql, gi.order(q))
g.set_cache_budget(int(w.adj_bytes * 0.01))
pos = 0


def take(nsmall):
    global pos
    part = w.batches[pos:pos + nsmall]
    pos += nsmall
    return (np.concatenate([p[0] for p in part]).astype(np.int32), np.concatenate([p[1] for p in part]).astype(np.int32))


g.apply_batch(*take(1))  # warm-up
for B in [1, 2, 4, 8, 16, 32, 64]:
    ins, dele = take(B)
    t = time.time()
    g.apply_batch(ins, dele)
    dt = time.time() - t
    rec = {"batch": len(ins) + len(dele), "wall_ms": round(dt * 1e3, 1),
           "updated_edges_per_s": round((len(ins) + len(dele)) / dt, 1)}
    for qi, q in enumerate(queries):
        st = g.query_stats(qi)
        rec[q] = {"added": st["added"], "removed": st["removed"], "ms_match": round(st["ms_match"], 1),
                  "ms_cache_step": round(st["ms_copy"], 1), "host_gb": round(st["host_copied_bytes"] / 1e9, 2)}
    print(json.dumps(rec), flush=True)
g.close()
