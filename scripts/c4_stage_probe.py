"""C4 probe: fetch-once staging variants, B_comp (distinct-list bytes), per-query match time and host bytes.

VARIANTS (env, comma list of name=ENV:VAL+ENV:VAL@budget_frac): default s1, s16, nostage, hbm (budget 100%).
The last batch of the first variant runs in B_comp measurement mode (gcsm_set_measure)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import gcsm_inputs as gi
from paper_conf_ipps_wei024_b200 import Gcsm

cfg = os.environ.get("CFG", "C4")
nb = int(os.environ.get("NB", "4"))
t = time.time()
w = gi.make_workload(cfg, n_batches=nb)
print(json.dumps({"gen_s": round(time.time() - t, 1), "n": w.n, "adj_gb": w.adj_bytes / 1e9}), flush=True)
spec = os.environ.get("VARIANTS", "s1=GCSM_STAGE_MIN:1,s16=GCSM_STAGE_MIN:16,nostage=GCSM_STAGE_MB:0,hbm=GCSM_STAGE_MIN:1@1.0")
queries = os.environ.get("QUERIES", ",".join(w.queries)).split(",")
first = True
for item in spec.split(","):
    name, rest = item.split("=", 1)
    frac = w.budget_frac
    if "@" in rest:
        rest, f = rest.split("@")
        frac = float(f)
    env = dict(kv.split(":") for kv in rest.split("+") if kv)
    saved = {k: os.environ.get(k) for k in ("GCSM_STAGE_MIN", "GCSM_STAGE_MB", "GCSM_WALK_STAGE", "GCSM_STAGE_POLICY",
                                            "GCSM_NO_FILTER3", "GCSM_NO_HOIST")}
    for k in saved:
        os.environ.pop(k, None)
    staging = 1 if env.get("GCSM_STAGE_MB") == "0" else 0
    env.pop("GCSM_STAGE_MB", None)
    os.environ.update(env)
    t = time.time()
    g = Gcsm(w.n, w.row_ptr, w.col, device=0, staging_bytes=staging)
    for qi, q in enumerate(queries):
        k, qe, ql = gi.query(q)
        (g.set_query if qi == 0 else g.add_query)(k, qe, ql, gi.order(q))
    g.set_cache_budget(int(w.adj_bytes * frac))
    create_s = time.time() - t
    for b, (ins, dele) in enumerate(w.batches):
        meas = first and b == len(w.batches) - 1
        if meas:
            g.set_measure(True)
        t = time.time()
        g.apply_batch(ins, dele)
        wall = time.time() - t
        for qi, q in enumerate(queries):
            st = g.query_stats(qi)
            rec = {"var": name, "q": q, "batch": b, "bcomp_mode": meas, "wall_ms": round(wall * 1e3, 1),
                   "ms_walks": round(st["ms_walks"], 2), "walk_fill_gb": st["walk_fill_bytes"] / 1e9,
                   "create_s": round(create_s, 1), "added": st["added"], "removed": st["removed"],
                   "ms_match": round(st["ms_match"], 2), "ms_extend": round(st["ms_extend"], 2),
                   "ms_copy": round(st["ms_copy"], 2), "frontier": st["frontier"],
                   "miss_gb": st["miss_bytes"] / 1e9, "hit_gb": st["hit_bytes"] / 1e9,
                   "copied_gb": st["host_copied_bytes"] / 1e9, "stage_fill_gb": st["stage_fill_bytes"] / 1e9,
                   "stage_lists": st["stage_lists"], "stage_hit_gb": st["stage_hit_bytes"] / 1e9,
                   "bcomp_hit_gb": st["bcomp_hit_bytes"] / 1e9, "bcomp_miss_gb": st["bcomp_miss_bytes"] / 1e9,
                   "bcomp_delta_gb": st["bcomp_delta_bytes"] / 1e9, "cache_mb": st["cache_bytes"] / 2**20}
            print(json.dumps(rec), flush=True)
    g.close()
    first = False
    for k, v in saved.items():
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = v
