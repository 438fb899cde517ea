#!/usr/bin/env python
"""bench.py — updated edges/sec of the GCSM hot path on BASELINE.json configs[1] (C2), B200.

Contract (driver): `python bench.py --gpus N --steps K --warmup W [--impl reference]`, one process per GPU under
torchrun for N > 1, one JSON line printed by rank 0.

A step = one batch of updated edges pushed through the whole hot path (normalise, overlay,
unit enumeration, random-walk estimation, cache packing + DMA, the matching kernels, the count allreduce, the host
merge) for every query of the config (C2: 4-clique and 4-cycle), each query with its own context (its own host
store and HBM cache). Weak scaling: each of the N GPUs gets a 4096-edge share of the step's global batch
(global batch = 4096 N); units are LPT-sharded inside the library and one ncclAllReduce sums the counts.

value = updated edges (normalised |I| + |D| of the global batches) / max-over-ranks device time of the K timed steps
        (CUDA events on the library's stream, barrier + synchronize on both sides);
e2e   = the same through the public Python API with host (numpy) buffers, host wall clock, max over ranks.
Inputs are larger than L2 (the 560 MB graph lives in pinned host memory, the cache is repacked each batch).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "updated edges/sec per batch (C2: LJ-shaped 4.19M-vertex / 70M-edge R-MAT, 4-clique + 4-cycle)"
METRICS = {"C1": "updated edges/sec per batch (C1: 1K-vertex / 8K-edge R-MAT, triangle)", "C2": METRIC,
           "C3": "updated edges/sec per batch (C3: Orkut-shaped 3M-vertex / 120M-edge R-MAT, 8 labels, 5-vertex "
                 "labelled patterns)",
           "C4": "updated edges/sec per batch (C4: FR-shaped 67M-vertex / 1.8B-edge R-MAT in pinned host memory, "
                 "6-vertex patterns, budget 1%)"}
UNIT = "updated_edges/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=16)
    ap.add_argument("--warmup", type=int, default=4)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C2")
    ap.add_argument("--queries", default=None, help="comma list (default: the config's queries)")
    ap.add_argument("--batch", type=int, default=4096, help="updated edges per GPU per step")
    ap.add_argument("--budget-frac", type=float, default=None, help="cache budget as a fraction of adjacency bytes")
    ap.add_argument("--cache-policy", default="estimator")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=20.0)
    ap.add_argument("--quick", action="store_true", help="profiling mode: no clocks sampler / cpu baseline")
    ap.add_argument("--emulate", action="store_true",
                    help="test the N>1 plumbing on one GPU: gloo process group, every rank on cuda:0, shard-local "
                         "counts (no NCCL communicator)")
    ap.add_argument("--serial", action="store_true",
                    help="synchronous apply_batch per step (default: pipelined submit/wait, so batch t+1's host "
                         "steps overlap batch t's kernels)")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks sampler (nvidia-smi during the timed region)

class Clocks:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append((time.perf_counter(), [x.strip() for x in line.split(",")]))

    def mark(self, t0, t1):
        """the timed region: samples taken inside it (or the nearest one) are reported"""
        self.t0, self.t1 = t0, t1

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        t0, t1 = getattr(self, "t0", 0.0), getattr(self, "t1", float("inf"))
        rows = [r for t, r in self.rows if t0 <= t <= t1 + 0.05]
        if not rows and self.rows:  # region shorter than the sampling period: the sample closest to it
            rows = [min(self.rows, key=lambda tr: abs(tr[0] - 0.5 * (t0 + t1)))[1]]
        self.rows = rows
        sm = [float(r[1]) for r in self.rows if len(r) >= 9 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) >= 9 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows if len(r) >= 9 for i in range(4) if "Active" in r[5 + i]
                          and "Not" not in r[5 + i]})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


# ------------------------------------------------------------------ helpers

def dist_setup(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    import torch
    if world > 1 and args.emulate:
        import torch.distributed as dist
        torch.cuda.set_device(0)
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("gloo")
        local = 0
    elif world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    elif torch.cuda.is_available():
        torch.cuda.set_device(local)
    return world, rank, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def allmax(world, x):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], device="cuda" if dist.get_backend() == "nccl" else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


def load_traffic(query):
    """dram bytes per launch of the dominant kernel from the committed ncu capture (profiles/), if any."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get(query)
    return None


def workload(args, world):
    import gcsm_inputs as gi
    steps = args.warmup + args.steps
    gb = args.batch * world
    w = gi.make_workload(args.config, batch=gb, n_stream=max(12 * 8192, steps * gb))
    return w


# ------------------------------------------------------------------ the oracle arm (reference) and cpu_baseline

def cpu_baseline(w, queries, seconds):
    """Time the oracle as it stands on a bounded sample of the workload: the first s updated edges of the first
    batch (s doubled until the run takes >= seconds/4), on all host cores."""
    import oracle
    import gcsm_inputs as gi
    ins, dele = w.batches[0]
    total = len(ins) + len(dele)
    s = 32
    best = None
    t_all = time.perf_counter()
    while True:
        si, sd = ins[: s * len(ins) // total], dele[: s * len(dele) // total]
        t = time.perf_counter()
        for q in queries:
            k, qe, ql = gi.query(q)
            oracle.delta(w.n, w.row_ptr, w.col, w.labels, k, qe, ql, si, sd)
        dt = time.perf_counter() - t
        best = (len(si) + len(sd), dt)
        if dt >= seconds / 4 or s >= total or time.perf_counter() - t_all > seconds:
            break
        s = min(total, s * 2)
    edges, dt = best
    return {"value": edges / dt, "unit": UNIT, "cores": os.cpu_count(), "kind": "oracle",
            "sample": f"first {edges} updated edges of batch 0 of {w.name} (oracle.delta O3 incl. its graph update) "
                      f"for queries {','.join(queries)}: {dt:.2f} s"}


def run_reference(args):
    world, rank, local = int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")), 0
    if rank != 0:
        return
    import gcsm_inputs as gi
    w = workload(argparse.Namespace(**{**vars(args), "batch": args.batch}), 1)
    queries = args.queries.split(",") if args.queries else w.queries
    import oracle
    ins, dele = w.batches[0]
    # each step: a bounded sample (256 updated edges) of the step's batch through the oracle
    per = 256
    times, edges = [], 0
    for step in range(args.warmup + args.steps):
        b_ins, b_del = w.batches[step % len(w.batches)]
        si, sd = b_ins[: per // 2], b_del[: per // 2]
        t = time.perf_counter()
        for q in queries:
            k, qe, ql = gi.query(q)
            oracle.delta(w.n, w.row_ptr, w.col, w.labels, k, qe, ql, si, sd)
        dt = time.perf_counter() - t
        if step >= args.warmup:
            times.append(dt)
            edges += len(si) + len(sd)
    T = sum(times)
    v = edges / T
    line = {"impl": "reference", "metric": METRICS.get(w.name, METRIC), "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * T / max(len(times), 1),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic", "config": {"workload": f"{w.name} (BASELINE configs[1])", "queries": queries,
                                             "global_batch": per, "graph_vertices": w.n,
                                             "graph_edges": int(w.row_ptr[-1] // 2), "parallelism": "host threads"},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": os.cpu_count(), "kind": "oracle",
                             "sample": f"{per} updated edges of each step's batch, oracle.delta (O3) on all cores"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ our arm

def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    world, rank, local = dist_setup(args)
    import torch
    import gcsm_inputs as gi
    import paper_conf_ipps_wei024_b200 as G

    # the host cores are shared by the ranks of one node
    per_rank = max(1, (os.cpu_count() or 1) // world)
    os.environ.setdefault("GCSM_GEN_THREADS", str(per_rank))
    t0 = time.perf_counter()
    w = workload(args, world)
    gen_s = time.perf_counter() - t0
    queries = args.queries.split(",") if args.queries else w.queries
    frac = w.budget_frac if args.budget_frac is None else args.budget_frac
    budget = int(w.adj_bytes * frac)
    nccl_id = G.distributed_nccl_id() if world > 1 and not args.emulate else None
    # one context per GPU holding every standing query of the config: the store, each batch's normalisation,
    # overlays and merge, and ONE cache under the per-GPU budget are shared (gcsm_add_query)
    g = G.Gcsm(w.n, w.row_ptr, w.col, w.labels, device=local, rank=rank, world=world, nccl_id=nccl_id,
               cache_policy=args.cache_policy, local_counts=bool(args.emulate and world > 1),
               host_threads=per_rank if world > 1 else 0)
    for i, q in enumerate(queries):
        k, qe, ql = gi.query(q)
        if i == 0:
            g.set_query(k, qe, ql, gi.order(q))
        else:
            g.add_query(k, qe, ql, gi.order(q))
    g.set_cache_budget(budget)
    steps = args.warmup + args.steps
    assert len(w.batches) >= steps, "stream too short"
    batches = [(np.ascontiguousarray(a, dtype=np.int32), np.ascontiguousarray(b, dtype=np.int32))
               for a, b in w.batches[:steps]]

    def collect():
        return [(q, *g.query_counts(i), g.query_stats(i)) for i, q in enumerate(queries)]

    def do_step(i):
        g.apply_batch(*batches[i])
        return collect()

    def timed_steps(lo, hi):
        """per-step records [[(q, added, removed, stats) per query] per batch]"""
        if args.serial:
            return [do_step(i) for i in range(lo, hi)]
        # pipelined: batch i+1's host steps overlap batch i's kernels (gcsm_submit_batch / gcsm_wait_batch)
        recs = []
        g.submit_batch(*batches[lo])
        for i in range(lo + 1, hi):
            g.submit_batch(*batches[i])
            g.wait_batch()
            recs.append(collect())
        g.wait_batch()
        recs.append(collect())
        return recs

    # the clocks sampler (nvidia-smi) starts before the warm-up: its start-up must not land in the timed region
    clocks = Clocks(local)
    if not args.quick and rank == 0:
        clocks.start()
        time.sleep(1.0)
    for i in range(args.warmup):
        do_step(i)

    streams = [torch.cuda.ExternalStream(g.stream_ptr())]
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier(world)
    torch.cuda.synchronize()
    ev0.record(streams[0])
    th0 = time.perf_counter()
    recs = timed_steps(args.warmup, steps)
    th1 = time.perf_counter()
    ev1.record(streams[-1])
    torch.cuda.synchronize()
    barrier(world)
    ms_dev = allmax(world, ev0.elapsed_time(ev1))
    ms_host = allmax(world, 1e3 * (th1 - th0))
    if not args.quick and rank == 0:
        clocks.mark(th0, th1)
    clk = clocks.stop() if (not args.quick and rank == 0) else None

    # per query aggregates over the timed steps
    per_q = {}
    edges = 0
    for step in recs:
        edges += step[0][3]["n_ins"] + step[0][3]["n_del"]
        for q, a, r, st in step:
            d = per_q.setdefault(q, {"added": 0, "removed": 0, "ms_total": 0.0, "ms_match": 0.0, "ms_level2": 0.0,
                                     "ms_extend": 0.0, "ms_normalize": 0.0, "ms_estimate": 0.0, "ms_pack": 0.0,
                                     "ms_copy": 0.0, "ms_allreduce": 0.0, "ms_merge": 0.0, "hit_bytes": 0,
                                     "miss_bytes": 0, "delta_bytes": 0, "hit_bytes_ext": 0, "miss_bytes_ext": 0,
                                     "delta_bytes_ext": 0, "host_copied_bytes": 0, "cache_bytes": 0, "cached_vertices": 0, "units": 0,
                                     "frontier": 0, "h2d_bytes": 0, "d2h_bytes": 0, "kernel_launches": 0})
            d["added"] += a
            d["removed"] += r
            for key in d:
                if key not in ("added", "removed"):
                    d[key] += st[key]
    K = args.steps
    shared = {x: per_q[queries[0]][x] for x in ("h2d_bytes", "d2h_bytes", "kernel_launches", "cache_bytes",
                                                 "cached_vertices")}
    value = edges / (ms_dev / 1e3)
    e2e_value = edges / (ms_host / 1e3)
    # dominant kernel: the last-level kernel (k_last4 / k_extend) of the heaviest query; algorithmic bytes = every
    # list byte it reads (cache + delta + zero-copy)
    dom_q = max(per_q, key=lambda q: per_q[q]["ms_extend"] + per_q[q]["ms_level2"])
    dq = per_q[dom_q]
    kern = "k_extend" if dq["ms_extend"] > 0 else "k_level2"
    if kern == "k_extend":
        if gi.query(dom_q)[0] == 4:
            kern = "k_last4"  # k = 4 count mode: the last level runs in the lean kernel
        alg = (dq["hit_bytes_ext"] + dq["delta_bytes_ext"] + dq["miss_bytes_ext"]) / K
        kms = dq["ms_extend"] / K
    else:
        alg = (dq["hit_bytes"] + dq["delta_bytes"] + dq["miss_bytes"]) / K
        kms = dq["ms_level2"] / K
    alg_host = dq["host_copied_bytes"] / K  # real zero-copy bytes: lists bulk-copied from host memory
    alg_hbm = alg
    peak, peak_kind = load_peaks()
    achieved = alg_hbm / (kms / 1e3) / 1e9 if kms > 0 else 0.0
    link = None
    if rank == 0 and not args.quick:
        try:
            zc, dma, hbm = G.measure_host_link(local, 1 << 30)
            link = {"zero_copy_gbs": zc, "dma_h2d_gbs": dma, "hbm_copy_gbs": hbm}
        except Exception as e:  # noqa: BLE001
            link = {"error": str(e)}
    host_ach = alg_host / (kms / 1e3) / 1e9 if kms > 0 else 0.0
    roofline = {"bound": "hbm", "kernel": f"{kern} ({dom_q})", "achieved": achieved, "peak": peak,
                "unit": "GB/s", "frac": achieved / peak, "traffic": load_traffic(dom_q),
                "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_kind})",
                "algorithmic_bytes_per_launch": alg_hbm, "launch_ms": kms,
                "bytes_note": "algorithmic = 4 B x list length for every list an intersection reads (SURVEY 8d "
                              "B_alg), cached + zero-copy + delta lists; every byte is served to the SMs from HBM/L2/"
                              "smem (zero-copy lists via their staged copies)",
                "host_link": {"achieved": host_ach, "bytes_per_launch": alg_host,
                              "bytes_note": "bytes actually bulk-copied from pinned host memory by the kernel",
                              "peak": (link or {}).get("zero_copy_gbs"), "unit": "GB/s",
                              "frac": host_ach / link["zero_copy_gbs"] if link and link.get("zero_copy_gbs") else None}}
    tot_hit = sum(d["hit_bytes"] + d["delta_bytes"] for d in per_q.values())
    tot_all = sum(d["hit_bytes"] + d["delta_bytes"] + d["miss_bytes"] for d in per_q.values())
    if rank != 0:
        return
    cpu = None
    if not args.no_cpu_baseline and not args.quick and world == 1:
        cpu = cpu_baseline(w, queries, args.cpu_seconds)
    h2d = shared["h2d_bytes"] / K + sum(8 * len(b[0]) + 8 * len(b[1]) for b in batches[args.warmup:]) / K
    d2h = shared["d2h_bytes"] / K
    line = {
        "metric": METRICS.get(w.name, METRIC), "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": args.warmup,
        "ms_per_step": ms_dev / K, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "int32", "data": "synthetic (seeded R-MAT graph + P:331 update stream, generated on the box)",
        "config": {"workload": f"{w.name} (BASELINE configs[{int(w.name[1:]) - 1}]): R-MAT s={w.meta['scale']}, "
                               f"{w.meta['n_edges'] / 1e6:.0f}M edges"
                               + (f" ({w.meta['planted'][0]} planted {w.meta['planted'][1]}-cliques)"
                                  if w.meta['planted'][0] else "")
                               + (f", {w.meta['L']} labels" if w.meta['L'] else "")
                               + f", queries {'+'.join(queries)}, {args.batch} mixed updates per GPU per step, "
                                 f"cache budget {frac:.0%} of adjacency", "queries": queries,
                   "global_batch": args.batch * world,
                   "graph_vertices": w.n, "graph_edges": int(w.row_ptr[-1] // 2), "budget_bytes": budget,
                   "cache_policy": args.cache_policy,
                   "cache_mb": shared["cache_bytes"] / K / 2**20,
                   "parallelism": f"units LPT-sharded over {world} GPU(s); one context per GPU with all queries "
                                  f"(shared store, batch steps and cache budget), "
                                  f"{'synchronous' if args.serial else 'pipelined submit/wait'} batches",
                   "l2": f"inputs larger than L2 ({w.adj_bytes / 1e6:.0f} MB pinned host graph; cache repacked "
                         f"every batch)"},
        "roofline": roofline,
        "cpu_baseline": cpu,
        "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h)},
        "gpu_launches": int(shared["kernel_launches"]),
        "clocks": clk,
        "cache_hit_rate": tot_hit / tot_all if tot_all else None,
        "host_link": link,
        "per_query": {q: {"added": d["added"], "removed": d["removed"],
                          "ms_per_batch": d["ms_total"] / K, "ms_match": d["ms_match"] / K,
                          "ms_level2": d["ms_level2"] / K, "ms_extend": d["ms_extend"] / K,
                          "breakdown_ms": {x: d[x] / K for x in ("ms_normalize", "ms_estimate", "ms_pack", "ms_copy",
                                                                 "ms_match", "ms_allreduce", "ms_merge")},
                          "hit_rate": (d["hit_bytes"] + d["delta_bytes"]) /
                          max(1, d["hit_bytes"] + d["delta_bytes"] + d["miss_bytes"]),
                          "cache_mb": d["cache_bytes"] / K / 2**20, "units": d["units"] / K,
                          "miss_gb": d["miss_bytes"] / K / 1e9, "host_copied_gb": d["host_copied_bytes"] / K / 1e9,
                          "frontier": d["frontier"] / K} for q, d in per_q.items()},
        "gen_seconds": gen_s,
    }
    print(json.dumps(line), flush=True)
    g.close()


if __name__ == "__main__":
    main()
