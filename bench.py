#!/usr/bin/env python
"""bench.py — updated edges/sec of the GCSM hot path on B200 (default: BASELINE.json configs[3], C4).

Contract (driver): `python bench.py --gpus N --steps K --warmup W [--impl reference]`, one process per GPU under
torchrun for N > 1 (started by this script itself when run as `python bench.py --gpus N` without torchrun), one
JSON line printed by rank 0.

Workload: BASELINE.json's metric names no config, so the N = 1 headline is the largest single-GPU config, C4
(FR-shaped 67M-vertex / 1.8B-edge R-MAT, 14.4 GB of adjacency in pinned host memory, 6-vertex queries prism6 +
K4+2tri6 + K6, cache budget 1% of the adjacency, 4096 mixed updates per GPU per step). `--config C2|C3|C1` selects
the others.

A step = one batch of updated edges pushed through the whole hot path (normalise, overlay,
unit enumeration, random-walk estimation, cache packing + DMA, the matching kernels, the count allreduce, the host
merge) for every standing query of the config, in ONE context per GPU (shared store, batch steps and cache budget).
Weak scaling: each GPU gets a 4096-edge share of the step's global batch (global batch = 4096 N); units are
LPT-sharded inside the library and one ncclAllReduce sums the counts.

value = updated edges (normalised |I| + |D| of the global batches) / max-over-ranks device time of the K timed steps
        (CUDA events on the library's stream, barrier + synchronize on both sides);
e2e   = the same through the public Python API with host (numpy) buffers, host wall clock, max over ranks.
Inputs are larger than L2 (the graph lives in pinned host memory, the cache is refilled each batch).
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

METRIC = "updated edges/sec per batch (C4: FR-shaped 67M-vertex / 1.8B-edge R-MAT in pinned host memory, " \
         "6-vertex patterns, budget 1%)"
METRICS = {"C1": "updated edges/sec per batch (C1: 1K-vertex / 8K-edge R-MAT, triangle)",
           "C2": "updated edges/sec per batch (C2: LJ-shaped 4.19M-vertex / 70M-edge R-MAT, 4-clique + 4-cycle)",
           "C3": "updated edges/sec per batch (C3: Orkut-shaped 3M-vertex / 120M-edge R-MAT, 8 labels, 5-vertex "
                 "labelled patterns)",
           "PA": "updated edges/sec per batch (PA: RoadNetPA-shaped 1.09M-vertex lattice, all 29 connected 3-5-vertex "
                 "motifs as standing queries)",
           "C4": "updated edges/sec per batch (C4: FR-shaped 67M-vertex / 1.8B-edge R-MAT in pinned host memory, "
                 "6-vertex patterns, budget 1%)"}
UNIT = "updated_edges/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C4")
    ap.add_argument("--queries", default=None, help="comma list (default: the config's queries)")
    ap.add_argument("--batch", type=int, default=4096, help="updated edges per GPU per step")
    ap.add_argument("--budget-frac", type=float, default=None, help="cache budget as a fraction of adjacency bytes")
    ap.add_argument("--cache-policy", default="estimator")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=20.0)
    ap.add_argument("--ref-step-seconds", type=float, default=8.0,
                    help="reference arm: the oracle's per-step sample is sized (during the warm-up) to about this")
    ap.add_argument("--parity-edges", type=int, default=64,
                    help="updated edges of batch 0 applied first through the library and checked against the oracle "
                         "(N = 1, rank 0; 0 = off)")
    ap.add_argument("--quick", action="store_true", help="profiling mode: no clocks sampler / cpu baseline")
    ap.add_argument("--emulate", action="store_true",
                    help="test the N>1 plumbing on one GPU: gloo process group, every rank on cuda:0, shard-local "
                         "counts (no NCCL communicator)")
    ap.add_argument("--private-store", action="store_true",
                    help="N > 1: every rank builds its own pinned store (default: ONE node-shared store, rank 0 "
                         "builds it, the others attach; SURVEY 8e)")
    ap.add_argument("--no-peer-cache", action="store_true",
                    help="N > 1 with the shared store: do not link the ranks' HBM caches (gcsm_link_store_peers)")
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


def load_traffic(config, query):
    """dram bytes (read + write) per launch of the dominant kernel from the committed ncu capture (profiles/)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        e = d.get(f"{config}:{query}", d.get(query) if config == "C2" else None)
        if isinstance(e, dict):
            return e.get("dram_bytes")
        return e
    return None


def workload(args, world, extra_steps=1):
    import gcsm_inputs as gi
    steps = args.warmup + args.steps + extra_steps
    gb = args.batch * world
    return gi.make_workload(args.config, batch=gb, n_stream=max(12 * 8192, steps * gb))


def workload_name(w):
    if w.meta.get("grid"):
        W, H, pk, pd = w.meta["grid"]
        return (f"{w.name} (RoadNetPA-shaped, Fig. 11 motif counting, SURVEY 8f NEXT-4): {W}x{H} lattice kept with "
                f"p={pk} plus cell diagonals p={pd}, {w.meta['n_edges'] / 1e6:.2f}M edges")
    return (f"{w.name} (BASELINE configs[{int(w.name[1:]) - 1}]): R-MAT s={w.meta['scale']}, "
            f"{w.meta['n_edges'] / 1e6:.0f}M edges"
            + (f" ({w.meta['planted'][0]} planted {w.meta['planted'][1]}-cliques)" if w.meta['planted'][0] else "")
            + (f", {w.meta['L']} labels" if w.meta['L'] else ""))


def mem_status():
    """This process's memory (GB): private anonymous resident, shared-memory resident, peak resident."""
    out = {}
    try:
        with open("/proc/self/status") as f:
            for line in f:
                k, _, v = line.partition(":")
                if k in ("RssAnon", "RssShmem", "VmHWM"):
                    out[{"RssAnon": "rss_anon_gb", "RssShmem": "rss_shmem_gb", "VmHWM": "peak_rss_gb"}[k]] = \
                        int(v.split()[0]) / 2**20
    except OSError:
        pass
    return out


def sample_of(ins, dele, s):
    """The first s updated edges of a batch, split between insertions and deletions in the batch's proportion."""
    total = len(ins) + len(dele)
    s = min(s, total)
    si = (s * len(ins) + total // 2) // max(total, 1)
    return np.ascontiguousarray(ins[:si]), np.ascontiguousarray(dele[:s - si])


def host_info():
    info = {"cores": os.cpu_count()}
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    info["cpu_model"] = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    try:
        nodes = sorted(d for d in os.listdir("/sys/devices/system/node") if d.startswith("node"))
        lay = {}
        for nd in nodes:
            with open(f"/sys/devices/system/node/{nd}/cpulist") as f:
                lay[nd] = f.read().strip()
        info["numa"] = lay
    except OSError:
        pass
    return info


# ------------------------------------------------------------------ the oracle arm (reference) and cpu_baseline

def oracle_step(w, queries, ins, dele, threads=None):
    """The oracle as it stands on one (sub-)batch: normalise, G_{t+1} once, then O3 per query (oracle.delta's
    definition, with its graph update shared by the queries). Returns {query: (added, removed)}."""
    import oracle
    import gcsm_inputs as gi
    I, D, _ = oracle.normalize_batch(w.n, w.row_ptr, w.col, ins, dele)
    rp1, col1 = oracle.apply_batch(w.n, w.row_ptr, w.col, I, D)
    out = {}
    for q in queries:
        k, qe, ql = gi.query(q)
        out[q] = (oracle.o3(w.n, rp1, col1, w.labels, k, qe, ql, I, threads),
                  oracle.o3(w.n, w.row_ptr, w.col, w.labels, k, qe, ql, D, threads))
    return out


def cpu_baseline(w, queries, seconds, ins, dele):
    """The oracle as it stands, timed on the host cores on a bounded sample of the workload: the first s updated
    edges of batch 0 (s doubled from 8 until one run takes >= seconds/4, at most `seconds` in all); plus a
    single-thread C1 run. Returns (record, the oracle's counts of the last sample, the sample)."""
    total = len(ins) + len(dele)
    s = 8
    best = None
    t_all = time.perf_counter()
    while True:
        si, sd = sample_of(ins, dele, s)
        t = time.perf_counter()
        counts = oracle_step(w, queries, si, sd)
        dt = time.perf_counter() - t
        best = (len(si) + len(sd), dt, counts, (si, sd))
        if dt >= seconds / 4 or s >= total or time.perf_counter() - t_all + 2 * dt > seconds:
            break
        s = min(total, s * 2)
    edges, dt, counts, smp = best
    rec = {"value": edges / dt, "unit": UNIT, **host_info(), "kind": "oracle",
           "threads": os.cpu_count(),
           "sample": f"first {edges} updated edges of batch 0 of {w.name} (oracle: normalise, G_t+1, O3 per query) for "
                     f"queries {','.join(queries)}: {dt:.2f} s on {os.cpu_count()} threads"}
    try:  # single-thread C1 (triangle, 256 insertions)
        import gcsm_inputs as gi
        c1 = gi.make_workload("C1")
        i1, d1 = c1.batches[0]
        t = time.perf_counter()
        oracle_step(c1, ["triangle"], i1, d1, threads=1)
        dt1 = time.perf_counter() - t
        rec["single_thread_c1"] = {"value": (len(i1) + len(d1)) / dt1, "unit": UNIT, "seconds": dt1}
    except Exception as e:  # noqa: BLE001
        rec["single_thread_c1"] = {"error": str(e)}
    return rec, counts, smp


def run_reference(args):
    """--impl reference: the oracle (there is no reference implementation; the reference is a paper), as it stands,
    on the host cores, on this arm's config and metric; each step a bounded sample of the step's batch, sized
    during the warm-up so that one step takes about --ref-step-seconds."""
    world, rank = int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    t0 = time.perf_counter()
    w = workload(args, 1, extra_steps=0)
    gen_s = time.perf_counter() - t0
    queries = args.queries.split(",") if args.queries else w.queries
    s = 8
    times, edges = [], 0
    for step in range(args.warmup + args.steps):
        b_ins, b_del = w.batches[step % len(w.batches)]
        si, sd = sample_of(b_ins, b_del, s)
        t = time.perf_counter()
        oracle_step(w, queries, si, sd)
        dt = time.perf_counter() - t
        if step >= args.warmup:
            times.append(dt)
            edges += len(si) + len(sd)
        elif dt < args.ref_step_seconds / 2 and s < len(b_ins) + len(b_del):
            s *= 2  # warm-up: grow the sample toward the step-time target
    T = sum(times)
    v = edges / T
    line = {"impl": "reference", "metric": METRICS.get(w.name, METRIC), "value": v, "unit": UNIT,
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * T / max(len(times), 1),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic (seeded R-MAT graph + P:331 update stream, generated on the box)",
            "config": {"workload": workload_name(w), "queries": queries,
                       "global_batch": s, "graph_vertices": w.n, "graph_edges": int(w.row_ptr[-1] // 2),
                       "parallelism": "host threads"},
            "cpu_baseline": {"value": v, "unit": UNIT, **host_info(), "kind": "oracle",
                             "sample": f"the first {s} updated edges of each step's batch (of {args.batch}); per "
                                       f"step: normalise, G_t+1, O3 per query on all cores"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "gen_seconds": gen_s}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ our arm

def spawn(args):
    """`python bench.py --gpus N` without torchrun: start N ranks (one per GPU) with torch.distributed.run."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn(args))
    if args.impl == "reference":
        run_reference(args)
        return
    world, rank, local = dist_setup(args)
    import torch
    import gcsm_inputs as gi
    import paper_conf_ipps_wei024_b200 as G

    # the host cores are shared by the ranks of one node
    per_rank = max(1, (os.cpu_count() or 1) // world)
    shared_store = world > 1 and not args.private_store
    # (with a shared store only rank 0 generates the graph, on every core)
    os.environ.setdefault("GCSM_GEN_THREADS", str(os.cpu_count() if shared_store else per_rank))
    steps = args.warmup + args.steps
    t0 = time.perf_counter()
    w = workload(args, world) if (rank == 0 or not shared_store) else None
    gen_s = time.perf_counter() - t0
    nccl_id = G.distributed_nccl_id() if world > 1 and not args.emulate else None
    # one context per GPU holding every standing query of the config: the store, each batch's normalisation,
    # overlays and merge, and ONE cache under the per-GPU budget are shared (gcsm_add_query)
    common = dict(device=local, rank=rank, world=world, nccl_id=nccl_id, cache_policy=args.cache_policy,
                  local_counts=bool(args.emulate and world > 1), host_threads=per_rank if world > 1 else 0)
    t0 = time.perf_counter()
    if not shared_store:
        g = G.Gcsm(w.n, w.row_ptr, w.col, w.labels, **common)
    else:
        # node-shared host store: rank 0 generates the graph and builds ONE pinned store; the other
        # ranks attach to it by handle and receive only the batches (no graph generation, no replica)
        import torch.distributed as dist
        if rank == 0:
            g = G.Gcsm(w.n, w.row_ptr, w.col, w.labels, store_rank=0, store_world=world, **common)
            meta = [dict(handle=g.store_handle(), n=w.n, name=w.name, meta=w.meta, queries=w.queries,
                         budget_frac=w.budget_frac, adj_bytes=w.adj_bytes, edges=int(w.row_ptr[-1]),
                         batches=[(np.asarray(a, np.int32), np.asarray(b, np.int32))
                                  for a, b in w.batches[:steps + 1]])]
            w.col = None  # the graph lives in the shared store now (parity / cpu_baseline run at N = 1 only)
        else:
            meta = [None]
        dist.broadcast_object_list(meta, src=0)
        m = meta[0]
        if rank > 0:
            import types
            w = types.SimpleNamespace(n=m["n"], name=m["name"], meta=m["meta"], queries=m["queries"],
                                      budget_frac=m["budget_frac"], adj_bytes=m["adj_bytes"],
                                      row_ptr=np.array([0, m["edges"]], np.int64), batches=m["batches"])
            g = G.Gcsm(w.n, None, None, store_rank=rank, store_world=world, store_handle=m["handle"], **common)
        barrier(world)
    create_s = time.perf_counter() - t0
    queries = args.queries.split(",") if args.queries else w.queries
    frac = w.budget_frac if args.budget_frac is None else args.budget_frac
    budget = int(w.adj_bytes * frac)
    for i, q in enumerate(queries):
        k, qe, ql = gi.query(q)
        if i == 0:
            g.set_query(k, qe, ql, gi.order(q))
        else:
            g.add_query(k, qe, ql, gi.order(q))
    g.set_cache_budget(budget)
    peer_linked = shared_store and not args.no_peer_cache and budget > 0
    if peer_linked:  # NEXT-3 across processes: misses probe the other GPUs' caches over NVLink before PCIe
        g.link_store_peers()
    assert len(w.batches) >= steps + 1, "stream too short"
    batches = [(np.ascontiguousarray(a, dtype=np.int32), np.ascontiguousarray(b, dtype=np.int32))
               for a, b in w.batches[:steps + 1]]

    # parity probe (before the warm-up, untimed): the first P updated edges of batch 0 as a batch of their own
    # through the library; the oracle checks the same sample on G_0 after the timed region (N = 1). Batch 0 then
    # runs as warm-up step 0 with those edges dropped as no-ops (R8), so the timed steps are unaffected.
    probe = None
    do_parity = args.parity_edges > 0 and world == 1 and not args.quick
    if do_parity:
        pi, pd = sample_of(*batches[0], args.parity_edges)
        g.apply_batch(pi, pd)
        probe = (pi, pd, {q: g.query_counts(i) for i, q in enumerate(queries)})

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

    # B_comp (untimed, one more batch in measurement mode): bytes of the distinct lists each query's kernels touch
    bcomp = None
    if not args.quick:
        g.set_measure(True)
        g.apply_batch(*batches[steps])
        g.set_measure(False)
        bcomp = {q: g.query_stats(i) for i, q in enumerate(queries)}

    # per query aggregates over the timed steps
    per_q = {}
    edges = 0
    keys = ("ms_total", "ms_match", "ms_level2", "ms_extend", "ms_normalize", "ms_estimate", "ms_pack", "ms_copy",
            "ms_allreduce", "ms_merge", "hit_bytes", "miss_bytes", "delta_bytes", "hit_bytes_ext", "miss_bytes_ext",
            "delta_bytes_ext", "host_copied_bytes", "cache_bytes", "cached_vertices", "units", "frontier",
            "h2d_bytes", "d2h_bytes", "kernel_launches", "stage_fill_bytes", "stage_lists", "stage_hit_bytes",
            "ms_walks", "walk_alg_bytes", "walk_fill_bytes", "peer_bytes")
    for step in recs:
        edges += step[0][3]["n_ins"] + step[0][3]["n_del"]
        for q, a, r, st in step:
            d = per_q.setdefault(q, {"added": 0, "removed": 0, **{x: 0 for x in keys}})
            d["added"] += a
            d["removed"] += r
            for key in keys:
                d[key] += st[key]
    K = args.steps
    shared = {x: per_q[queries[0]][x] for x in ("h2d_bytes", "d2h_bytes", "kernel_launches", "cache_bytes",
                                                 "cached_vertices")}
    value = edges / (ms_dev / 1e3)
    e2e_value = edges / (ms_host / 1e3)
    # dominant kernel (CUDA-event times): the matching extension (k_last4 / k_extend) of a query, or a query's GPU
    # random walks (k_walks_l1 + k_walks, step 2)
    cands = []
    for q, d in per_q.items():
        cands.append((d["ms_extend"], q, "ext"))
        cands.append((d["ms_walks"], q, "walks"))
    _, dom_q, dom_kind = max(cands)
    dq = per_q[dom_q]
    if dom_kind == "walks":
        kern = "k_walks"
        hit, miss, dlt = dq["walk_alg_bytes"], 0, 0  # walks' list bytes (arena / cache / U lists: HBM-resident)
        kms = dq["ms_walks"] / K
    else:
        kern = "k_last4" if gi.query(dom_q)[0] == 4 else "k_extend"  # k = 4: the lean last-level kernel (§5)
        hit, miss, dlt = dq["hit_bytes_ext"], dq["miss_bytes_ext"], dq["delta_bytes_ext"]
        kms = dq["ms_extend"] / K
    # per link: algorithmic list bytes served from HBM (the cache, the batch's device-resident delta
    # data and lists of U, and lists staged in the batch arena) vs the HBM peak; bytes that really crossed the host
    # link (bulk copies of zero-copy lists: the arena fills and the warps' staging) vs the measured zero-copy peak
    stage_hit = dq["stage_hit_bytes"] if dom_kind == "ext" else 0
    b_hbm = (hit + dlt + stage_hit) / K
    b_alg = (hit + dlt + miss) / K
    b_host = (dq["host_copied_bytes"] if dom_kind == "ext" else dq["walk_fill_bytes"]) / K
    peak, peak_kind = load_peaks()
    sec = kms / 1e3 if kms > 0 else float("inf")
    link = None
    if rank == 0 and not args.quick:
        try:
            zc, dma, hbm = G.measure_host_link(local, 1 << 30)
            link = {"zero_copy_gbs": zc, "dma_h2d_gbs": dma, "hbm_copy_gbs": hbm}
        except Exception as e:  # noqa: BLE001
            link = {"error": str(e)}
    zc_peak = (link or {}).get("zero_copy_gbs")
    hbm_ach = b_hbm / sec / 1e9
    host_ach = b_host / sec / 1e9
    hbm_obj = {"achieved": hbm_ach, "peak": peak, "unit": "GB/s", "frac": hbm_ach / peak,
               "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_kind})", "bytes_per_launch": b_hbm,
               "bytes_note": "algorithmic list bytes (4 B x list length per read, SURVEY 8d B_alg) served from HBM: "
                             "cache hits + device-resident delta / U lists + lists staged once in the batch arena"}
    link_obj = {"achieved": host_ach, "peak": zc_peak, "unit": "GB/s",
                "frac": host_ach / zc_peak if zc_peak else None, "bytes_per_launch": b_host,
                "peak_source": "gcsm_measure_host_link zero-copy streaming read, measured in this run",
                "bytes_note": "bytes the kernel bulk-copied from pinned host memory (arena fills + warp staging)"}
    hf, lf = hbm_obj["frac"], link_obj["frac"] or 0.0
    bound = "host_link" if lf >= hf else "hbm"
    top = link_obj if bound == "host_link" else hbm_obj
    bq = (bcomp or {}).get(dom_q)
    roofline = {"bound": bound, "kernel": f"{kern} ({dom_q})", "achieved": top["achieved"], "peak": top["peak"],
                "unit": "GB/s", "frac": top["frac"],
                "traffic": load_traffic(w.name, dom_q + (":walks" if dom_kind == "walks" else "")),
                "launch_ms": kms, "algorithmic_bytes_per_launch": b_alg,
                "hbm": hbm_obj, "host_link": link_obj,
                "b_comp": None if bq is None else {
                    "hit_bytes": bq["bcomp_hit_bytes"], "miss_bytes": bq["bcomp_miss_bytes"],
                    "delta_bytes": bq["bcomp_delta_bytes"],
                    "host_bytes_same_batch": bq["host_copied_bytes"],
                    "host_over_bcomp_miss": bq["host_copied_bytes"] / bq["bcomp_miss_bytes"]
                    if bq["bcomp_miss_bytes"] else None,
                    "note": "bytes of the DISTINCT main lists the query's kernels touched (SURVEY 8d lower bound), by "
                            "home, measured on one extra untimed batch (gcsm_set_measure)"}}
    # per-rank host work and memory (shared store: overlays / merges split by vertex owner, one graph per node)
    q0 = per_q[queries[0]]
    me = {"rank": rank, "ms_host_per_batch": sum(q0[x] for x in ("ms_normalize", "ms_estimate", "ms_pack",
                                                                   "ms_merge")) / K,
          "ms_normalize": q0["ms_normalize"] / K, "ms_merge": q0["ms_merge"] / K, **mem_status()}
    ranks_host = [me]
    if world > 1:
        import torch.distributed as dist
        ranks_host = [None] * world
        dist.all_gather_object(ranks_host, me)
    tot_hit = sum(d["hit_bytes"] + d["delta_bytes"] for d in per_q.values())
    tot_all = sum(d["hit_bytes"] + d["delta_bytes"] + d["miss_bytes"] for d in per_q.values())
    if rank != 0:
        g.close()
        return
    cpu = parity = None
    if not args.no_cpu_baseline and not args.quick and world == 1:
        cpu, counts, smp = cpu_baseline(w, queries, args.cpu_seconds, *batches[0])
        if probe is not None:
            want = counts if len(smp[0]) + len(smp[1]) == len(probe[0]) + len(probe[1]) and \
                np.array_equal(smp[0], probe[0]) and np.array_equal(smp[1], probe[1]) else \
                oracle_step(w, queries, probe[0], probe[1])
            parity = {"sample_edges": len(probe[0]) + len(probe[1]), "batch": 0,
                      "library": {q: list(probe[2][q]) for q in queries},
                      "oracle": {q: [int(x) for x in want[q]] for q in queries},
                      "ok": all(tuple(probe[2][q]) == tuple(want[q]) for q in queries)}
    h2d = shared["h2d_bytes"] / K + sum(8 * len(b[0]) + 8 * len(b[1]) for b in batches[args.warmup:steps]) / K
    d2h = shared["d2h_bytes"] / K
    line = {
        "metric": METRICS.get(w.name, METRIC), "value": value, "unit": UNIT, "n_gpus": world, "steps": K,
        "warmup": args.warmup, "ms_per_step": ms_dev / K, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "int32",
        "data": "synthetic (seeded R-MAT graph + P:331 update stream, generated on the box)",
        "config": {"workload": workload_name(w),
                   "detail": f"queries {'+'.join(queries)}, {args.batch} mixed updates per GPU per step, "
                             f"cache budget {frac:.0%} of adjacency", "queries": queries,
                   "global_batch": args.batch * world,
                   "graph_vertices": w.n, "graph_edges": int(w.row_ptr[-1] // 2), "budget_bytes": budget,
                   "cache_policy": args.cache_policy,
                   "cache_mb": shared["cache_bytes"] / K / 2**20,
                   "parallelism": f"units LPT-sharded over {world} GPU(s); one context per GPU with all queries "
                                  f"(shared store, batch steps and cache budget), "
                                  f"{'synchronous' if args.serial else 'pipelined submit/wait'} batches",
                   "l2": f"inputs larger than L2 ({w.adj_bytes / 1e6:.0f} MB pinned host graph; cache refilled "
                         f"every batch)"},
        "roofline": roofline,
        "cpu_baseline": cpu,
        "parity": parity,
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
                          "stage_fill_gb": d["stage_fill_bytes"] / K / 1e9,
                          "stage_hit_gb": d["stage_hit_bytes"] / K / 1e9,
                          "ms_walks": d["ms_walks"] / K, "walk_alg_gb": d["walk_alg_bytes"] / K / 1e9,
                          "peer_gb": d["peer_bytes"] / K / 1e9,
                          "bcomp_miss_gb": None if bcomp is None else bcomp[q]["bcomp_miss_bytes"] / 1e9,
                          "bcomp_hit_gb": None if bcomp is None else bcomp[q]["bcomp_hit_bytes"] / 1e9,
                          "frontier": d["frontier"] / K} for q, d in per_q.items()},
        "gen_seconds": gen_s, "create_seconds": create_s,
        "peer_cache": "linked (CUDA IPC, gcsm_link_store_peers)" if peer_linked else None,
        "host_store": "node-shared (one pinned store, rank 0 builds, ranks attach)" if shared_store else
                      ("private per rank" if world > 1 else "private"),
        "ranks_host": ranks_host,
    }
    print(json.dumps(line), flush=True)
    g.close()


if __name__ == "__main__":
    main()
