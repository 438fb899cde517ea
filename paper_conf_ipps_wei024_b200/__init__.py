"""B200-native GCSM incremental-matching hot path — Python binding of libgcsm.so.

Argument marshalling only: every step of the path (normalise, estimate, pack,
match, allreduce, merge) runs inside libgcsm.so (C++ host code + sm_100a CUDA
kernels). PyTorch is used only for process groups (the ncclUniqueId broadcast)
and, optionally, to time the library's stream.

    from paper_conf_ipps_wei024_b200 import Gcsm
    g = Gcsm(n, row_ptr, col)                  # G_0 as symmetric CSR
    g.set_query(3, [(0, 1), (0, 2), (1, 2)])  # triangle
    g.set_cache_budget(64 << 20)
    added, removed = g.apply_batch(ins, dele)  # embeddings
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _lib
from ._lib import Options, Stats, STATUS

__all__ = ["Gcsm", "GcsmError", "plan_inspect", "shard", "nccl_unique_id", "measure_host_link", "CACHE_POLICIES"]

CACHE_POLICIES = {"estimator": 0, "degree": 1, "none": 2}
FLAG_LOCAL_COUNTS = 1
FLAG_NO_SYMMETRY = 2


class GcsmError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status
        self.name = STATUS.get(status, str(status))


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _i32(a, shape=None):
    if a is None:
        return None
    a = np.ascontiguousarray(np.asarray(a, dtype=np.int32))
    return a.reshape(shape) if shape is not None else a


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    s = _lib.load().gcsm_nccl_unique_id(buf)
    if s:
        raise GcsmError(s, "ncclGetUniqueId failed")
    return buf.raw


class Gcsm:
    """One GCSM context (one GPU, one process). See include/gcsm.h for the semantics."""

    def __init__(self, n, row_ptr, col, labels=None, *, device=-1, rank=0, world=1, nccl_id=None, seed=0x6C53,
                 host_threads=0, cache_policy="estimator", walks_override=0, local_counts=False, symmetry=True,
                 staging_bytes=0, vertex_capacity=0, store_rank=0, store_world=1, store_handle=None):
        """store_world > 1: a node-shared host store (gcsm.h gcsm_options.store_*): store_rank 0 creates it from
        the CSR and exposes `store_handle()`; the other local ranks pass that string as store_handle (row_ptr /
        col / labels may then be None)."""
        lib = _lib.load()
        self._lib = lib
        opt = Options()
        lib.gcsm_default_options(ctypes.byref(opt))
        opt.device, opt.rank, opt.world = device, rank, world
        self._nccl_buf = None
        if nccl_id is not None:
            self._nccl_buf = ctypes.create_string_buffer(bytes(nccl_id), 128)
            opt.nccl_id = ctypes.cast(self._nccl_buf, ctypes.c_void_p)
        opt.seed = seed & (2**64 - 1)
        opt.host_threads = host_threads
        opt.cache_policy = CACHE_POLICIES[cache_policy] if isinstance(cache_policy, str) else int(cache_policy)
        opt.walks_override = walks_override
        opt.staging_bytes = int(staging_bytes)
        opt.vertex_capacity = int(vertex_capacity)
        opt.flags = (FLAG_LOCAL_COUNTS if local_counts else 0) | (0 if symmetry else FLAG_NO_SYMMETRY)
        opt.store_rank, opt.store_world = int(store_rank), int(store_world)
        self._handle_buf = None
        if store_handle is not None:
            self._handle_buf = store_handle.encode() if isinstance(store_handle, str) else bytes(store_handle)
            opt.store_handle = self._handle_buf
        self.n = int(n)
        attach = store_handle is not None
        self._rp = None if attach else np.ascontiguousarray(row_ptr, dtype=np.int64)
        self._col = None if attach else np.ascontiguousarray(col, dtype=np.int32)
        lab = None if attach else _i32(labels)
        h = ctypes.c_void_p()
        s = lib.gcsm_create(self.n, _ptr(self._rp), _ptr(self._col), _ptr(lab), ctypes.byref(opt), ctypes.byref(h))
        self._rp = self._col = None  # copied into the library's store: the caller may free the CSR
        if s:
            raise GcsmError(s, "gcsm_create failed")
        self._h = h
        self.k = None

    # ------------------------------------------------------------------ API
    def link_store_peers(self):
        """Cross-process peer cache over the node-shared store (collective over the store's ranks; after
        set_cache_budget): misses probe the other ranks' HBM caches (over NVLink) before zero-copy."""
        self._check(self._lib.gcsm_link_store_peers(self._h), "link_store_peers")

    def store_handle(self) -> str:
        """The node-shared store's handle (store_rank 0 of a store_world > 1 context)."""
        buf = ctypes.create_string_buffer(4096)
        self._check(self._lib.gcsm_store_handle(self._h, buf, len(buf)), "store_handle")
        return buf.value.decode()

    def _check(self, s, what):
        if s:
            msg = self._lib.gcsm_last_error(self._h)
            raise GcsmError(s, f"{what}: {msg.decode() if msg else ''}")

    def set_query(self, k, qedges, qlabels=None, order=None):
        qe = _i32(qedges).reshape(-1, 2)
        self._check(self._lib.gcsm_set_query(self._h, int(k), len(qe), _ptr(qe), _ptr(_i32(qlabels)),
                                             _ptr(_i32(order))), "set_query")
        self.k = int(k)

    def add_query(self, k, qedges, qlabels=None, order=None) -> int:
        """Another standing query sharing the store, the batch steps and the cache budget; returns its id."""
        qe = _i32(qedges).reshape(-1, 2)
        qid = ctypes.c_int32()
        self._check(self._lib.gcsm_add_query(self._h, int(k), len(qe), _ptr(qe), _ptr(_i32(qlabels)),
                                             _ptr(_i32(order)), ctypes.byref(qid)), "add_query")
        return qid.value

    def num_queries(self) -> int:
        return int(self._lib.gcsm_num_queries(self._h))

    def query_stats(self, qid: int) -> dict:
        st = Stats()
        self._check(self._lib.gcsm_get_query_stats(self._h, int(qid), ctypes.byref(st)), "get_query_stats")
        return {name: getattr(st, name) for name, _ in Stats._fields_}

    def query_counts(self, qid: int):
        st = self.query_stats(qid)
        return st["added"], st["removed"]

    def set_measure(self, bcomp: bool):
        """Measurement mode (gcsm_set_measure): B_comp of the following batches in stats()['bcomp_*_bytes']."""
        self._check(self._lib.gcsm_set_measure(self._h, 1 if bcomp else 0), "set_measure")

    def set_cache_budget(self, nbytes: int):
        self._check(self._lib.gcsm_set_cache_budget(self._h, int(nbytes)), "set_cache_budget")

    def apply_batch(self, ins, dele):
        ins = _i32(ins).reshape(-1, 2)
        dele = _i32(dele).reshape(-1, 2)
        a, r = ctypes.c_uint64(), ctypes.c_uint64()
        self._check(self._lib.gcsm_apply_batch(self._h, len(ins), _ptr(ins), len(dele), _ptr(dele), ctypes.byref(a),
                                               ctypes.byref(r)), "apply_batch")
        return a.value, r.value

    def submit_batch(self, ins, dele):
        """Pipelined: host steps + enqueue + merge; the counts come from wait_batch (at most 2 outstanding)."""
        ins = _i32(ins).reshape(-1, 2)
        dele = _i32(dele).reshape(-1, 2)
        self._check(self._lib.gcsm_submit_batch(self._h, len(ins), _ptr(ins), len(dele), _ptr(dele)), "submit_batch")

    def wait_batch(self):
        a, r = ctypes.c_uint64(), ctypes.c_uint64()
        self._check(self._lib.gcsm_wait_batch(self._h, ctypes.byref(a), ctypes.byref(r)), "wait_batch")
        return a.value, r.value

    def apply_batch_list(self, ins, dele, added_cap=1 << 16, removed_cap=1 << 16):
        """Returns (added, removed, added_tuples[k], removed_tuples[k]); raises GcsmError(ETRUNC) if truncated."""
        ins = _i32(ins).reshape(-1, 2)
        dele = _i32(dele).reshape(-1, 2)
        ta = np.zeros((max(added_cap, 1), self.k), np.int32)
        tr = np.zeros((max(removed_cap, 1), self.k), np.int32)
        a, r = ctypes.c_uint64(), ctypes.c_uint64()
        s = self._lib.gcsm_apply_batch_list(self._h, len(ins), _ptr(ins), len(dele), _ptr(dele), _ptr(ta), added_cap,
                                            _ptr(tr), removed_cap, ctypes.byref(a), ctypes.byref(r))
        self._check(s, "apply_batch_list")
        return a.value, r.value, ta[:min(a.value, added_cap)], tr[:min(r.value, removed_cap)]

    def stats(self) -> dict:
        st = Stats()
        self._check(self._lib.gcsm_get_stats(self._h, ctypes.byref(st)), "get_stats")
        return {name: getattr(st, name) for name, _ in Stats._fields_}

    def automorphisms(self) -> int:
        return int(self._lib.gcsm_query_automorphisms(self._h))

    def num_vertices(self) -> int:
        return int(self._lib.gcsm_num_vertices(self._h))

    def add_vertices(self, count, labels=None) -> int:
        """count new isolated vertices; returns the first new id."""
        first = ctypes.c_int32()
        lab = None if labels is None else _i32(labels)
        self._check(self._lib.gcsm_add_vertices(self._h, int(count), _ptr(lab), ctypes.byref(first)), "add_vertices")
        return first.value

    def export_csr(self):
        rp = np.zeros(self.num_vertices() + 1, np.int64)
        self._lib.gcsm_export_csr(self._h, _ptr(rp), None, 0)
        col = np.zeros(int(rp[-1]), np.int32)
        self._check(self._lib.gcsm_export_csr(self._h, _ptr(rp), _ptr(col), len(col)), "export_csr")
        return rp, col

    def estimates(self):
        """Last batch's estimator output: (ids, levcnt[len(ids), 8])."""
        n = ctypes.c_uint64()
        self._lib.gcsm_get_estimates(self._h, None, None, 0, ctypes.byref(n))
        ids = np.zeros(n.value, np.int32)
        lev = np.zeros((n.value, 8), np.uint64)
        self._check(self._lib.gcsm_get_estimates(self._h, _ptr(ids), _ptr(lev), n.value, ctypes.byref(n)),
                    "get_estimates")
        return ids, lev

    def cached(self):
        n = ctypes.c_uint64()
        self._lib.gcsm_get_cached(self._h, None, 0, ctypes.byref(n))
        ids = np.zeros(n.value, np.int32)
        self._check(self._lib.gcsm_get_cached(self._h, _ptr(ids), n.value, ctypes.byref(n)), "get_cached")
        return ids

    def stream_ptr(self) -> int:
        p = ctypes.c_void_p()
        self._check(self._lib.gcsm_get_stream(self._h, ctypes.byref(p)), "get_stream")
        return p.value or 0

    def close(self):
        if getattr(self, "_h", None):
            self._lib.gcsm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def plan_inspect(k, qedges, order=None):
    """The library's per-term plan (pure host; no GPU needed)."""
    qe = _i32(qedges).reshape(-1, 2)
    m = len(qe)
    seed = np.zeros(2 * m, np.int32)
    order_out = np.zeros(m * k, np.int32)
    nb = np.zeros(m * k, np.int32)
    bq = np.full(m * k * 8, -1, np.int32)
    view = np.full(2 * m * k * 8, -1, np.int32)
    s = _lib.load().gcsm_plan_inspect(k, m, _ptr(qe), _ptr(_i32(order)), _ptr(seed), _ptr(order_out), _ptr(nb),
                                      _ptr(bq), _ptr(view))
    if s:
        raise GcsmError(s, "bad query")
    return dict(seed=seed.reshape(m, 2), order=order_out.reshape(m, k), nb=nb.reshape(m, k), bq=bq.reshape(m, k, 8),
                view=view.reshape(2, m, k, 8))


def query_restrictions(k, qedges, qlabels=None, order=None):
    """(pairs [(u, w): f(u) < f(w)], |Aut_L|) of the library's symmetry breaking (pure host)."""
    qe = _i32(qedges).reshape(-1, 2)
    out = np.zeros(2 * 64, np.int32)
    n = ctypes.c_int32()
    aut = ctypes.c_uint64()
    s = _lib.load().gcsm_query_restrictions(k, len(qe), _ptr(qe), _ptr(_i32(qlabels)), _ptr(_i32(order)), _ptr(out),
                                            64, ctypes.byref(n), ctypes.byref(aut))
    if s:
        raise GcsmError(s, "bad query")
    return [tuple(out[2 * i:2 * i + 2].tolist()) for i in range(n.value)], aut.value


def shard(cost, world):
    """Rank of each unit under the library's LPT sharding (pure host)."""
    c = np.ascontiguousarray(cost, dtype=np.uint64)
    out = np.zeros(len(c), np.int32)
    s = _lib.load().gcsm_shard(len(c), _ptr(c), int(world), _ptr(out))
    if s:
        raise GcsmError(s, "bad shard arguments")
    return out


def link_peers(contexts):
    """NVLink peer cache (gcsm_link_peers): the contexts read each other's HBM caches; drive each from its own
    host thread, in lockstep. An empty or one-element list unlinks."""
    arr = (ctypes.c_void_p * max(len(contexts), 1))(*[c._h.value if hasattr(c._h, "value") else c._h
                                                       for c in contexts])
    s = _lib.load().gcsm_link_peers(arr, len(contexts))
    if s:
        raise GcsmError(s, "gcsm_link_peers")


def binomial_samples(key0, n, p, count):
    """The estimator's host binomial sampler (gcsm_binomial_samples): count draws of Bin(n, p)."""
    out = np.zeros(int(count), np.int64)
    s = _lib.load().gcsm_binomial_samples(int(key0) & (2**64 - 1), int(n), float(p), int(count), _ptr(out))
    if s:
        raise GcsmError(s, "gcsm_binomial_samples")
    return out


def measure_host_link(device=-1, nbytes=1 << 30):
    """(zero-copy read GB/s, H2D DMA GB/s, HBM copy GB/s) measured by the library's micro-benchmarks."""
    z, d, h = ctypes.c_double(), ctypes.c_double(), ctypes.c_double()
    s = _lib.load().gcsm_measure_host_link(device, nbytes, ctypes.byref(z), ctypes.byref(d), ctypes.byref(h))
    if s:
        raise GcsmError(s, "gcsm_measure_host_link failed")
    return z.value, d.value, h.value


def distributed_nccl_id():
    """Rank 0 creates the ncclUniqueId; torch.distributed broadcasts it (plumbing only)."""
    import torch.distributed as dist
    obj = [nccl_unique_id() if dist.get_rank() == 0 else None]
    dist.broadcast_object_list(obj, src=0)
    return obj[0]
