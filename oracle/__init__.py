"""GCSM oracle — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package. It
shares no code with ``paper_conf_ipps_wei024_b200`` (the product) and never
imports it; the product never imports this.

A plain, slow, obviously-correct CPU implementation of what the GCSM hot path
computes, each function citing the PAPER.md passage it follows (``P:<line>``)
and the DESIGN.md reading (``R<n>``) it takes where the paper is silent.

Functions (pins in tests/test_oracle_*.py):
  normalize_batch  a0  R8 set semantics                       (pinned: brute force, hand cases)
  apply_batch      a7  G_{t+1} = (E \\ D) ∪ I                 (pinned: numpy set algebra + invariants)
  delta            a5  added/removed by definition (O3)        (pinned: O1 brute force, networkx, closed forms, Fig. 1)
  static_count     O2  |Emb(Q, G)|                             (pinned: K_n / stars / K_ab closed forms)
  ivm_count        a5  eq. (1) terms with stable split (R7)    (pinned: equals delta on fuzz cases)
  access_counts    a3  exact C_v of the execution trees        (pinned: brute-force tree walk in Python)
  estimate         a3  M plain random walks of §IV-A, eq. (3) (pinned: eq. (6) unbiasedness vs the exact C_v,
                                                                 eq. (7) variance bound, ">= |ΔE|" property,
                                                                 a one-unit closed form of the walk distribution)
  select_cache     a4  top-K prefix under a byte budget (R23)  (pinned: brute-force prefix search)
"""
from __future__ import annotations

import ctypes
import itertools
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(HERE, "oracle.c")
    if not force and os.path.exists(LIB_PATH) and os.path.getmtime(LIB_PATH) >= os.path.getmtime(src):
        return LIB_PATH
    subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-fPIC", "-shared", "-pthread", src, "-o",
                           LIB_PATH + ".tmp", "-lm"])
    os.replace(LIB_PATH + ".tmp", LIB_PATH)
    return LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(LIB_PATH)
        P, I32, I64, U64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64
        lib.o3_delta.restype = ctypes.c_int
        lib.o3_delta.argtypes = [I32, P, P, P, I32, I32, P, P, I64, P, I32, P, P, I64, P]
        lib.o2_static.restype = ctypes.c_int
        lib.o2_static.argtypes = [I32, P, P, P, I32, I32, P, P, I32, P]
        lib.ivm_plan.restype = ctypes.c_int
        lib.ivm_plan.argtypes = [I32, I32, P, P, P, P, P, P, P]
        lib.ivm_units.restype = I64
        lib.ivm_units.argtypes = [I32, I32, P, P, P, P, I64, P, I64, P, P, I64]
        lib.ivm_run.restype = ctypes.c_int
        lib.ivm_run.argtypes = [I32, I32, P, P, P, P, P, P, P, I32, I32, P, P, P, I64, P, I32, U64, I64, I64,
                                P, P, P]
        lib.o_apply.restype = ctypes.c_int
        lib.o_apply.argtypes = [I32, P, P, I64, P, I64, P, P, P]
        _lib = lib
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _i32(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.int32)


def _threads(threads):
    return threads if threads else (os.cpu_count() or 1)


# ------------------------------------------------------------------ graphs

def edges_of(rp, col) -> np.ndarray:
    """Canonical (u<v) edge list of a symmetric CSR, sorted by (u, v)."""
    n = len(rp) - 1
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(rp))
    dst = col.astype(np.int64)
    keep = src < dst
    return np.stack([src[keep], dst[keep]], axis=1).astype(np.int32)


def csr(n, uv):
    """Symmetric CSR with sorted rows from a canonical edge list (plain numpy)."""
    uv = np.asarray(uv, dtype=np.int64).reshape(-1, 2)
    src = np.concatenate([uv[:, 0], uv[:, 1]])
    dst = np.concatenate([uv[:, 1], uv[:, 0]])
    order = np.lexsort((dst, src))
    src, dst = src[order], dst[order]
    rp = np.concatenate([[0], np.cumsum(np.bincount(src, minlength=n))]).astype(np.int64)
    return rp, dst.astype(np.int32)


def _keys(uv):
    uv = np.asarray(uv, dtype=np.int64).reshape(-1, 2)
    return (np.minimum(uv[:, 0], uv[:, 1]) << 32) | np.maximum(uv[:, 0], uv[:, 1])


def _unkey(keys):
    keys = np.asarray(keys, dtype=np.int64)
    return np.stack([keys >> 32, keys & 0xFFFFFFFF], axis=1).astype(np.int32)


def has_edges(rp, col, uv):
    """Membership of each pair (u, v) in the graph (binary search of row u)."""
    uv = np.asarray(uv, dtype=np.int64).reshape(-1, 2)
    out = np.zeros(len(uv), dtype=bool)
    for i, (u, v) in enumerate(uv.tolist()):
        row = col[rp[u]:rp[u + 1]]
        j = np.searchsorted(row, v)
        out[i] = j < len(row) and row[j] == v
    return out


def normalize_batch(n, rp, col, ins, dele):
    """a0, reading R8: set semantics E' = (E \\ D) ∪ I.

    Raises ValueError (the library's EINVAL) on a self loop, an id outside
    [0, n), or an edge both inserted and deleted. Duplicates collapse; an
    insertion of an existing edge and a deletion of an absent edge are dropped
    (no-ops). Returns (I, D, n_dropped) as canonical sorted int32 [*,2] arrays.
    """
    ins = np.asarray(ins, dtype=np.int64).reshape(-1, 2)
    dele = np.asarray(dele, dtype=np.int64).reshape(-1, 2)
    for a in (ins, dele):
        if len(a) and (a.min() < 0 or a.max() >= n):
            raise ValueError("vertex id out of range")
        if len(a) and np.any(a[:, 0] == a[:, 1]):
            raise ValueError("self loop")
    ki, kd = np.unique(_keys(ins)), np.unique(_keys(dele))
    if len(np.intersect1d(ki, kd)):
        raise ValueError("edge both inserted and deleted")
    ei, ed = has_edges(rp, col, _unkey(ki)), has_edges(rp, col, _unkey(kd))
    ki_new, kd_real = ki[~ei], kd[ed]
    dropped = (len(ki) - len(ki_new)) + (len(kd) - len(kd_real))
    return _unkey(ki_new), _unkey(kd_real), int(dropped)


def apply_batch(n, rp, col, I, D):
    """a7: CSR of G_{t+1} = (E \\ D) ∪ I for a normalised batch (row-by-row, oracle.c)."""
    I = _i32(np.asarray(I).reshape(-1, 2))
    D = _i32(np.asarray(D).reshape(-1, 2))
    rp2 = np.zeros(n + 1, np.int64)
    col2 = np.zeros(int(rp[-1]) + 2 * len(I) - 2 * len(D), np.int32)
    _load().o_apply(n, _p(np.ascontiguousarray(rp, dtype=np.int64)), _p(np.ascontiguousarray(col, dtype=np.int32)),
                    len(I), _p(I), len(D), _p(D), _p(rp2), _p(col2))
    return rp2, col2


def apply_batch_setalgebra(n, rp, col, I, D):
    """The same as apply_batch by plain numpy set algebra on edge keys (small graphs; pins apply_batch)."""
    e = _keys(edges_of(rp, col))
    e = np.union1d(np.setdiff1d(e, _keys(D)), _keys(I))
    return csr(n, _unkey(e))


def stable_graph(n, rp, col, D):
    """CSR of the stable edge set S = E ∩ E' = E \\ D (§8 notation)."""
    return apply_batch(n, rp, col, np.zeros((0, 2), np.int32), D)


# ------------------------------------------------------------------ counts

def _u128(lo, hi):
    return int(lo) | (int(hi) << 64)


def o3(n, rp, col, labels, k, qe, ql, chg, threads=None, listing=False, tuple_cap=0):
    lib = _load()
    qe = _i32(qe)
    ql = _i32(ql)
    labels = _i32(labels)
    chg = _i32(np.asarray(chg).reshape(-1, 2))
    out = np.zeros(2, dtype=np.uint64)
    ntup = np.zeros(1, dtype=np.int64)
    tuples = None
    if listing:
        tuples = np.zeros((max(tuple_cap, 1), k), dtype=np.int32)
    r = lib.o3_delta(n, _p(rp), _p(col), _p(labels), k, len(qe), _p(qe), _p(ql), len(chg), _p(chg),
                     1 if listing else _threads(threads), _p(out), _p(tuples), tuple_cap, _p(ntup))
    if r:
        raise ValueError("bad query")
    cnt = _u128(out[0], out[1])
    if listing:
        return cnt, tuples[:min(int(ntup[0]), tuple_cap)]
    return cnt


def delta(n, rp, col, labels, k, qe, ql, ins, dele, threads=None, listing=False, tuple_cap=0):
    """(added, removed) embeddings for one batch (definition).

    added   = |Emb(Q, G_{t+1}) \\ Emb(Q, G_t)|: embeddings in G_{t+1} using >= 1 inserted edge;
    removed = |Emb(Q, G_t) \\ Emb(Q, G_{t+1})|: embeddings in G_t using >= 1 deleted edge.
    With listing=True returns ((added, tuples), (removed, tuples)).
    """
    I, D, _ = normalize_batch(n, rp, col, ins, dele)
    rp2, col2 = apply_batch(n, rp, col, I, D)
    a = o3(n, rp2, col2, labels, k, qe, ql, I, threads, listing, tuple_cap)
    r = o3(n, rp, col, labels, k, qe, ql, D, threads, listing, tuple_cap)
    return a, r


def static_count(n, rp, col, labels, k, qe, ql, threads=None):
    """|Emb(Q, G)| by plain backtracking."""
    qe, ql, labels = _i32(qe), _i32(ql), _i32(labels)
    out = np.zeros(2, dtype=np.uint64)
    if _load().o2_static(n, _p(rp), _p(col), _p(labels), k, len(qe), _p(qe), _p(ql), _threads(threads), _p(out)):
        raise ValueError("bad query")
    return _u128(out[0], out[1])


# ------------------------------------------------------------------ IVM algorithm

def plan(k, qe, user_order=None):
    """Per-term order / backward positions / views (readings R7, R11, R12; Fig. 2)."""
    qe = _i32(qe)
    m = len(qe)
    uo = _i32(user_order)
    order = np.zeros(m * k, np.int32)
    nb = np.zeros(m * k, np.int32)
    bq = np.full(m * k * 8, -1, np.int32)
    view = np.full(2 * m * k * 8, -1, np.int32)
    seed = np.zeros(2 * m, np.int32)
    if _load().ivm_plan(k, m, _p(qe), _p(uo), _p(order), _p(nb), _p(bq), _p(view), _p(seed)):
        raise ValueError("bad query")
    return dict(order=order.reshape(m, k), nb=nb.reshape(m, k), bq=bq.reshape(m, k, 8),
                view=view.reshape(2, m, k, 8), seed=seed.reshape(m, 2))


def units(k, qe, ql, labels, I, D, user_order=None):
    """Level-1 units (term, kind, a, b): every term, every changed edge, both orientations, label-filtered."""
    qe, ql, labels = _i32(qe), _i32(ql), _i32(labels)
    I, D = _i32(np.asarray(I).reshape(-1, 2)), _i32(np.asarray(D).reshape(-1, 2))
    uo = _i32(user_order)
    lib = _load()
    cap = 2 * len(qe) * (len(I) + len(D))
    out = np.zeros((max(cap, 1), 4), np.int32)
    nu = lib.ivm_units(k, len(qe), _p(qe), _p(ql), _p(uo), _p(labels), len(I), _p(I), len(D), _p(D), _p(out), cap)
    return out[:nu]


class _Views:
    def __init__(self, n, rp, col, I, D):
        self.n = n
        self.old = (rp, col)
        self.new = apply_batch(n, rp, col, I, D)
        self.stable = stable_graph(n, rp, col, D)

    def max_degree(self):
        """D (reading R19): max list length over G_t ∪ G_{t+1}."""
        return int(max(np.diff(self.old[0]).max(initial=0), np.diff(self.new[0]).max(initial=0), 1))


def _ivm(mode, n, rp, col, labels, k, qe, ql, ins, dele, user_order=None, unit_filter=None, threads=None,
         seed=0, M=None, D=None):
    I, Dl, _ = normalize_batch(n, rp, col, ins, dele)
    V = _Views(n, rp, col, I, Dl)
    U = units(k, qe, ql, labels, I, Dl, user_order)
    if unit_filter is not None:
        U = U[unit_filter(U)]
    U = np.ascontiguousarray(U, dtype=np.int32)
    qe, ql, labels, uo = _i32(qe), _i32(ql), _i32(labels), _i32(user_order)
    Dv = V.max_degree() if D is None else D
    out = np.zeros(4, np.uint64)
    access = np.zeros(n, np.uint64) if mode == 1 else None
    lev = np.zeros(n * max(k - 2, 1), np.uint64) if mode == 2 else None
    if M is None:
        M = walks(len(U), Dv, k)
    r = _load().ivm_run(mode, n, _p(V.stable[0]), _p(V.stable[1]), _p(V.old[0]), _p(V.old[1]), _p(V.new[0]),
                        _p(V.new[1]), _p(labels), k, len(qe), _p(qe), _p(ql), _p(uo), len(U), _p(U),
                        _threads(threads), seed & (2**64 - 1), int(M), Dv, _p(out), _p(access), _p(lev))
    if r:
        raise ValueError("bad query")
    return dict(added=_u128(out[0], out[1]), removed=_u128(out[2], out[3]), access=access,
                levcnt=None if lev is None else lev.reshape(n, max(k - 2, 1)), N1=len(U), D=Dv, M=int(M))


def ivm_count(n, rp, col, labels, k, qe, ql, ins, dele, user_order=None, threads=None):
    """(added, removed) via the eq. (1) terms as Fig. 2b-f nested loops, stable split R7."""
    r = _ivm(0, n, rp, col, labels, k, qe, ql, ins, dele, user_order, threads=threads)
    return r["added"], r["removed"]


def access_counts(n, rp, col, labels, k, qe, ql, ins, dele, user_order=None, threads=None, unit_filter=None):
    """Exact C_v: number of execution-tree nodes (levels 1..k-2, all terms) reading v's list (R17)."""
    return _ivm(1, n, rp, col, labels, k, qe, ql, ins, dele, user_order, unit_filter, threads)["access"]


def walks(N1: int, D: int, k: int) -> int:
    """M = |ΔE| D^{n-2} / 32^n, |ΔE| = N1 (R15); integer floor, clamped to [1, 2^62] (R21)."""
    if N1 <= 0:
        return 1
    return int(min(max((N1 * D ** max(k - 2, 0)) // 32 ** k, 1), 2 ** 62))


def estimate(n, rp, col, labels, k, qe, ql, ins, dele, seed, M=None, user_order=None, threads=None,
             unit_filter=None):
    """Access-frequency estimate by M plain random walks (§IV-A), one walk at a time.

    A walk picks one level-1 unit (term, sign, oriented changed edge; R15/R16) with probability 1/|ΔE|
    (|ΔE| = N1), records the lists its node accesses (R17), computes the candidate set V of the next position,
    picks one element with probability 1/|V| and continues with probability |V|/D (D of R19). Drawn from the
    oracle's own PCG32 streams (one per walk index, `seed`), never the product's generator.

    Returns dict(levcnt=[n, k-2] number of walks whose level-l node read v's list, N1, D, M,
    est=[n] float64) where est_v = (1/M) Σ_l |ΔE| D^(l-1) levcnt[v, l-1]  (eq. (3), averaged over M).
    """
    r = _ivm(2, n, rp, col, labels, k, qe, ql, ins, dele, user_order, unit_filter, threads, seed, M)
    lev = r["levcnt"].astype(np.float64)
    est = np.zeros(n)
    if k > 2:
        for l in range(1, k - 1):
            est += float(r["N1"]) * float(r["D"]) ** (l - 1) * lev[:, l - 1]
        est /= float(r["M"])
    r["est"] = est
    return r


def estimate_from_levels(levcnt, k, N1, D, M):
    """eq. (3) averaged over M for per-level sums (rows of any estimator's output): Σ_l N1 D^(l-1) lev[:, l-1] / M."""
    lev = np.asarray(levcnt, dtype=np.float64)
    est = np.zeros(lev.shape[0])
    for l in range(1, k - 1):
        est += float(N1) * float(D) ** (l - 1) * lev[:, l - 1]
    return est / float(M)


# ------------------------------------------------------------------ cache selection

def select_cache(score, list_bytes, budget, exclude=None):
    """a4 (reading R23): order vertices with score > 0 by (score desc, id asc);
    keep the longest prefix whose list bytes fit the budget. Returns sorted ids.

    exclude: vertices that take no part in the ranking. Reading R32: on the GPU path the stable lists of the
    batch's updated vertices U travel with the batch into HBM, so they compete for no budget; pass U there.
    The paper's own rule ranks every vertex (exclude=None)."""
    ex = set() if exclude is None else {int(v) for v in np.asarray(exclude).ravel()}
    ids = [v for v in range(len(score)) if score[v] > 0 and v not in ex]
    ids.sort(key=lambda v: (-score[v], v))
    used, keep = 0, []
    for v in ids:
        if used + list_bytes[v] > budget:
            break
        used += list_bytes[v]
        keep.append(v)
    return sorted(keep)


# ------------------------------------------------------------------ brute force (O1)

def brute_embeddings(n, edges, labels, k, qe, ql):
    """Every injective, label- and edge-preserving map V(Q) -> V(G) (Def. 1 read as R1-R3), as a set of tuples."""
    E = {(int(a), int(b)) for a, b in edges} | {(int(b), int(a)) for a, b in edges}
    out = set()
    for f in itertools.permutations(range(n), k):
        if ql is not None and any((0 if labels is None else labels[f[u]]) != ql[u] for u in range(k)):
            continue
        if all((f[u], f[w]) in E for u, w in qe):
            out.add(f)
    return out


def brute_delta(n, g0_edges, labels, k, qe, ql, ins, dele):
    """O1: set difference of brute-force embeddings before/after the batch."""
    E0 = {tuple(sorted(map(int, e))) for e in g0_edges}
    E1 = (E0 - {tuple(sorted(map(int, e))) for e in dele}) | {tuple(sorted(map(int, e))) for e in ins}
    A = brute_embeddings(n, E0, labels, k, qe, ql)
    B = brute_embeddings(n, E1, labels, k, qe, ql)
    return len(B - A), len(A - B), B - A, A - B


def automorphisms(k, qe, ql=None):
    """|Aut_L(Q)|: label-preserving permutations of V(Q) mapping E(Q) onto itself."""
    E = {tuple(sorted(e)) for e in map(tuple, np.asarray(qe).tolist())}
    cnt = 0
    for p in itertools.permutations(range(k)):
        if ql is not None and any(ql[p[u]] != ql[u] for u in range(k)):
            continue
        if {tuple(sorted((p[a], p[b]))) for a, b in E} == E:
            cnt += 1
    return cnt
