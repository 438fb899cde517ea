"""CPU tests of the boundary: libgcsm.so loads, exports every symbol include/gcsm.h declares, and its pure-host
logic (plan builder vs Fig. 2, LPT sharding) is right. No compute call needs a GPU here."""
import os
import re
import subprocess

import numpy as np
import pytest

import gcsm_inputs as gi
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def pkg():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_wei024_b200 as p
    return p


def header_symbols():
    src = open(os.path.join(ROOT, "include", "gcsm.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gcsm_[a-z_0-9]+)\s*\(", src)))


def test_exports_every_header_symbol(pkg):
    lib = pkg._lib.load()
    syms = header_symbols()
    assert len(syms) >= 17
    out = subprocess.run(["nm", "-D", "--defined-only", pkg._lib.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (gcsm_\w+)", out))
    for s in syms:
        assert s in exported, s
        assert hasattr(lib, s)
    assert sorted(pkg._lib.SYMBOLS) == syms


def test_library_is_sm100a(pkg):
    out = subprocess.run(["cuobjdump", "--list-elf", pkg._lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_plan_matches_fig2_and_oracle(pkg):
    for name in ["diamond", "triangle", "c4", "k4", "house5u", "prism6", "k6", "star3"]:
        k, qe, _ = gi.query(name)
        a = pkg.plan_inspect(k, qe)
        b = oracle.plan(k, qe)
        assert np.array_equal(a["seed"], b["seed"])
        assert np.array_equal(a["order"], b["order"])
        assert np.array_equal(a["nb"], b["nb"])
        for t in range(len(qe)):
            for p in range(k):
                nb = a["nb"][t, p]
                ga = {int(a["order"][t, q]): (int(a["view"][0, t, p, i]), int(a["view"][1, t, p, i]))
                      for i, q in enumerate(a["bq"][t, p, :nb])}
                gb = {int(b["order"][t, q]): (int(b["view"][0, t, p, i]), int(b["view"][1, t, p, i]))
                      for i, q in enumerate(b["bq"][t, p, :nb])}
                assert ga == gb, (name, t, p)
    # Fig. 2e: ΔM_4 of the diamond: order u1,u3,u0,u2; x2 ∈ S(x0) ∩ S(x1) ∩ N'(x3)
    k, qe, _ = gi.query("diamond")
    a = pkg.plan_inspect(k, qe)
    assert a["order"][3].tolist() == [1, 3, 0, 2]
    views = {int(a["order"][3, q]): int(a["view"][0, 3, 3, i]) for i, q in enumerate(a["bq"][3, 3, :3])}
    assert views == {1: 0, 3: 2, 0: 0}


def test_plan_rejects_bad_queries(pkg):
    with pytest.raises(pkg.GcsmError):
        pkg.plan_inspect(4, [(0, 1), (2, 3)])        # disconnected
    with pytest.raises(pkg.GcsmError):
        pkg.plan_inspect(3, [(0, 0), (1, 2)])        # self loop
    with pytest.raises(pkg.GcsmError):
        pkg.plan_inspect(9, [(i, i + 1) for i in range(8)])  # k > 8


def test_shard_disjoint_cover_and_balance(pkg):
    rng = np.random.default_rng(0)
    cost = rng.integers(1, 10000, size=5000).astype(np.uint64)
    for world in (1, 2, 4, 8):
        r = pkg.shard(cost, world)
        assert r.min() >= 0 and r.max() < world
        loads = np.bincount(r, weights=cost.astype(float) + 1, minlength=world)
        assert loads.max() <= loads.mean() + cost.max() + 1  # LPT bound
        assert np.array_equal(r, pkg.shard(cost, world))      # deterministic


def test_no_cpu_fallback(pkg):
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    w = gi.make_workload("C1", scale=6, n_edges=100, batch=8)
    with pytest.raises(pkg.GcsmError) as ei:
        pkg.Gcsm(w.n, w.row_ptr, w.col)
    assert ei.value.name in ("GCSM_EDEVICE", "GCSM_ENOMEM")


@pytest.mark.parametrize("name", ["edge", "wedge", "triangle", "c4", "diamond", "k4", "star3", "path4", "house5u",
                                  "house5", "bowtie5", "k5e", "k5", "prism6", "k4tri6"])
def test_symmetry_breaking_restrictions_brute_force(pkg, name):
    """Exactly one embedding per Aut_L orbit satisfies the library's restrictions:
    |{f in Emb : f(u) < f(w) for all (u, w)}| * |Aut_L| = |Emb|, by brute force on random small graphs."""
    k, qe, ql = gi.query(name)
    pairs, aut = pkg.query_restrictions(k, qe, ql)
    assert aut == oracle.automorphisms(k, qe, ql)
    rng = np.random.default_rng(len(name))
    for trial in range(3):
        n = 7 if k <= 5 else 8
        edges = gi.random_graph(n, 0.6, 1000 * trial + k)
        labels = rng.integers(0, 3, n).astype(np.int32) if ql is not None else None
        emb = oracle.brute_embeddings(n, edges, labels, k, qe.tolist(), ql)
        canon = [f for f in emb if all(f[u] < f[w] for u, w in pairs)]
        assert len(canon) * aut == len(emb)
    # a random user order changes the restrictions, not their property
    order = rng.permutation(k).astype(np.int32)
    pairs2, aut2 = pkg.query_restrictions(k, qe, ql, order)
    emb = oracle.brute_embeddings(7, gi.random_graph(7, 0.7, 5), None if ql is None else np.zeros(7, np.int32),
                                  k, qe.tolist(), None if ql is None else np.zeros(k, np.int32))
    if ql is None:
        assert len([f for f in emb if all(f[u] < f[w] for u, w in pairs2)]) * aut2 == len(emb)


def test_generator_planted_cliques():
    """C4's planted 8-cliques: exactly n_edges unique edges, every planted group a clique, deterministic, and the
    R-MAT part unchanged when nothing is planted (C2 / C3 inputs are the same as before)."""
    import numpy as np
    import gcsm_inputs as gi
    uv = gi.rmat_edges(12, 20000, 0.42, 0.176, 0.176, 7, planted=(50, 8))
    assert len(uv) == 20000 and (uv[:, 0] < uv[:, 1]).all()
    keys = uv[:, 0].astype(np.int64) * (1 << 32) + uv[:, 1]
    assert len(np.unique(keys)) == len(keys)
    assert np.array_equal(uv, gi.rmat_edges(12, 20000, 0.42, 0.176, 0.176, 7, planted=(50, 8)))
    # the planted edges come first in generation order: the first group's distinct members form a clique
    first = uv[:28]
    verts = np.unique(first)
    assert len(first) == len(verts) * (len(verts) - 1) // 2
    plain = gi.rmat_edges(12, 20000, 0.42, 0.176, 0.176, 7)
    assert not np.array_equal(plain[:28], first)
    w = gi.make_workload("C4", scale=12, n_edges=30000, batch=64, n_batches=1)
    assert w.meta["planted"][0] > 0 and int(w.row_ptr[-1]) > 0


def test_catalogue_orders_are_valid(pkg):
    """The catalogue's matching orders are permutations the plan builder accepts (connected per-term orders)."""
    import gcsm_inputs as gi
    for name in gi.ORDERS:
        k, qe, _ = gi.query(name)
        o = gi.order(name)
        assert sorted(o.tolist()) == list(range(k))
        pkg.plan_inspect(k, qe, o)
