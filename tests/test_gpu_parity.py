"""GPU parity: the CUDA path through the C ABI vs the oracle, bit-exact (integer counts, tuples, estimator sums).

Sizes: small enough for the oracle to finish in seconds, large enough to span many warps/units, ragged tails,
multi-segment lists (updated vertices), hub lists and the level-2 frontier; plus degenerate cases.
"""
import math

import numpy as np
import pytest

import gcsm_inputs as gi
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def G():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_wei024_b200 as pkg
    return pkg


def tuples_set(t):
    return sorted(map(tuple, np.asarray(t).tolist()))


def lib_run(G, n, rp, col, labels, name_or_q, batches, budget_frac=0.1, listing=False, **kw):
    k, qe, ql = gi.query(name_or_q) if isinstance(name_or_q, str) else name_or_q
    g = G.Gcsm(n, rp, col, labels, device=0, **kw)
    g.set_query(k, qe, ql)
    g.set_cache_budget(int(4 * rp[-1] * budget_frac))
    out = []
    for ins, dele in batches:
        if listing:
            a, r, ta, tr = g.apply_batch_list(ins, dele, 1 << 18, 1 << 18)
            out.append((a, r, tuples_set(ta), tuples_set(tr)))
        else:
            out.append(g.apply_batch(ins, dele))
    st = g.stats()
    rp2, col2 = g.export_csr()
    g.close()
    return out, st, (rp2, col2)


def oracle_run(n, rp, col, labels, name_or_q, batches, listing=False):
    k, qe, ql = gi.query(name_or_q) if isinstance(name_or_q, str) else name_or_q
    out = []
    for ins, dele in batches:
        if listing:
            (a, ta), (r, tr) = oracle.delta(n, rp, col, labels, k, qe, ql, ins, dele, listing=True, tuple_cap=1 << 18)
            out.append((a, r, tuples_set(ta), tuples_set(tr)))
        else:
            out.append(oracle.delta(n, rp, col, labels, k, qe, ql, ins, dele))
        I, D, _ = oracle.normalize_batch(n, rp, col, ins, dele)
        rp, col = oracle.apply_batch(n, rp, col, I, D)
    return out, (rp, col)


# ------------------------------------------------------------------ C1 (BASELINE configs[0])

@pytest.mark.parametrize("budget", [0.0, 0.1, 1.0])
def test_c1_triangle_budgets(G, budget):
    w = gi.make_workload("C1")
    want, (rp1, col1) = oracle_run(w.n, w.row_ptr, w.col, None, "triangle", w.batches, listing=True)
    got, st, (rp2, col2) = lib_run(G, w.n, w.row_ptr, w.col, None, "triangle", w.batches, budget, listing=True)
    assert got == want
    assert want[0][0] > 0
    assert np.array_equal(rp1, rp2) and np.array_equal(col1, col2)
    if budget == 0:  # no cache; a triangle reads only the updated vertices' lists, uploaded with the batch
        assert st["hit_bytes"] == 0 and st["cached_vertices"] == 0 and st["delta_bytes"] > 0
    if budget == 1.0:  # every list a triangle reads belongs to U: device-resident with the batch (R32), no misses
        assert st["miss_bytes"] == 0


# ------------------------------------------------------------------ fuzz

FUZZ = ["edge", "wedge", "triangle", "path4", "c4", "diamond", "k4", "star3", "house5u", "k5", "prism6", "k4tri6",
        "wheel7", "k4k4_7", "k7", "cube8", "k8"]


@pytest.mark.parametrize("seed", range(51))
def test_fuzz_small_graphs(G, seed):
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(8, 14))
    n_, g0, ins, dele = gi.small_random_case(1000 + seed, n=n, p=float(rng.uniform(0.25, 0.7)),
                                             n_ins=int(rng.integers(0, 7)), n_del=int(rng.integers(0, 7)))
    name = FUZZ[seed % len(FUZZ)]
    k, qe, _ = gi.query(name)
    labels = ql = None
    if seed % 3 == 1:
        labels = rng.integers(0, 2, n).astype(np.int32)
        ql = rng.integers(0, 2, k).astype(np.int32)
    order = rng.permutation(k).astype(np.int32) if seed % 4 == 2 else None
    rp, col = oracle.csr(n, g0)
    if k >= 7:  # 7- and 8-vertex patterns: counts (their tuple lists on dense graphs run to millions)
        want, _ = oracle_run(n, rp, col, labels, (k, qe, ql), [(ins, dele)])
        for sym in (True, False):
            g = G.Gcsm(n, rp, col, labels, device=0, symmetry=sym)
            g.set_query(k, qe, ql, order)
            g.set_cache_budget([0, 64, 1 << 20][seed % 3])
            assert g.apply_batch(ins, dele) == want[0]
            g.close()
        return
    want, _ = oracle_run(n, rp, col, labels, (k, qe, ql), [(ins, dele)], listing=True)
    g = G.Gcsm(n, rp, col, labels, device=0)
    g.set_query(k, qe, ql, order)
    g.set_cache_budget([0, 64, 1 << 20][seed % 3])
    a, r, ta, tr = g.apply_batch_list(ins, dele, 1 << 16, 1 << 16)
    g.close()
    assert (a, r, tuples_set(ta), tuples_set(tr)) == want[0]


@pytest.mark.parametrize("name", ["wheel7", "k4k4_7", "k7", "cube8"])
def test_seven_eight_vertex_lists(G, name):
    """k = 7 / 8 in list mode (every tuple, no symmetry breaking) on a sparse graph with planted cliques."""
    w = gi.make_workload("C4", scale=9, n_edges=2_500, batch=64, n_batches=2)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, name, w.batches, listing=True)
    got, _, _ = lib_run(G, w.n, w.row_ptr, w.col, None, name, w.batches, 0.05, listing=True)
    assert got == want


def test_degenerate_cases(G):
    k, qe, _ = gi.query("triangle")
    # empty batch; empty graph; complete graph built in one batch; all edges deleted
    n = 7
    E = [(i, j) for i in range(n) for j in range(i + 1, n)]
    rp0, col0 = oracle.csr(n, np.zeros((0, 2), np.int32))
    g = G.Gcsm(n, rp0, col0, device=0)
    g.set_query(k, qe)
    g.set_cache_budget(1 << 20)
    assert g.apply_batch(np.zeros((0, 2)), np.zeros((0, 2))) == (0, 0)
    assert g.apply_batch(E, []) == (n * (n - 1) * (n - 2), 0)
    assert g.apply_batch([], E) == (0, n * (n - 1) * (n - 2))
    # no-ops are dropped and counted (R8)
    g.apply_batch([(0, 1)], [])
    assert g.apply_batch([(0, 1), (1, 0)], [(2, 3)]) == (0, 0)
    assert g.stats()["dropped"] == 2
    # EINVAL leaves the graph unchanged
    before = g.export_csr()
    for ins, dele in [([(1, 1)], []), ([(0, 99)], []), ([(2, 4)], [(4, 2)])]:
        with pytest.raises(G.GcsmError) as ei:
            g.apply_batch(ins, dele)
        assert ei.value.name == "GCSM_EINVAL"
        after = g.export_csr()
        assert all(np.array_equal(x, y) for x, y in zip(before, after))
    g.close()
    # apply before set_query -> ESTATE
    g = G.Gcsm(n, rp0, col0, device=0)
    with pytest.raises(G.GcsmError) as ei:
        g.apply_batch([(0, 1)], [])
    assert ei.value.name == "GCSM_ESTATE"
    g.close()


def test_bad_graph_rejected(G):
    rp = np.array([0, 1, 1], np.int64)
    col = np.array([1], np.int32)  # not symmetric
    with pytest.raises(G.GcsmError) as ei:
        G.Gcsm(2, rp, col, device=0)
    assert ei.value.name == "GCSM_EINVAL"


def test_list_truncation(G):
    n = 6
    E = [(i, j) for i in range(n) for j in range(i + 1, n)]
    rp0, col0 = oracle.csr(n, np.zeros((0, 2), np.int32))
    g = G.Gcsm(n, rp0, col0, device=0)
    g.set_query(*gi.query("triangle")[:2])
    with pytest.raises(G.GcsmError) as ei:
        g.apply_batch_list(E, [], 5, 5)
    assert ei.value.name == "GCSM_ETRUNC"
    assert g.stats()["added"] == 120
    g.close()


# ------------------------------------------------------------------ streams (multi-batch state, store ① / ⑤)

@pytest.mark.parametrize("name", ["diamond", "k4", "c4", "house5u"])
def test_stream_of_mixed_batches(G, name):
    w = gi.make_workload("C2", scale=11, n_edges=12000, batch=200)
    batches = w.batches[:5]
    want, (rp1, col1) = oracle_run(w.n, w.row_ptr, w.col, None, name, batches)
    got, st, (rp2, col2) = lib_run(G, w.n, w.row_ptr, w.col, None, name, batches, 0.1)
    assert got == want
    assert any(a + r > 0 for a, r in want)
    assert np.array_equal(rp1, rp2) and np.array_equal(col1, col2)


@pytest.mark.parametrize("order", [None, [3, 2, 1, 0], [2, 0, 3, 1]])
def test_matching_order_invariance(G, order):
    w = gi.make_workload("C2", scale=11, n_edges=12000, batch=300)
    k, qe, _ = gi.query("diamond")
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, "diamond", w.batches[:2])
    g = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
    g.set_query(k, qe, None, order)
    g.set_cache_budget(w.adj_bytes // 20)
    assert [g.apply_batch(*b) for b in w.batches[:2]] == want
    g.close()


# ------------------------------------------------------------------ scaled configs C2 / C3

@pytest.mark.parametrize("name", ["k4", "c4"])
@pytest.mark.parametrize("budget", [0.0, 0.1, 1.0])
def test_c2_shaped(G, name, budget):
    w = gi.make_workload("C2", scale=16, n_edges=600_000, batch=1024, n_batches=2)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, name, w.batches)
    got, st, _ = lib_run(G, w.n, w.row_ptr, w.col, None, name, w.batches, budget)
    assert got == want


@pytest.mark.parametrize("name", ["house5", "bowtie5", "k5e"])
def test_c3_shaped_labelled(G, name):
    w = gi.make_workload("C3", scale=14, n_edges=200_000, batch=1024, n_batches=2)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, w.labels, name, w.batches)
    got, st, _ = lib_run(G, w.n, w.row_ptr, w.col, w.labels, name, w.batches, 0.1)
    assert got == want


@pytest.mark.parametrize("name", ["prism6", "k4tri6", "k6"])
def test_six_vertex_queries(G, name):
    w = gi.make_workload("C2", scale=12, n_edges=40_000, batch=256, n_batches=2)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, name, w.batches)
    got, _, _ = lib_run(G, w.n, w.row_ptr, w.col, None, name, w.batches, 0.05)
    assert got == want


@pytest.mark.parametrize("name", ["prism6", "k4tri6", "k6", "wheel7", "k4k4_7"])
def test_c4_shaped_planted(G, name):
    """C4-shaped (FR R-MAT parameters + planted 8-cliques): the 6-vertex counts are non-zero, budget << graph."""
    w = gi.make_workload("C4", scale=13, n_edges=60_000, batch=256, n_batches=2)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, name, w.batches)
    assert any(a or r for a, r in want)
    got, _, _ = lib_run(G, w.n, w.row_ptr, w.col, None, name, w.batches, 0.01)
    assert got == want


@pytest.mark.parametrize("overlap", ["8", "5"])
def test_c4_shaped_pipelined_multi_query(G, overlap, monkeypatch):
    """The bench's C4 layout on a C4-shaped graph: ONE context holding prism6 + K4+2tri6 + K6, pipelined
    submit / wait, 1 % budget; with the cache step of batch t+1 beside the matching of batch t (GCSM_OVERLAP_KMAX=8,
    the default) and without (5). Every query's counts equal the oracle's on every batch, and the final graph too."""
    monkeypatch.setenv("GCSM_OVERLAP_KMAX", overlap)
    w = gi.make_workload("C4", scale=13, n_edges=60_000, batch=256, n_batches=4)
    names = ["prism6", "k4tri6", "k6"]
    want = {q: oracle_run(w.n, w.row_ptr, w.col, None, q, w.batches)[0] for q in names}
    g = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
    for i, q in enumerate(names):
        k, qe, ql = gi.query(q)
        (g.set_query if i == 0 else g.add_query)(k, qe, ql, gi.order(q))
    g.set_cache_budget(w.adj_bytes // 100)
    got = {q: [] for q in names}

    def collect():
        g.wait_batch()
        for i, q in enumerate(names):
            got[q].append(g.query_counts(i))

    g.submit_batch(*w.batches[0])
    for b in w.batches[1:]:
        g.submit_batch(*b)
        collect()
    collect()
    assert got == want
    _, (rp1, col1) = oracle_run(w.n, w.row_ptr, w.col, None, "edge", w.batches)
    rp2, col2 = g.export_csr()
    assert np.array_equal(rp1, rp2) and np.array_equal(col1, col2)
    g.close()


@pytest.mark.parametrize("r", [1, 2, 3])
def test_star_closed_form_at_scale(G, r):
    """SURVEY §8c degree closed form for K_{1,r}: added = Σ_U P(d',r) - P(s,r), removed = Σ_U P(d,r) - P(s,r)."""
    w = gi.make_workload("C2", scale=18, n_edges=3_000_000, batch=4096, n_batches=2)
    k = r + 1
    qe = np.array([(0, i) for i in range(1, k)], np.int32)
    g = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
    g.set_query(k, qe)
    g.set_cache_budget(w.adj_bytes // 10)
    rp, col = w.row_ptr, w.col

    def P(x):
        out = np.ones_like(x, dtype=object)
        for i in range(r):
            out = out * (x - i)
        return out

    for ins, dele in w.batches:
        I, D, _ = oracle.normalize_batch(w.n, rp, col, ins, dele)
        rp1, col1 = oracle.apply_batch(w.n, rp, col, I, D)
        rps, _ = oracle.stable_graph(w.n, rp, col, D)
        U = np.unique(np.concatenate([I.ravel(), D.ravel()]))
        d, d1, s = (np.diff(x)[U].astype(object) for x in (rp, rp1, rps))
        want = (int((P(d1) - P(s)).sum()), int((P(d) - P(s)).sum()))
        assert g.apply_batch(ins, dele) == want
        rp, col = rp1, col1
    g.close()


# ------------------------------------------------------------------ estimator ② and packer ③
# The oracle estimates by plain walks (§IV-A) with its own generator, so the product's merged walks (§IV-B) are
# pinned STATISTICALLY against the exact access counts C_v (eq. (6)/(7)), while the host walker (the paper's
# CPU placement, GCSM_HOST_EST=1) and the GPU walker are compared bit-exactly with each other (product-internal).

def updated_vertices(I, D):
    return np.unique(np.concatenate([np.asarray(I).ravel(), np.asarray(D).ravel()]))


def host_est_ctx(G, *args, **kw):
    import os
    os.environ["GCSM_HOST_EST"] = "1"
    try:
        return G.Gcsm(*args, **kw)
    finally:
        del os.environ["GCSM_HOST_EST"]


def product_estimate(g, n, k):
    """eq. (3) over the product's per-level sums (query 0), as a dense vector."""
    st = g.stats()
    ids, lev = g.estimates()
    est = np.zeros(n)
    est[ids] = oracle.estimate_from_levels(lev[:, :k - 2], k, st["n1"], st["max_degree"], st["walks"])
    return est, ids, lev, st


def _eq6_case():
    w = gi.make_workload("C1", scale=8, n_edges=1500, batch=24)
    ins = w.batches[0][0][:12]
    E = oracle.edges_of(w.row_ptr, w.col)
    dele = E[np.random.default_rng(9).choice(len(E), 8, replace=False)]
    return w, ins, dele


@pytest.mark.parametrize("name", ["diamond", "house5u", "k4", "prism6"])
def test_gpu_estimator_unbiased_eq6(G, name):
    """The DEVICE walker (merged walks, §IV-B) against the oracle's exact C_v: the mean of eq. (3) over 60 seeds lies
    within 5 standard errors of C_v (eq. (6)), the spread respects eq. (7) (merged walks: independent binomials,
    R20, so a factor 2 of slack), every estimated vertex is accessed in the exact trees, and every sampled vertex's
    un-averaged estimate is >= |ΔE|."""
    w, ins, dele = _eq6_case()
    k, qe, ql = gi.query(name)
    C = oracle.access_counts(w.n, w.row_ptr, w.col, None, k, qe, ql, ins, dele).astype(float)
    I, D, _ = oracle.normalize_batch(w.n, w.row_ptr, w.col, ins, dele)
    N1 = len(oracle.units(k, qe, ql, None, I, D))
    R, M = 60, 3000
    ests = []
    for r in range(R):
        g = G.Gcsm(w.n, w.row_ptr, w.col, None, device=0, seed=1000 + r, walks_override=M)
        g.set_query(k, qe, ql)
        g.set_cache_budget(w.adj_bytes // 10)
        assert g.apply_batch(ins, dele) == oracle.delta(w.n, w.row_ptr, w.col, None, k, qe, ql, ins, dele)
        est, ids, lev, st = product_estimate(g, w.n, k)
        g.close()
        assert (st["n1"], st["walks"]) == (N1, M)
        Dmax = st["max_degree"]
        ests.append(est)
    ests = np.array(ests)
    mean, sd = ests.mean(0), ests.std(0, ddof=1)
    hot = C > 0
    bound7 = np.sqrt((k - 1) * N1 * float(Dmax) ** (k - 2) * C / M)
    se = np.maximum(sd, bound7 / 4) / np.sqrt(R)
    z = np.abs(mean[hot] - C[hot]) / se[hot]
    assert np.mean(z < 5) > 0.995 and z.max() < 8, (z.max(), np.mean(z < 5))
    assert np.all(ests[:, ~hot] == 0)
    assert np.all(sd[hot] ** 2 <= 2.0 * bound7[hot] ** 2 + 1e-9)
    for row in ests:
        s_ = row > 0
        assert np.all(row[s_] * M >= N1 * (1 - 1e-12))


@pytest.mark.parametrize("name,labelled", [("diamond", False), ("k4", False), ("house5u", False), ("house5", True),
                                           ("prism6", False)])
def test_gpu_walker_equals_host_walker(G, name, labelled):
    """Product-internal: the device walker draws exactly what the host walker draws (R30), batch after batch; the
    two packers select by R23 (GPU path: over the vertices not updated by the batch, R32) — checked against the
    oracle's independent ranking on the product's own estimates; counts equal the oracle's."""
    w = gi.make_workload("C3" if labelled else "C2", scale=12, n_edges=30_000, batch=256, n_batches=2)
    labels = w.labels if labelled else None
    k, qe, ql = gi.query(name)
    seed = 0xBEEF
    budget = w.adj_bytes // 25
    g = G.Gcsm(w.n, w.row_ptr, w.col, labels, device=0, seed=seed)
    h = host_est_ctx(G, w.n, w.row_ptr, w.col, labels, device=0, seed=seed)
    for c in (g, h):
        c.set_query(k, qe, ql)
        c.set_cache_budget(budget)
    rp, col = w.row_ptr, w.col
    for t, (ins, dele) in enumerate(w.batches):
        want = oracle.delta(w.n, rp, col, labels, k, qe, ql, ins, dele)
        assert g.apply_batch(ins, dele) == want
        assert h.apply_batch(ins, dele) == want
        I, D, _ = oracle.normalize_batch(w.n, rp, col, ins, dele)
        eg, ids_g, lev_g, st_g = product_estimate(g, w.n, k)
        eh, ids_h, lev_h, st_h = product_estimate(h, w.n, k)
        N1 = len(oracle.units(k, qe, ql, labels, I, D))
        Dmax = oracle._Views(w.n, rp, col, I, D).max_degree()
        assert (st_g["n1"], st_g["max_degree"], st_g["walks"]) == (N1, Dmax, oracle.walks(N1, Dmax, k))
        assert (st_h["n1"], st_h["max_degree"], st_h["walks"]) == (st_g["n1"], st_g["max_degree"], st_g["walks"])
        assert np.array_equal(ids_g, ids_h)
        assert np.array_equal(lev_g[:, :k - 2], lev_h[:, :k - 2])
        # every estimated vertex is one the exact execution trees access (eq. (6) support)
        C = oracle.access_counts(w.n, rp, col, labels, k, qe, ql, ins, dele)
        assert np.all(C[ids_g] > 0)
        rps, _ = oracle.stable_graph(w.n, rp, col, D)
        sz = 16 * ((np.diff(rps) + 3) // 4)
        assert np.array_equal(g.cached(), oracle.select_cache(eg, sz, budget & ~15, exclude=updated_vertices(I, D)))
        assert np.array_equal(h.cached(), oracle.select_cache(eh, sz, budget & ~15))
        rp, col = oracle.apply_batch(w.n, rp, col, I, D)
    g.close()
    h.close()


@pytest.mark.parametrize("name,M", [("k4", 10**9), ("house5u", 10**9), ("prism6", 10**9)])
def test_gpu_walker_btrd_range(G, name, M):
    """Walk budgets large enough that children draw B' ~ Bin(B, 1/D) with B/D >= 10 (BTRD, R20) on the device: the
    per-vertex per-level sums still equal the host walker's, and the cached set is R23 on them."""
    w = gi.make_workload("C2", scale=11, n_edges=12_000, batch=96, n_batches=1)
    k, qe, ql = gi.query(name)
    seed = 0x5EED
    budget = w.adj_bytes // 20
    g = G.Gcsm(w.n, w.row_ptr, w.col, None, device=0, seed=seed, walks_override=M)
    h = host_est_ctx(G, w.n, w.row_ptr, w.col, None, device=0, seed=seed, walks_override=M)
    ins, dele = w.batches[0]
    want = oracle.delta(w.n, w.row_ptr, w.col, None, k, qe, ql, ins, dele)
    for c in (g, h):
        c.set_query(k, qe, ql)
        c.set_cache_budget(budget)
        assert c.apply_batch(ins, dele) == want
    eg, ids_g, lev_g, st = product_estimate(g, w.n, k)
    _, ids_h, lev_h, _ = product_estimate(h, w.n, k)
    assert st["walks"] == M
    assert M // st["n1"] >= 10 * st["max_degree"]  # level-1 children are in BTRD's range
    assert np.array_equal(ids_g, ids_h)
    assert np.array_equal(lev_g[:, :k - 2], lev_h[:, :k - 2])
    I, D, _ = oracle.normalize_batch(w.n, w.row_ptr, w.col, ins, dele)
    rps, _ = oracle.stable_graph(w.n, w.row_ptr, w.col, D)
    sz = 16 * ((np.diff(rps) + 3) // 4)
    assert np.array_equal(g.cached(), oracle.select_cache(eg, sz, budget & ~15, exclude=updated_vertices(I, D)))
    g.close()
    h.close()


@pytest.mark.parametrize("name", ["house5u", "prism6", "k4tri6", "wheel7"])
def test_walk_lane_path_equals_warp_dfs(G, name, monkeypatch):
    """Product-internal: the level k-3 walk nodes walked one per lane (walk_leaf_parent, default) record exactly the
    sums of the warp-wide DFS (GCSM_WALK_LANE=0) on a C4-shaped planted graph. M is chosen so that level k-3 nodes
    carry B ~ 2 (M = 2 N1 D^(k-4): B_l ~ M / (N1 D^(l-1))), i.e. they are in BINV's domain AND draw children."""
    w = gi.make_workload("C4", scale=13, n_edges=60_000, batch=256, n_batches=1)
    k, qe, ql = gi.query(name)
    ins, dele = w.batches[0]
    probe = G.Gcsm(w.n, w.row_ptr, w.col, None, device=0)
    probe.set_query(k, qe, ql, gi.order(name))
    probe.apply_batch(ins, dele)
    st = probe.stats()
    probe.close()
    M = 2 * st["n1"] * st["max_degree"] ** (k - 4)
    out = []
    for lane in ("1", "0"):
        monkeypatch.setenv("GCSM_WALK_LANE", lane)
        g = G.Gcsm(w.n, w.row_ptr, w.col, None, device=0, seed=0xA11, walks_override=M)
        g.set_query(k, qe, ql, gi.order(name))
        g.set_cache_budget(w.adj_bytes // 100)
        cnt = g.apply_batch(ins, dele)
        _, ids, lev, st = product_estimate(g, w.n, k)
        out.append((cnt, ids, lev[:, :k - 2], g.cached()))
        g.close()
    assert out[0][0] == out[1][0]
    assert np.array_equal(out[0][1], out[1][1]) and np.array_equal(out[0][2], out[1][2])
    assert np.array_equal(out[0][3], out[1][3])
    assert out[0][2][:, k - 3].sum() > 0  # level k-2 records exist: level k-3 nodes drew children


def test_degree_policy_cached_set(G):
    """Naive ablation (degree-ranked cache): the device ranking is R23 applied to the stable degrees."""
    w = gi.make_workload("C2", scale=12, n_edges=30_000, batch=256, n_batches=2)
    k, qe, ql = gi.query("k4")
    budget = w.adj_bytes // 10
    g = G.Gcsm(w.n, w.row_ptr, w.col, None, device=0, cache_policy="degree")
    g.set_query(k, qe, ql)
    g.set_cache_budget(budget)
    rp, col = w.row_ptr, w.col
    for ins, dele in w.batches:
        g.apply_batch(ins, dele)
        I, D, _ = oracle.normalize_batch(w.n, rp, col, ins, dele)
        rps, _ = oracle.stable_graph(w.n, rp, col, D)
        deg = np.diff(rps).astype(np.float64)
        sz = 16 * ((np.diff(rps) + 3) // 4)
        assert np.array_equal(g.cached(), oracle.select_cache(deg, sz, budget & ~15, exclude=updated_vertices(I, D)))
        rp, col = oracle.apply_batch(w.n, rp, col, I, D)
    g.close()


def test_budget_change_between_batches(G):
    """Growing the budget reallocates the cache buffers: descriptors of the old selection must not dangle."""
    w = gi.make_workload("C2", scale=12, n_edges=30_000, batch=256, n_batches=4)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, "c4", w.batches)
    k, qe, ql = gi.query("c4")
    g = G.Gcsm(w.n, w.row_ptr, w.col, None, device=0)
    g.set_query(k, qe, ql)
    got = []
    for i, (ins, dele) in enumerate(w.batches):
        g.set_cache_budget([w.adj_bytes // 50, w.adj_bytes // 5, 0, w.adj_bytes][i])
        got.append(g.apply_batch(ins, dele))
    g.close()
    assert got == want


# ------------------------------------------------------------------ multi-GPU sharding, emulated world on one GPU

@pytest.mark.parametrize("world", [2, 4, 8])
def test_emulated_world_sums(G, world):
    w = gi.make_workload("C2", scale=13, n_edges=60_000, batch=512, n_batches=2)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, "k4", w.batches)
    tot = [[0, 0] for _ in w.batches]
    units = 0
    for rank in range(world):
        got, st, _ = lib_run(G, w.n, w.row_ptr, w.col, None, "k4", w.batches, 0.1, rank=rank, world=world,
                             local_counts=True)
        for i, (a, r) in enumerate(got):
            tot[i][0] += a
            tot[i][1] += r
    assert [tuple(x) for x in tot] == want


def test_interleaved_contexts(G):
    """Two live contexts with different queries (per-context plans and caches) applied alternately."""
    w = gi.make_workload("C2", scale=12, n_edges=30_000, batch=256, n_batches=3)
    want = {q: oracle_run(w.n, w.row_ptr, w.col, None, q, w.batches)[0] for q in ("k4", "c4", "house5u")}
    ctx = {}
    for q in want:
        k, qe, ql = gi.query(q)
        ctx[q] = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
        ctx[q].set_query(k, qe, ql)
        ctx[q].set_cache_budget(w.adj_bytes // 10)
    got = {q: [] for q in want}
    for b in w.batches:
        for q in want:
            got[q].append(ctx[q].apply_batch(*b))
    for g in ctx.values():
        g.close()
    assert got == want


def test_cache_policies_same_counts(G):
    w = gi.make_workload("C2", scale=14, n_edges=150_000, batch=512, n_batches=2)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, "k4", w.batches)
    for pol in ("estimator", "degree", "none"):
        got, st, _ = lib_run(G, w.n, w.row_ptr, w.col, None, "k4", w.batches, 0.05, cache_policy=pol)
        assert got == want, pol
        if pol == "none":
            assert st["hit_bytes"] == 0 or st["cached_vertices"] == 0


# ------------------------------------------------------------------ pipelined submit / wait (NEXT-2)

@pytest.mark.parametrize("name", ["k4", "c4", "house5u"])
def test_pipelined_submit_wait(G, name):
    """Batch t+1's host steps overlap batch t's kernels; counts, final graph and state rules are unchanged."""
    w = gi.make_workload("C2", scale=12, n_edges=40_000, batch=256, n_batches=6)
    want, (rp1, col1) = oracle_run(w.n, w.row_ptr, w.col, None, name, w.batches)
    k, qe, ql = gi.query(name)
    g = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
    g.set_query(k, qe, ql)
    g.set_cache_budget(w.adj_bytes // 10)
    got = []
    g.submit_batch(*w.batches[0])
    for b in w.batches[1:]:
        g.submit_batch(*b)
        got.append(g.wait_batch())
    got.append(g.wait_batch())
    assert got == want
    rp2, col2 = g.export_csr()
    assert np.array_equal(rp1, rp2) and np.array_equal(col1, col2)
    # state rules
    with pytest.raises(G.GcsmError) as ei:
        g.wait_batch()
    assert ei.value.name == "GCSM_ESTATE"
    g.submit_batch(np.zeros((0, 2)), np.zeros((0, 2)))
    g.submit_batch(np.zeros((0, 2)), np.zeros((0, 2)))
    for call in (lambda: g.submit_batch(np.zeros((0, 2)), np.zeros((0, 2))), lambda: g.set_query(k, qe, ql),
                 lambda: g.set_cache_budget(1 << 20)):
        with pytest.raises(G.GcsmError) as ei:
            call()
        assert ei.value.name == "GCSM_ESTATE"
    assert g.wait_batch() == (0, 0) and g.wait_batch() == (0, 0)
    # apply_batch drains outstanding submissions first
    g.submit_batch(np.zeros((0, 2)), np.zeros((0, 2)))
    assert g.apply_batch(np.zeros((0, 2)), np.zeros((0, 2))) == (0, 0)
    g.close()


# ------------------------------------------------------------------ full-size configs, bench launch configuration

@pytest.mark.parametrize("cfg,queries", [("C2", ["k4", "c4"]), ("C3", ["house5", "bowtie5", "k5e"])])
def test_full_size_sampled(G, cfg, queries):
    """BASELINE configs[1]/[2] at full size (70M / 120M edges) with bench.py's launch configuration (default grid,
    10 % budget, estimator cache): a sampled sub-batch (the first 256 updated edges of batch 0) against the oracle."""
    w = gi.make_workload(cfg, n_batches=2)
    ins, dele = w.batches[0]
    si, sd = ins[:128], dele[:128]
    g = G.Gcsm(w.n, w.row_ptr, w.col, w.labels, device=0)  # bench.py: one context holding every query
    for i, q in enumerate(queries):
        k, qe, ql = gi.query(q)
        (g.set_query if i == 0 else g.add_query)(k, qe, ql)
    g.set_cache_budget(int(w.adj_bytes * w.budget_frac))
    g.apply_batch(si, sd)
    for i, q in enumerate(queries):
        k, qe, ql = gi.query(q)
        want = oracle.delta(w.n, w.row_ptr, w.col, w.labels, k, qe, ql, si, sd)
        assert g.query_counts(i) == want, q
        st = g.query_stats(i)
        assert st["cached_vertices"] > 0 and st["hit_bytes"] > 0
    g.close()


@pytest.mark.parametrize("r", [2, 3])
def test_full_size_star_closed_form(G, r):
    """Whole C2 batches at full size (4096 mixed updates, 70M edges) against the K_{1,r} degree closed form."""
    w = gi.make_workload("C2", n_batches=2)
    k = r + 1
    qe = np.array([(0, i) for i in range(1, k)], np.int32)
    g = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
    g.set_query(k, qe)
    g.set_cache_budget(w.adj_bytes // 10)
    rp, col = w.row_ptr, w.col

    def P(x):
        out = np.ones_like(x, dtype=object)
        for i in range(r):
            out = out * (x - i)
        return out

    for ins, dele in w.batches:
        I, D, _ = oracle.normalize_batch(w.n, rp, col, ins, dele)
        rp1, col1 = oracle.apply_batch(w.n, rp, col, I, D)
        U = np.unique(np.concatenate([I.ravel(), D.ravel()]))
        d, d1 = np.diff(rp)[U].astype(object), np.diff(rp1)[U].astype(object)
        # stable degree: old degree minus deleted incident edges
        s = d - np.array([int(np.count_nonzero(D == u)) for u in U], dtype=object)
        want = (int((P(d1) - P(s)).sum()), int((P(d) - P(s)).sum()))
        assert g.apply_batch(ins, dele) == want
        rp, col = rp1, col1
    g.close()


def test_nccl_single_rank_allreduce(G):
    """The NCCL path on one GPU: a one-rank communicator from gcsm_nccl_unique_id; the counts go through
    ncclAllReduce on the kernel stream and come back unchanged."""
    w = gi.make_workload("C2", scale=12, n_edges=30_000, batch=256, n_batches=2)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, "diamond", w.batches)
    got, st, _ = lib_run(G, w.n, w.row_ptr, w.col, None, "diamond", w.batches, 0.1, nccl_id=G.nccl_unique_id())
    assert got == want
    assert st["ms_allreduce"] > 0


@pytest.mark.parametrize("name", ["triangle", "k4", "c4", "diamond", "house5u", "prism6", "k4tri6"])
def test_symmetry_breaking_on_off(G, name):
    """Count mode walks one embedding per Aut_L orbit and scales by |Aut_L| (default); both settings equal the
    oracle on a mixed stream."""
    w = gi.make_workload("C2", scale=12, n_edges=40_000, batch=256, n_batches=3)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, name, w.batches)
    on, _, _ = lib_run(G, w.n, w.row_ptr, w.col, None, name, w.batches, 0.1, symmetry=True)
    off, _, _ = lib_run(G, w.n, w.row_ptr, w.col, None, name, w.batches, 0.1, symmetry=False)
    assert on == want and off == want


# ------------------------------------------------------------------ standing queries sharing one context

@pytest.mark.parametrize("policy", ["estimator", "degree", "none"])
def test_multi_query_context(G, policy):
    """gcsm_add_query: several queries share the store, the batch steps and one cache budget; every query's
    counts equal the oracle's on every batch (mixed k, labels off, pipelined submit/wait)."""
    names = ["k4", "c4", "triangle", "house5u", "path4"]
    w = gi.make_workload("C2", scale=12, n_edges=40_000, batch=256, n_batches=4)
    want = {q: oracle_run(w.n, w.row_ptr, w.col, None, q, w.batches)[0] for q in names}
    g = G.Gcsm(w.n, w.row_ptr, w.col, device=0, cache_policy=policy)
    k, qe, ql = gi.query(names[0])
    g.set_query(k, qe, ql)
    for i, q in enumerate(names[1:], 1):
        k, qe, ql = gi.query(q)
        assert g.add_query(k, qe, ql) == i
    assert g.num_queries() == len(names)
    g.set_cache_budget(w.adj_bytes // 10)
    got = {q: [] for q in names}
    g.submit_batch(*w.batches[0])
    for b in list(w.batches[1:]) + [None]:
        if b is not None:
            g.submit_batch(*b)
        a0 = g.wait_batch()
        for i, q in enumerate(names):
            got[q].append(g.query_counts(i))
        assert a0 == got[names[0]][-1]
    assert got == want
    st = g.query_stats(1)
    assert st["cache_bytes"] <= w.adj_bytes // 10 and st["units"] > 0
    with pytest.raises(G.GcsmError) as ei:
        g.apply_batch_list(np.zeros((0, 2)), np.zeros((0, 2)))
    assert ei.value.name == "GCSM_EINVAL"
    # set_query resets to one query
    k, qe, ql = gi.query("triangle")
    g.set_query(k, qe, ql)
    assert g.num_queries() == 1
    g.close()


def test_multi_query_limits(G):
    w = gi.make_workload("C2", scale=10, n_edges=5_000, batch=64, n_batches=1)
    g = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
    k, qe, ql = gi.query("triangle")
    with pytest.raises(G.GcsmError) as ei:
        g.add_query(k, qe, ql)  # before set_query
    assert ei.value.name == "GCSM_ESTATE"
    g.set_query(k, qe, ql)
    for _ in range(31):
        g.add_query(k, qe, ql)
    with pytest.raises(G.GcsmError) as ei:
        g.add_query(k, qe, ql)
    assert ei.value.name == "GCSM_EINVAL"
    a = g.apply_batch(*w.batches[0])
    assert all(g.query_counts(i) == a for i in range(32))
    g.close()


@pytest.mark.parametrize("name", ["c4", "k4"])
def test_sampled_index_on_off(G, name, monkeypatch):
    """The sampled index only narrows which slice of a zero-copy x2 list crosses PCIe: counts equal the
    oracle with it on and off over a 4-batch stream (the previous batch's updated vertices get their samples
    refreshed), and with it on the kernels never copy more bytes from host memory than with it off."""
    w = gi.make_workload("C2", scale=16, n_edges=600_000, batch=1024, n_batches=4)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, name, w.batches)
    k, qe, ql = gi.query(name)
    copied = {}
    for mode in ("on", "off"):
        if mode == "off":
            monkeypatch.setenv("GCSM_NO_SIDX", "1")
        g = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
        g.set_query(k, qe, ql)
        g.set_cache_budget(w.adj_bytes // 20)
        got, cb = [], 0
        for ins, dele in w.batches:
            got.append(g.apply_batch(ins, dele))
            cb += g.stats()["host_copied_bytes"]
        g.close()
        assert got == want, mode
        copied[mode] = cb
    monkeypatch.delenv("GCSM_NO_SIDX", raising=False)
    assert copied["on"] <= copied["off"], copied


@pytest.mark.parametrize("overlap", ["on", "off"])
def test_pipelined_cache_step_overlap(G, overlap, monkeypatch):
    """Batch t+1's GPU cache step runs on its own stream beside batch t's matching (DESIGN.md §1c step 6; off:
    GCSM_NO_OVERLAP=1 at create). Two standing queries, C2-shaped graph, 5 pipelined batches: each query's counts
    equal the oracle's and the final graph equals the oracle's either way."""
    if overlap == "off":
        monkeypatch.setenv("GCSM_NO_OVERLAP", "1")
    w = gi.make_workload("C2", scale=16, n_edges=600_000, batch=2048, n_batches=5)
    names = ["k4", "c4"]
    g = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
    g.set_query(*gi.query(names[0]))
    qids = [0] + [g.add_query(*gi.query(nm)) for nm in names[1:]]
    g.set_cache_budget(w.adj_bytes // 10)
    got = {nm: [] for nm in names}

    def collect():
        g.wait_batch()
        for nm, qi in zip(names, qids):
            got[nm].append(g.query_counts(qi))

    g.submit_batch(*w.batches[0])
    for b in w.batches[1:]:
        g.submit_batch(*b)
        collect()
    collect()
    rp2, col2 = g.export_csr()
    g.close()
    for nm in names:
        want, (rp1, col1) = oracle_run(w.n, w.row_ptr, w.col, None, nm, w.batches)
        assert got[nm] == want, nm
    assert np.array_equal(rp1, rp2) and np.array_equal(col1, col2)


# ------------------------------------------------------------------ NEXT-4: motif counting (Fig. 11)

def test_motif_census_road_net(G):
    """All 29 connected 3-, 4- and 5-vertex motifs as standing queries of ONE context on a road-net-shaped graph
    (low skew): every motif's (added, removed) equals the oracle's, over a 3-batch stream, and the
    final graph equals the oracle's G_t."""
    w = gi.make_workload("PA", scale=14, batch=512, n_batches=3)
    names = gi.MOTIFS[3] + gi.MOTIFS[4] + gi.MOTIFS[5]
    g = G.Gcsm(w.n, w.row_ptr, w.col, device=0)
    for i, q in enumerate(names):
        k, qe, ql = gi.query(q)
        (g.set_query if i == 0 else g.add_query)(k, qe, ql)
    g.set_cache_budget(w.adj_bytes // 10)
    rp, col = w.row_ptr, w.col
    nonzero = 0
    for ins, dele in w.batches:
        g.apply_batch(ins, dele)
        for i, q in enumerate(names):
            k, qe, ql = gi.query(q)
            want = oracle.delta(w.n, rp, col, None, k, qe, ql, ins, dele)
            assert g.query_counts(i) == want, q
            nonzero += want != (0, 0)
        I, D, _ = oracle.normalize_batch(w.n, rp, col, ins, dele)
        rp, col = oracle.apply_batch(w.n, rp, col, I, D)
    assert nonzero >= 30
    rp2, col2 = g.export_csr()
    assert np.array_equal(rp, rp2) and np.array_equal(col, col2)
    g.close()


# ------------------------------------------------------------------ NEXT-4: vertex-id growth

def _growth_batches(w, n0, ncap, seed, n_batches=3):
    """Mixed batches that also attach new ids in [n0, ncap): a new vertex x gets edges to both endpoints of an
    existing edge (a, b), so it closes triangles / diamonds / K4s at once; later batches join new ids together
    and delete some of their edges again."""
    rng = np.random.default_rng(seed)
    E = oracle.edges_of(w.row_ptr, w.col)
    out = []
    nxt = n0
    joined = []
    for t in range(n_batches):
        ins, dele = [tuple(e) for e in w.batches[t][0]], [tuple(e) for e in w.batches[t][1]]
        for _ in range(40):
            if nxt >= ncap:
                break
            a, b = E[rng.integers(len(E))]
            ins += [(nxt, int(a)), (int(b), nxt)]
            joined.append(nxt)
            nxt += 1
        if len(joined) >= 4:
            for _ in range(10):
                x, y = rng.choice(joined, 2, replace=False)
                ins.append((int(x), int(y)))
        out.append((np.array(sorted(set(ins)), np.int32).reshape(-1, 2), np.array(dele, np.int32).reshape(-1, 2)))
    return out


@pytest.mark.parametrize("name", ["triangle", "diamond", "k4", "house5u"])
def test_vertex_growth(G, name):
    """Insertions naming ids in [n, vertex_capacity) add vertices, each with an empty list of the average
    degree's capacity; the oracle sees the same ids as isolated vertices of the capacity-sized universe
    (reading R9), so the counts and the final graph must agree batch by batch."""
    w = gi.make_workload("C2", scale=11, n_edges=12000, batch=200)
    n0, ncap = w.n, w.n + 150
    batches = _growth_batches(w, n0, ncap, 11)
    rp = np.concatenate([w.row_ptr, np.full(ncap - n0, w.row_ptr[-1], np.int64)])
    want, (rp1, col1) = oracle_run(ncap, rp, w.col, None, name, batches)
    k, qe, ql = gi.query(name)
    g = G.Gcsm(n0, w.row_ptr, w.col, device=0, vertex_capacity=ncap)
    g.set_query(k, qe, ql)
    g.set_cache_budget(w.adj_bytes // 10)
    got = [g.apply_batch(*b) for b in batches]
    assert got == want
    assert any(a for a, _ in want)
    n1 = g.num_vertices()
    assert n0 < n1 <= ncap
    rp2, col2 = g.export_csr()
    assert np.array_equal(rp2, rp1[:n1 + 1]) and np.array_equal(col2, col1) and rp1[n1] == rp1[-1]
    # a deletion naming a vertex that does not exist, or an id beyond the capacity: EINVAL, nothing changes
    bad = [([(0, ncap)], [])] + ([([], [(0, ncap - 1)])] if n1 < ncap else [])
    for ins, dele in bad:
        with pytest.raises(G.GcsmError) as ei:
            g.apply_batch(ins, dele)
        assert ei.value.name == "GCSM_EINVAL"
    assert g.num_vertices() == n1
    g.close()


def test_add_vertices_labelled(G):
    """gcsm_add_vertices with labels, then edges to them: labelled house5 counts equal the oracle's."""
    w = gi.make_workload("C3", scale=11, n_edges=12000, batch=200, n_batches=2)
    n0, extra = w.n, 80
    lab_new = np.random.default_rng(5).integers(0, 8, extra).astype(np.int32)
    labels = np.concatenate([w.labels, lab_new])
    k, qe, ql = gi.query("house5")
    g = G.Gcsm(n0, w.row_ptr, w.col, w.labels, device=0, vertex_capacity=n0 + extra)
    g.set_query(k, qe, ql)
    g.set_cache_budget(w.adj_bytes // 10)
    assert g.add_vertices(extra, lab_new) == n0 and g.num_vertices() == n0 + extra
    with pytest.raises(G.GcsmError):
        g.add_vertices(1)  # capacity exhausted
    batches = _growth_batches(w, n0, n0 + extra, 12, n_batches=2)
    rp = np.concatenate([w.row_ptr, np.full(extra, w.row_ptr[-1], np.int64)])
    want, _ = oracle_run(n0 + extra, rp, w.col, labels, "house5", batches)
    assert [g.apply_batch(*b) for b in batches] == want
    g.close()


# ------------------------------------------------------------------ NEXT-3: NVLink peer cache

@pytest.mark.parametrize("name", ["c4", "house5u", "prism6"])
def test_peer_cache_two_contexts(G, name):
    """Two contexts on one GPU (an emulated 2-rank world: each counts its own shard of the units) link their HBM
    caches (gcsm_link_peers): a list missing from one context's cache is read from the other's. Each context is
    driven by its own host thread in lockstep; the shard counts sum to the oracle's, batch by batch, and some
    list bytes are served by the peer."""
    import threading
    w = gi.make_workload("C2" if name != "prism6" else "C4", scale=13, n_edges=60_000, batch=512, n_batches=3)
    k, qe, ql = gi.query(name)
    want, _ = oracle_run(w.n, w.row_ptr, w.col, None, name, w.batches)
    ctxs = [G.Gcsm(w.n, w.row_ptr, w.col, device=0, rank=r, world=2, local_counts=True, seed=0x77 + r)
            for r in range(2)]
    for c in ctxs:
        c.set_query(k, qe, ql, gi.order(name))
        c.set_cache_budget(w.adj_bytes // 20)
    G.link_peers(ctxs)
    out = [[], []]
    errs = []

    def drive(r):
        try:
            for ins, dele in w.batches:
                out[r].append((ctxs[r].apply_batch(ins, dele), ctxs[r].stats()["peer_bytes"]))
        except Exception as e:  # noqa: BLE001
            errs.append(e)

    th = [threading.Thread(target=drive, args=(r,)) for r in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not errs, errs
    got = [(a0 + a1, r0 + r1) for ((a0, r0), _), ((a1, r1), _) in zip(out[0], out[1])]
    assert got == want
    assert sum(p for _, p in out[0]) + sum(p for _, p in out[1]) > 0
    G.link_peers([])
    G.link_peers(ctxs[:1])  # unlink (n < 2) is accepted
    for c in ctxs:
        c.close()


def _star_closed_form(n, rp, col, ins, dele, r):
    """K_{1,r} added = Σ_U P(d',r) - P(s,r), removed = Σ_U P(d,r) - P(s,r) (O(|U|) arithmetic)."""
    I, D, _ = oracle.normalize_batch(n, rp, col, ins, dele)
    U = np.unique(np.concatenate([I.ravel(), D.ravel()]))
    d = np.diff(rp)[U].astype(object)
    cnt = lambda E: np.array([0 if len(E) == 0 else int(np.count_nonzero(E == u)) for u in U], dtype=object)
    di, dd = cnt(I), cnt(D)
    s, d1 = d - dd, d - dd + di

    def P(x):
        out = np.ones_like(x, dtype=object)
        for i in range(r):
            out = out * (x - i)
        return out
    return (int((P(d1) - P(s)).sum()), int((P(d) - P(s)).sum())), (I, D)


def test_full_size_c2_whole_batch(G):
    """One WHOLE 4096-update C2 batch (70M edges, bench launch configuration: one context holding K4 + C4 with the
    catalogue orders, 10 % budget) against the oracle."""
    w = gi.make_workload("C2", n_batches=1)
    ins, dele = w.batches[0]
    queries = ["k4", "c4"]
    g = G.Gcsm(w.n, w.row_ptr, w.col, None, device=0)
    for i, q in enumerate(queries):
        k, qe, ql = gi.query(q)
        (g.set_query if i == 0 else g.add_query)(k, qe, ql, gi.order(q))
    g.set_cache_budget(int(w.adj_bytes * w.budget_frac))
    g.apply_batch(ins, dele)
    for i, q in enumerate(queries):
        k, qe, ql = gi.query(q)
        assert g.query_counts(i) == oracle.delta(w.n, w.row_ptr, w.col, None, k, qe, ql, ins, dele), q
    g.close()


def test_full_size_c4(G):
    """BASELINE configs[3] at FULL size (67M vertices, 1.8B edges in pinned host memory, planted 8-cliques, 1 %
    budget, bench.py's context: prism6 + K4+2tri6 + K6 with the catalogue orders, plus a K_{1,3} star): on two
    batches, a sampled sub-batch (64 updated edges) against the oracle for every 6-vertex query, and the rest of
    the batch against the star's degree closed form."""
    w = gi.make_workload("C4", n_batches=2)
    queries = ["prism6", "k4tri6", "k6"]
    star = (4, np.array([(0, 1), (0, 2), (0, 3)], np.int32), None)
    g = G.Gcsm(w.n, w.row_ptr, w.col, None, device=0)
    for i, q in enumerate(queries):
        k, qe, ql = gi.query(q)
        (g.set_query if i == 0 else g.add_query)(k, qe, ql, gi.order(q))
    g.add_query(*star)
    g.set_cache_budget(int(w.adj_bytes * w.budget_frac))
    rp, col = w.row_ptr, w.col
    nonzero = 0
    for t, (ins, dele) in enumerate(w.batches):
        si, sd = ins[:32], dele[:32]
        ri, rd = ins[32:], dele[32:]
        g.apply_batch(si, sd)
        for i, q in enumerate(queries):
            k, qe, ql = gi.query(q)
            want = oracle.delta(w.n, rp, col, None, k, qe, ql, si, sd)
            assert g.query_counts(i) == want, (t, q)
            nonzero += want != (0, 0)
        cf, (I, D) = _star_closed_form(w.n, rp, col, si, sd, 3)
        assert g.query_counts(3) == cf
        rp, col = oracle.apply_batch(w.n, rp, col, I, D)
        g.apply_batch(ri, rd)  # the rest of the batch, on the star closed form
        cf, (I, D) = _star_closed_form(w.n, rp, col, ri, rd, 3)
        assert g.query_counts(3) == cf
        assert g.query_stats(0)["stage_fill_bytes"] > 0  # the fetch-once staging ran at full size
        if t + 1 < len(w.batches):
            rp, col = oracle.apply_batch(w.n, rp, col, I, D)
    assert nonzero >= 2
    g.close()
