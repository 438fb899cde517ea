"""Pins of the oracle's plan, access counts and estimator (M plain random walks, §IV-A).

* plan vs the Fig. 2b-f listing under readings R7/R11/R12;
* exact access counts C_v vs a brute force over all partial maps (tiny graphs);
* eq. (6) unbiasedness E[C~_v] = C_v of the plain walks against the brute-force-pinned C_v,
  and the eq. (7) variance bound;
* every sampled vertex has an (un-averaged) estimate >= |ΔE|;
* a hand-computed walk distribution on a one-unit instance.
(The product's merged-walk binomial sampler is pinned in tests/test_product_sampler.py.)
"""
import itertools

import numpy as np
import pytest

import gcsm_inputs as gi
import oracle

S, OLD, NEW = 0, 1, 2


def test_plan_matches_fig2():
    """Fig. 2b-f for the diamond (user order u0..u3, R1..R5 = 01,02,12,13,23).

    Term orders follow the listing; the views are the paper's N (j<i) -> S and N' (j>i) -> N' / N by sign (R7).
    """
    k, qe, _ = gi.query("diamond")
    p = oracle.plan(k, qe)
    assert p["seed"].tolist() == [[0, 1], [0, 2], [1, 2], [1, 3], [2, 3]]
    assert p["order"].tolist() == [[0, 1, 2, 3], [0, 2, 1, 3], [1, 2, 0, 3], [1, 3, 0, 2], [2, 3, 0, 1]]
    # (positions of backward neighbours, views for + terms) per term, for order positions 2 and 3
    expect = {
        0: {2: ([0, 1], [NEW, NEW]), 3: ([1, 2], [NEW, NEW])},          # ΔM_1: x2∈N'(x0)∩N'(x1); x3∈N'(x1)∩N'(x2)
        1: {2: ([0, 1], [S, NEW]), 3: ([1, 2], [NEW, NEW])},            # ΔM_2: x1∈N(x0)∩N'(x2); x3∈N'(x1)∩N'(x2)
        2: {2: ([0, 1], [S, S]), 3: ([0, 1], [NEW, NEW])},              # ΔM_3: x0∈N(x1)∩N(x2); x3∈N'(x1)∩N'(x2)
        3: {2: ([0], [S]), 3: ([0, 1, 2], [S, NEW, S])},                # ΔM_4: x0∈N(x1); x2∈N(x0)∩N(x1)∩N'(x3)
        4: {2: ([0], [S]), 3: ([0, 1, 2], [S, S, S])},                  # ΔM_5: x0∈N(x2); x1∈N(x0)∩N(x2)∩N(x3)
    }
    for t, lv in expect.items():
        for pos, (bq, views) in lv.items():
            nb = p["nb"][t, pos]
            got_bq = p["bq"][t, pos, :nb].tolist()
            # compare as (backward query vertex -> view) maps
            got = {int(p["order"][t, q]): int(p["view"][0, t, pos, i]) for i, q in enumerate(got_bq)}
            want = {int(p["order"][t, q]): v for q, v in zip(bq, views)}
            assert got == want, (t, pos)
            # - terms read N (old) instead of N' for j > i
            got_m = {int(p["order"][t, q]): int(p["view"][1, t, pos, i]) for i, q in enumerate(got_bq)}
            assert got_m == {u: (OLD if v == NEW else v) for u, v in want.items()}


def _brute_access(n, g0, labels, k, qe, ql, ins, dele):
    """C_v by enumerating every partial map of each term's positions (no DFS, no intersections)."""
    rp, col = oracle.csr(n, g0)
    I, D, _ = oracle.normalize_batch(n, rp, col, ins, dele)
    E = {tuple(sorted(map(int, e))) for e in g0}
    Dset = {tuple(sorted(map(int, e))) for e in D}
    Iset = {tuple(sorted(map(int, e))) for e in I}
    views = {S: E - Dset, OLD: E, NEW: (E - Dset) | Iset}
    pl = oracle.plan(k, qe)
    m = len(qe)
    C = np.zeros(n, np.int64)

    def lab_ok(u, v):
        return ql is None or (0 if labels is None else labels[v]) == ql[u]

    for t in range(m):
        order = pl["order"][t]
        for kind, edges in ((0, I), (1, D)):
            for a0, b0 in edges.tolist():
                for a, b in ((a0, b0), (b0, a0)):
                    if not (lab_ok(order[0], a) and lab_ok(order[1], b)):
                        continue
                    for lvl in range(1, k - 1):  # node at level lvl has positions 0..lvl matched
                        for rest in itertools.permutations([v for v in range(n) if v not in (a, b)], lvl - 1):
                            f = [a, b, *rest]
                            ok = True
                            for pos in range(2, lvl + 1):
                                if not lab_ok(order[pos], f[pos]):
                                    ok = False
                                    break
                                for i in range(pl["nb"][t, pos]):
                                    q = pl["bq"][t, pos, i]
                                    v = pl["view"][kind, t, pos, i]
                                    if tuple(sorted((f[q], f[pos]))) not in views[v]:
                                        ok = False
                                if not ok:
                                    break
                            if not ok:
                                continue
                            nxt = lvl + 1
                            for i in range(pl["nb"][t, nxt]):
                                C[f[pl["bq"][t, nxt, i]]] += 1
    return C


@pytest.mark.parametrize("seed", range(8))
def test_access_counts_vs_brute_force(seed):
    names = ["triangle", "diamond", "c4", "house5u"]
    name = names[seed % 4]
    k, qe, _ = gi.query(name)
    n, g0, ins, dele = gi.small_random_case(400 + seed, n=7, p=0.55, n_ins=2, n_del=2)
    labels = ql = None
    if seed % 2:
        rng = np.random.default_rng(seed)
        labels = rng.integers(0, 2, n).astype(np.int32)
        ql = rng.integers(0, 2, k).astype(np.int32)
    rp, col = oracle.csr(n, g0)
    got = oracle.access_counts(n, rp, col, labels, k, qe, ql, ins, dele)
    assert got.astype(np.int64).tolist() == _brute_access(n, g0, labels, k, qe, ql, ins, dele).tolist()


def _estimator_case():
    w = gi.make_workload("C1", scale=8, n_edges=1500, batch=24)
    ins = w.batches[0][0][:12]
    E = oracle.edges_of(w.row_ptr, w.col)
    dele = E[np.random.default_rng(9).choice(len(E), 8, replace=False)]
    return w.n, w.row_ptr, w.col, ins, dele


@pytest.mark.parametrize("name", ["diamond", "house5u", "k4"])
def test_estimator_unbiased_eq6(name):
    """Plain walks: E[C~_v] = C_v (eq. (6)); Var per walk <= (n-1)|ΔE| D^{n-2} C_v (eq. (7))."""
    n, rp, col, ins, dele = _estimator_case()
    k, qe, _ = gi.query(name)
    C = oracle.access_counts(n, rp, col, None, k, qe, None, ins, dele).astype(float)
    R, M = 60, 3000
    ests = []
    for r in range(R):
        e = oracle.estimate(n, rp, col, None, k, qe, None, ins, dele, seed=1000 + r, M=M)
        ests.append(e["est"])
        N1, D = e["N1"], e["D"]
    ests = np.array(ests)
    mean = ests.mean(0)
    sd = ests.std(0, ddof=1)
    hot = C > 0
    bound7 = np.sqrt((k - 1) * N1 * float(D) ** (k - 2) * C / M)  # eq. (7) per-walk sd / sqrt(M)
    se = np.maximum(sd, bound7 / 4) / np.sqrt(R)
    z = np.abs(mean[hot] - C[hot]) / se[hot]
    assert np.mean(z < 5) > 0.995 and z.max() < 8, (z.max(), np.mean(z < 5))
    assert np.all(ests[:, ~hot] == 0)  # never-accessed vertices are never estimated
    # eq. (7) holds for single walks exactly; the sample variance of 60 draws stays under 1.6x of it
    assert np.all(sd[hot] ** 2 <= 1.6 * bound7[hot] ** 2 + 1e-9)
    # a sampled vertex's un-averaged estimate M * C~_v >= |ΔE|
    for row in ests:
        s = row > 0
        assert np.all(row[s] * M >= N1 * (1 - 1e-12))


def test_walk_distribution_one_unit():
    """Hand-computed distribution of §IV-A's walk on one unit: the diamond's term ΔM_1 seeded by an inserted edge
    (0,1) whose endpoints share the common neighbours {2, 3} (and 0 has a private neighbour 4): the level-1 node
    reads N'(0), N'(1) (weight |ΔE| = N1); V = {2, 3}, so each level-2 child (0,1,x2) is reached with probability
    (1/|V|)(|V|/D) = 1/D and reads the lists of x3's backward neighbours (x1 and x2: weight N1 D)."""
    n = 6
    g0 = [(0, 2), (0, 3), (0, 4), (1, 2), (1, 3), (2, 5)]
    rp, col = oracle.csr(n, g0)
    ins = np.array([[0, 1]], np.int32)
    dele = np.zeros((0, 2), np.int32)
    k, qe, _ = gi.query("diamond")
    only_term0_plus = lambda U: (U[:, 0] == 0) & (U[:, 2] == 0)  # term 0, orientation (0, 1)
    M = 200_000
    e = oracle.estimate(n, rp, col, None, k, qe, None, ins, dele, seed=7, M=M, unit_filter=only_term0_plus)
    N1, D, lev = e["N1"], e["D"], e["levcnt"]
    assert N1 == 1 and D == 4  # degrees after the insertion: 0 -> {1,2,3,4}
    assert lev[0, 0] == M and lev[1, 0] == M  # the one unit is drawn by every walk (probability 1/N1 = 1)
    plan = oracle.plan(k, qe)
    assert plan["order"][0].tolist() == [0, 1, 2, 3]
    # level 2: (0,1,x2) for x2 in {2,3} w.p. 1/D each; it reads the lists of x3's backward neighbours 1 and x2
    p2 = 2.0 / D
    assert abs(lev[1, 1] / M - p2) < 5 * np.sqrt(p2 * (1 - p2) / M)
    for x2 in (2, 3):
        p = 1.0 / D
        assert abs(lev[x2, 1] / M - p) < 5 * np.sqrt(p * (1 - p) / M)
    assert lev[[4, 5], :].sum() == 0 and lev[0, 1] == 0
    # eq. (3) then gives the exact C_v in expectation: C_1 = 1 (level 1) + 2 (two level-2 nodes)
    C = oracle.access_counts(n, rp, col, None, k, qe, None, ins, dele, unit_filter=only_term0_plus)
    assert C.tolist() == [1, 3, 1, 1, 0, 0]
    assert abs(e["est"][1] - 3.0) < 0.05


def test_estimator_deterministic_and_thread_independent():
    n, rp, col, ins, dele = _estimator_case()
    k, qe, _ = gi.query("diamond")
    a = oracle.estimate(n, rp, col, None, k, qe, None, ins, dele, seed=5, threads=1)
    b = oracle.estimate(n, rp, col, None, k, qe, None, ins, dele, seed=5, threads=7)
    c = oracle.estimate(n, rp, col, None, k, qe, None, ins, dele, seed=6, threads=7)
    assert np.array_equal(a["levcnt"], b["levcnt"])
    assert not np.array_equal(a["levcnt"], c["levcnt"])
    assert a["M"] == oracle.walks(a["N1"], a["D"], k)


def test_walk_budget_formula():
    """M = |ΔE| D^{n-2} / 32^n — SURVEY appendix A numbers (|ΔE| = 4096)."""
    assert oracle.walks(4096, 5214, 5) == 4096 * 5214 ** 3 // 32 ** 5
    assert abs(oracle.walks(4096, 5214, 5) / 1.7e7 - 1) < 0.05
    assert abs(oracle.walks(4096, 5214, 6) / 2.8e9 - 1) < 0.05
    assert oracle.walks(3, 2, 3) == 1


def test_select_cache_prefix():
    score = np.array([0.0, 5.0, 9.0, 5.0, 1.0])
    size = np.array([16, 32, 48, 16, 16])
    assert oracle.select_cache(score, size, 0) == []
    assert oracle.select_cache(score, size, 48) == [2]
    assert oracle.select_cache(score, size, 80) == [1, 2]        # ties by id: 1 before 3
    assert oracle.select_cache(score, size, 95) == [1, 2]        # 3 does not fit -> stop (prefix)
    assert oracle.select_cache(score, size, 96) == [1, 2, 3]
    assert oracle.select_cache(score, size, 10**9) == [1, 2, 3, 4]  # score 0 never cached
    # R32: excluded vertices (the batch's updated set on the GPU path) take no part in the ranking
    assert oracle.select_cache(score, size, 80, exclude=[2]) == [1, 3, 4]
