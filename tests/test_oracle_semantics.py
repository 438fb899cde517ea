"""Pins of the oracle's counting functions against things other than itself.

* O1 brute force over all injective maps (itertools) on <= 9-vertex graphs;
* networkx's GraphMatcher monomorphisms (independent library routine);
* closed forms on K_n, K_n - e, stars, K_{a,b} (SURVEY §8c "Closed forms");
* the Fig. 1 reconstruction (tests/golden/fig1.txt);
* invariants: telescoping eq. (1), insert-then-delete negation,
  relabelling, label-sum, |Aut| divisibility, batch normalisation (R8).
"""
import itertools
import math

import numpy as np
import pytest

import gcsm_inputs as gi
import oracle
from conftest import load_golden


def _csr(n, edges):
    return oracle.csr(n, np.asarray(edges, dtype=np.int32).reshape(-1, 2))


def _complete(n):
    return [(i, j) for i in range(n) for j in range(i + 1, n)]


def falling(x, r):
    out = 1
    for i in range(r):
        out *= (x - i)
    return out


# ------------------------------------------------------------------ worked example

def test_fig1_reconstruction():
    g = load_golden("fig1.txt")
    n = g["n"][0][0]
    qe = np.array(g["query"][0]).reshape(-1, 2)
    E0 = np.array(g["g0"][0]).reshape(-1, 2)
    ins = np.array(g["ins"][0]).reshape(-1, 2)
    dele = np.array(g["del"][0]).reshape(-1, 2)
    rp, col = _csr(n, E0)
    a, r = oracle.delta(n, rp, col, None, 4, qe, None, ins, dele)
    assert (a, r) == (g["added"][0][0], g["removed"][0][0])
    assert oracle.automorphisms(4, qe) == g["aut"][0][0]
    # Fig. 4a: the level-2 child of each ΔM_1 seed is N'(x0) ∩ N'(x1)
    rp1, col1 = oracle.apply_batch(n, rp, col, ins, dele)
    for x0, x1, child in g["fig4a"]:
        s = set(col1[rp1[x0]:rp1[x0 + 1]]) & set(col1[rp1[x1]:rp1[x1 + 1]])
        assert s == {child}
    # Fig. 6: v3's old list and appended new neighbours; v4 old list (before the deletion mark)
    assert list(col[rp[3]:rp[4]]) == g["fig6_v3_old"][0]
    assert sorted(set(col1[rp1[3]:rp1[4]]) - set(col[rp[3]:rp[4]])) == g["fig6_v3_new"][0]
    assert list(col[rp[4]:rp[5]]) == g["fig6_v4_old"][0]


# ------------------------------------------------------------------ brute force (O1)

FUZZ_QUERIES = ["edge", "wedge", "triangle", "path4", "c4", "diamond", "k4", "star3", "house5u"]


@pytest.mark.parametrize("seed", range(24))
def test_delta_vs_brute_force(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(6, 9))
    n_, g0, ins, dele = gi.small_random_case(seed, n=n, p=float(rng.uniform(0.3, 0.7)),
                                             n_ins=int(rng.integers(0, 5)), n_del=int(rng.integers(0, 5)))
    name = FUZZ_QUERIES[seed % len(FUZZ_QUERIES)]
    k, qe, _ = gi.query(name)
    labelled = seed % 3 == 0
    labels = rng.integers(0, 2, size=n).astype(np.int32) if labelled else None
    ql = rng.integers(0, 2, size=k).astype(np.int32) if labelled else None
    rp, col = _csr(n, g0)
    ba, br, bA, bR = oracle.brute_delta(n, g0, labels, k, qe, ql, ins, dele)
    a, r = oracle.delta(n, rp, col, labels, k, qe, ql, ins, dele)
    assert (a, r) == (ba, br)
    # the IVM algorithm (eq. (1), stable split R7) gives the same per-sign counts
    assert oracle.ivm_count(n, rp, col, labels, k, qe, ql, ins, dele) == (ba, br)
    # listing: exactly the brute-force embedding sets
    (a2, ta), (r2, tr) = oracle.delta(n, rp, col, labels, k, qe, ql, ins, dele, listing=True, tuple_cap=10**5)
    assert {tuple(t) for t in ta.tolist()} == bA and len(ta) == a2
    assert {tuple(t) for t in tr.tolist()} == bR and len(tr) == r2


@pytest.mark.parametrize("seed", range(6))
def test_ivm_invariant_to_user_order(seed):
    """Reading R11: counts do not depend on the matching order / edge numbering."""
    rng = np.random.default_rng(100 + seed)
    n, g0, ins, dele = gi.small_random_case(100 + seed, n=8, p=0.5, n_ins=3, n_del=3)
    k, qe, _ = gi.query(["diamond", "c4", "house5u"][seed % 3])
    rp, col = _csr(n, g0)
    ref = oracle.delta(n, rp, col, None, k, qe, None, ins, dele)
    for _ in range(3):
        uo = rng.permutation(k).astype(np.int32)
        assert oracle.ivm_count(n, rp, col, None, k, qe, None, ins, dele, user_order=uo) == ref


def test_paper_form_overcounts_mixed_batches():
    """Reading R7: with a deletion and a later-numbered insertion in one embedding, eq. (1)'s per-sign sums with the
    paper's N (j<i) / N' (j>i) views over-count, but its net is exact."""
    # triangle 0-1-2 where (0,1) is deleted and (1,2) inserted: appears in G_t? no ((1,2) missing) — build explicitly
    n = 4
    g0 = [(0, 1), (0, 2), (2, 3)]
    ins, dele = [(1, 2)], [(0, 1)]
    k, qe, _ = gi.query("triangle")
    rp, col = _csr(n, g0)
    a, r = oracle.delta(n, rp, col, None, k, qe, None, ins, dele)
    assert (a, r) == (0, 0)  # no triangle before or after
    assert oracle.ivm_count(n, rp, col, None, k, qe, None, ins, dele) == (0, 0)


# ------------------------------------------------------------------ networkx

def test_delta_vs_networkx():
    nx = pytest.importorskip("networkx")
    from networkx.algorithms import isomorphism as iso
    for seed in range(6):
        n, g0, ins, dele = gi.small_random_case(200 + seed, n=10, p=0.45, n_ins=4, n_del=4)
        for name in ["triangle", "c4", "diamond", "prism6"]:
            k, qe, _ = gi.query(name)
            Q = nx.Graph()
            Q.add_nodes_from(range(k))
            Q.add_edges_from(qe.tolist())

            def emb(edges):
                G = nx.Graph()
                G.add_nodes_from(range(n))
                G.add_edges_from(np.asarray(edges).tolist())
                M = iso.GraphMatcher(G, Q)
                return {tuple(inv[u] for u in range(k))
                        for inv in ({v: u for u, v in mm.items()} for mm in M.subgraph_monomorphisms_iter())}

            E0 = {tuple(sorted(e)) for e in g0.tolist()}
            E1 = (E0 - {tuple(sorted(e)) for e in dele.tolist()}) | {tuple(sorted(e)) for e in ins.tolist()}
            A, B = emb(sorted(E0)), emb(sorted(E1))
            rp, col = _csr(n, g0)
            assert oracle.delta(n, rp, col, None, k, qe, None, ins, dele) == (len(B - A), len(A - B))


# ------------------------------------------------------------------ closed forms

@pytest.mark.parametrize("name", ["triangle", "c4", "k4", "diamond", "house5u", "prism6"])
@pytest.mark.parametrize("n", [6, 7])
def test_complete_graph_static(name, n):
    k, qe, _ = gi.query(name)
    rp, col = _csr(n, _complete(n))
    assert oracle.static_count(n, rp, col, None, k, qe, None) == math.factorial(n) // math.factorial(n - k)


@pytest.mark.parametrize("n", [5, 6, 8])
def test_complete_minus_edge_insert(n):
    E = _complete(n)
    e = (0, n - 1)
    g0 = [x for x in E if x != e]
    rp, col = _csr(n, g0)
    expect = {"triangle": 6 * (n - 2), "k4": 24 * math.comb(n - 2, 2), "c4": 8 * (n - 2) * (n - 3)}
    for name, val in expect.items():
        k, qe, _ = gi.query(name)
        assert oracle.delta(n, rp, col, None, k, qe, None, [e], []) == (val, 0)
    # deletion of the edge from K_n: the negatives
    rpk, colk = _csr(n, E)
    for name, val in expect.items():
        k, qe, _ = gi.query(name)
        assert oracle.delta(n, rpk, colk, None, k, qe, None, [], [e]) == (0, val)
    # general k-clique gains k! C(n-2, k-2)
    k, qe, _ = gi.query("k5")
    if n >= 5:
        assert oracle.delta(n, rp, col, None, k, qe, None, [e], [])[0] == math.factorial(5) * math.comb(n - 2, 3)


@pytest.mark.parametrize("n", [4, 5, 6])
def test_empty_to_complete_one_batch(n):
    rp, col = _csr(n, np.zeros((0, 2), np.int32))
    rpk, colk = _csr(n, _complete(n))
    for name in ["triangle", "c4", "k4", "diamond"]:
        k, qe, _ = gi.query(name)
        val = math.factorial(n) // math.factorial(n - k)
        assert oracle.delta(n, rp, col, None, k, qe, None, _complete(n), []) == (val, 0)
        assert oracle.ivm_count(n, rp, col, None, k, qe, None, _complete(n), []) == (val, 0)
        assert oracle.delta(n, rpk, colk, None, k, qe, None, [], _complete(n)) == (0, val)
        assert oracle.ivm_count(n, rpk, colk, None, k, qe, None, [], _complete(n)) == (0, val)


@pytest.mark.parametrize("n", [5, 7])
def test_star_graph(n):
    star = [(0, i) for i in range(1, n)]
    rp, col = _csr(n, star)
    k, qe, _ = gi.query("triangle")
    assert oracle.static_count(n, rp, col, None, k, qe, None) == 0
    assert oracle.delta(n, rp, col, None, k, qe, None, [(1, 2)], []) == (6, 0)
    k, qe, _ = gi.query("wedge")
    assert oracle.static_count(n, rp, col, None, k, qe, None) == (n - 1) * (n - 2)


@pytest.mark.parametrize("a,b", [(2, 3), (3, 3), (3, 4)])
def test_complete_bipartite(a, b):
    E = [(i, a + j) for i in range(a) for j in range(b)]
    rp, col = _csr(a + b, E)
    assert oracle.static_count(a + b, rp, col, None, *gi.query("triangle")) == 0
    assert oracle.static_count(a + b, rp, col, None, *gi.query("c4")) == 2 * a * (a - 1) * b * (b - 1)


@pytest.mark.parametrize("seed", range(8))
@pytest.mark.parametrize("r", [1, 2, 3])
def test_star_query_degree_closed_form(seed, r):
    """for Q = K_{1,r}, added = Σ_U P(d',r) - P(s,r), removed = Σ_U P(d,r) - P(s,r)."""
    n, g0, ins, dele = gi.small_random_case(300 + seed, n=12, p=0.4, n_ins=4, n_del=4)
    qe = np.array([(0, i) for i in range(1, r + 1)], np.int32)
    k = r + 1
    rp, col = _csr(n, g0)
    I, D, _ = oracle.normalize_batch(n, rp, col, ins, dele)
    rp1, _ = oracle.apply_batch(n, rp, col, I, D)
    rps, _ = oracle.stable_graph(n, rp, col, D)
    d, d1, s = np.diff(rp), np.diff(rp1), np.diff(rps)
    U = np.unique(np.concatenate([I.ravel(), D.ravel()]))
    add = sum(falling(int(d1[v]), r) - falling(int(s[v]), r) for v in U)
    rem = sum(falling(int(d[v]), r) - falling(int(s[v]), r) for v in U)
    assert oracle.delta(n, rp, col, None, k, qe, None, ins, dele) == (add, rem)


# ------------------------------------------------------------------ invariants

def test_telescoping_over_a_stream():
    """Eq. (1) verified by subtraction: Σ nets over a stream = static recount difference."""
    w = gi.make_workload("C1", scale=7, n_edges=500, batch=16)
    rng = np.random.default_rng(5)
    n, rp, col = w.n, w.row_ptr, w.col
    k, qe, _ = gi.query("diamond")
    start = oracle.static_count(n, rp, col, None, k, qe, None)
    net = 0
    E = oracle.edges_of(rp, col)
    for t in range(4):
        dele = E[rng.choice(len(E), 5, replace=False)]
        ins = w.batches[t][0]
        a, r = oracle.delta(n, rp, col, None, k, qe, None, ins, dele)
        net += a - r
        I, D, _ = oracle.normalize_batch(n, rp, col, ins, dele)
        rp, col = oracle.apply_batch(n, rp, col, I, D)
        E = oracle.edges_of(rp, col)
    assert oracle.static_count(n, rp, col, None, k, qe, None) - start == net


def test_insert_then_delete_negation_and_relabel():
    n, g0, ins, _ = gi.small_random_case(7, n=11, p=0.5, n_ins=6, n_del=0)
    k, qe, _ = gi.query("diamond")
    rp, col = _csr(n, g0)
    a, r = oracle.delta(n, rp, col, None, k, qe, None, ins, [])
    rp1, col1 = oracle.apply_batch(n, rp, col, *oracle.normalize_batch(n, rp, col, ins, [])[:2])
    assert oracle.delta(n, rp1, col1, None, k, qe, None, [], ins) == (r, a)
    perm = np.random.default_rng(1).permutation(n).astype(np.int32)
    g0p = np.sort(perm[g0], axis=1)
    rpp, colp = _csr(n, g0p)
    assert oracle.delta(n, rpp, colp, None, k, qe, None, perm[ins], []) == (a, r)


def test_label_sum_and_aut_divisibility():
    """R5: Σ over all L^k query labelings of the labelled count = the unlabelled count; emb divisible by |Aut_L|."""
    n, g0, ins, dele = gi.small_random_case(11, n=9, p=0.55, n_ins=3, n_del=3)
    rng = np.random.default_rng(3)
    L = 2
    labels = rng.integers(0, L, size=n).astype(np.int32)
    rp, col = _csr(n, g0)
    k, qe, _ = gi.query("diamond")
    ua, ur = oracle.delta(n, rp, col, labels, k, qe, None, ins, dele)
    sa = sr = 0
    for lab in itertools.product(range(L), repeat=k):
        ql = np.array(lab, np.int32)
        a, r = oracle.delta(n, rp, col, labels, k, qe, ql, ins, dele)
        sa += a
        sr += r
        s = oracle.static_count(n, rp, col, labels, k, qe, ql)
        assert s % oracle.automorphisms(k, qe, ql) == 0
    assert (sa, sr) == (ua, ur)


def test_automorphism_table():
    """|Aut| of the catalogue, pinned by K_n: |Emb(Q, K_k)| = k! = |Aut(Q)| only for Q = K_k."""
    expect = {"triangle": 6, "diamond": 4, "k4": 24, "c4": 8, "house5": 2, "k5e": 2, "bowtie5": 4,
              "prism6": 12, "k4tri6": 8, "k6": 720}
    for name, val in expect.items():
        k, qe, ql = gi.query(name)
        assert oracle.automorphisms(k, qe, ql) == val


def test_normalize_batch_r8():
    rp, col = _csr(5, [(0, 1), (1, 2)])
    I, D, dropped = oracle.normalize_batch(5, rp, col, [(3, 2), (2, 3), (1, 0)], [(2, 1), (4, 3)])
    assert I.tolist() == [[2, 3]] and D.tolist() == [[1, 2]] and dropped == 2
    for bad in [([(1, 1)], []), ([(0, 5)], []), ([(0, 2)], [(2, 0)]), ([], [(-1, 2)])]:
        with pytest.raises(ValueError):
            oracle.normalize_batch(5, rp, col, *bad)


@pytest.mark.parametrize("seed", range(10))
def test_apply_batch_vs_set_algebra(seed):
    """The row-by-row graph update (oracle.c o_apply) equals plain numpy set algebra on edge keys."""
    n, g0, ins, dele = gi.small_random_case(500 + seed, n=30, p=0.2, n_ins=12, n_del=12)
    rp, col = _csr(n, g0)
    I, D, _ = oracle.normalize_batch(n, rp, col, ins, dele)
    a = oracle.apply_batch(n, rp, col, I, D)
    b = oracle.apply_batch_setalgebra(n, rp, col, I, D)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    s = oracle.stable_graph(n, rp, col, D)
    e = {tuple(x) for x in oracle.edges_of(*s).tolist()}
    assert e == {tuple(x) for x in g0.tolist()} - {tuple(x) for x in D.tolist()}


def test_motif_catalogue():
    """Fig. 11 counts 'all size-3, 4, and 5 motifs': the connected simple graphs on 3, 4, 5 vertices up
    to isomorphism number 2, 6 and 21 (OEIS A001349); each is connected and no two are isomorphic (networkx)."""
    nx = pytest.importorskip("networkx")
    for size, want in ((3, 2), (4, 6), (5, 21)):
        cat = gi.motifs(size)
        assert len(cat) == want
        graphs = []
        for name, edges in cat:
            h = nx.Graph()
            h.add_nodes_from(range(size))
            h.add_edges_from(edges)
            assert nx.is_connected(h), name
            graphs.append(h)
        for i in range(len(graphs)):
            for j in range(i + 1, len(graphs)):
                assert not nx.is_isomorphic(graphs[i], graphs[j])
    assert gi.MOTIFS[3] == ["m3_0", "m3_1"]
    assert gi.query("m3_1")[1].tolist() == [[0, 1], [0, 2], [1, 2]]  # the triangle


def test_road_net_shape():
    """PA-shaped input (Table I RoadNetPA: 1.09M vertices, 1.54M edges, small degrees): low skew, small max degree."""
    w = gi.make_workload("PA", scale=14, n_batches=1, batch=256)
    deg = np.diff(w.row_ptr)
    assert deg.max() <= 8 and 2.0 < deg.mean() < 3.5
    assert w.n == 128 * 128
