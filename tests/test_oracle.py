"""Pins for the CPU oracle (oracle/): every function is checked against something
other than itself — hand-computed examples, closed forms, the exact parallel
characterisation of Alg 3 (derived), a library routine (scipy
P A P^T), conservation/symmetry invariants, the matching bound
 and the known answers of an independent model."""
import itertools
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp

import graphgen as gg
import oracle as o

SEED = 0x5EED


# ----------------------------------------------------------------- helpers
def csr_of(c):
    return c.row_ptr, c.col, c.wgt


def digest_graph(c):
    return gg.sha16(c.row_ptr, c.col, c.wgt)


def lower_child_rounds(H, pr):
    """The round formulation of SURVEY §8(c) (scatter only from ACTIVE_NEW), written
    as plain Python over sets.  This is the scheme the GPU implements; here it is
    checked against Alg 3 (the oracle) on exhaustive visit orders."""
    n = len(H)
    UNDEC, ACTIVE_NEW, ACTIVE, ROOT = 0, 1, 2, 3
    status = [ROOT if H[u] == u else UNDEC for u in range(n)]
    lower = [H[y] != y and pr[y] < pr[H[y]] for y in range(n)]
    rootflag = [False] * n
    blocked = [0] * n
    r = 0
    while any(s == UNDEC for s in status):
        r += 1
        for y in range(n):
            if not lower[y]:
                continue
            x = H[y]
            if status[y] == ACTIVE_NEW:
                rootflag[x] = True
            elif status[y] == UNDEC:
                blocked[x] = r
        for y in range(n):
            if status[y] == ACTIVE_NEW:
                status[y] = ACTIVE
        for u in range(n):
            if status[u] == UNDEC:
                if rootflag[u]:
                    status[u] = ROOT
                elif blocked[u] != r:
                    status[u] = ACTIVE_NEW
    roots = sorted(u for u in range(n) if status[u] == ROOT)
    label = {x: i for i, x in enumerate(roots)}
    M = []
    for u in range(n):
        x = u
        while status[x] != ROOT:
            x = H[x]
        M.append(label[x])
    return M, len(roots), r


def random_graph(n, rng, p=0.5, wmax=3):
    edges = [(u, v, int(rng.integers(1, wmax + 1)))
             for u in range(n) for v in range(u + 1, n) if rng.random() < p]
    return gg.from_edges(n, edges)


def dense_adj(g):
    A = np.zeros((g.n, g.n), np.int64)
    for u in range(g.n):
        for e in range(g.row_ptr[u], g.row_ptr[u + 1]):
            A[u, g.col[e]] = g.wgt[e]
    return A


def check_mapping_invariants(g, H, M, nc, root):
    """SURVEY §8(c) pin M3."""
    n = g.n
    assert M.min(initial=0) >= 0 and (n == 0 or M.max() == nc - 1)
    assert len(np.unique(M)) == nc                       # every label used
    roots = np.nonzero(root)[0]
    assert len(roots) == nc                              # one root per aggregate
    assert np.array_equal(M[roots], np.arange(nc))       # ids ordered by root id (Z3)
    nonroot = np.nonzero(root == 0)[0]
    assert np.array_equal(M[nonroot], M[H[nonroot]])     # M[u] = M[H[u]]
    deg = np.diff(g.row_ptr)
    if n and deg.min() > 0:
        sizes = np.bincount(M, minlength=nc)
        assert sizes.min() >= 2                          # aggregates have >= 2 members
        assert nc <= n // 2                              # ratio >= 2 (matching bound, L61)


def check_coarse_invariants(g, M, nc, c):
    """SURVEY §8(c) pin C3: conservation, symmetry, no loops, ascending, W_c > 0."""
    assert c.row_ptr[0] == 0 and c.row_ptr[-1] == c.nnz
    assert int(c.vwgt.astype(np.int64).sum()) == int(g.vwgt.astype(np.int64).sum())
    assert int(c.wgt.astype(np.int64).sum()) + c.intra == int(g.wgt.astype(np.int64).sum())
    rows = np.repeat(np.arange(nc), np.diff(c.row_ptr))
    assert not np.any(rows == c.col)
    assert np.all(c.wgt > 0)
    d = np.diff(c.col.astype(np.int64))
    assert np.all(d[rows[1:] == rows[:-1]] > 0)
    A = sp.csr_matrix((c.wgt, c.col, c.row_ptr), shape=(nc, nc))
    assert (A != A.T).nnz == 0


def scipy_PAPt(g, M, nc):
    """Library routine pin C1: P A P^T with P(M[u], u) = 1, diagonal removed (L280)."""
    n = g.n
    A = sp.csr_matrix((g.wgt.astype(np.int64), g.col, g.row_ptr), shape=(n, n))
    P = sp.csr_matrix((np.ones(n, np.int64), (M, np.arange(n))), shape=(nc, n))
    Ac = (P @ A @ P.T).tocsr()
    Ac.setdiag(0)
    Ac.eliminate_zeros()
    Ac.sort_indices()
    return Ac


# --------------------------------------------------------------- R3 order
def test_splitmix64_known_answers(golden_dir):
    ka = json.load(open(os.path.join(golden_dir, "survey_known_answers.json")))
    for x, v in ka["splitmix64"].items():
        assert o.splitmix64(int(x)) == int(v, 16)
    assert o.splitmix64(SEED) == int(ka["prio"]["s_0"], 16)
    assert [int(p) for p in o.prio(SEED, 0, 4)] == [int(v, 16) for v in ka["prio"]["prio_0"]]


def test_prio_is_total_order_and_carries_id():
    pr = o.prio(123, 3, 100000)
    assert len(np.unique(pr)) == len(pr)
    assert np.array_equal(pr & np.uint64(0xFFFFFFFF), np.arange(100000, dtype=np.uint64))
    assert not np.array_equal(pr, o.prio(123, 4, 100000))  # fresh per level


# ----------------------------------------------------------- R2 heavy nbr
def test_heavy_grid_closed_form():
    """Unit weights: H[u] = min N(u) (first max of the strict '>' scan, L116)."""
    g = gg.grid2d(64, 64)
    H = o.heavy(g)
    for i in range(64):
        for j in range(64):
            exp = (i - 1, j) if i > 0 else ((0, j - 1) if j > 0 else (0, 1))
            assert H[i * 64 + j] == exp[0] * 64 + exp[1]


def test_heavy_brute_force_and_isolated():
    rng = np.random.default_rng(0)
    for t in range(50):
        n = int(rng.integers(1, 9))
        g = random_graph(n, rng, p=0.4, wmax=3)
        A = dense_adj(g)
        H = o.heavy(g)
        for u in range(n):
            if A[u].max() == 0:
                assert H[u] == u
            else:
                assert H[u] == int(np.flatnonzero(A[u] == A[u].max())[0])


def test_heavy_pseudoforest_only_2cycles():
    """Under R2 the functional graph of H has only 2-cycles (derived)."""
    rng = np.random.default_rng(1)
    for t in range(200):
        g = random_graph(int(rng.integers(2, 12)), rng, p=0.5, wmax=2)
        H = o.heavy(g)
        for u in range(g.n):
            seen = []
            x = u
            while x not in seen:
                seen.append(x)
                x = int(H[x])
            cyc = seen[seen.index(x):]
            assert len(cyc) in (1, 2)
            if len(cyc) == 1:
                assert g.row_ptr[x + 1] == g.row_ptr[x]  # only isolated vertices self-map


# --------------------------------------------------------- hand examples
def test_hand_examples(golden_dir):
    ex = json.load(open(os.path.join(golden_dir, "hand_examples.json")))
    g6 = ex["G6"]
    g = gg.from_edges(g6["n"], g6["edges"])
    assert o.heavy(g).tolist() == g6["H"]
    for run in g6["runs"]:
        M, nc, root = o.mapping(g, o.prio_from_order(run["order"]))
        assert M.tolist() == run["M"] and nc == run["n_c"]
        assert np.nonzero(root)[0].tolist() == run["roots"]
        c = o.coarsen(g, M, nc)
        cc = g6["coarse"]
        assert c.row_ptr.tolist() == cc["row_ptr"] and c.col.tolist() == cc["col"]
        assert c.wgt.tolist() == cc["wgt"] and c.vwgt.tolist() == cc["vwgt"]
        assert c.intra == cc["intra_directed"]
        assert int(c.wgt.sum()) + c.intra == cc["total_directed"]
    p4 = ex["P4w"]
    g = gg.from_edges(p4["n"], p4["edges"])
    assert o.heavy(g).tolist() == p4["H"]
    for run in p4["runs"]:
        M, nc, _ = o.mapping(g, o.prio_from_order(run["order"]))
        assert M.tolist() == run["M"] and nc == run["n_c"]
        c = o.coarsen(g, M, nc)
        assert c.row_ptr.tolist() == run["coarse"]["row_ptr"]
        assert c.col.tolist() == run["coarse"]["col"] and c.wgt.tolist() == run["coarse"]["wgt"]


# ------------------------------------------------------- R4 closed forms
def path(n, w=None):
    return gg.from_edges(n, [(i, i + 1, 1 if w is None else w[i]) for i in range(n - 1)])


@pytest.mark.parametrize("n", [2, 3, 4, 7, 10, 11])
def test_path_closed_forms(n):
    g = path(n)
    M, nc, _ = o.mapping(g, o.prio_from_order(range(n)))          # identity order
    assert nc == 1 and set(M.tolist()) == {0}
    if n % 2 == 0:
        M, nc, _ = o.mapping(g, o.prio_from_order(range(n - 1, -1, -1)))  # reversed
        assert nc == n // 2
        assert M.tolist() == [u // 2 for u in range(n)]                   # pairs {2k, 2k+1}


def test_star_and_clique_single_aggregate():
    rng = np.random.default_rng(2)
    star = gg.from_edges(9, [(0, i, 1) for i in range(1, 9)])
    clique = gg.from_edges(7, [(u, v, 1) for u in range(7) for v in range(u + 1, 7)])
    for g in (star, clique):
        for t in range(30):
            M, nc, _ = o.mapping(g, o.prio_from_order(rng.permutation(g.n)))
            assert nc == 1


def test_ladder_rungs():
    """Ladder with rung weight 2 > rail weight 1: M = the rungs for every order."""
    k = 6
    e = [(2 * i, 2 * i + 1, 2) for i in range(k)]
    e += [(2 * i, 2 * i + 2, 1) for i in range(k - 1)] + [(2 * i + 1, 2 * i + 3, 1) for i in range(k - 1)]
    g = gg.from_edges(2 * k, e)
    rng = np.random.default_rng(3)
    for t in range(30):
        M, nc, _ = o.mapping(g, o.prio_from_order(rng.permutation(g.n)))
        assert nc == k and M.tolist() == [u // 2 for u in range(2 * k)]


# ------------------------------------------- R4 exhaustive + characterisation
def test_exhaustive_orders_match_round_formulation():
    """All n! visit orders on random small graphs with tied weights (n <= 7):
    Alg 3 (oracle) == the exact parallel characterisation (round formulation)."""
    rng = np.random.default_rng(4)
    cases = 0
    for t in range(14):
        n = 5 if t < 8 else 7
        g = random_graph(n, rng, p=0.45, wmax=2)
        if t % 5 == 0 and n > 1:  # include an isolated vertex
            keep = [(u, g.col[e], g.wgt[e]) for u in range(n - 1)
                    for e in range(g.row_ptr[u], g.row_ptr[u + 1]) if u < g.col[e] < n - 1]
            g = gg.from_edges(n, keep)
        H = o.heavy(g).tolist()
        for order in itertools.permutations(range(n)):
            pr = o.prio_from_order(order)
            M, nc, root = o.mapping(g, pr)
            M2, nc2, _ = lower_child_rounds(H, [int(p) for p in pr])
            assert nc == nc2 and M.tolist() == M2
            cases += 1
    assert cases > 30000


def test_mapping_invariants_random():
    rng = np.random.default_rng(5)
    for t in range(40):
        g = random_graph(int(rng.integers(2, 40)), rng, p=0.2, wmax=4)
        H = o.heavy(g)
        M, nc, root = o.mapping(g, o.prio(int(rng.integers(1 << 30)), 0, g.n))
        check_mapping_invariants(g, H, M, nc, root)


def test_mapping_rejects_non_total_order():
    g = path(4)
    with pytest.raises(o.OracleError) as e:
        o.mapping(g, np.array([0, 1, 1, 2], np.uint64))
    assert e.value.code == o.EINVAL


# ------------------------------------------------------ R5 construction
def test_coarsen_matches_scipy_and_dense():
    rng = np.random.default_rng(6)
    for t in range(30):
        g = random_graph(int(rng.integers(2, 30)), rng, p=0.3, wmax=5)
        g.vwgt = rng.integers(1, 4, g.n).astype(np.int32)
        nc = int(rng.integers(1, g.n + 1))
        M = rng.integers(0, nc, g.n).astype(np.int32)
        M[:nc] = np.arange(nc)  # every label used
        c = o.coarsen(g, M, nc)
        Ac = scipy_PAPt(g, M, nc)
        assert np.array_equal(c.row_ptr, Ac.indptr) and np.array_equal(c.col, Ac.indices)
        assert np.array_equal(c.wgt, Ac.data)
        # dense pin C2
        P = np.zeros((nc, g.n), np.int64)
        P[M, np.arange(g.n)] = 1
        D = P @ dense_adj(g) @ P.T
        intra = int(np.trace(D))
        np.fill_diagonal(D, 0)
        assert np.array_equal(D, dense_adj_c(c, nc)) and intra == c.intra
        assert np.array_equal(c.vwgt, np.bincount(M, weights=g.vwgt, minlength=nc).astype(np.int32))
        check_coarse_invariants(g, M, nc, c)


def dense_adj_c(c, nc):
    D = np.zeros((nc, nc), np.int64)
    for a in range(nc):
        for e in range(c.row_ptr[a], c.row_ptr[a + 1]):
            D[a, c.col[e]] = c.wgt[e]
    return D


def test_coarsen_c1_levels_match_scipy():
    g = gg.config(1)
    H = o.hierarchy(g, 50, SEED)
    cur = g
    for lv in H.levels:
        Ac = scipy_PAPt(cur, lv.M, lv.n_c)
        c = lv.graph
        assert np.array_equal(c.row_ptr, Ac.indptr) and np.array_equal(c.col, Ac.indices)
        assert np.array_equal(c.wgt, Ac.data)
        check_coarse_invariants(cur, lv.M, lv.n_c, c)
        cur = c


def test_coarsen_overflow_detected():
    big = 2**31 - 1
    g = gg.from_edges(3, [(0, 2, big), (1, 2, big)])
    M = np.array([0, 0, 1], np.int32)
    with pytest.raises(o.OracleError) as e:
        o.coarsen(g, M, 2)
    assert e.value.code == o.EOVERFLOW


def test_coarsen_rejects_bad_labels():
    g = path(3)
    with pytest.raises(o.OracleError):
        o.coarsen(g, np.array([0, 2, 1], np.int32), 2)


# -------------------------------------------------------- R6 hierarchy
def _hier_answers(H):
    out = []
    for lv in H.levels:
        out.append((lv.n_c, lv.graph.nnz, int(lv.graph.wgt.astype(np.int64).sum())))
    return out


def test_hierarchy_c1_known_answers(golden_dir):
    ka = json.load(open(os.path.join(golden_dir, "survey_known_answers.json")))["C1"]
    g = gg.config(1)
    H = o.hierarchy(g, 50, SEED)
    assert [lv.n_c for lv in H.levels] == ka["n_c"]
    assert [lv.graph.nnz for lv in H.levels] == ka["nnz_c"]
    assert [int(lv.graph.wgt.sum()) for lv in H.levels] == ka["sum_wc"]
    assert gg.sha16(H.levels[0].M) == ka["sha_M1"]
    assert digest_graph(H.levels[0].graph) == ka["sha_G1"]
    assert H.stop_reason == o.STOP_CUTOFF
    # rounds of the parallel formulation (independent model's count)
    cur = g
    rounds = []
    for lv, level in zip(H.levels, range(len(H.levels))):
        Hh = o.heavy(cur).tolist()
        M2, nc2, r = lower_child_rounds(Hh, [int(p) for p in o.prio(SEED, level, cur.n)])
        assert M2 == lv.M.tolist() and nc2 == lv.n_c
        rounds.append(r)
        cur = lv.graph
    assert rounds == ka["rounds"]


@pytest.mark.parametrize("idx", [0, 1, 2, 3])
def test_hierarchy_rmat_known_answers(golden_dir, idx):
    r = json.load(open(os.path.join(golden_dir, "survey_known_answers.json")))["rmat"][idx]
    g = gg.rmat(r["scale"], r["ef"])
    H = o.hierarchy(g, 50, SEED)
    assert len(H.levels) == len(r["levels"])
    for lv, exp in zip(H.levels, r["levels"]):
        n, nc, nnzc, rounds, shaM, shaG, swc = exp
        assert (lv.n_c, lv.graph.nnz, int(lv.graph.wgt.sum())) == (nc, nnzc, swc)
        assert gg.sha16(lv.M) == shaM and digest_graph(lv.graph) == shaG
    if r["discarded"] is None:
        assert H.stop_reason == o.STOP_CUTOFF
    else:
        assert H.stop_reason == o.STOP_DISCARD and H.discarded_n_c == r["discarded"]


def test_hierarchy_c2_known_answers(golden_dir):
    ka = json.load(open(os.path.join(golden_dir, "survey_known_answers.json")))["C2"]
    g = gg.config(2)
    H = o.hierarchy(g, 1000, SEED)
    assert [lv.n_c for lv in H.levels] == ka["n_c"]
    assert [lv.graph.nnz for lv in H.levels] == ka["nnz_c"]
    assert int(H.levels[0].graph.wgt.sum()) == ka["sum_wc_L1"]
    assert gg.sha16(H.levels[0].M) == ka["sha_M1"]
    assert digest_graph(H.levels[0].graph) == ka["sha_G1"]
    # each level shrinks and the per-level ratio respects the matching bound (L61)
    ns = [g.n] + ka["n_c"]
    assert all(a >= 2 * b for a, b in zip(ns, ns[1:]))


def test_hierarchy_edge_cases():
    empty = gg.Graph(np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0, np.int32),
                     np.zeros(0, np.int32))
    H = o.hierarchy(empty, 50, SEED)
    assert H.levels == [] and H.stop_reason == o.STOP_CUTOFF
    small = path(20)
    assert o.hierarchy(small, 50, SEED).levels == []
    # all isolated -> n_c == n -> stall
    iso = gg.Graph(np.zeros(61, np.int64), np.zeros(0, np.int32), np.zeros(0, np.int32),
                   np.ones(60, np.int32))
    H = o.hierarchy(iso, 50, SEED)
    assert H.levels == [] and H.stop_reason == o.STOP_STALL
    # a star of 60 collapses to 1 < 10 in one step -> discard
    star = gg.from_edges(60, [(0, i, 1) for i in range(1, 60)])
    H = o.hierarchy(star, 50, SEED)
    assert H.levels == [] and H.stop_reason == o.STOP_DISCARD and H.discarded_n_c == 1
    # max levels
    H = o.hierarchy(gg.config(1), 50, SEED, max_levels=2)
    assert len(H.levels) == 2 and H.stop_reason == o.STOP_MAX_LEVELS
