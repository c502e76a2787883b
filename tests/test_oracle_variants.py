"""Pins of the oracle's other mapping methods, -m "not gpu":
HEC3 (Alg 5) and HEM (Alg 2).  Hand-computed
examples, closed forms, an independent formulation of each (union-find
components for HEC3; a round-based parallel characterisation for HEM, checked
on every visit order of small graphs), and the invariants the paper states
(HEM is a matching: coarsening ratio <= 2)."""
import itertools

import numpy as np
import pytest

import graphgen as gg
import oracle as o

G6 = [(0, 1, 3), (1, 2, 1), (2, 3, 2), (3, 4, 2), (4, 5, 1), (1, 4, 1), (0, 5, 1)]


def path(n, w=1):
    return gg.from_edges(n, [(i, i + 1, w) for i in range(n - 1)])


def canon(M):
    """Partition of the vertices as a canonical label array (first occurrence order)."""
    seen, out = {}, []
    for x in M:
        out.append(seen.setdefault(int(x), len(seen)))
    return out


def random_graph(n, rng, p=0.4, wmax=3, isolated=0):
    edges = [(u, v, int(rng.integers(1, wmax + 1)))
             for u in range(n - isolated) for v in range(u + 1, n - isolated) if rng.random() < p]
    return gg.from_edges(n, edges)


# ------------------------------------------------------------------ HEC3
def test_hec3_hand_example():
    g = gg.from_edges(6, G6)
    M, nc, root = o.mapping_hec3(g)
    # H = [1,0,3,2,3,0]: mutual pairs (0,1) -> root 0 and (2,3) -> root 2;
    # 4 and 5 (in-degree 0) inherit from 3 and 0
    assert nc == 2 and M.tolist() == [0, 0, 1, 1, 1, 0] and root.tolist() == [1, 0, 1, 0, 0, 0]


@pytest.mark.parametrize("n", [4, 5, 9, 50])
def test_hec3_path_closed_form(n):
    """Unit path: H[0] = 1, H[u] = u - 1 -> {0,1}, {2}, ..., {n-3}, {n-2, n-1}."""
    M, nc, _ = o.mapping_hec3(path(n))
    exp = [0, 0] + list(range(1, n - 3)) + [n - 3, n - 3]
    assert nc == n - 2 and M.tolist() == exp


def test_hec3_star_clique_ladder():
    star = gg.from_edges(9, [(0, v, 1) for v in range(1, 9)])
    assert o.mapping_hec3(star)[1] == 1
    clique = gg.from_edges(7, [(u, v, 1) for u in range(7) for v in range(u + 1, 7)])
    assert o.mapping_hec3(clique)[1] == 1
    k = 10  # rungs (2k, 2k+1) of weight 2, rails of weight 1: H = rung partner, all mutual
    ladder = gg.from_edges(2 * k, [(2 * i, 2 * i + 1, 2) for i in range(k)]
                           + [(2 * i, 2 * i + 2, 1) for i in range(k - 1)]
                           + [(2 * i + 1, 2 * i + 3, 1) for i in range(k - 1)])
    M, nc, _ = o.mapping_hec3(ladder)
    assert nc == k and M.tolist() == [i // 2 for i in range(2 * k)]


def test_hec3_union_find_formulation():
    """Independent formulation: the aggregates are the connected components of
    {u, H[u]} over vertices of in-degree 0 in the heavy-neighbour pseudoforest,
    plus the mutual pairs."""
    rng = np.random.default_rng(7)
    for t in range(60):
        n = int(rng.integers(1, 40))
        g = random_graph(n, rng, p=0.15, wmax=4, isolated=int(rng.integers(0, 3)))
        H = o.heavy(g)
        indeg = np.bincount(H[H != np.arange(n)], minlength=n) if n else np.zeros(0, int)
        parent = list(range(n))

        def find(x):
            while parent[x] != x:
                parent[x] = parent[parent[x]]
                x = parent[x]
            return x
        for u in range(n):
            v = int(H[u])
            if v != u and (indeg[u] == 0 or H[v] == u):
                parent[find(u)] = find(v)
        M, nc, root = o.mapping_hec3(g)
        comp = [find(u) for u in range(n)]
        assert canon(M) == canon(comp) and nc == len(set(comp))
        # one root per aggregate, never a vertex of in-degree 0 (unless isolated),
        # coarse ids ascending with the root (FINDUNIQANDRELABEL, reading Z3)
        roots = np.flatnonzero(root)
        assert len(roots) == nc and M[roots].tolist() == list(range(nc))
        assert all(indeg[r] > 0 or H[r] == r for r in roots)


# ------------------------------------------------------------------- HEM
def test_hem_hand_examples():
    g = gg.from_edges(6, G6)
    M, nc, _ = o.mapping_hem(g, o.prio_from_order(range(6)))
    assert nc == 3 and M.tolist() == [0, 0, 1, 1, 2, 2]
    M, nc, _ = o.mapping_hem(g, o.prio_from_order([5, 4, 3, 2, 1, 0]))
    # 5 takes 0 (tie 0/4 -> smaller id), 4 takes 3, 2 takes 1: roots 2, 4, 5
    assert nc == 3 and M.tolist() == [2, 0, 0, 1, 1, 2]


@pytest.mark.parametrize("n", [2, 7, 10])
def test_hem_path_and_star_closed_forms(n):
    M, nc, _ = o.mapping_hem(path(n), o.prio_from_order(range(n)))
    assert nc == (n + 1) // 2 and M.tolist() == [i // 2 for i in range(n)]
    k = n
    star = gg.from_edges(k + 1, [(0, v, 1) for v in range(1, k + 1)])
    for order in (range(k + 1), list(range(1, k + 1)) + [0]):
        M, nc, _ = o.mapping_hem(star, o.prio_from_order(order))
        assert nc == k  # one leaf pairs with the centre, the rest stay single


def hem_rounds(g, pr):
    """Round-based characterisation (independent of Alg 2's loop): an undecided
    u is decided once no undecided lower-priority vertex is adjacent to u, nor
    to u's heaviest undecided neighbour x (first maximum: smallest id); it then
    pairs with x (or stays single).  Coarse ids by ascending root (the decider)."""
    n = g.n
    adj = [[(int(g.col[e]), int(g.wgt[e])) for e in range(g.row_ptr[u], g.row_ptr[u + 1])] for u in range(n)]
    state = [-1] * n  # -1 undecided, else root id
    while -1 in state:
        und = [u for u in range(n) if state[u] == -1]
        minp = {u: min([pr[v] for v, _ in adj[u] if state[v] == -1] + [2**64]) for u in und}
        dec = []
        for u in und:
            if minp[u] < pr[u]:
                continue
            best, x = 0, -1
            for v, w in adj[u]:
                if state[v] == -1 and w > best:
                    best, x = w, v
            if x >= 0 and min(pr[y] for y, _ in adj[x] if state[y] == -1) < pr[u]:
                continue
            dec.append((u, x))
        assert dec, "no progress"
        for u, x in dec:
            state[u] = u
            if x >= 0:
                state[x] = u
    roots = sorted(set(state))
    return np.array([roots.index(r) for r in state], np.int32), len(roots)


def test_hem_rounds_match_alg2_all_orders():
    rng = np.random.default_rng(11)
    cases = 0
    for t in range(6):
        n = 6
        g = random_graph(n, rng, p=0.5, wmax=2, isolated=t % 2)
        for order in itertools.permutations(range(n)):
            pr = o.prio_from_order(order)
            M, nc, _ = o.mapping_hem(g, pr)
            Mr, ncr = hem_rounds(g, [int(x) for x in pr])
            assert nc == ncr and np.array_equal(M, Mr)
            cases += 1
    assert cases == 6 * 720


def test_hem_is_a_maximal_matching():
    rng = np.random.default_rng(12)
    for t in range(40):
        n = int(rng.integers(2, 60))
        g = random_graph(n, rng, p=0.1, wmax=5, isolated=int(rng.integers(0, 3)))
        pr = o.prio(0x5EED, t, n)
        M, nc, _ = o.mapping_hem(g, pr)
        sizes = np.bincount(M, minlength=nc)
        assert sizes.max() <= 2 and nc >= (n + 1) // 2  # coarsening ratio <= 2
        edges = {(u, int(v)) for u in range(n) for v in g.col[g.row_ptr[u]:g.row_ptr[u + 1]]}
        for c in np.flatnonzero(sizes == 2):
            a, b = np.flatnonzero(M == c)
            assert (int(a), int(b)) in edges  # pairs are edges
        single = sizes[M] == 1
        for u, v in edges:
            assert not (single[u] and single[v])  # maximal


def test_variant_hierarchies_conserve_and_shrink():
    g = gg.config(1)
    for method in ("hec3", "hem"):
        H = o.hierarchy(g, 50, gg.COARSEN_SEED, method=method)
        n = g.n
        for lv in H.levels:
            assert lv.n_c < n and int(lv.graph.vwgt.sum()) == g.n
            n = lv.n_c
        assert H.levels and (n <= 50 or H.stop_reason != o.STOP_CUTOFF)
