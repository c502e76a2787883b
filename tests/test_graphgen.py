"""Input generators: closed-form counts, G-spec hashes, determinism,
and the graph-model invariants of PAPER.md:L59 (undirected, no self-loops, no
parallel edges, positive weights) plus connectivity (LCC, L336)."""
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp
import scipy.sparse.csgraph as csg

import graphgen as gg


def check_graph_model(g):
    n = g.n
    rp, col = g.row_ptr, g.col
    assert rp[0] == 0 and rp[-1] == g.nnz and np.all(np.diff(rp) >= 0)
    assert col.min(initial=0) >= 0 and col.max(initial=-1) < n
    rows = np.repeat(np.arange(n), np.diff(rp))
    assert not np.any(rows == col), "self-loop"
    # strictly ascending within rows
    d = np.diff(col.astype(np.int64))
    same_row = rows[1:] == rows[:-1]
    assert np.all(d[same_row] > 0), "unsorted or duplicate columns"
    A = sp.csr_matrix((g.wgt, col, rp), shape=(n, n))
    assert (A != A.T).nnz == 0, "not symmetric"
    return A


def test_grid2d_counts():
    g = gg.grid2d(64, 64)
    assert g.n == 4096 and g.nnz == 16128  # 2*(2*64*63)
    A = check_graph_model(g)
    deg = np.diff(g.row_ptr)
    assert sorted(set(deg.tolist())) == [2, 3, 4]
    assert int((deg == 2).sum()) == 4 and int((deg == 3).sum()) == 4 * 62
    assert csg.connected_components(A, directed=False)[0] == 1


def test_mesh27_counts_small():
    for shape in [(3, 3, 3), (4, 5, 6), (1, 1, 7)]:
        g = gg.mesh27(*shape)
        nx, ny, nz = shape
        # closed form: per axis, the number of ordered (i,i') pairs with |i-i'|<=1 is 3n-2
        tot = (3 * nx - 2) * (3 * ny - 2) * (3 * nz - 2) - nx * ny * nz
        assert g.nnz == tot
        check_graph_model(g)


def test_mesh27_c2_size():
    g = gg.mesh27(128, 128, 128)
    assert g.n == 2097152 and g.nnz == 53645816
    assert (3 * 128 - 2) ** 3 - 128 ** 3 == 53645816


def test_rmat_known_hashes(golden_dir):
    ka = json.load(open(os.path.join(golden_dir, "survey_known_answers.json")))
    for r in ka["rmat"]:
        if r["scale"] > 16:
            continue
        g = gg.rmat(r["scale"], r["ef"])
        assert (g.n, g.nnz) == (r["n"], r["nnz"])
        assert int(np.diff(g.row_ptr).max()) == r["maxdeg"]
        assert gg.sha16(g.row_ptr, g.col) == r["sha_G0"]


def test_rmat_thread_count_independent():
    a = gg.rmat(12, 8, seed=7, threads=1)
    b = gg.rmat(12, 8, seed=7, threads=8)
    assert np.array_equal(a.row_ptr, b.row_ptr) and np.array_equal(a.col, b.col)
    c = gg.rmat(12, 8, seed=8)
    assert not (c.nnz == a.nnz and np.array_equal(c.col, a.col))


def test_rmat_graph_model_and_lcc():
    g = gg.rmat(14, 16)
    A = check_graph_model(g)
    assert csg.connected_components(A, directed=False)[0] == 1
    deg = np.diff(g.row_ptr)
    assert deg.min() >= 1
    # skewed: max degree far above average (Table I's skew measure Δ/(2m/n), L343)
    assert deg.max() / deg.mean() > 20


def test_from_edges():
    g = gg.from_edges(3, [(0, 1, 5), (1, 2, 7)])
    assert g.row_ptr.tolist() == [0, 1, 3, 4]
    assert g.col.tolist() == [1, 0, 2, 1] and g.wgt.tolist() == [5, 5, 7, 7]
