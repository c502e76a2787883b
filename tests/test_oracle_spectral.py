"""Pins of the multilevel spectral bisection oracle (PAPER.md
L330 / L367): closed forms (a path's Fiedler ordering and cut 1; two cliques
joined by one edge split along the bridge; the 64x64 grid's second eigenvalue
2 - 2 cos(pi / 64)), the eigen-residual of the converged vector, exact balance."""
import numpy as np

import graphgen as gg
import oracle as o
from oracle import spectral as S


def path(n):
    return gg.from_edges(n, [(i, i + 1, 1) for i in range(n - 1)])


def test_path_single_level():
    g = path(40)
    part, x, cut, iters = S.spectral_bisection(g, [], max_iter=200000, tol=1e-12)
    assert cut == 1 and int((part == 0).sum()) == 20
    assert (part[:20] == part[0]).all() and (part[20:] != part[0]).all()
    assert np.all(np.diff(x) > 0) or np.all(np.diff(x) < 0)  # monotone along the path


def test_barbell_cut_is_the_bridge():
    k = 12
    edges = [(u, v, 1) for u in range(k) for v in range(u + 1, k)]
    edges += [(k + u, k + v, 1) for u in range(k) for v in range(u + 1, k)] + [(k - 1, k, 1)]
    g = gg.from_edges(2 * k, edges)
    part, _, cut, _ = S.spectral_bisection(g, [], max_iter=100000, tol=1e-12)
    assert cut == 1 and len(set(part[:k])) == 1 and len(set(part[k:])) == 1


def test_grid_fiedler_value_and_residual():
    """64x64 grid: lambda_2 = 2 - 2 cos(pi/64) (a product of two paths), and the
    converged iterate satisfies L x = lambda x."""
    g = gg.config(1)
    H = o.hierarchy(g, 50, gg.COARSEN_SEED)
    part, x, cut, iters = S.spectral_bisection(g, [(lv.M, lv.graph) for lv in H.levels], max_iter=200000, tol=1e-13)
    A, d = S.laplacian_parts(g.row_ptr, g.col, g.wgt)
    Lx = d * x - A @ x
    lam = float(x @ Lx)
    assert abs(lam - (2 - 2 * np.cos(np.pi / 64))) < 1e-8
    assert np.linalg.norm(Lx - lam * x) < 1e-5
    assert int((part == 0).sum()) == g.n // 2
    assert cut == 64  # a straight cut through the middle of the grid


def test_interpolation_uses_the_mapping():
    g = gg.config(1)
    H = o.hierarchy(g, 50, gg.COARSEN_SEED)
    levels = [(lv.M, lv.graph) for lv in H.levels]
    # zero iterations on every level: x0 of the coarsest graph, carried down by M
    part, x, _, iters = S.spectral_bisection(g, levels, max_iter=0)
    xc = S.start_vector(levels[-1][1].n, 0x5EED)
    xc = (xc - xc.mean()) / np.linalg.norm(xc - xc.mean())
    for M, _ in reversed(levels):
        xc = xc[M]
        xc = (xc - xc.mean()) / np.linalg.norm(xc - xc.mean())
    assert np.allclose(x, xc) and iters == [0] * (len(levels) + 1)
