"""Multilevel spectral bisection -- TEST INFRASTRUCTURE ONLY.

Plain fp64 numpy / scipy, following PAPER.md §III-C (L330) and L367 step by
step; only tests/ and bench.py's reference legs may import it.

  * Laplacian L = D - A of each level's weighted graph (reading Z18: the plain
    combinatorial Laplacian; vertex weights are not used).
  * Power iteration for the eigenvector of the second-smallest eigenvalue of L
    (L330): x <- (sigma I - L) x with sigma = 2 max weighted degree (>= the
    largest eigenvalue, Gershgorin), projected off the constant null vector
    (x <- x - mean(x)) and normalised every iteration.
  * Stop when the 2-norm of the difference of successive iterates is below tol
    (L367: 1e-10; reading Z18: ||x_{k+1} - x_k||_2, the iterates being unit
    vectors), or after max_iter iterations per level.
  * Coarsest level first from a seeded start vector x0[u] = (splitmix64(seed ^
    u) >> 11) * 2^-53 - 1/2; interpolation x_fine[u] = x_coarse[M[u]] (L330:
    "the interpolation step ... uses the mapping vectors").
  * Bisection without imbalance (L330): the n // 2 vertices with the smallest
    (x, id) form part 0.  Edge cut = sum of the weights of undirected edges
    whose ends lie in different parts.
"""
from __future__ import annotations

import numpy as np
import scipy.sparse as sp

from . import splitmix64


def start_vector(n: int, seed: int) -> np.ndarray:
    x = np.empty(n, np.float64)
    for u in range(n):
        x[u] = (splitmix64((seed ^ u) & 0xFFFFFFFFFFFFFFFF) >> 11) * (1.0 / (1 << 53)) - 0.5
    return x


def laplacian_parts(row_ptr, col, wgt):
    n = row_ptr.shape[0] - 1
    A = sp.csr_matrix((wgt.astype(np.float64), col, row_ptr), shape=(n, n))
    d = np.asarray(A.sum(axis=1)).ravel()
    return A, d


def fiedler_power(row_ptr, col, wgt, x, max_iter: int, tol: float):
    """Power iteration on (sigma I - L) from x; returns (x, iterations, last delta)."""
    A, d = laplacian_parts(row_ptr, col, wgt)
    sigma = 2.0 * (d.max() if d.size else 0.0)
    x = x - x.mean()
    nx = np.linalg.norm(x)
    if nx > 0:
        x = x / nx
    delta, it = np.inf, 0
    for it in range(1, max_iter + 1):
        y = (sigma - d) * x + A @ x   # (sigma I - L) x with L x = d x - A x
        y = y - y.mean()
        ny = np.linalg.norm(y)
        if ny > 0:
            y = y / ny
        delta = np.linalg.norm(y - x)
        x = y
        if delta < tol:
            break
    return x, it, delta


def bisect(x: np.ndarray) -> np.ndarray:
    n = x.shape[0]
    order = np.lexsort((np.arange(n), x))   # by value, ties by vertex id
    part = np.ones(n, np.uint8)
    part[order[: n // 2]] = 0
    return part


def edge_cut(row_ptr, col, wgt, part) -> int:
    rows = np.repeat(np.arange(row_ptr.shape[0] - 1), np.diff(row_ptr))
    cut = part[rows] != part[col]
    return int(wgt[cut].astype(np.int64).sum()) // 2


def spectral_bisection(g0, levels, max_iter: int = 1000, tol: float = 1e-10, seed: int = 0x5EED):
    """g0: the fine graph; levels: [(M_i, G_i)] of the hierarchy (M_i maps
    G_{i-1} -> G_i).  Returns (part u8[n0], x f64[n0], cut, iterations per level
    from the coarsest)."""
    graphs = [(g0.row_ptr, g0.col, g0.wgt)] + [(G.row_ptr, G.col, G.wgt) for _, G in levels]
    x = start_vector(graphs[-1][0].shape[0] - 1, seed)
    iters = []
    for lvl in range(len(graphs) - 1, -1, -1):
        x, it, _ = fiedler_power(*graphs[lvl], x, max_iter, tol)
        iters.append(it)
        if lvl > 0:
            x = x[levels[lvl - 1][0]]   # interpolation with the mapping vector
    part = bisect(x)
    return part, x, edge_cut(g0.row_ptr, g0.col, g0.wgt, part), iters
