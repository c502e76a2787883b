"""Multilevel spectral bisection on the GPU against the fp64
oracle (oracle/spectral.py): same hierarchy, same start vector, same
iteration counts (tol = 0 runs exactly max_iter per level) -> the iterates
agree to 1e-9 (different summation orders only), the split is exactly
balanced and equal to the oracle's away from near-ties; closed-form cuts for a
path and a barbell; the tolerance stop (L367) converges to the same vector."""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle as o
from oracle import spectral as S

pytestmark = pytest.mark.gpu
SEED = 0x5EED


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_gilbertabmr21_b200 as P
    return P


@pytest.fixture(scope="module")
def ctx(P):
    c = P.Context()
    yield c
    c.close()


def run_both(P, ctx, g, cutoff, max_iter, tol):
    H = P.coarsen_hierarchy(ctx, P.DeviceGraph.from_host(g), cutoff, SEED)
    part, x, cut, iters = P.spectral_bisection(ctx, P.DeviceGraph.from_host(g), H, max_iter, tol, SEED)
    ref = o.hierarchy(g, cutoff, SEED)
    rp, rx, rcut, riters = S.spectral_bisection(g, [(lv.M, lv.graph) for lv in ref.levels], max_iter, tol, SEED)
    out = part.cpu().numpy(), x.cpu().numpy(), cut, iters, rp, rx, rcut, riters
    H.free()
    return out


@pytest.mark.parametrize("which,cutoff", [("c1", 50), ("mesh27_16", 50), ("rmat12", 50)])
def test_spectral_fixed_iterations(P, ctx, which, cutoff):
    g = {"c1": lambda: gg.config(1), "mesh27_16": lambda: gg.mesh27(16, 16, 16),
         "rmat12": lambda: gg.rmat(12, 16)}[which]()
    part, x, cut, iters, rp, rx, rcut, riters = run_both(P, ctx, g, cutoff, 200, 0.0)
    assert iters == riters == [200] * len(iters)
    assert np.max(np.abs(x - rx)) < 1e-9
    assert int((part == 0).sum()) == g.n // 2
    xm = np.sort(rx)[g.n // 2]
    clear = np.abs(rx - xm) > 1e-7  # away from the median, the sides must agree
    assert np.array_equal(part[clear], rp[clear])
    assert cut == S.edge_cut(g.row_ptr, g.col, g.wgt, part)


def test_spectral_tolerance_stop(P, ctx):
    g = gg.config(1)
    part, x, cut, iters, rp, rx, rcut, riters = run_both(P, ctx, g, 50, 20000, 1e-10)
    assert all(abs(a - b) <= 2 for a, b in zip(iters, riters))
    assert np.max(np.abs(x - rx)) < 1e-6
    assert cut == rcut == 64  # the grid's straight middle cut


def test_spectral_closed_forms(P, ctx):
    for g in (gg.from_edges(40, [(i, i + 1, 1) for i in range(39)]),
              gg.from_edges(24, [(u, v, 1) for u in range(12) for v in range(u + 1, 12)]
                            + [(12 + u, 12 + v, 1) for u in range(12) for v in range(u + 1, 12)] + [(11, 12, 1)])):
        H = P.coarsen_hierarchy(P.Context(), P.DeviceGraph.from_host(g), 10 ** 9, SEED)  # no levels: G0 only
        part, x, cut, iters = P.spectral_bisection(ctx, P.DeviceGraph.from_host(g), H, 200000, 1e-12, SEED)
        assert cut == 1 and int((part == 0).sum()) == g.n // 2
