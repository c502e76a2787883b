"""Parity of the other mapping methods on the GPU against
the oracle, bit for bit: HEC3 (Alg 5) and HEM (Alg 2), single levels and whole
hierarchies (the same construction), every visit order of small graphs for HEM,
and full-size single levels of C3/C4 against sampled oracle properties."""
import itertools

import numpy as np
import pytest
import torch

import graphgen as gg
import oracle as o

pytestmark = pytest.mark.gpu
SEED = 0x5EED


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_gilbertabmr21_b200 as P
    assert torch.cuda.is_available()
    return P


@pytest.fixture(scope="module")
def ctx(P):
    c = P.Context()
    yield c
    c.close()


def dev(P, g):
    return P.DeviceGraph.from_host(g)


def random_graph(n, rng, p=0.3, wmax=3, isolated=0):
    edges = [(u, v, int(rng.integers(1, wmax + 1)))
             for u in range(n - isolated) for v in range(u + 1, n - isolated) if rng.random() < p]
    return gg.from_edges(n, edges)


def prio_tensor(pr):
    return torch.from_numpy(pr.view(np.int64).copy()).cuda()


GRAPHS = {"c1": lambda: gg.config(1), "c2": lambda: gg.config(2), "rmat14": lambda: gg.rmat(14, 16),
          "rmat17": lambda: gg.rmat(17, 16), "mesh27_20": lambda: gg.mesh27(20, 20, 20)}


@pytest.mark.parametrize("which", list(GRAPHS))
@pytest.mark.parametrize("method", ["hec3", "hem"])
def test_mapping_method_parity(P, ctx, which, method):
    g = GRAPHS[which]()
    dg = dev(P, g)
    for level in (0, 2):
        M, nc = P.hec_find_mapping_method(ctx, dg, method, SEED, level)
        Mo, nco, _ = o.map_level(g, SEED, level, method)
        assert nc == nco and np.array_equal(M.cpu().numpy(), Mo)


def test_mapping_methods_random_graphs(P, ctx):
    rng = np.random.default_rng(51)
    for t in range(30):
        g = random_graph(int(rng.integers(1, 150)), rng, p=0.05, wmax=4, isolated=int(rng.integers(0, 3)))
        dg = dev(P, g)
        for method in ("hec3", "hem"):
            M, nc = P.hec_find_mapping_method(ctx, dg, method, SEED, t)
            Mo, nco, _ = o.map_level(g, SEED, t, method)
            assert nc == nco and np.array_equal(M.cpu().numpy(), Mo), (t, method)


def test_hem_all_visit_orders(P, ctx):
    rng = np.random.default_rng(52)
    for t in range(3):
        g = random_graph(6, rng, p=0.5, wmax=2, isolated=t % 2)
        dg = dev(P, g)
        for order in itertools.permutations(range(6)):
            pr = o.prio_from_order(order)
            M, nc = P.hec_find_mapping_method(ctx, dg, "hem", prio=prio_tensor(pr))
            Mo, nco, _ = o.mapping_hem(g, pr)
            assert nc == nco and np.array_equal(M.cpu().numpy(), Mo)


@pytest.mark.parametrize("method", ["hec3", "hem"])
@pytest.mark.parametrize("which,cutoff", [("c1", 50), ("rmat14", 50), ("mesh27_20", 100)])
def test_method_hierarchies(P, ctx, method, which, cutoff):
    g = GRAPHS[which]()
    H = P.coarsen_hierarchy(ctx, dev(P, g), cutoff, SEED, method=method)
    ref = o.hierarchy(g, cutoff, SEED, method=method)
    assert len(H.levels) == len(ref.levels) and H.stop_reason == ref.stop_reason
    for lv, lo in zip(H.levels, ref.levels):
        rp, col, wgt, vw = lv.graph.to_host()
        assert np.array_equal(lv.M.cpu().numpy(), lo.M)
        assert np.array_equal(rp, lo.graph.row_ptr) and np.array_equal(col, lo.graph.col)
        assert np.array_equal(wgt, lo.graph.wgt) and np.array_equal(vw, lo.graph.vwgt)
    H.free()


@pytest.mark.parametrize("method", ["hec3", "hem"])
def test_method_full_size_c3(P, ctx, method):
    """C3 level 0 (2.4M vertices, 128M entries): the whole M against the oracle."""
    g = gg.config(3)
    M, nc = P.hec_find_mapping_method(ctx, dev(P, g), method, SEED, 0)
    Mo, nco, _ = o.map_level(g, SEED, 0, method)
    assert nc == nco and np.array_equal(M.cpu().numpy(), Mo)
