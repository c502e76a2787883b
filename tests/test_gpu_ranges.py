"""Range variants of the C-ABI (the multi-GPU building blocks) reproduce the
whole-graph calls exactly when their ranges are stitched together."""
import ctypes

import numpy as np
import pytest
import torch

import graphgen as gg

pytestmark = pytest.mark.gpu
SEED = 0x5EED


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_gilbertabmr21_b200 as P
    return P


def split(n, parts):
    from paper_conf_ipps_gilbertabmr21_b200.dist import even_ranges
    return even_ranges(n, parts)


@pytest.mark.parametrize("which", ["c1", "rmat14"])
def test_heavy_and_mapping_ranges(P, which):
    L = P.load()
    g = gg.config(1) if which == "c1" else gg.rmat(14, 16)
    ctx = P.Context()
    dg = P.DeviceGraph.from_host(g)
    gc = dg.c()
    H_full = P.hec_debug_heavy(ctx, dg)
    H = torch.full((g.n,), -7, dtype=torch.int32, device="cuda")
    for lo, hi in split(g.n, 3):
        assert L.hec_heavy_range(ctx.h, ctypes.byref(gc), lo, hi, H.data_ptr()) == 0, L.hec_last_error()
    torch.cuda.synchronize()
    assert torch.equal(H, H_full)
    M_full, nc_full = P.hec_find_mapping(ctx, dg, SEED, 2)
    M = torch.full((g.n,), -7, dtype=torch.int32, device="cuda")
    for lo, hi in split(g.n, 3):
        nc = ctypes.c_int64()
        assert L.hec_mapping_from_heavy(ctx.h, ctypes.byref(gc), H.data_ptr(), SEED, 2, lo, hi, M.data_ptr(),
                                        ctypes.byref(nc)) == 0, L.hec_last_error()
        assert nc.value == nc_full
    torch.cuda.synchronize()
    assert torch.equal(M, M_full)


@pytest.mark.parametrize("which,parts", [("c1", 2), ("c1", 5), ("rmat14", 3), ("rmat17", 4)])
def test_construction_ranges(P, which, parts):
    L = P.load()
    g = {"c1": lambda: gg.config(1), "rmat14": lambda: gg.rmat(14, 16), "rmat17": lambda: gg.rmat(17, 16)}[which]()
    ctx = P.Context()
    dg = P.DeviceGraph.from_host(g)
    gc = dg.c()
    M, nc = P.hec_find_mapping(ctx, dg, SEED, 0)
    full = P.build_coarse_graph(ctx, dg, M, nc).graph
    rp, col, wgt, vw = full.to_host()
    bounds = (ctypes.c_int64 * (parts + 1))()
    assert L.hec_balance_rows(ctx.h, ctypes.byref(gc), M.data_ptr(), nc, parts, bounds) == 0, L.hec_last_error()
    b = list(bounds)
    assert b[0] == 0 and b[-1] == nc and all(x <= y for x, y in zip(b, b[1:]))
    off = 0
    for r in range(parts):
        a0, a1 = b[r], b[r + 1]
        rows = a1 - a0
        counts = torch.empty(max(rows, 1), dtype=torch.int64, device="cuda")
        k = ctypes.c_int64()
        assert L.hec_build_rows_count(ctx.h, ctypes.byref(gc), M.data_ptr(), nc, a0, a1, counts.data_ptr(),
                                      ctypes.byref(k)) == 0, L.hec_last_error()
        k = k.value
        assert k == rp[a1] - rp[a0]
        if rows:
            assert np.array_equal(counts[:rows].cpu().numpy(), np.diff(rp[a0:a1 + 1]))
        orp = torch.empty(rows + 1, dtype=torch.int64, device="cuda")
        ocol = torch.empty(max(k, 1), dtype=torch.int32, device="cuda")
        owgt = torch.empty(max(k, 1), dtype=torch.int32, device="cuda")
        ovw = torch.empty(max(rows, 1), dtype=torch.int32, device="cuda")
        assert L.hec_build_rows_write(ctx.h, off, orp.data_ptr(), ocol.data_ptr(), owgt.data_ptr(),
                                      ovw.data_ptr()) == 0, L.hec_last_error()
        assert np.array_equal(orp.cpu().numpy(), rp[a0:a1 + 1])
        assert np.array_equal(ocol[:k].cpu().numpy(), col[rp[a0]:rp[a1]])
        assert np.array_equal(owgt[:k].cpu().numpy(), wgt[rp[a0]:rp[a1]])
        if rows:
            assert np.array_equal(ovw[:rows].cpu().numpy(), vw[a0:a1])
        off += k
