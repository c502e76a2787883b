"""Partitioned hierarchy on the GPU: two ranks (gloo, both on
cuda:0 — the driver's box has one GPU) run coarsen_hierarchy_dist; every level
must equal the single-GPU coarsen_hierarchy bit for bit."""
import os

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

from dist_helpers import free_port, init

pytestmark = pytest.mark.gpu
SEED = 0x5EED


def _graph(which):
    import graphgen as gg
    if which == "c1":
        return gg.config(1), 50
    if which == "rmat14":
        return gg.rmat(14, 16), 50
    return gg.mesh27(24, 24, 24), 100


def _worker(rank, world, port, which, outdir, q):
    import torch.distributed as dist
    import paper_conf_ipps_gilbertabmr21_b200 as P
    from paper_conf_ipps_gilbertabmr21_b200.dist import coarsen_hierarchy_dist
    try:
        torch.cuda.set_device(0)
        init(rank, world, port, "gloo")
        g, cutoff = _graph(which)
        ctx = P.Context()
        H = coarsen_hierarchy_dist(ctx, P.DeviceGraph.from_host(g), cutoff, SEED)
        if rank == 0:
            arrs = {"stop": np.array([H.stop_reason, H.discarded_n_c]), "nlev": np.array([len(H.levels)])}
            for i, lv in enumerate(H.levels):
                rp, col, wgt, vw = lv.graph.to_host()
                arrs.update({f"M{i}": lv.M.cpu().numpy(), f"rp{i}": rp, f"col{i}": col, f"wgt{i}": wgt,
                             f"vw{i}": vw})
            np.savez(os.path.join(outdir, f"{which}.npz"), **arrs)
        dist.barrier()
        ctx.close()
        q.put((rank, "ok"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        if torch.distributed.is_initialized():
            torch.distributed.destroy_process_group()


@pytest.mark.parametrize("which", ["c1", "rmat14", "mesh27"])
def test_dist_hierarchy_matches_single_gpu(which, tmp_path):
    import paper_conf_ipps_gilbertabmr21_b200 as P
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, which, str(tmp_path), q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res
    d = np.load(tmp_path / f"{which}.npz")
    g, cutoff = _graph(which)
    c = P.Context()
    H = P.coarsen_hierarchy(c, P.DeviceGraph.from_host(g), cutoff, SEED)
    assert int(d["nlev"][0]) == len(H.levels) and int(d["stop"][0]) == H.stop_reason
    for i, lv in enumerate(H.levels):
        rp, col, wgt, vw = lv.graph.to_host()
        assert np.array_equal(d[f"M{i}"], lv.M.cpu().numpy())
        assert np.array_equal(d[f"rp{i}"], rp) and np.array_equal(d[f"col{i}"], col)
        assert np.array_equal(d[f"wgt{i}"], wgt) and np.array_equal(d[f"vw{i}"], vw)
