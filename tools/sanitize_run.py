"""Small hierarchies for compute-sanitizer (memcheck / racecheck / synccheck):
C1 (grid2d 64x64), R-MAT s12 and a mesh27 16^3, every level compared with the
oracle.  Run by tools/gpu.sh sanitize; test infrastructure (imports oracle/)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import graphgen as gg  # noqa: E402
import oracle as o  # noqa: E402
import paper_conf_ipps_gilbertabmr21_b200 as P  # noqa: E402


def main():
    import torch
    torch.cuda.set_device(0)
    ctx = P.Context(torch_alloc=False)
    cases = [("c1", gg.config(1), 50), ("rmat12", gg.rmat(12, 16), 50), ("mesh27_16", gg.mesh27(16, 16, 16), 50)]
    # second pass: the next level's heavy keys fused into every placement (test hooks)
    for fused in (False, True):
        if fused:
            os.environ["HEC_FUSE_HEAVY_ALL"] = "1"
            os.environ["HEC_PLACE_ONE_SLICE"] = "1"
        for name, g, cut in cases:
            h = P.coarsen_hierarchy(ctx, P.DeviceGraph.from_host(g), cut, gg.COARSEN_SEED)
            ref = o.hierarchy(g, cut, gg.COARSEN_SEED)
            assert len(h.levels) == len(ref.levels), name
            for lv, lo in zip(h.levels, ref.levels):
                rp, col, wgt, vw = lv.graph.to_host()
                assert np.array_equal(lv.M.cpu().numpy(), lo.M), name
                assert np.array_equal(rp, lo.graph.row_ptr) and np.array_equal(col, lo.graph.col), name
                assert np.array_equal(wgt, lo.graph.wgt) and np.array_equal(vw, lo.graph.vwgt), name
            print(name, "fused" if fused else "", "levels", len(h.levels), "bit-exact", flush=True)
            h.free()
    ctx.close()
    print("sanitize_run ok")


if __name__ == "__main__":
    main()
