"""Ablation of the paper's alternatives on B200:
mapping HEC / HEC3 / HEM and construction hash / sort / one-end for whole
hierarchies, and the multilevel spectral bisection consumer (SpMV rate).
Every variant is bit-exact with the oracle (tests/); this measures speed.

usage: python tools/ablation.py [--configs 2 3 4] [--steps 5] [--out gpurun_out/ablation.json]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def timed(fn, steps, warmup=2):
    import torch
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", type=int, nargs="+", default=[2, 3, 4])
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--spectral-iters", type=int, default=100)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "ablation.json"))
    args = ap.parse_args()
    import torch
    import graphgen as gg
    import paper_conf_ipps_gilbertabmr21_b200 as P
    torch.cuda.set_device(0)
    ctx = P.Context()
    rows = []
    for cfg in args.configs:
        c = gg.CONFIGS[cfg]
        t0 = time.time()
        g = gg.config(cfg)
        dg = P.DeviceGraph.from_host(g)
        print(f"C{cfg} {c['name']}: n={g.n} nnz={g.nnz} (gen {time.time() - t0:.0f} s)", flush=True)
        variants = [("hec", "hash"), ("hec", "sort"), ("hec", "one_end"), ("hec", "auto"), ("hec3", "hash")]
        if c["kind"] != "rmat":  # HEM on R-MAT runs into the 200-level cap (Table IV: 201 levels)
            variants.append(("hem", "hash"))
        for method, build in variants:
            levels = []

            def run():
                h = P.coarsen_hierarchy(ctx, dg, c["cutoff"], gg.COARSEN_SEED, method=method, build=build)
                levels[:] = [lv.graph.n for lv in h.levels]
                h.free()
            try:
                ms = timed(run, args.steps)
            except Exception as e:  # noqa: BLE001
                print(f"  {method}/{build}: FAILED {e}", flush=True)
                continue
            r = {"config": f"C{cfg}", "mapping": method, "construction": build, "ms": ms,
                 "edges_per_s": (g.nnz // 2) / (ms / 1e3), "levels": list(levels)}
            rows.append(r)
            print(f"  {method:5s} {build:8s} {ms:9.3f} ms  {r['edges_per_s'] / 1e9:6.2f} G edges/s  "
                  f"levels {levels}", flush=True)
        # single-level mappings (level 0): HEC / HEC3 / HEM
        for method in ("hec", "hec3", "hem"):
            ms = timed(lambda: P.hec_find_mapping_method(ctx, dg, method, gg.COARSEN_SEED, 0), args.steps, warmup=1)
            _, nc = P.hec_find_mapping_method(ctx, dg, method, gg.COARSEN_SEED, 0)
            rows.append({"config": f"C{cfg}", "mapping_level0": method, "ms": ms, "n_c": nc,
                         "GBps_algorithmic": (8 * g.nnz + 12 * g.n) / (ms / 1e3) / 1e9})
            print(f"  level-0 mapping {method:5s} {ms:8.3f} ms  n -> n_c {g.n} -> {nc}", flush=True)
        # spectral bisection on the HEC hierarchy: fixed iterations -> SpMV rate
        h = P.coarsen_hierarchy(ctx, dg, c["cutoff"], gg.COARSEN_SEED)
        it = args.spectral_iters
        ms = timed(lambda: P.spectral_bisection(ctx, dg, h, it, 0.0), 2, warmup=1)
        spmv = it * (len(h.levels) + 1)
        # per iteration on G0: col + wgt (8 B / entry) + x gathers (8 B / entry, L2) + d, x, y (24 B / vertex)
        nnz_all = g.nnz + sum(lv.graph.nnz for lv in h.levels)
        n_all = g.n + sum(lv.graph.n for lv in h.levels)
        gbs = it * (16 * nnz_all + 40 * n_all) / (ms / 1e3) / 1e9
        _, _, cut, _ = P.spectral_bisection(ctx, dg, h, it, 0.0)
        rows.append({"config": f"C{cfg}", "spectral_ms": ms, "iterations_per_level": it, "spmv_launches": spmv,
                     "GBps_algorithmic": gbs, "cut": cut})
        print(f"  spectral ({it} it/level, {len(h.levels) + 1} levels): {ms:.2f} ms, {gbs:.0f} GB/s algorithmic, "
              f"cut {cut}", flush=True)
        h.free()
        del dg
    json.dump(rows, open(args.out, "w"), indent=1)
    ctx.close()


if __name__ == "__main__":
    main()
