"""Host-overhead probe for small hierarchies (GPU box): per config, ms per
hierarchy with torch's allocator callbacks vs cudaMallocAsync, with and
without phase profiling, plus levels and kernel launches per hierarchy, and
the cost of one allocator callback.  Usage: python tools/small_levels.py [CFG ...]"""
import ctypes
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_ipps_gilbertabmr21_b200 as P  # noqa: E402


def run(cfg, torch_alloc, profiling, reps=20):
    c = gg.CONFIGS[cfg]
    g = gg.config(cfg)
    dg = P.DeviceGraph.from_host(g, device="cuda:0")
    ctx = P.Context(torch_alloc=torch_alloc)
    ctx.set_profiling(profiling)

    def step():
        h = P.coarsen_hierarchy(ctx, dg, c["cutoff"], gg.COARSEN_SEED)
        nl = len(h.levels)
        h.free()
        return nl

    for _ in range(3):
        nl = step()
    torch.cuda.synchronize()
    l0 = ctx.launches()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record()
    for _ in range(reps):
        step()
    e1.record()
    torch.cuda.synchronize()
    wall = (time.perf_counter() - t0) / reps * 1e3
    launches = (ctx.launches() - l0) / reps
    dev_sum = 0.0
    if profiling:
        prof = ctx.profile(by_level=True)
        dev_sum = sum(v["ms"] for (k, _), v in prof.items() if k == "level") / (reps + 3)
    ctx.close()
    return {"cfg": cfg, "torch_alloc": torch_alloc, "profiling": profiling, "levels": nl,
            "ms": e0.elapsed_time(e1) / reps, "wall_ms": wall, "launches": launches,
            "level_event_ms": dev_sum}


def alloc_cost(n=2000):
    ctx = P.Context(torch_alloc=True)
    cb = ctx._alloc_cb
    fr = ctx._free_cb
    t0 = time.perf_counter()
    for _ in range(n):
        p = cb(4096, None, None)
        fr(p, None, None)
    dt = (time.perf_counter() - t0) / n * 1e6
    ctx.close()
    return dt


if __name__ == "__main__":
    cfgs = [int(a) for a in sys.argv[1:]] or [2, 3]
    print(f"alloc+free callback: {alloc_cost():.1f} us")
    for cfg in cfgs:
        for ta in (True, False):
            for pr in (False, True):
                print(run(cfg, ta, pr), flush=True)
