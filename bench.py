#!/usr/bin/env python
"""Benchmark of the HEC coarsening hot path on B200.

One step = one full HEC hierarchy (Alg 1: mapping + coarse
construction at every level until n_l <= C, discard rule L367) of the
workload's G0, which is resident in HBM when the timed region starts.

  metric  fine edges coarsened/sec (undirected G0 edges m0 / time-to-cutoff)
  value   whole job: with N > 1 ranks (torchrun) every level of the one hierarchy
          is partitioned over the ranks (strong scaling)
  e2e     same metric through the C-ABI call with host buffers: pinned-host ->
          device copy of G0 and a device -> host read of the coarsest graph and
          the level sizes inside the timed region
  roofline  the dominant part (mapping or construction of one level): SURVEY
          §8(d) compulsory bytes / its CUDA-event device time, vs the measured HBM
          copy bandwidth in MEASURED_PEAKS.json; `levels` gives B_l / T_l per level
  cpu_baseline  the CPU oracle (single thread) on a bounded sample

usage: python bench.py [--gpus N] [--steps K] [--warmup W] [--config 4] [--impl ours|reference]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "fine edges coarsened/sec and time-to-cutoff per hierarchy; HBM GB/s vs peak"
UNIT = "edges/s"
SAMPLE = dict(kind="rmat", scale=19, ef=32, cutoff=50)  # oracle sample: G-spec R-MAT, 1/32 of C4's vertex range


def env_rank():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("LOCAL_RANK", 0)),
            int(os.environ.get("WORLD_SIZE", 1)))


def make_graph(cfg):
    import graphgen as gg
    if isinstance(cfg, dict):
        return gg.rmat(cfg["scale"], cfg["ef"], gg.GEN_SEED)
    return gg.config(cfg)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.FIELDS}",
                                       "--format=csv,noheader,nounits", "-lms", "50"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.p = None
        time.sleep(0.15)
        return self

    def __exit__(self, *a):
        self.out = ""
        if self.p:
            self.p.terminate()
            try:
                self.out = self.p.communicate(timeout=5)[0]
            except subprocess.TimeoutExpired:
                self.p.kill()

    def summary(self):
        rows = []
        for line in (self.out or "").splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                rows.append(dict(sm=float(f[1]), smax=float(f[2]), power=float(f[3]),
                                 hw=f[5] == "Active", hwt=f[6] == "Active", swt=f[7] == "Active",
                                 cap=f[8] == "Active"))
            except ValueError:
                continue
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        load = [r for r in rows if r["power"] > 200] or rows
        reasons = sorted({name for r in rows for name, k in
                          (("hw_slowdown", "hw"), ("hw_thermal_slowdown", "hwt"),
                           ("sw_thermal_slowdown", "swt"), ("sw_power_cap", "cap")) if r[k]})
        return {"sm_mhz": statistics.median(r["sm"] for r in load), "sm_max_mhz": rows[0]["smax"],
                "reasons": reasons, "samples": len(rows)}


MAPPING_PHASES = ("heavy", "rounds", "relabel")
CONSTRUCTION_PHASES = ("bucket", "expand", "rows_skew", "rows", "place")


def level_bytes(levels, g0_n, g0_nnz):
    """B_l = 16 nnz + 8 nnz_c + 28 n + 12 n_c per built level."""
    tot = 0.0
    n, nnz = g0_n, g0_nnz
    for (nc, nnzc) in levels:
        tot += 16 * nnz + 8 * nnzc + 28 * n + 12 * nc
        n, nnz = nc, nnzc
    return tot


def mapping_bytes(n, nnz):
    """a1-a5 compulsory bytes: col + wgt once, row_ptr, M written."""
    return 8.0 * nnz + 12.0 * n


def construction_bytes(n, nnz, nc, nnzc):
    """a7-a10 compulsory bytes: col + wgt once, col_c + wgt_c once,
    row_ptr, M, vwgt in; row_ptr_c, vwgt_c out."""
    return 8.0 * nnz + 8.0 * nnzc + 16.0 * n + 12.0 * nc


def source_stamp():
    """sha256[:16] over the CUDA sources: ties a committed ncu capture to the code it measured."""
    import glob
    import hashlib
    h = hashlib.sha256()
    for f in sorted(glob.glob(os.path.join(ROOT, "paper_conf_ipps_gilbertabmr21_b200", "csrc", "*.cu*"))):
        h.update(open(f, "rb").read())
    return h.hexdigest()[:16]


def traffic_from_profiles(config, level, part):
    """ncu dram bytes (read + write) of one hierarchy's `part` ("mapping" /
    "construction") at `level`, from the committed capture of this workload
    (profiles/ncu_traffic.json, written by tools/ncu_traffic.py).  A capture
    of other CUDA sources is stale and ignored (returns None)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None, None
    d = json.load(open(p)).get(f"C{config}")
    if not d or d.get("source_stamp") != source_stamp():
        return None, (d or {}).get("source_stamp")
    lv = d.get("levels", [])
    if level >= len(lv):
        return None, d.get("source_stamp")
    return lv[level].get(f"{part}_dram"), d.get("source_stamp")


def run_oracle_sample(reps):
    import oracle as o
    g = make_graph(SAMPLE)
    ts = []
    for _ in range(reps):
        H = o.hierarchy(g, SAMPLE["cutoff"], 0x5EED)
        ts.append(H.t_total)
    return g, ts


def reference_arm(args, rank, world):
    """The base contract's reference arm: the CPU oracle as it stands, on a bounded
    sample of the workload (this tier has no runnable reference implementation)."""
    if rank != 0:
        return 0
    import oracle as o
    g = make_graph(SAMPLE)
    m0 = g.nnz // 2
    for _ in range(args.warmup):
        o.hierarchy(g, SAMPLE["cutoff"], 0x5EED)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        H = o.hierarchy(g, SAMPLE["cutoff"], 0x5EED)
    dt = (time.perf_counter() - t0) / args.steps
    val = m0 / dt
    sample = f"oracle hierarchy (C=50) of rmat_s{SAMPLE['scale']}_ef{SAMPLE['ef']} (G-spec, n={g.n}, nnz={g.nnz})"
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": workload_name(args.config), "sample": sample,
                       "levels": [lv.n_c for lv in H.levels]},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def workload_name(cfg):
    import graphgen as gg
    c = gg.CONFIGS[cfg]
    return f"C{cfg} {c['name']} HEC hierarchy to C={c['cutoff']} (seed 0x5EED)"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--prof-steps", type=int, default=-1,
                    help="steps of the instrumented per-level pass (default min(steps, 5); 0: none, e.g. under ncu)")
    ap.add_argument("--method", default="hec", choices=["hec", "hec3", "hem"],
                    help="mapping method of every level (SURVEY 8(f) f2/f4 ablation; default HEC, the north star)")
    ap.add_argument("--build", default="hash", choices=["hash", "sort", "one_end", "auto"],
                    help="construction method (SURVEY 8(f) f1 ablation)")
    args = ap.parse_args()
    rank, local_rank, world = env_rank()
    if args.impl == "reference":
        return reference_arm(args, rank, world)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # one process per GPU: re-exec under torchrun (the driver's launch form)
        import torch
        have = torch.cuda.device_count()
        if have < args.gpus:
            print(json.dumps({"error": f"--gpus {args.gpus} requested but only {have} CUDA device(s) visible"}),
                  flush=True)
            return 2
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", str(29500 + os.getpid() % 1000),
               os.path.abspath(__file__)] + sys.argv[1:]
        return subprocess.call(cmd)
    if world != args.gpus:
        print(json.dumps({"error": f"--gpus {args.gpus} but WORLD_SIZE={world}"}), flush=True)
        return 2

    import numpy as np
    import torch
    import graphgen as gg
    import paper_conf_ipps_gilbertabmr21_b200 as P

    if world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    else:
        dist = None
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    cfg = gg.CONFIGS[args.config]
    t0 = time.time()
    g = make_graph(args.config)
    t_gen = time.time() - t0
    m0 = g.nnz // 2
    dg = P.DeviceGraph.from_host(g, device=dev)
    stream = torch.cuda.current_stream()
    ctx = P.Context(stream=stream)

    def barrier():
        if dist:
            dist.barrier()

    comm = None
    if world > 1:
        from paper_conf_ipps_gilbertabmr21_b200 import dist as D
        comm = D.Comm(None, dev)

    def hierarchy(graph):
        """One full hierarchy: single GPU, or (N > 1) the levels of >= 64M fine
        entries partitioned over the ranks inside libhec (coarsen_hierarchy_dist:
        H / M all-gathers, coarse-row ranges, slices all-gathered so every rank
        holds G_{l+1}); smaller levels replicated."""
        if world > 1:
            return D.coarsen_hierarchy_dist(ctx, graph, cfg["cutoff"], gg.COARSEN_SEED, comm=comm)
        return P.coarsen_hierarchy(ctx, graph, cfg["cutoff"], gg.COARSEN_SEED, method=args.method,
                                   build=args.build)

    def step():
        h = hierarchy(dg)
        sizes = [(lv.graph.n, lv.graph.nnz) for lv in h.levels]
        h.free()
        return sizes

    for _ in range(args.warmup):
        levels = step()
    torch.cuda.synchronize()
    # ---- timed region (no instrumentation: per-phase events only in the pass below)
    ctx.profile_reset()  # (also resets the launch counter)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    with ClockSampler(torch.cuda.current_device()) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            levels = step()
        ev1.record(stream)
        torch.cuda.synchronize()
    barrier()
    ms = ev0.elapsed_time(ev1) / args.steps
    launches = ctx.launches()
    # ---- instrumented pass (same step, per-phase / per-level CUDA events): the
    # per-level breakdown and the roofline come from here
    prof_steps = max(1, min(args.steps, 5)) if args.prof_steps < 0 else args.prof_steps
    ctx.set_profiling(True)
    ctx.profile_reset()
    torch.cuda.synchronize()
    ep0, ep1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ep0.record(stream)
    for _ in range(prof_steps):
        step()
    ep1.record(stream)
    torch.cuda.synchronize()
    ms_prof = ep0.elapsed_time(ep1) / prof_steps if prof_steps else 0.0
    prof_steps = max(prof_steps, 1)  # (divisor of the empty profile below)
    prof = ctx.profile()
    prof_lv = ctx.profile(by_level=True)
    ctx.set_profiling(False)
    if dist:
        t = torch.tensor([ms], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    # strong scaling: one graph per job, every level partitioned over the ranks
    value = m0 / (ms / 1e3)

    # ---- per-level records and the roofline (SURVEY §8(d) compulsory bytes)
    peak, peak_src = peaks()
    B = level_bytes(levels, g.n, g.nnz)
    B_fused = 0.0
    per_level = []
    parts = []  # (ms per step, level, part, algorithmic bytes)
    n_l, nnz_l = g.n, g.nnz
    n_levels = max([lv for (_, lv) in prof_lv] + [-1]) + 1
    for l in range(n_levels):
        built = l < len(levels)
        nc, nnzc = levels[l] if built else (None, None)
        t_l = prof_lv.get(("level", l), {}).get("ms", 0.0) / prof_steps
        t_map = sum(prof_lv.get((k, l), {}).get("ms", 0.0) for k in MAPPING_PHASES) / prof_steps
        t_con = sum(prof_lv.get((k, l), {}).get("ms", 0.0) for k in CONSTRUCTION_PHASES) / prof_steps
        # fused a1: the heavy keys of G_l were kept by the previous level's placement,
        # so this mapping reads 8 B of keys per vertex instead of G_l (libhec's
        # "heavy" phase then declares 20 n bytes)
        hv = prof_lv.get(("heavy", l), {})
        fused = l > 0 and hv.get("calls", 0) > 0 and hv["bytes"] / hv["calls"] < 8 * nnz_l
        b_map = 20.0 * n_l if fused else mapping_bytes(n_l, nnz_l)
        b_l = (b_map + construction_bytes(n_l, nnz_l, nc, nnzc)) if built else b_map
        B_fused += b_l
        rec = {"level": l, "n": n_l, "nnz": nnz_l, "n_c": nc, "nnz_c": nnzc, "built": built, "heavy_fused": fused,
               "ms": t_l, "B": b_l, "GBps": b_l / (t_l / 1e3) / 1e9 if t_l else None,
               "frac": (b_l / (t_l / 1e3) / 1e9 / peak) if t_l else None,
               "mapping_ms": t_map, "construction_ms": t_con if built else 0.0}
        per_level.append(rec)
        parts.append((t_map, l, "mapping", b_map))
        if built:
            parts.append((t_con, l, "construction", construction_bytes(n_l, nnz_l, nc, nnzc)))
            n_l, nnz_l = nc, nnzc
    if B_fused > 0:
        B = B_fused  # the bytes this (fused) path must move, discarded level's mapping included
    t_dom, l_dom, part_dom, b_dom = max(parts) if parts else (0.0, 0, "mapping", 0.0)
    achieved = b_dom / (t_dom / 1e3) / 1e9 if t_dom > 0 else 0.0
    traffic, stamp = traffic_from_profiles(args.config, l_dom, part_dom)
    phases = {k: {"ms_per_step": v["ms"] / prof_steps, "GBps": (v["bytes"] / (v["ms"] / 1e3) / 1e9) if v["ms"] else 0,
                  "share": v["ms"] / (ms_prof * prof_steps) if ms_prof else 0.0}
              for k, v in sorted(prof.items(), key=lambda kv: -kv[1]["ms"]) if k != "level"}

    # ---- e2e through host buffers
    e2e = None
    if args.e2e_steps > 0:
        host = [torch.from_numpy(a).pin_memory() for a in (g.row_ptr, g.col, g.wgt, g.vwgt)]
        bi = sum(t.numel() * t.element_size() for t in host)
        bo = 0
        # a user's resident buffers: device inputs and pinned result staging are
        # allocated once (outside the timed region) and refilled every step; the
        # result sizes come from the (deterministic) hierarchy already timed above
        del dg
        d_in = [torch.empty_like(t, device=dev) for t in host]
        last_n, last_nnz = (levels[-1][0], levels[-1][1]) if levels else (g.n, g.nnz)
        out_h = [torch.empty(last_n + 1, dtype=torch.int64).pin_memory(),
                 torch.empty(last_nnz, dtype=torch.int32).pin_memory(),
                 torch.empty(last_nnz, dtype=torch.int32).pin_memory()]
        torch.cuda.synchronize()
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.e2e_steps):
            for d, t in zip(d_in, host):
                d.copy_(t, non_blocking=True)
            hg = P.DeviceGraph(*d_in)
            h = hierarchy(hg)
            last = h.levels[-1].graph if h.levels else hg
            outs = [o[: x.numel()] for o, x in zip(out_h, (last.row_ptr, last.col, last.wgt))]
            for o, x in zip(outs, (last.row_ptr, last.col, last.wgt)):
                o.copy_(x, non_blocking=True)
            sizes = torch.tensor([lv.graph.n for lv in h.levels], dtype=torch.int64)
            bo = sum(t.numel() * t.element_size() for t in outs) + sizes.numel() * 8
            h.free()
            del hg
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        ems = e0.elapsed_time(e1) / args.e2e_steps
        if dist:
            t = torch.tensor([ems], device=dev, dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        e2e = {"value": m0 / (ems / 1e3), "unit": UNIT, "h2d_bytes_per_step": bi, "d2h_bytes_per_step": bo,
               "ms_per_step": ems}

    # ---- CPU oracle baseline (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        sg, ts = run_oracle_sample(2)
        tmed = statistics.median(ts)
        cpu = {"value": (sg.nnz // 2) / tmed, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"oracle hierarchy (C=50, seed 0x5EED) of rmat_s{SAMPLE['scale']}_ef{SAMPLE['ef']} "
                         f"(G-spec, n={sg.n}, nnz={sg.nnz}), median of 2 runs, {tmed:.2f} s each; "
                         f"host nproc={os.cpu_count()}"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong" if world > 1 else "weak",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": workload_name(args.config), "n": g.n, "nnz": g.nnz, "m0": m0,
                       "mapping": args.method, "construction": args.build,
                       "cutoff": cfg["cutoff"], "seed": gg.COARSEN_SEED,
                       "parallelism": (f"partitioned x{world} (levels with >= 64M fine entries): fine-vertex "
                                       "slices for heavy/M, coarse-row ranges for construction, NCCL all-gathers "
                                       "through libhec's collective callback (gather_ms: their share)")
                       if world > 1 else "single",
                       "l2": f"inputs {(g.nnz * 8 + g.n * 12) / 1e9:.1f} GB > 126 MB L2 (no flush needed)",
                       "levels": [n for n, _ in levels], "gen_s": round(t_gen, 1)},
            "time_to_cutoff_ms": ms,
            "hierarchy_GBps": B / (ms / 1e3) / 1e9,
            "hierarchy_frac_of_peak": B / (ms / 1e3) / 1e9 / peak,
            "roofline": {"bound": "hbm", "kernel": f"{part_dom} of level {l_dom}", "achieved": achieved,
                         "peak": peak, "unit": "GB/s", "frac": achieved / peak, "traffic": traffic,
                         "algorithmic_bytes": b_dom, "ms": t_dom,
                         "bytes_rule": ("SURVEY 8(d): mapping 8 nnz + 12 n (20 n when its heavy keys were fused "
                                        "into the previous level's placement); construction 8 nnz + 8 nnz_c + "
                                        "16 n + 12 n_c"),
                         "traffic_source": (f"profiles/ncu_traffic.json (source stamp {stamp})" if traffic
                                            else f"no ncu capture of these sources ({source_stamp()})"),
                         "peak_source": peak_src},
            "levels": per_level,
            "levels_source": (f"separate instrumented pass ({prof_steps} steps with per-phase CUDA events, "
                              f"{ms_prof:.3f} ms per step); ms_per_step is measured without them"),
            "ms_per_step_instrumented": ms_prof,
            "gather_ms": prof.get("gather", {}).get("ms", 0.0) / prof_steps,
            "phases": phases,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "gpu_launches_per_step": launches / args.steps,
            "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    ctx.close()
    if dist:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
