"""Multi-GPU HEC hierarchy: one process per GPU.

Per level, on every rank (the collectives are torch.distributed; NCCL over
NVLink on a GPU box, gloo in the CPU tests):

  1. heavy neighbours of the rank's fine-vertex slice (the edge-streaming part
     of the mapping, a1)                           -> all-gather H
  2. resolution rounds + relabel (replicated: vertex-only, cheap), M for the
     rank's fine slice                             -> all-gather M
  3. identical coarse-row ranges balanced by member-edge volume (hec_balance_rows)
  4. the rank's coarse rows are constructed        -> all-gather row counts
  5. each rank writes its slice at its global offset; the slices are
     all-gathered so that every rank holds G_{l+1} for the next level.

The result is bit-identical to the single-GPU coarsen_hierarchy (tests).
Every compute step runs in libhec; this module only marshals arguments and
calls collectives.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass, field

import torch
import torch.distributed as dist

from . import _lib
from ._lib import HecGraph, check, load
from .hec import Context, DeviceGraph

DISCARD_BELOW = 10
MAX_LEVELS = 200


def even_ranges(n: int, parts: int) -> list[tuple[int, int]]:
    """[lo, hi) of `parts` contiguous, nearly equal pieces of range(n)."""
    q, r = divmod(n, parts)
    out, lo = [], 0
    for k in range(parts):
        hi = lo + q + (1 if k < r else 0)
        out.append((lo, hi))
        lo = hi
    return out


def all_gather_uneven(t: torch.Tensor, sizes: list[int], group=None) -> torch.Tensor:
    """Concatenate the ranks' 1-D tensors (rank r holds sizes[r] elements).

    Padded to the largest piece so that the collective is a plain all-gather
    (NCCL all_gather_into_tensor); gloo goes through host memory."""
    world = len(sizes)
    m = max(sizes) if sizes else 0
    dev = t.device
    backend = dist.get_backend(group)
    work = t if backend == "nccl" else t.cpu()
    pad = torch.zeros(m, dtype=t.dtype, device=work.device)
    pad[: work.numel()] = work
    if backend == "nccl":
        out = torch.empty(world * m, dtype=t.dtype, device=work.device)
        dist.all_gather_into_tensor(out, pad, group=group)
        pieces = [out[r * m: r * m + sizes[r]] for r in range(world)]
    else:
        outs = [torch.empty(m, dtype=t.dtype, device=work.device) for _ in range(world)]
        dist.all_gather(outs, pad, group=group)
        pieces = [outs[r][: sizes[r]] for r in range(world)]
    return torch.cat(pieces).to(dev)


def all_gather_scalars(values: list[int], group=None, device="cpu") -> list[list[int]]:
    """All-gather a small list of int64 per rank."""
    world = dist.get_world_size(group)
    backend = dist.get_backend(group)
    dev = device if backend == "nccl" else "cpu"
    t = torch.tensor(values, dtype=torch.int64, device=dev)
    outs = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(outs, t, group=group)
    return [o.cpu().tolist() for o in outs]


@dataclass
class DistLevel:
    graph: DeviceGraph   # G_l+1, replicated on every rank
    M: torch.Tensor      # M_l+1 (full), replicated
    n_fine: int
    rows: tuple[int, int]  # this rank's coarse rows
    nnz_slice: int


@dataclass
class DistHierarchy:
    levels: list = field(default_factory=list)
    stop_reason: int = _lib.STOP_CUTOFF
    discarded_n_c: int = -1


def coarsen_level_dist(ctx: Context, g: DeviceGraph, seed: int, level: int, group=None,
                       gather_graph: bool = True):
    """One partitioned level.  Returns (M, n_c, DistLevel or None if n_c needs no build)."""
    L = load()
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    n = g.n
    gc = g.c()
    fine = even_ranges(n, world)
    u0, u1 = fine[rank]
    sizes = [hi - lo for lo, hi in fine]
    # 1. heavy neighbours of the slice -> all-gather H
    H = torch.empty(max(n, 1), dtype=torch.int32, device=ctx.device)
    check(L.hec_heavy_range(ctx.h, ctypes.byref(gc), u0, u1, H.data_ptr()), "hec_heavy_range")
    H = all_gather_uneven(H[u0:u1], sizes, group)
    # 2. rounds + relabel (replicated), M for the slice -> all-gather M
    M = torch.empty(max(n, 1), dtype=torch.int32, device=ctx.device)
    nc = ctypes.c_int64()
    check(L.hec_mapping_from_heavy(ctx.h, ctypes.byref(gc), H.data_ptr(), seed & 0xFFFFFFFFFFFFFFFF, level,
                                   u0, u1, M.data_ptr(), ctypes.byref(nc)), "hec_mapping_from_heavy")
    M = all_gather_uneven(M[u0:u1], sizes, group)
    return M, int(nc.value)


def build_level_dist(ctx: Context, g: DeviceGraph, M: torch.Tensor, n_c: int, group=None) -> DistLevel:
    """Partitioned construction of G_c = P A P^T; the slices are all-gathered."""
    L = load()
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    gc = g.c()
    # 3. coarse-row ranges balanced by member-edge volume (identical on all ranks)
    bounds = (ctypes.c_int64 * (world + 1))()
    check(L.hec_balance_rows(ctx.h, ctypes.byref(gc), M.data_ptr(), n_c, world, bounds), "hec_balance_rows")
    b = [int(x) for x in bounds]
    a0, a1 = b[rank], b[rank + 1]
    rows = a1 - a0
    # 4. the rank's coarse rows -> all-gather the row counts
    counts = torch.empty(max(rows, 1), dtype=torch.int64, device=ctx.device)
    nnz_slice = ctypes.c_int64()
    check(L.hec_build_rows_count(ctx.h, ctypes.byref(gc), M.data_ptr(), n_c, a0, a1, counts.data_ptr(),
                                 ctypes.byref(nnz_slice)), "hec_build_rows_count")
    row_sizes = [b[r + 1] - b[r] for r in range(world)]
    all_counts = all_gather_uneven(counts[:rows], row_sizes, group)  # coarse row lengths, all rows
    nnz_all = [v[0] for v in all_gather_scalars([int(nnz_slice.value)], group, ctx.device)]
    offset = sum(nnz_all[:rank])
    # 5. write the slice at its global offset, then replicate G_c
    k = int(nnz_slice.value)
    rp = torch.empty(rows + 1, dtype=torch.int64, device=ctx.device)
    col = torch.empty(max(k, 1), dtype=torch.int32, device=ctx.device)
    wgt = torch.empty(max(k, 1), dtype=torch.int32, device=ctx.device)
    vw = torch.empty(max(rows, 1), dtype=torch.int32, device=ctx.device)
    check(L.hec_build_rows_write(ctx.h, offset, rp.data_ptr(), col.data_ptr(), wgt.data_ptr(), vw.data_ptr()),
          "hec_build_rows_write")
    col_all = all_gather_uneven(col[:k], nnz_all, group)
    wgt_all = all_gather_uneven(wgt[:k], nnz_all, group)
    vw_all = all_gather_uneven(vw[:rows], row_sizes, group)
    # global row pointers: each rank's slice starts are already global offsets
    rp_all = all_gather_uneven(rp[:rows], row_sizes, group)
    total = torch.tensor([sum(nnz_all)], dtype=torch.int64, device=ctx.device)
    row_ptr = torch.cat([rp_all, total])
    G = DeviceGraph(row_ptr.contiguous(), col_all.contiguous(), wgt_all.contiguous(), vw_all.contiguous())
    lvl = DistLevel(G, M, g.n, (a0, a1), k)
    lvl.row_counts = all_counts
    return lvl


def coarsen_hierarchy_dist(ctx: Context, g0: DeviceGraph, cutoff: int, seed: int, group=None,
                           discard_below: int = DISCARD_BELOW, max_levels: int = MAX_LEVELS) -> DistHierarchy:
    """Alg 1 (cutoff/discard L367) with every level partitioned."""
    out = DistHierarchy()
    cur = g0
    level = 0
    while True:
        if cur.n <= cutoff:
            out.stop_reason = _lib.STOP_CUTOFF
            break
        if level >= max_levels:
            out.stop_reason = _lib.STOP_MAX_LEVELS
            break
        M, nc = coarsen_level_dist(ctx, cur, seed, level, group)
        if nc < discard_below:
            out.stop_reason = _lib.STOP_DISCARD
            out.discarded_n_c = nc
            break
        if nc == cur.n:
            out.stop_reason = _lib.STOP_STALL
            break
        lvl = build_level_dist(ctx, cur, M, nc, group)
        out.levels.append(lvl)
        cur = lvl.graph
        level += 1
    return out
