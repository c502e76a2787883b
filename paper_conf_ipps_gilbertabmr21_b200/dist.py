"""Multi-GPU calls of libhec: one process per GPU.

libhec does the partitioned work itself (include/hec.h: hec_find_mapping_dist,
build_coarse_graph_dist, coarsen_hierarchy_dist -- slice ranges, global row
offsets and the stitching of the gathered CSR are computed in C).  Its only
exchange step is an all-gather of equal-size byte blocks, which this module
supplies as a callback over a torch.distributed process group: NCCL
(all_gather_into_tensor over NVLink) on a GPU box, gloo in the tests.
Marshalling only: no computation of the method happens here.
"""
from __future__ import annotations

import ctypes
import traceback

import torch
import torch.distributed as dist

from . import _lib
from ._lib import HecComm, HecGraph, check, load
from .hec import CoarseGraph, Context, DeviceGraph, Hierarchy

DISCARD_BELOW = 10
MAX_LEVELS = 200
# levels with fewer fine entries run replicated on every rank (launch-bound;
# SURVEY §8(d) applies the bandwidth target from 64M entries up)
PARTITION_MIN_NNZ = 64 << 20


def even_ranges(n: int, parts: int) -> list[tuple[int, int]]:
    """[lo, hi) of `parts` contiguous, nearly equal pieces of range(n) (the
    fine-vertex slices libhec's dist mapping uses)."""
    q, r = divmod(n, parts)
    out, lo = [], 0
    for k in range(parts):
        hi = lo + q + (1 if k < r else 0)
        out.append((lo, hi))
        lo = hi
    return out


class _CudaBytes:
    """__cuda_array_interface__ view of `n` bytes at a device pointer."""

    def __init__(self, ptr: int, n: int):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "|u1", "data": (ptr, False), "version": 3,
                                         "strides": None, "stream": None}


def byte_view(ptr: int, n: int, device: torch.device) -> torch.Tensor:
    """uint8 tensor over n bytes at ptr (device memory, or host memory for device 'cpu')."""
    if n == 0:
        return torch.empty(0, dtype=torch.uint8, device=device)
    if device.type == "cuda":
        return torch.as_tensor(_CudaBytes(ptr, n), device=device)
    return torch.frombuffer((ctypes.c_uint8 * n).from_address(ptr), dtype=torch.uint8)


def allgather_bytes(send: int, recv: int, nbytes: int, group=None, device: torch.device | None = None):
    """recv[r * nbytes : (r + 1) * nbytes] = rank r's send block, on every rank."""
    world = dist.get_world_size(group)
    device = device or torch.device("cpu")
    s = byte_view(send, nbytes, device)
    r = byte_view(recv, nbytes * world, device)
    if dist.get_backend(group) == "nccl":
        dist.all_gather_into_tensor(r, s, group=group)
    else:  # gloo: through host memory
        outs = [torch.empty(nbytes, dtype=torch.uint8) for _ in range(world)]
        dist.all_gather(outs, s.cpu(), group=group)
        r.copy_(torch.cat(outs).to(r.device))


class Comm:
    """hec_comm over a torch.distributed process group (the all-gather callback)."""

    def __init__(self, group=None, device: torch.device | None = None):
        self.group = group
        self.rank, self.world = dist.get_rank(group), dist.get_world_size(group)
        self.device = device or torch.device("cuda", torch.cuda.current_device())
        self.error = None
        self.calls = 0  # collective calls made by libhec through this communicator

        def _cb(send, recv, nbytes, stream, user):
            self.calls += 1
            try:
                allgather_bytes(send, recv, int(nbytes), self.group, self.device)
                return 0
            except Exception:  # noqa: BLE001 -- reported through the library's error code
                self.error = traceback.format_exc()
                return 1

        self._cb = _lib.ALLGATHER_FN(_cb)
        self.c = HecComm(self.rank, self.world, self._cb, None)


def hec_find_mapping_dist(ctx: Context, g: DeviceGraph, seed: int, level: int, comm: Comm):
    """FINDCOARSEMAPPING partitioned over the ranks: (M complete on every rank, n_c)."""
    M = torch.empty(g.n, dtype=torch.int32, device=ctx.device)
    nc = ctypes.c_int64()
    gc = g.c()
    check(load().hec_find_mapping_dist(ctx.h, ctypes.byref(gc), seed & 0xFFFFFFFFFFFFFFFF, level,
                                       ctypes.byref(comm.c), M.data_ptr() if g.n else None, ctypes.byref(nc)),
          "hec_find_mapping_dist")
    return M, int(nc.value)


class CoarseSlice(CoarseGraph):
    """build_coarse_graph_dist result; .rows / .entry_offset / .nnz_total place a slice."""

    def __init__(self, ctx: Context, handle: ctypes.c_void_p):
        super().__init__(ctx, handle)
        a0, a1, off, tot = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        check(load().hec_csr_dist_slice(handle, ctypes.byref(a0), ctypes.byref(a1), ctypes.byref(off),
                                        ctypes.byref(tot)), "hec_csr_dist_slice")
        self.rows = (int(a0.value), int(a1.value))
        self.entry_offset, self.nnz_total = int(off.value), int(tot.value)


def build_coarse_graph_dist(ctx: Context, g: DeviceGraph, M: torch.Tensor, n_c: int, comm: Comm,
                            gather_full: bool = True) -> CoarseSlice:
    """CONSTRUCTCOARSEGRAPH partitioned by coarse-row range (whole G_c on every
    rank with gather_full, else the rank's slice)."""
    h = ctypes.c_void_p()
    gc = g.c()
    check(load().build_coarse_graph_dist(ctx.h, ctypes.byref(gc), M.data_ptr() if g.n else None, n_c,
                                         ctypes.byref(comm.c), int(gather_full), ctypes.byref(h)),
          "build_coarse_graph_dist")
    return CoarseSlice(ctx, h)


def coarsen_hierarchy_dist(ctx: Context, g0: DeviceGraph, cutoff: int, seed: int, group=None,
                           comm: Comm | None = None, partition_min_nnz: int = PARTITION_MIN_NNZ,
                           discard_below: int = DISCARD_BELOW, max_levels: int = MAX_LEVELS) -> Hierarchy:
    """Alg 1 (cutoff/discard L367) with the levels of at least
    partition_min_nnz fine entries partitioned over the ranks; every rank
    receives the whole hierarchy (identical to coarsen_hierarchy)."""
    comm = comm or Comm(group, ctx.device)
    h = ctypes.c_void_p()
    gc = g0.c()
    check(load().coarsen_hierarchy_dist(ctx.h, ctypes.byref(gc), cutoff, seed & 0xFFFFFFFFFFFFFFFF, discard_below,
                                        max_levels, ctypes.byref(comm.c), partition_min_nnz, ctypes.byref(h)),
          "coarsen_hierarchy_dist")
    return Hierarchy(ctx, h)


__all__ = ["Comm", "even_ranges", "allgather_bytes", "byte_view", "hec_find_mapping_dist",
           "build_coarse_graph_dist", "coarsen_hierarchy_dist", "CoarseSlice", "HecGraph"]
