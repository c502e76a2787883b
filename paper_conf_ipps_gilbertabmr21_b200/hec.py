"""Python binding of libhec with the C-ABI's names (include/hec.h).

Marshalling only: every step of the hot path runs in libhec's sm_100a kernels.
torch supplies device memory (through the allocator callbacks, so outputs are
torch tensors), the stream and, for the multi-GPU path, process groups.

PAPER.md references: Alg 1 (L37-53) = coarsen_hierarchy, HEC (Alg 3 L99-130,
Alg 4) = hec_find_mapping, Alg 6 / P A P^T (L141, L280-324) =
build_coarse_graph.
"""
from __future__ import annotations

import ctypes
import weakref
from dataclasses import dataclass

import torch

from . import _lib
from ._lib import HecGraph, HecStats, check, load


@dataclass
class DeviceGraph:
    """CSR on the GPU: row_ptr int64[n+1], col int32[nnz], wgt int32[nnz], vwgt int32[n]|None."""
    row_ptr: torch.Tensor
    col: torch.Tensor
    wgt: torch.Tensor
    vwgt: torch.Tensor | None = None

    @property
    def n(self) -> int:
        return int(self.row_ptr.numel() - 1)

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    def c(self) -> HecGraph:
        for t, dt in ((self.row_ptr, torch.int64), (self.col, torch.int32), (self.wgt, torch.int32)):
            if t.dtype != dt or not t.is_cuda or not t.is_contiguous():
                raise TypeError("DeviceGraph arrays must be contiguous CUDA tensors "
                                "(row_ptr int64, col/wgt/vwgt int32)")
        if self.vwgt is not None and (self.vwgt.dtype != torch.int32 or not self.vwgt.is_cuda):
            raise TypeError("vwgt must be an int32 CUDA tensor")
        return HecGraph(self.n, self.nnz, self.row_ptr.data_ptr(), self.col.data_ptr() if self.nnz else 0,
                        self.wgt.data_ptr() if self.nnz else 0,
                        self.vwgt.data_ptr() if self.vwgt is not None else None)

    @staticmethod
    def from_host(g, device="cuda", non_blocking=False) -> "DeviceGraph":
        """From a host graph with numpy arrays row_ptr/col/wgt/vwgt (graphgen.Graph)."""
        def t(a):
            x = torch.from_numpy(a)
            if non_blocking:
                x = x.pin_memory()
            return x.to(device, non_blocking=non_blocking)
        return DeviceGraph(t(g.row_ptr), t(g.col), t(g.wgt), t(g.vwgt) if g.vwgt is not None else None)

    def to_host(self):
        return (self.row_ptr.cpu().numpy(), self.col.cpu().numpy(), self.wgt.cpu().numpy(),
                None if self.vwgt is None else self.vwgt.cpu().numpy())


class Context:
    """hec_ctx bound to the current CUDA device and a stream (default: torch's current stream).

    torch_alloc=True routes library allocations through torch's caching allocator
    (outputs become torch tensors without copies); False uses cudaMallocAsync and
    outputs are copied into torch tensors when materialised."""

    def __init__(self, stream: torch.cuda.Stream | None = None, torch_alloc: bool = True,
                 validate: bool = False):
        L = load()
        self.stream = stream or torch.cuda.current_stream()
        self.device = self.stream.device
        self._blocks: dict[int, torch.Tensor] = {}
        if torch_alloc:
            def _alloc(nbytes, stream, user):
                with torch.cuda.device(self.device), torch.cuda.stream(self.stream):
                    t = torch.empty(max(int(nbytes), 16), dtype=torch.uint8, device=self.device)
                p = t.data_ptr()
                self._blocks[p] = t
                return p

            def _free(ptr, stream, user):
                self._blocks.pop(int(ptr), None)

            self._alloc_cb = _lib.ALLOC_FN(_alloc)
            self._free_cb = _lib.FREE_FN(_free)
        else:
            self._alloc_cb = ctypes.cast(None, _lib.ALLOC_FN)
            self._free_cb = ctypes.cast(None, _lib.FREE_FN)
        self.torch_alloc = torch_alloc
        h = ctypes.c_void_p()
        with torch.cuda.device(self.device):
            check(L.hec_ctx_create(ctypes.c_void_p(self.stream.cuda_stream), self._alloc_cb,
                                   self._free_cb, None, ctypes.byref(h)), "hec_ctx_create")
        self.h = h
        self._owned = weakref.WeakSet()  # live results: freed before the context
        if validate:
            self.set_validate(True)

    def set_validate(self, on: bool):
        check(load().hec_ctx_set_validate(self.h, int(on)), "hec_ctx_set_validate")

    def stats(self) -> dict:
        s = HecStats()
        check(load().hec_ctx_last_stats(self.h, ctypes.byref(s)), "hec_ctx_last_stats")
        return {k: getattr(s, k) for k, _ in HecStats._fields_}

    # --- profiling (CUDA events on the context stream, inside libhec) ---------
    def set_profiling(self, on: bool):
        check(load().hec_ctx_set_profiling(self.h, int(on)), "hec_ctx_set_profiling")

    def profile_reset(self):
        check(load().hec_ctx_profile_reset(self.h), "hec_ctx_profile_reset")

    def profile(self, by_level: bool = False) -> dict:
        """{phase: {"ms": summed device ms, "calls": n, "bytes": algorithmic bytes}}
        (summed over levels), or with by_level {(phase, level): {...}}."""
        L = load()
        cap = 512
        arr = (_lib.HecPhaseTime * cap)()
        cnt = ctypes.c_int()
        check(L.hec_ctx_profile(self.h, arr, cap, ctypes.byref(cnt)), "hec_ctx_profile")
        out: dict = {}
        for i in range(min(cnt.value, cap)):
            key = (arr[i].name.decode(), int(arr[i].level)) if by_level else arr[i].name.decode()
            d = out.setdefault(key, {"ms": 0.0, "calls": 0, "bytes": 0.0})
            d["ms"] += arr[i].ms
            d["calls"] += arr[i].calls
            d["bytes"] += arr[i].bytes
        return out

    def launches(self) -> int:
        return int(load().hec_ctx_launches(self.h))

    def close(self):
        if getattr(self, "h", None):
            for r in list(getattr(self, "_owned", ())):
                r.free()  # results use the context's allocator: free them first
            load().hec_ctx_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # --- device buffer views -------------------------------------------------
    def _view(self, ptr: int, count: int, dtype: torch.dtype) -> torch.Tensor:
        """torch tensor over library-owned memory (zero-copy with torch_alloc)."""
        if count == 0:
            return torch.empty(0, dtype=dtype, device=self.device)
        if self.torch_alloc:
            nbytes = count * torch.empty(0, dtype=dtype).element_size()
            ptr = int(ptr)
            base = self._blocks.get(ptr)
            if base is not None:
                return base[:nbytes].view(dtype)
            # small hierarchy outputs are sub-allocated from shared slab chunks
            for p0, blk in self._blocks.items():
                if p0 <= ptr and ptr + nbytes <= p0 + blk.numel():
                    return blk[ptr - p0:ptr - p0 + nbytes].view(dtype)
            raise RuntimeError("pointer not owned by this context's allocator")
        out = torch.empty(count, dtype=dtype, device=self.device)
        cudart = _cudart()
        nbytes = count * out.element_size()
        cudart.cudaMemcpyAsync(ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(ptr),
                               ctypes.c_size_t(nbytes), 3, ctypes.c_void_p(self.stream.cuda_stream))
        return out


_CUDART = None


def _cudart():
    global _CUDART
    if _CUDART is None:
        import glob
        import os
        cands = glob.glob(os.path.join(os.path.dirname(torch.__file__), "lib", "libcudart*.so*"))
        cands += glob.glob("/usr/local/cuda/lib64/libcudart.so*")
        _CUDART = ctypes.CDLL(cands[0])
    return _CUDART


def hec_prio(seed: int, level: int, u: int) -> int:
    return int(load().hec_prio(seed & 0xFFFFFFFFFFFFFFFF, level, u))


def hec_find_mapping(ctx: Context, g: DeviceGraph, seed: int, level: int, M: torch.Tensor | None = None):
    """FINDCOARSEMAPPING (HEC): returns (M int32[n] on the device, n_c)."""
    if M is None:
        M = torch.empty(g.n, dtype=torch.int32, device=ctx.device)
    nc = ctypes.c_int64()
    gc = g.c()
    check(load().hec_find_mapping(ctx.h, ctypes.byref(gc), seed & 0xFFFFFFFFFFFFFFFF, level,
                                  M.data_ptr() if g.n else None, ctypes.byref(nc)),
          "hec_find_mapping")
    return M, int(nc.value)


def hec_find_mapping_method(ctx: Context, g: DeviceGraph, method: str, seed: int = 0, level: int = 0,
                            prio: torch.Tensor | None = None):
    """FINDCOARSEMAPPING by "hec" (Alg 3), "hec3" (Alg 5) or "hem" (Alg 2):
    (M int32[n] on the device, n_c).  prio: explicit visit order (test hook)."""
    M = torch.empty(g.n, dtype=torch.int32, device=ctx.device)
    nc = ctypes.c_int64()
    gc = g.c()
    m = _lib.MAP_METHODS[method]
    L = load()
    if prio is None:
        rc = L.hec_find_mapping_method(ctx.h, ctypes.byref(gc), m, seed & 0xFFFFFFFFFFFFFFFF, level,
                                       M.data_ptr() if g.n else None, ctypes.byref(nc))
    else:
        rc = L.hec_find_mapping_method_prio(ctx.h, ctypes.byref(gc), m, prio.data_ptr() if g.n else None,
                                            M.data_ptr() if g.n else None, ctypes.byref(nc))
    check(rc, "hec_find_mapping_method")
    return M, int(nc.value)


def hec_find_mapping_prio(ctx: Context, g: DeviceGraph, prio: torch.Tensor, M: torch.Tensor | None = None):
    """Mapping under explicit priorities (uint64 bit patterns in an int64 CUDA tensor)."""
    if M is None:
        M = torch.empty(g.n, dtype=torch.int32, device=ctx.device)
    nc = ctypes.c_int64()
    gc = g.c()
    check(load().hec_find_mapping_prio(ctx.h, ctypes.byref(gc), prio.data_ptr() if g.n else None,
                                       M.data_ptr() if g.n else None, ctypes.byref(nc)),
          "hec_find_mapping_prio")
    return M, int(nc.value)


def hec_debug_heavy(ctx: Context, g: DeviceGraph) -> torch.Tensor:
    H = torch.empty(g.n, dtype=torch.int32, device=ctx.device)
    gc = g.c()
    check(load().hec_debug_heavy(ctx.h, ctypes.byref(gc), H.data_ptr() if g.n else None), "hec_debug_heavy")
    return H


def hec_debug_roots(ctx: Context, g: DeviceGraph, seed: int = 0, level: int = 0,
                    prio: torch.Tensor | None = None):
    root = torch.empty(g.n, dtype=torch.uint8, device=ctx.device)
    rounds = ctypes.c_int()
    gc = g.c()
    check(load().hec_debug_roots(ctx.h, ctypes.byref(gc), prio.data_ptr() if prio is not None else None,
                                 seed & 0xFFFFFFFFFFFFFFFF, level, root.data_ptr() if g.n else None,
                                 ctypes.byref(rounds)), "hec_debug_roots")
    return root, int(rounds.value)


def _graph_from_view(ctx: Context, v: HecGraph) -> DeviceGraph:
    return DeviceGraph(ctx._view(v.row_ptr, v.n + 1, torch.int64),
                       ctx._view(v.col, v.nnz, torch.int32),
                       ctx._view(v.wgt, v.nnz, torch.int32),
                       ctx._view(v.vwgt, v.n, torch.int32) if v.n else
                       torch.empty(0, dtype=torch.int32, device=ctx.device))


class CoarseGraph:
    """Owned result of build_coarse_graph (hec_csr_owned); .graph is a DeviceGraph view."""

    def __init__(self, ctx: Context, handle: ctypes.c_void_p):
        self.ctx, self.h = ctx, handle
        ctx._owned.add(self)
        v = HecGraph()
        check(load().hec_csr_view(handle, ctypes.byref(v)), "hec_csr_view")
        self.graph = _graph_from_view(ctx, v)

    def free(self):
        if self.h:
            load().hec_csr_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def build_coarse_graph(ctx: Context, g: DeviceGraph, M: torch.Tensor, n_c: int, method: str = "hash") -> CoarseGraph:
    """CONSTRUCTCOARSEGRAPH: G_c = P A P^T without the diagonal, rows sorted, weights summed.
    method: "hash" (default), "sort", "one_end" (Alg 6's degree-based one-end storage) or "auto"."""
    h = ctypes.c_void_p()
    gc = g.c()
    L = load()
    Mp = M.data_ptr() if g.n else None
    if method == "hash":
        rc = L.build_coarse_graph(ctx.h, ctypes.byref(gc), Mp, n_c, ctypes.byref(h))
    else:
        rc = L.build_coarse_graph_ex(ctx.h, ctypes.byref(gc), Mp, n_c, _lib.BUILD_METHODS[method], ctypes.byref(h))
    check(rc, "build_coarse_graph")
    return CoarseGraph(ctx, h)


@dataclass
class Level:
    graph: DeviceGraph   # G_i
    M: torch.Tensor      # M_i: G_{i-1} -> G_i
    n_fine: int
    rounds: int


class Hierarchy:
    """Owned result of coarsen_hierarchy (hec_hierarchy)."""

    def __init__(self, ctx: Context, handle: ctypes.c_void_p):
        L = load()
        self.ctx, self.h = ctx, handle
        ctx._owned.add(self)
        self.stop_reason = L.hec_hierarchy_stop_reason(handle)
        self.discarded_n_c = int(L.hec_hierarchy_discarded_n_c(handle))
        self.levels: list[Level] = []
        for i in range(1, L.hec_hierarchy_levels(handle) + 1):
            v = HecGraph()
            mp = ctypes.c_void_p()
            nf = ctypes.c_int64()
            check(L.hec_hierarchy_level(handle, i, ctypes.byref(v), ctypes.byref(mp), ctypes.byref(nf)),
                  "hec_hierarchy_level")
            self.levels.append(Level(_graph_from_view(ctx, v), ctx._view(mp.value, nf.value, torch.int32),
                                     int(nf.value), int(L.hec_hierarchy_rounds(handle, i))))

    def free(self):
        if self.h:
            self.levels = []
            load().hec_hierarchy_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def coarsen_hierarchy(ctx: Context, g0: DeviceGraph, cutoff: int, seed: int, discard_below: int = 10,
                      max_levels: int = 200, method: str = "hec", build: str = "hash") -> Hierarchy:
    """Alg 1: G_1..G_l until n_l <= cutoff (discard rule of PAPER.md:L367), every
    level mapped by `method` ("hec" Alg 3, "hec3" Alg 5, "hem" Alg 2) and built
    by `build` ("hash", "sort", "one_end", "auto")."""
    h = ctypes.c_void_p()
    gc = g0.c()
    L = load()
    if method == "hec" and build == "hash":
        rc = L.coarsen_hierarchy(ctx.h, ctypes.byref(gc), cutoff, seed & 0xFFFFFFFFFFFFFFFF, discard_below,
                                 max_levels, ctypes.byref(h))
    else:
        rc = L.coarsen_hierarchy_ex(ctx.h, ctypes.byref(gc), cutoff, seed & 0xFFFFFFFFFFFFFFFF, discard_below,
                                    max_levels, _lib.MAP_METHODS[method], _lib.BUILD_METHODS[build],
                                    ctypes.byref(h))
    check(rc, "coarsen_hierarchy")
    return Hierarchy(ctx, h)


def spectral_bisection(ctx: Context, g0: DeviceGraph, hier: Hierarchy, max_iter: int = 1000, tol: float = 1e-10,
                       seed: int = 0x5EED):
    """Multilevel spectral bisection on a hierarchy of g0:
    (part uint8[n0], x float64[n0] on the device, edge cut, iterations per level
    from the coarsest)."""
    part = torch.empty(g0.n, dtype=torch.uint8, device=ctx.device)
    x = torch.empty(g0.n, dtype=torch.float64, device=ctx.device)
    cut = ctypes.c_int64()
    iters = (ctypes.c_int64 * (len(hier.levels) + 1))()
    opts = _lib.HecSpectralOpts(max_iter, tol, seed & 0xFFFFFFFFFFFFFFFF)
    gc = g0.c()
    check(load().hec_spectral_bisection(ctx.h, ctypes.byref(gc), hier.h, ctypes.byref(opts),
                                        part.data_ptr() if g0.n else None, x.data_ptr() if g0.n else None,
                                        ctypes.byref(cut), iters), "hec_spectral_bisection")
    return part, x, int(cut.value), list(iters)
