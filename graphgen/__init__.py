"""Seeded synthetic input graphs (SURVEY.md §8(d) "Concrete synthetic inputs").

Shared by the oracle and the CUDA path; contains none of the coarsening
method's arithmetic.  Every graph is undirected, unit edge weights, unit vertex
weights, CSR with int64 ``row_ptr``, ascending int32 ``col``, no self-loops and
no duplicate edges (PAPER.md:L59 graph model; L336/L361 "LCC + relabel").

Configs (BASELINE.json ``configs``):
  C1 grid2d 64x64, C=50      C2 mesh27 128^3, C=1000
  C3 R-MAT s22 ef16, C=50    C4 R-MAT s24 ef32, C=50    C5 R-MAT s26 ef16, C=50
"""
from __future__ import annotations

import ctypes
import hashlib
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

# cutoff C per config
CONFIGS = {
    1: dict(kind="grid2d", shape=(64, 64), cutoff=50, name="grid2d_64x64"),
    2: dict(kind="mesh27", shape=(128, 128, 128), cutoff=1000, name="mesh27_128^3"),
    3: dict(kind="rmat", scale=22, ef=16, cutoff=50, name="rmat_s22_ef16"),
    4: dict(kind="rmat", scale=24, ef=32, cutoff=50, name="rmat_s24_ef32"),
    5: dict(kind="rmat", scale=26, ef=16, cutoff=50, name="rmat_s26_ef16"),
}
GEN_SEED = 1          # seed_g of the R-MAT G-spec
COARSEN_SEED = 0x5EED  # hierarchy seed (R3)


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libgraphgen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make -C {os.path.dirname(_HERE)} graphgen`")
        L = ctypes.CDLL(path)
        i64, p = ctypes.c_int64, ctypes.c_void_p
        L.gg_hash.restype = ctypes.c_uint64
        L.gg_hash.argtypes = [ctypes.c_uint64]
        L.gg_grid2d_nnz.restype = i64
        L.gg_grid2d_nnz.argtypes = [i64, i64]
        L.gg_grid2d.argtypes = [i64, i64, p, p]
        L.gg_mesh27_nnz.restype = i64
        L.gg_mesh27_nnz.argtypes = [i64, i64, i64]
        L.gg_mesh27.argtypes = [i64, i64, i64, p, p]
        L.gg_rmat.restype = p
        L.gg_rmat.argtypes = [ctypes.c_int, i64, ctypes.c_uint64, ctypes.c_int]
        L.gg_n.restype = i64
        L.gg_n.argtypes = [p]
        L.gg_nnz.restype = i64
        L.gg_nnz.argtypes = [p]
        L.gg_copy.argtypes = [p, p, p]
        L.gg_free.argtypes = [p]
        _LIB = L
    return _LIB


@dataclass
class Graph:
    """Host CSR graph: row_ptr int64[n+1], col int32[nnz], wgt int32[nnz], vwgt int32[n]."""
    row_ptr: np.ndarray
    col: np.ndarray
    wgt: np.ndarray
    vwgt: np.ndarray

    @property
    def n(self) -> int:
        return int(self.row_ptr.shape[0] - 1)

    @property
    def nnz(self) -> int:
        return int(self.col.shape[0])


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def _unit(row_ptr, col) -> Graph:
    n = row_ptr.shape[0] - 1
    return Graph(row_ptr, col, np.ones(col.shape[0], np.int32), np.ones(n, np.int32))


def grid2d(nx: int, ny: int) -> Graph:
    L = lib()
    nnz = L.gg_grid2d_nnz(nx, ny)
    rp = np.empty(nx * ny + 1, np.int64)
    col = np.empty(nnz, np.int32)
    L.gg_grid2d(nx, ny, _ptr(rp), _ptr(col))
    return _unit(rp, col)


def mesh27(nx: int, ny: int, nz: int) -> Graph:
    L = lib()
    nnz = L.gg_mesh27_nnz(nx, ny, nz)
    rp = np.empty(nx * ny * nz + 1, np.int64)
    col = np.empty(nnz, np.int32)
    L.gg_mesh27(nx, ny, nz, _ptr(rp), _ptr(col))
    return _unit(rp, col)


def rmat(scale: int, ef: int, seed: int = GEN_SEED, threads: int = 0) -> Graph:
    L = lib()
    h = L.gg_rmat(scale, ef, seed, threads)
    if not h:
        raise MemoryError("gg_rmat failed")
    try:
        n, nnz = L.gg_n(h), L.gg_nnz(h)
        rp = np.empty(n + 1, np.int64)
        col = np.empty(nnz, np.int32)
        L.gg_copy(h, _ptr(rp), _ptr(col))
    finally:
        L.gg_free(h)
    return _unit(rp, col)


def config(k: int) -> Graph:
    c = CONFIGS[k]
    if c["kind"] == "grid2d":
        return grid2d(*c["shape"])
    if c["kind"] == "mesh27":
        return mesh27(*c["shape"])
    return rmat(c["scale"], c["ef"], GEN_SEED)


def sha16(*arrays: np.ndarray) -> str:
    """sha256 over the little-endian bytes of the arrays, first 16 hex digits."""
    h = hashlib.sha256()
    for a in arrays:
        h.update(np.ascontiguousarray(a).tobytes())
    return h.hexdigest()[:16]


def from_edges(n: int, edges, symmetric_weights=True) -> Graph:
    """Build a CSR graph from a list of undirected (u, v, w) triples (tests)."""
    adj = [dict() for _ in range(n)]
    for (u, v, w) in edges:
        assert u != v
        adj[u][v] = w
        adj[v][u] = w
    rp = np.zeros(n + 1, np.int64)
    cols, ws = [], []
    for u in range(n):
        for v in sorted(adj[u]):
            cols.append(v)
            ws.append(adj[u][v])
        rp[u + 1] = len(cols)
    return Graph(rp, np.array(cols, np.int32), np.array(ws, np.int32), np.ones(n, np.int32))
