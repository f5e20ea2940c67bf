"""Seeded synthetic CSR generators (ctypes binding to libsgr_gen.so, include/sgr_gen.h).

The generator is the one module both the CPU oracle tests and the CUDA path consume: it
produces graphs and holds none of the coloring arithmetic. Workloads follow PAPER.md P:234
(R-MAT) and Table I, and BASELINE.json's configs (SURVEY §8(d) "Concrete
synthetic inputs"):

  cfg1  rmat(16, 8, .57, .19, .19, seed=1)        cfg4  rmat(24, 8, .57, .19, .19, seed=4)
  cfg2  stencil3d(104, 104, 104, 27)              cfg5  rmat(27, 8, .57, .19, .19, seed=5)
  cfg3  er(2**24, 8 * 2**24, seed=3)
"""
from __future__ import annotations

import ctypes
import weakref
from dataclasses import dataclass
from pathlib import Path

import numpy as np

_LIBPATH = Path(__file__).resolve().parent.parent / "lib" / "libsgr_gen.so"
_lib = None


class _CGraph(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.POINTER(ctypes.c_int64)),
                ("col_idx", ctypes.POINTER(ctypes.c_int32))]


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not _LIBPATH.exists():
        from .. import _build
        _build.build_gen()
    lib = ctypes.CDLL(str(_LIBPATH))
    P = ctypes.POINTER(_CGraph)
    i64, i32, u64, dbl = ctypes.c_int64, ctypes.c_int, ctypes.c_uint64, ctypes.c_double
    lib.sgr_gen_rmat.argtypes = [i32, i64, dbl, dbl, dbl, u64, i32, P]
    lib.sgr_gen_er.argtypes = [i64, i64, u64, P]
    lib.sgr_gen_stencil2d.argtypes = [i64, i64, i32, P]
    lib.sgr_gen_stencil3d.argtypes = [i64, i64, i64, i32, P]
    lib.sgr_gen_from_edges.argtypes = [i64, i64, ctypes.c_void_p, ctypes.c_void_p, P]
    lib.sgr_gen_permute.argtypes = [P, u64, P]
    lib.sgr_gen_validate.argtypes = [ctypes.c_void_p, ctypes.c_void_p, i64, i64]
    lib.sgr_gen_free.argtypes = [P]
    lib.sgr_gen_free.restype = None
    lib.sgr_gen_splitmix64.argtypes = [u64]
    lib.sgr_gen_splitmix64.restype = u64
    _lib = lib
    return lib


@dataclass
class Graph:
    """Host CSR: symmetric, rows sorted ascending, no self-loops, no duplicates."""
    n: int
    nnz: int
    row_ptr: np.ndarray  # int64, n+1
    col_idx: np.ndarray  # int32, nnz
    name: str = ""

    @property
    def degrees(self) -> np.ndarray:
        return np.diff(self.row_ptr)

    def validate(self) -> int:
        return validate(self.row_ptr, self.col_idx)


def _wrap(cg: _CGraph, name: str) -> Graph:
    """Adopt the malloc'd arrays without copying; free them when both arrays are gone."""
    lib = _load()
    n, nnz = int(cg.n), int(cg.nnz)
    owner = _Owner(_CGraph(cg.n, cg.nnz, cg.row_ptr, cg.col_idx))
    weakref.finalize(owner, lib.sgr_gen_free, ctypes.byref(owner.holder))
    rp = np.asarray(_View(np.ctypeslib.as_array(cg.row_ptr, shape=(n + 1,)), owner))
    if nnz > 0:
        ci = np.asarray(_View(np.ctypeslib.as_array(cg.col_idx, shape=(nnz,)), owner))
    else:
        ci = np.zeros(0, np.int32)
    return Graph(n, nnz, rp, ci, name)


class _Owner:
    """Owns the generator's malloc'd buffers; freed by a finalizer when unreferenced."""

    def __init__(self, holder):
        self.holder = holder


class _View:
    """Array-interface shim: np.asarray(_View) has .base = the _View, which holds the owner."""

    def __init__(self, arr: np.ndarray, owner: _Owner):
        self._owner = owner
        self.__array_interface__ = arr.__array_interface__


def _check(rc: int, what: str):
    if rc == -1:
        raise ValueError(f"{what}: invalid arguments")
    if rc == -2:
        raise MemoryError(f"{what}: allocation failed")
    if rc != 0:
        raise RuntimeError(f"{what}: error {rc}")


def rmat(scale: int, edge_factor: int = 8, a: float = 0.57, b: float = 0.19, c: float = 0.19,
         seed: int = 1, permute: bool = False) -> Graph:
    """R-MAT [36]: n = 2**scale, edge_factor*n pairs, symmetrized."""
    cg = _CGraph()
    _check(_load().sgr_gen_rmat(scale, edge_factor, a, b, c, seed, int(permute),
                                ctypes.byref(cg)), "rmat")
    return _wrap(cg, f"rmat-s{scale}-ef{edge_factor}-seed{seed}{'-perm' if permute else ''}")


def er(n: int, pairs: int, seed: int = 3) -> Graph:
    """Erdos-Renyi: `pairs` uniform vertex pairs, symmetrized (avg degree ~ 2*pairs/n)."""
    cg = _CGraph()
    _check(_load().sgr_gen_er(n, pairs, seed, ctypes.byref(cg)), "er")
    return _wrap(cg, f"er-n{n}-p{pairs}-seed{seed}")


def stencil2d(nx: int, ny: int, points: int = 5) -> Graph:
    cg = _CGraph()
    _check(_load().sgr_gen_stencil2d(nx, ny, points, ctypes.byref(cg)), "stencil2d")
    return _wrap(cg, f"stencil2d-{points}pt-{nx}x{ny}")


def stencil3d(nx: int, ny: int, nz: int, points: int = 27) -> Graph:
    """3D stencil, natural order, no diagonal (HPCG-style for points=27)."""
    cg = _CGraph()
    _check(_load().sgr_gen_stencil3d(nx, ny, nz, points, ctypes.byref(cg)), "stencil3d")
    return _wrap(cg, f"stencil3d-{points}pt-{nx}x{ny}x{nz}")


def from_edges(n: int, edges) -> Graph:
    """CSR from an undirected edge list [(u, v), ...]: symmetrize, drop loops, dedupe, sort."""
    e = np.asarray(list(edges) if not isinstance(edges, np.ndarray) else edges,
                   dtype=np.int64).reshape(-1, 2)
    src = np.ascontiguousarray(e[:, 0])
    dst = np.ascontiguousarray(e[:, 1])
    cg = _CGraph()
    _check(_load().sgr_gen_from_edges(n, len(e), src.ctypes.data, dst.ctypes.data,
                                      ctypes.byref(cg)), "from_edges")
    return _wrap(cg, f"edges-n{n}-m{len(e)}")


def permute(g: Graph, seed: int) -> Graph:
    """Seeded relabeling of `g` (same permutation family as rmat(permute=True))."""
    cin = _CGraph(g.n, g.nnz, g.row_ptr.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                  g.col_idx.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)))
    cg = _CGraph()
    _check(_load().sgr_gen_permute(ctypes.byref(cin), seed, ctypes.byref(cg)), "permute")
    return _wrap(cg, g.name + f"-perm{seed}")


def validate(row_ptr: np.ndarray, col_idx: np.ndarray) -> int:
    """Bitmask of CSR contract violations (0 = valid); see include/sgr_gen.h."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(col_idx, dtype=np.int32)
    return int(_load().sgr_gen_validate(rp.ctypes.data, ci.ctypes.data if len(ci) else None,
                                        len(rp) - 1, len(ci)))


def splitmix64(x: int) -> int:
    return int(_load().sgr_gen_splitmix64(x))


def config(idx: int) -> Graph:
    """The BASELINE.json configs (1-based), exact recipes of SURVEY §8(d)."""
    if idx == 1:
        return rmat(16, 8, 0.57, 0.19, 0.19, seed=1)
    if idx == 2:
        return stencil3d(104, 104, 104, 27)
    if idx == 3:
        return er(1 << 24, 8 << 24, seed=3)
    if idx == 4:
        return rmat(24, 8, 0.57, 0.19, 0.19, seed=4)
    if idx == 5:
        return rmat(27, 8, 0.57, 0.19, 0.19, seed=5)
    # extra workloads beyond BASELINE.json
    if idx == 6:  # Table I rmat-er: R-MAT (.25,.25,.25,.25), 2^20 vertices, edge factor 10
        return rmat(20, 10, 0.25, 0.25, 0.25, seed=6)
    if idx == 7:  # Table I rmat-g: R-MAT (.45,.15,.15,.25), 2^20 vertices, edge factor 10
        return rmat(20, 10, 0.45, 0.15, 0.15, seed=7)
    if idx == 8:  # cfg4 with Graph500-style relabeling ("--permute")
        return rmat(24, 8, 0.57, 0.19, 0.19, seed=4, permute=True)
    if idx == 9:  # cfg5's shape with edge factor 9: nnz ~ 2.39e9 > 2^31 (cfg5's 2.126e9 is
        # just below), so the int64 row offsets (reading C17) really exceed 32 bits
        return rmat(27, 9, 0.57, 0.19, 0.19, seed=9)
    raise ValueError(idx)


CONFIG_NAMES = {
    1: "rmat-s16-ef8 (a=.57,b=c=.19) seed 1",
    2: "stencil3d-27pt-104^3",
    3: "er-n2^24-pairs8n seed 3",
    4: "rmat-s24-ef8 (a=.57,b=c=.19) seed 4",
    5: "rmat-s27-ef8 (a=.57,b=c=.19) seed 5",
    6: "rmat-er-s20-ef10 (a=b=c=.25, Table I) seed 6",
    7: "rmat-g-s20-ef10 (a=.45,b=c=.15, Table I) seed 7",
    8: "rmat-s24-ef8 (a=.57,b=c=.19) seed 4, permuted",
    9: "rmat-s27-ef9 (a=.57,b=c=.19) seed 9 (nnz > 2^31)",
}
