"""CPU oracle for deterministic SGR coloring — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package. The product path
(``paper_conf_ipps_licqfsty16_b200``, ``libsgr.so``) never imports it, and the two share
no code: the only common module is the seeded input generator
(``paper_conf_ipps_licqfsty16_b200.gen``), which holds none of the method's arithmetic.

Two implementations, written independently from PAPER.md:
  * ``liboracle.so`` (sgr_oracle.c): plain C, single-threaded by default, used at every
    size (optionally OpenMP over the per-vertex loops of a round, which are independent
    given the snapshot).
  * ``pyoracle`` : a ~60-line pure-Python twin for tiny graphs (tests only).

"parity unpinned": none — every function is pinned in tests/test_oracle.py.
"""
from __future__ import annotations

import ctypes
import subprocess
from pathlib import Path

import numpy as np

_DIR = Path(__file__).resolve().parent
_LIBPATH = _DIR / "liboracle.so"
_lib = None

TIEBREAK_LOWID_KEEPS = 0
TIEBREAK_PAPER = 1


class Round(ctypes.Structure):
    _fields_ = [("w_size", ctypes.c_int64), ("w_edges", ctypes.c_int64),
                ("next_size", ctypes.c_int64), ("max_color", ctypes.c_int32),
                ("pad", ctypes.c_int32)]


def _load():
    global _lib
    if _lib is not None:
        return _lib
    src = _DIR / "sgr_oracle.c"
    if not _LIBPATH.exists() or _LIBPATH.stat().st_mtime < src.stat().st_mtime:
        subprocess.run(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-fopenmp", "-Wall",
                        "-Wextra", "-o", str(_LIBPATH), str(src)], check=True)
    lib = ctypes.CDLL(str(_LIBPATH))
    vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
    lib.oracle_alg1.argtypes = [vp, vp, i64, vp]
    lib.oracle_jacobi.argtypes = [vp, vp, i64, i32, i32, i32, i64, vp, vp, i64, vp]
    lib.oracle_assign.argtypes = [vp, vp, i64, vp, i64, vp, vp]
    lib.oracle_detect.argtypes = [vp, vp, i64, vp, i64, vp, i32, vp]
    lib.oracle_jacobi_partitioned.argtypes = [vp, vp, i64, i32, i32, vp, vp, vp]
    lib.oracle_gauss_seidel.argtypes = [vp, vp, i64, i32, i64, i32, i64, vp, vp, i64, vp]
    lib.oracle_max_threads.argtypes = []
    _lib = lib
    return lib


def _ptr(a):
    return a.ctypes.data if a is not None and a.size else None


def _csr(g):
    rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(g.col_idx, dtype=np.int32)
    return rp, ci, len(rp) - 1


def _check(rc, what):
    if rc < 0:
        raise RuntimeError(f"oracle {what} failed: {rc}")
    return rc


def alg1(g) -> np.ndarray:
    """O1 — Algorithm 1 in natural vertex order; returns int32 colors (1-based)."""
    rp, ci, n = _csr(g)
    color = np.zeros(n, np.int32)
    _check(_load().oracle_alg1(_ptr(rp), _ptr(ci), n, _ptr(color)), "alg1")
    return color


class JacobiResult:
    def __init__(self, colors, rounds, trace, converged):
        self.colors = colors
        self.rounds = rounds
        self.trace = trace  # structured array: w_size, w_edges, next_size, max_color
        self.converged = converged

    @property
    def num_colors(self) -> int:
        return int(self.colors.max()) if len(self.colors) else 0

    @property
    def round_sizes(self) -> np.ndarray:
        return self.trace["w_size"].copy()

    @property
    def edges_scanned(self) -> int:
        return int(self.trace["w_edges"].sum())

    @property
    def vertices_processed(self) -> int:
        return int(self.trace["w_size"].sum())


def jacobi(g, tiebreak: int = TIEBREAK_LOWID_KEEPS, detect_over_v: bool = False,
           nthreads: int = 1, max_rounds: int = 0, trace_cap: int | None = None) -> JacobiResult:
    """O2 — Algorithm 5 with Jacobi rounds; see oracle/sgr_oracle.h."""
    rp, ci, n = _csr(g)
    color = np.zeros(n, np.int32)
    cap = (n + 1) if trace_cap is None else trace_cap
    if max_rounds > 0:
        cap = min(cap, max_rounds)
    trace = (Round * max(cap, 1))()
    rounds = ctypes.c_int64(0)
    rc = _check(_load().oracle_jacobi(_ptr(rp), _ptr(ci), n, tiebreak, int(detect_over_v),
                                      nthreads, max_rounds, _ptr(color),
                                      ctypes.cast(trace, ctypes.c_void_p), cap,
                                      ctypes.byref(rounds)), "jacobi")
    r = rounds.value
    dt = np.dtype([("w_size", np.int64), ("w_edges", np.int64), ("next_size", np.int64),
                   ("max_color", np.int32), ("pad", np.int32)])
    tr = np.frombuffer(trace, dtype=dt, count=min(r, cap)).copy()
    return JacobiResult(color, r, tr, rc == 0)


def gauss_seidel(g, substeps: int, partition: int = 0, tiebreak: int = TIEBREAK_LOWID_KEEPS,
                 max_rounds: int = 0, trace_cap: int | None = None) -> JacobiResult:
    """O3 — K-sub-step Gauss-Seidel rounds; partition 0 = strided
    (v mod K), 1 = blocked (floor(v K / n)). See oracle/sgr_oracle.h."""
    rp, ci, n = _csr(g)
    color = np.zeros(n, np.int32)
    cap = (n + 1) if trace_cap is None else trace_cap
    if max_rounds > 0:
        cap = min(cap, max_rounds)
    trace = (Round * max(cap, 1))()
    rounds = ctypes.c_int64(0)
    rc = _check(_load().oracle_gauss_seidel(_ptr(rp), _ptr(ci), n, tiebreak, int(substeps),
                                            int(partition), max_rounds, _ptr(color),
                                            ctypes.cast(trace, ctypes.c_void_p), cap,
                                            ctypes.byref(rounds)), "gauss_seidel")
    r = rounds.value
    dt = np.dtype([("w_size", np.int64), ("w_edges", np.int64), ("next_size", np.int64),
                   ("max_color", np.int32), ("pad", np.int32)])
    tr = np.frombuffer(trace, dtype=dt, count=min(r, cap)).copy()
    return JacobiResult(color, r, tr, rc == 0)


def assign(g, wl, snapshot) -> np.ndarray:
    """One assignment step (Alg. 5 l.4-10) of the listed vertices against `snapshot`."""
    rp, ci, n = _csr(g)
    wl = np.ascontiguousarray(wl, dtype=np.int32)
    snap = np.ascontiguousarray(snapshot, dtype=np.int32)
    tent = np.zeros(len(wl), np.int32)
    _check(_load().oracle_assign(_ptr(rp), _ptr(ci), n, _ptr(wl), len(wl), _ptr(snap),
                                 _ptr(tent)), "assign")
    return tent


def detect(g, wl, colors, tiebreak: int = TIEBREAK_LOWID_KEEPS) -> np.ndarray:
    """One detection step (Alg. 5 l.12-18) of the listed vertices; returns uint8 flags."""
    rp, ci, n = _csr(g)
    wl = np.ascontiguousarray(wl, dtype=np.int32)
    col = np.ascontiguousarray(colors, dtype=np.int32)
    out = np.zeros(len(wl), np.uint8)
    _check(_load().oracle_detect(_ptr(rp), _ptr(ci), n, _ptr(wl), len(wl), _ptr(col),
                                 tiebreak, _ptr(out)), "detect")
    return out


def jacobi_partitioned(g, P: int, tiebreak: int = TIEBREAK_LOWID_KEEPS, ranges=None):
    """O2 on P logical ranks with explicit (v, color) exchange; returns (colors, rounds)."""
    rp, ci, n = _csr(g)
    color = np.zeros(n, np.int32)
    rounds = ctypes.c_int64(0)
    rg = None if ranges is None else np.ascontiguousarray(ranges, dtype=np.int64)
    rc = _load().oracle_jacobi_partitioned(_ptr(rp), _ptr(ci), n, tiebreak, P,
                                           None if rg is None else rg.ctypes.data,
                                           _ptr(color), ctypes.byref(rounds))
    _check(rc, "jacobi_partitioned")
    return color, rounds.value


def max_threads() -> int:
    return int(_load().oracle_max_threads())
