"""ctypes loader for libsgr.so (include/sgr.h). Argument marshalling only.

There is no fallback: if the CUDA library is missing or fails to load, every call raises.
"""
from __future__ import annotations

import ctypes
import os
from pathlib import Path

LIBPATH = Path(__file__).resolve().parent / "lib" / "libsgr.so"
# experiments only (tools/variants.py): load an alternative build of the same library
if os.environ.get("SGR_LIBPATH"):
    LIBPATH = Path(os.environ["SGR_LIBPATH"])

SGR_K_COUNT = 4
KERNEL_CLASSES = ("first", "round", "control", "final")
BINS = ("thread", "group", "chunk")


class Csr(ctypes.Structure):
    _fields_ = [("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p)]


class Opts(ctypes.Structure):
    _fields_ = [("tiebreak", ctypes.c_int32), ("max_rounds", ctypes.c_int32),
                ("loop_mode", ctypes.c_int32), ("color_bits", ctypes.c_int32),
                ("bin_small_max", ctypes.c_int32), ("bin_med_max", ctypes.c_int32),
                ("stream", ctypes.c_void_p), ("round_sizes", ctypes.c_void_p),
                ("round_edges", ctypes.c_void_p), ("round_cap", ctypes.c_int32),
                ("validate", ctypes.c_int32), ("rounds_per_batch", ctypes.c_int32),
                ("profile", ctypes.c_int32), ("round_ms", ctypes.c_void_p),
                ("round_ns", ctypes.c_void_p), ("color_cap", ctypes.c_int32),
                ("block_size", ctypes.c_int32), ("unsorted_rows", ctypes.c_int32),
                ("flat_bin0", ctypes.c_int32)]


class Stats(ctypes.Structure):
    _fields_ = [("rounds", ctypes.c_int32), ("num_colors", ctypes.c_int32),
                ("vertices_processed", ctypes.c_int64), ("edges_scanned", ctypes.c_int64),
                ("entries_read", ctypes.c_int64),
                ("bytes_algorithmic", ctypes.c_int64), ("elapsed_ms", ctypes.c_float),
                ("launches", ctypes.c_int32),
                ("kernel_ms", ctypes.c_float * SGR_K_COUNT),
                ("kernel_launches", ctypes.c_int64 * SGR_K_COUNT),
                ("kernel_bytes", ctypes.c_int64 * SGR_K_COUNT),
                ("bin_vertices", ctypes.c_int64 * 3), ("bin_edges", ctypes.c_int64 * 3),
                ("chunk_items", ctypes.c_int64), ("bin_warp_cycles", ctypes.c_int64 * 3),
                ("grid_blocks", ctypes.c_int32),
                ("color_bits", ctypes.c_int32), ("entries_written", ctypes.c_int64),
                ("transport", ctypes.c_int32)]

    def as_dict(self) -> dict:
        d = {k: getattr(self, k) for k in ("rounds", "num_colors", "vertices_processed",
                                             "edges_scanned", "entries_read", "bytes_algorithmic",
                                             "elapsed_ms", "launches")}
        d["kernel_ms"] = dict(zip(KERNEL_CLASSES, list(self.kernel_ms)))
        d["kernel_launches"] = dict(zip(KERNEL_CLASSES, list(self.kernel_launches)))
        d["kernel_bytes"] = dict(zip(KERNEL_CLASSES, list(self.kernel_bytes)))
        d["bin_vertices"] = dict(zip(BINS, list(self.bin_vertices)))
        d["bin_edges"] = dict(zip(BINS, list(self.bin_edges)))
        d["chunk_items"] = self.chunk_items
        d["bin_warp_cycles"] = dict(zip(BINS, list(self.bin_warp_cycles)))
        d["grid_blocks"] = self.grid_blocks
        d["entries_written"] = self.entries_written
        d["color_bits"] = self.color_bits
        d["transport"] = ("none", "device", "allgather")[self.transport] if 0 <= self.transport < 3 else self.transport
        return d


_lib = None

EXPORTS = ("sgr_opts_default", "sgr_workspace_bytes", "sgr_color", "sgr_color_ex",
           "sgr_color_host", "sgr_color_host_batch", "sgr_color_topo", "sgr_color_gs", "sgr_assign", "sgr_commit", "sgr_detect", "sgr_compact",
           "sgr_validate_csr", "sgr_partition", "sgr_nccl_unique_id", "sgr_comm_init",
           "sgr_comm_destroy", "sgr_color_dist", "sgr_color_partitioned", "sgr_strerror",
           "sgr_last_error", "sgr_version")


def load():
    """Load libsgr.so (raises if it is missing: there is no CPU fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not LIBPATH.exists():
        raise ImportError(f"CUDA library {LIBPATH} is not built; run "
                          "`python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(str(LIBPATH))
    vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
    P = ctypes.POINTER
    lib.sgr_opts_default.argtypes = [P(Opts)]
    lib.sgr_opts_default.restype = None
    lib.sgr_workspace_bytes.argtypes = [i64, i64, P(Opts)]
    lib.sgr_workspace_bytes.restype = ctypes.c_size_t
    lib.sgr_color.argtypes = [P(Csr), i64, i64, vp, P(Stats)]
    lib.sgr_color_ex.argtypes = [P(Csr), i64, i64, vp, P(Stats), P(Opts), vp, ctypes.c_size_t]
    lib.sgr_color_host.argtypes = [vp, vp, i64, i64, vp, P(Stats), P(Opts)]
    lib.sgr_color_host_batch.argtypes = [P(vp), P(vp), P(i64), P(i64), P(vp), i32, P(Stats), P(Opts)]
    lib.sgr_color_topo.argtypes = [P(Csr), i64, i64, vp, P(Stats), P(Opts)]
    lib.sgr_color_gs.argtypes = [P(Csr), i64, i64, i32, i32, vp, P(Stats), P(Opts)]
    lib.sgr_assign.argtypes = [P(Csr), i64, vp, i64, vp, vp, P(Opts)]
    lib.sgr_commit.argtypes = [vp, vp, i64, vp, P(Opts)]
    lib.sgr_detect.argtypes = [P(Csr), i64, vp, i64, vp, vp, P(Opts)]
    lib.sgr_compact.argtypes = [vp, vp, i64, vp, vp, P(Opts)]
    lib.sgr_validate_csr.argtypes = [P(Csr), i64, i64, P(i32), vp]
    lib.sgr_partition.argtypes = [vp, i64, i32, vp]
    lib.sgr_nccl_unique_id.argtypes = [vp]
    lib.sgr_comm_init.argtypes = [P(vp), i32, i32, vp, i32]
    lib.sgr_comm_destroy.argtypes = [vp]
    lib.sgr_color_dist.argtypes = [vp, P(Csr), i64, i64, i64, i64, vp, P(Stats), P(Opts)]
    lib.sgr_color_partitioned.argtypes = [P(Csr), i64, i64, i32, vp, vp, P(Stats), P(Opts)]
    lib.sgr_strerror.argtypes = [i32]
    lib.sgr_strerror.restype = ctypes.c_char_p
    lib.sgr_last_error.argtypes = []
    lib.sgr_last_error.restype = ctypes.c_char_p
    lib.sgr_version.argtypes = []
    lib.sgr_version.restype = ctypes.c_char_p
    for name in EXPORTS:
        if name not in ("sgr_opts_default", "sgr_workspace_bytes", "sgr_strerror",
                        "sgr_last_error", "sgr_version"):
            getattr(lib, name).restype = i32
    _lib = lib
    return lib


class SgrError(RuntimeError):
    def __init__(self, status: int, what: str):
        lib = load()
        msg = lib.sgr_strerror(status).decode()
        detail = lib.sgr_last_error().decode()
        super().__init__(f"{what}: {msg} ({status}) {detail}")
        self.status = status


def check(status: int, what: str):
    if status != 0:
        raise SgrError(status, what)
