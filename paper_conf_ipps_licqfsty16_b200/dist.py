"""Multi-GPU binding: one process per GPU, torch.distributed for bootstrap.

The round loop and every exchange run inside libsgr.so (sgr_color_dist, NCCL); Python only
broadcasts the 128-byte ncclUniqueId and slices the rank's owned rows.
"""
from __future__ import annotations

import ctypes

import numpy as np

from ._lib import Csr, Stats, check, load


class Comm:
    """NCCL communicator owned by libsgr (created from a torch.distributed process group)."""

    def __init__(self, rank: int, world: int, device: int, group=None):
        import torch
        import torch.distributed as dist
        lib = load()
        uid = torch.zeros(128, dtype=torch.uint8)
        if rank == 0:
            buf = (ctypes.c_uint8 * 128)()
            check(lib.sgr_nccl_unique_id(ctypes.cast(buf, ctypes.c_void_p)), "sgr_nccl_unique_id")
            uid.copy_(torch.frombuffer(bytearray(buf), dtype=torch.uint8))
        backend = dist.get_backend(group)
        if backend == "nccl":
            t = uid.cuda(device)
            dist.broadcast(t, 0, group=group)
            uid = t.cpu()
        else:
            dist.broadcast(uid, 0, group=group)
        raw = (ctypes.c_uint8 * 128)(*uid.tolist())
        self.ptr = ctypes.c_void_p()
        check(lib.sgr_comm_init(ctypes.byref(self.ptr), rank, world,
                                ctypes.cast(raw, ctypes.c_void_p), device), "sgr_comm_init")
        self.rank, self.world, self.device = rank, world, device

    def close(self):
        if self.ptr:
            load().sgr_comm_destroy(self.ptr)
            self.ptr = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def local_rows(row_ptr: np.ndarray, col_idx: np.ndarray, v_begin: int, v_end: int):
    """Owned rows [v_begin, v_end) with local offsets and global column ids (host)."""
    lo, hi = int(row_ptr[v_begin]), int(row_ptr[v_end])
    return (row_ptr[v_begin:v_end + 1] - lo).astype(np.int64), col_idx[lo:hi]


def color_dist(comm: Comm, local_row_ptr, local_col_idx, n_global: int, v_begin: int,
               v_end: int, tiebreak="lowid", *, stream=None, **opt_kw):
    """Collective over comm: every rank passes its owned rows (device tensors); returns the
    full coloring (device int32, n_global) on every rank plus stats."""
    import torch
    from . import ColorResult, make_opts
    colors = torch.empty(n_global, dtype=torch.int32, device=local_row_ptr.device)
    opts = make_opts(tiebreak, stream, **opt_kw)
    nnz_local = local_col_idx.numel()
    csr = Csr(local_row_ptr.data_ptr(), local_col_idx.data_ptr() if nnz_local else None)
    st = Stats()
    check(load().sgr_color_dist(comm.ptr, ctypes.byref(csr), n_global, v_begin, v_end,
                                nnz_local, colors.data_ptr() if n_global else None,
                                ctypes.byref(st), ctypes.byref(opts)), "sgr_color_dist")
    return ColorResult(colors, st.as_dict())
