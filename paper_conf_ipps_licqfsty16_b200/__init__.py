"""paper_conf_ipps_licqfsty16_b200 — deterministic speculative-greedy (SGR) graph coloring on
B200 (sm_100a), after Li et al., "High Performance Parallel Graph Coloring on GPGPUs"
(IPDPS-W 2016; Algorithm 5).

Thin Python binding over the C ABI of libsgr.so (include/sgr.h): argument marshalling only,
every step of the coloring runs in the library's CUDA kernels. PyTorch provides device
memory, streams and (for multi-GPU) the process group; there is no CPU fallback — calls
raise if the CUDA library is not built or no GPU is present.

    import torch, paper_conf_ipps_licqfsty16_b200 as sgr
    g = sgr.gen.config(4)                                   # RMAT scale-24 (host CSR)
    rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
    res = sgr.color(rp, ci)                                  # Jacobi-SGR, LOWID_KEEPS
    res.colors, res.stats["rounds"], res.stats["num_colors"]
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass, field

import numpy as np

from . import gen  # noqa: F401  (seeded input generators; no coloring arithmetic)
from ._lib import Csr, Opts, Stats, check, load

TIEBREAK = {"lowid": 0, "lowid_keeps": 0, "paper": 1}
LOOP = {"auto": 0, "graph": 1, "persistent": 2, "host": 3}

__all__ = ["color", "color_host", "color_host_batch", "color_topo", "color_gs", "color_partitioned", "color_dist", "assign", "commit",
           "detect", "compact", "validate_csr", "partition", "workspace_bytes", "gen",
           "ColorResult", "TIEBREAK"]


def _torch():
    import torch
    return torch


def _tb(tiebreak) -> int:
    if isinstance(tiebreak, str):
        return TIEBREAK[tiebreak.lower()]
    return int(tiebreak)


def _stream_ptr(stream):
    torch = _torch()
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _require_cuda(*tensors):
    torch = _torch()
    for t in tensors:
        if not isinstance(t, torch.Tensor) or not t.is_cuda:
            raise TypeError("expected CUDA tensors (the library has no CPU path)")
        if not t.is_contiguous():
            raise ValueError("tensors must be contiguous")


def _check_csr(row_ptr, col_idx):
    torch = _torch()
    _require_cuda(row_ptr, col_idx)
    if row_ptr.dtype != torch.int64 or col_idx.dtype != torch.int32:
        raise TypeError("row_ptr must be int64 and col_idx int32")


def make_opts(tiebreak="lowid", stream=None, max_rounds=0, loop_mode="auto", color_bits=0,
              bin_small_max=0, bin_med_max=0, validate=False, rounds_per_batch=0,
              profile=False, round_sizes=None, round_edges=None, round_cap=0,
              round_ms=None, color_cap=0, round_ns=None, block_size=0,
              unsorted_rows=False, flat_bin0=0) -> Opts:
    o = Opts()
    load().sgr_opts_default(ctypes.byref(o))
    o.tiebreak = _tb(tiebreak)
    o.max_rounds = int(max_rounds)
    o.loop_mode = LOOP[loop_mode] if isinstance(loop_mode, str) else int(loop_mode)
    o.color_bits = int(color_bits)
    o.bin_small_max = int(bin_small_max)
    o.bin_med_max = int(bin_med_max)
    o.stream = _stream_ptr(stream)
    o.validate = int(bool(validate))
    o.rounds_per_batch = int(rounds_per_batch)
    o.profile = int(bool(profile))
    o.round_sizes = round_sizes.data_ptr() if round_sizes is not None else None
    o.round_edges = round_edges.data_ptr() if round_edges is not None else None
    o.round_cap = int(round_cap)
    o.round_ms = round_ms.ctypes.data if round_ms is not None else None
    o.color_cap = int(color_cap)
    o.round_ns = round_ns.data_ptr() if round_ns is not None else None
    o.block_size = int(block_size)
    o.unsorted_rows = int(bool(unsorted_rows))
    o.flat_bin0 = int(flat_bin0)
    return o


@dataclass
class ColorResult:
    colors: object                       # torch.int32 CUDA tensor (or numpy for color_host)
    stats: dict
    round_sizes: np.ndarray | None = None  # |W_r|, r = 1..R (trace=True)
    round_edges: np.ndarray | None = None  # sum deg(W_r)
    extra: dict = field(default_factory=dict)


def workspace_bytes(n: int, nnz: int) -> int:
    return int(load().sgr_workspace_bytes(n, nnz, None))


def color(row_ptr, col_idx, tiebreak="lowid", *, out=None, stream=None, trace=False,
          workspace=None, sync_stats=True, **opt_kw) -> ColorResult:
    """Color a device CSR (row_ptr int64[n+1], col_idx int32[nnz], symmetric, sorted rows).

    Returns colors (int32, 1-based, proper) and stats (rounds, num_colors, ...). With
    trace=True also the per-round worklist sizes |W_r| and scanned entries."""
    torch = _torch()
    _check_csr(row_ptr, col_idx)
    n = row_ptr.numel() - 1
    nnz = col_idx.numel()
    colors = out if out is not None else torch.empty(n, dtype=torch.int32, device=row_ptr.device)
    _require_cuda(colors)
    rs = re = None
    if trace:
        rs = torch.zeros(n + 2, dtype=torch.int32, device=row_ptr.device)
        re = torch.zeros(n + 2, dtype=torch.int64, device=row_ptr.device)
    rms = np.zeros(n + 2, np.float32) if trace else None
    opts = make_opts(tiebreak, stream, round_sizes=rs, round_edges=re,
                     round_cap=(n + 2) if trace else 0, round_ms=rms, **opt_kw)
    csr = Csr(row_ptr.data_ptr(), col_idx.data_ptr() if nnz else None)
    st = Stats()
    ws_ptr, ws_len = None, 0
    if workspace is not None:
        ws_ptr, ws_len = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    check(load().sgr_color_ex(ctypes.byref(csr), n, nnz, colors.data_ptr() if n else None,
                              ctypes.byref(st), ctypes.byref(opts), ws_ptr, ws_len),
          "sgr_color_ex")
    res = ColorResult(colors, st.as_dict())
    if trace:
        R = res.stats["rounds"]
        res.round_sizes = rs[:R].cpu().numpy()
        res.round_edges = re[:R].cpu().numpy()
        res.extra["round_ms"] = rms[:R]
    return res


def color_topo(row_ptr, col_idx, tiebreak="lowid", *, out=None, stream=None, trace=False,
               **opt_kw) -> ColorResult:
    """Topology-driven mapping (the paper's Algorithm 4, T-base): every iteration visits all
    vertices, one thread each, and the host reads the `changed` count. Same result as
    color() (colors, rounds, |W_r|); the comparison mapping, not the fast path."""
    torch = _torch()
    _check_csr(row_ptr, col_idx)
    n = row_ptr.numel() - 1
    nnz = col_idx.numel()
    colors = out if out is not None else torch.empty(n, dtype=torch.int32, device=row_ptr.device)
    _require_cuda(colors)
    rs = torch.zeros(n + 2, dtype=torch.int32, device=row_ptr.device) if trace else None
    opts = make_opts(tiebreak, stream, round_sizes=rs, round_cap=(n + 2) if trace else 0, **opt_kw)
    csr = Csr(row_ptr.data_ptr(), col_idx.data_ptr() if nnz else None)
    st = Stats()
    check(load().sgr_color_topo(ctypes.byref(csr), n, nnz, colors.data_ptr() if n else None,
                                ctypes.byref(st), ctypes.byref(opts)), "sgr_color_topo")
    res = ColorResult(colors, st.as_dict())
    if trace:
        res.round_sizes = rs[:res.stats["rounds"]].cpu().numpy()
    return res


GS_PARTITION = {"strided": 0, "blocked": 1, "inplace": 2}


def color_gs(row_ptr, col_idx, substeps=16, partition="strided", tiebreak="lowid", *, out=None,
             stream=None, trace=False, **opt_kw) -> ColorResult:
    """Reduced-round variant (include/sgr.h sgr_color_gs): each round's
    assignment runs as `substeps` ordered sub-steps ("strided": v mod K, "blocked":
    floor(v K / n)), a sub-step seeing the earlier ones' colors; "inplace" is the paper's
    nondeterministic in-place mode. Different semantics (fewer rounds, more colors) from
    color(); substeps=1 equals it."""
    torch = _torch()
    _check_csr(row_ptr, col_idx)
    n = row_ptr.numel() - 1
    nnz = col_idx.numel()
    colors = out if out is not None else torch.empty(n, dtype=torch.int32, device=row_ptr.device)
    _require_cuda(colors)
    rs = re = None
    if trace:
        rs = torch.zeros(n + 2, dtype=torch.int32, device=row_ptr.device)
        re = torch.zeros(n + 2, dtype=torch.int64, device=row_ptr.device)
    opts = make_opts(tiebreak, stream, round_sizes=rs, round_edges=re,
                     round_cap=(n + 2) if trace else 0, **opt_kw)
    part = GS_PARTITION[partition] if isinstance(partition, str) else int(partition)
    csr = Csr(row_ptr.data_ptr(), col_idx.data_ptr() if nnz else None)
    st = Stats()
    check(load().sgr_color_gs(ctypes.byref(csr), n, nnz, int(substeps), part,
                              colors.data_ptr() if n else None, ctypes.byref(st),
                              ctypes.byref(opts)), "sgr_color_gs")
    res = ColorResult(colors, st.as_dict())
    if trace:
        R = res.stats["rounds"]
        res.round_sizes = rs[:R].cpu().numpy()
        res.round_edges = re[:R].cpu().numpy()
    return res


def color_host(row_ptr: np.ndarray, col_idx: np.ndarray, tiebreak="lowid", *, out=None,
               stream=None, **opt_kw) -> ColorResult:
    """End to end from HOST arrays (pinned for full speed): H2D, color, D2H, in the library."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64) if isinstance(row_ptr, np.ndarray) else row_ptr
    ci = np.ascontiguousarray(col_idx, dtype=np.int32) if isinstance(col_idx, np.ndarray) else col_idx
    n = (rp.numel() if hasattr(rp, "numel") else len(rp)) - 1
    nnz = ci.numel() if hasattr(ci, "numel") else len(ci)
    if out is None:
        out = np.zeros(n, np.int32)
    ptr = (lambda a: a.data_ptr() if hasattr(a, "data_ptr") else a.ctypes.data)
    opts = make_opts(tiebreak, stream, **opt_kw)
    st = Stats()
    check(load().sgr_color_host(ptr(rp), ptr(ci) if nnz else None, n, nnz,
                                ptr(out) if n else None, ctypes.byref(st), ctypes.byref(opts)),
          "sgr_color_host")
    return ColorResult(out, st.as_dict())


def color_host_batch(graphs, tiebreak="lowid", *, outs=None, stream=None, **opt_kw):
    """Pipelined end to end over a list of HOST graphs [(row_ptr, col_idx), ...] (pinned
    torch tensors or numpy arrays): graph i+1's upload and graph i-1's download overlap the
    coloring of graph i, in the library (sgr_color_host_batch). Returns one ColorResult
    per graph."""
    ptr = (lambda a: a.data_ptr() if hasattr(a, "data_ptr") else a.ctypes.data)
    size = (lambda a: a.numel() if hasattr(a, "numel") else len(a))
    cnt = len(graphs)
    keep, rps, cis, ns, nnzs = [], [], [], [], []
    for rp, ci in graphs:
        if isinstance(rp, np.ndarray):
            rp = np.ascontiguousarray(rp, dtype=np.int64)
        if isinstance(ci, np.ndarray):
            ci = np.ascontiguousarray(ci, dtype=np.int32)
        keep += [rp, ci]
        ns.append(size(rp) - 1)
        nnzs.append(size(ci))
        rps.append(ptr(rp))
        cis.append(ptr(ci) if nnzs[-1] else None)
    if outs is None:
        outs = [np.zeros(n, np.int32) for n in ns]
    VP, I64 = ctypes.c_void_p, ctypes.c_int64
    st = (Stats * max(cnt, 1))()
    opts = make_opts(tiebreak, stream, **opt_kw)
    check(load().sgr_color_host_batch((VP * max(cnt, 1))(*rps), (VP * max(cnt, 1))(*cis),
                                      (I64 * max(cnt, 1))(*ns), (I64 * max(cnt, 1))(*nnzs),
                                      (VP * max(cnt, 1))(*[ptr(o) if n else None for o, n in zip(outs, ns)]),
                                      cnt, st, ctypes.byref(opts)),
          "sgr_color_host_batch")
    return [ColorResult(outs[i], st[i].as_dict()) for i in range(cnt)]


def assign(row_ptr, col_idx, wl, colors_in, *, out=None, stream=None, **opt_kw):
    """Alg. 5 l.4-10 step: tent[i] = first-fit of wl[i] against the snapshot colors_in."""
    torch = _torch()
    _check_csr(row_ptr, col_idx)
    _require_cuda(wl, colors_in)
    tent = out if out is not None else torch.empty(wl.numel(), dtype=torch.int32, device=wl.device)
    csr = Csr(row_ptr.data_ptr(), col_idx.data_ptr() if col_idx.numel() else None)
    o = make_opts(stream=stream, **opt_kw)
    check(load().sgr_assign(ctypes.byref(csr), row_ptr.numel() - 1,
                            wl.data_ptr() if wl.numel() else None, wl.numel(),
                            colors_in.data_ptr() if colors_in.numel() else None,
                            tent.data_ptr() if tent.numel() else None, ctypes.byref(o)),
          "sgr_assign")
    return tent


def commit(wl, tent, colors, *, stream=None, **opt_kw):
    """Alg. 5 l.9 applied after the step: colors[wl[i]] = tent[i] (in place)."""
    _require_cuda(wl, tent, colors)
    o = make_opts(stream=stream, **opt_kw)
    check(load().sgr_commit(wl.data_ptr() if wl.numel() else None,
                            tent.data_ptr() if tent.numel() else None, wl.numel(),
                            colors.data_ptr() if colors.numel() else None, ctypes.byref(o)),
          "sgr_commit")
    return colors


def detect(row_ptr, col_idx, wl, colors, tiebreak="lowid", *, out=None, stream=None, **opt_kw):
    """Alg. 5 l.13-14 step: uint8 flag per listed vertex (1 = v loses a conflict)."""
    torch = _torch()
    _check_csr(row_ptr, col_idx)
    _require_cuda(wl, colors)
    flags = out if out is not None else torch.empty(wl.numel(), dtype=torch.uint8, device=wl.device)
    csr = Csr(row_ptr.data_ptr(), col_idx.data_ptr() if col_idx.numel() else None)
    o = make_opts(tiebreak, stream, **opt_kw)
    check(load().sgr_detect(ctypes.byref(csr), row_ptr.numel() - 1,
                            wl.data_ptr() if wl.numel() else None, wl.numel(),
                            colors.data_ptr() if colors.numel() else None,
                            flags.data_ptr() if flags.numel() else None, ctypes.byref(o)),
          "sgr_detect")
    return flags


def compact(wl, flags, *, stream=None):
    """Alg. 5 l.15 / P:228-230: order-preserving compaction; returns the new worklist."""
    torch = _torch()
    _require_cuda(wl, flags)
    out = torch.empty(max(wl.numel(), 1), dtype=torch.int32, device=wl.device)
    cnt = torch.zeros(1, dtype=torch.int64, device=wl.device)
    o = make_opts(stream=stream)
    check(load().sgr_compact(wl.data_ptr() if wl.numel() else None,
                             flags.data_ptr() if flags.numel() else None, wl.numel(),
                             out.data_ptr(), cnt.data_ptr(), ctypes.byref(o)), "sgr_compact")
    return out[: int(cnt.item())]


def validate_csr(row_ptr, col_idx, *, stream=None) -> int:
    """Device check of the CSR contract: bitmask (1 offsets, 2 range, 4 unsorted), 0 = ok."""
    _check_csr(row_ptr, col_idx)
    csr = Csr(row_ptr.data_ptr(), col_idx.data_ptr() if col_idx.numel() else None)
    v = ctypes.c_int32(0)
    check(load().sgr_validate_csr(ctypes.byref(csr), row_ptr.numel() - 1, col_idx.numel(),
                                  ctypes.byref(v), _stream_ptr(stream)), "sgr_validate_csr")
    return v.value


def partition(row_ptr: np.ndarray, P: int) -> np.ndarray:
    """nnz-balanced contiguous vertex ranges (host): P+1 boundaries."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    out = np.zeros(P + 1, np.int64)
    check(load().sgr_partition(rp.ctypes.data, len(rp) - 1, P, out.ctypes.data), "sgr_partition")
    return out


def color_partitioned(row_ptr, col_idx, P: int, ranges=None, tiebreak="lowid", *, stream=None,
                      **opt_kw) -> ColorResult:
    """P logical partitions on one GPU with the distributed exchange protocol (testing)."""
    torch = _torch()
    _check_csr(row_ptr, col_idx)
    n = row_ptr.numel() - 1
    nnz = col_idx.numel()
    if ranges is None:
        ranges = partition(row_ptr.cpu().numpy(), P)
    rg = np.ascontiguousarray(ranges, dtype=np.int64)
    colors = torch.empty(n, dtype=torch.int32, device=row_ptr.device)
    opts = make_opts(tiebreak, stream, **opt_kw)
    csr = Csr(row_ptr.data_ptr(), col_idx.data_ptr() if nnz else None)
    st = Stats()
    check(load().sgr_color_partitioned(ctypes.byref(csr), n, nnz, P, rg.ctypes.data,
                                       colors.data_ptr() if n else None, ctypes.byref(st),
                                       ctypes.byref(opts)), "sgr_color_partitioned")
    return ColorResult(colors, st.as_dict(), extra={"ranges": rg})


def version() -> str:
    return load().sgr_version().decode()


from .dist import color_dist  # noqa: E402
