"""C-ABI checks that need no GPU (-m "not gpu"): libsgr.so loads, exports every symbol that
include/sgr.h declares, host-only entry points work, and the product path refuses to run
without CUDA tensors (there is no CPU fallback)."""
from __future__ import annotations

import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared(header: str):
    src = open(os.path.join(ROOT, "include", header)).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sgr_[a-z0-9_]+)\s*\(", src)))


def test_libsgr_exports_everything_in_sgr_h():
    from paper_conf_ipps_licqfsty16_b200 import _lib
    lib = _lib.load()
    names = declared("sgr.h")
    assert "sgr_color" in names and "sgr_color_dist" in names and "sgr_compact" in names
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    nm = subprocess.run(["nm", "-D", "--defined-only", str(_lib.LIBPATH)], capture_output=True,
                        text=True, check=True).stdout
    for n in names:
        assert re.search(rf"\bT {n}\b", nm), n


def test_libsgr_is_sm100a():
    from paper_conf_ipps_licqfsty16_b200 import _lib
    out = subprocess.run(["cuobjdump", "--list-elf", str(_lib.LIBPATH)], capture_output=True,
                         text=True, check=True).stdout
    assert "sm_100a" in out


def test_generator_exports_everything_in_sgr_gen_h():
    from paper_conf_ipps_licqfsty16_b200 import gen
    lib = gen._load()
    for n in declared("sgr_gen.h"):
        assert hasattr(lib, n), n


def test_host_entry_points_without_gpu():
    import paper_conf_ipps_licqfsty16_b200 as sgr
    lib = sgr._lib.load()
    assert b"sm_100a" in lib.sgr_version()
    assert lib.sgr_strerror(-1) == b"invalid argument"
    rp = np.array([0, 5, 10, 10, 12, 30], np.int64)  # nnz = 30
    r = sgr.partition(rp, 3)
    assert r.tolist() == [0, 2, 5, 5]  # targets 10, 20 -> first v with row_ptr[v] >= target
    assert r[0] == 0 and r[-1] == 5 and np.all(np.diff(r) >= 0)
    # default options
    o = sgr._lib.Opts()
    lib.sgr_opts_default(ctypes.byref(o))
    assert o.tiebreak == 0 and o.loop_mode == 0
    assert o.unsorted_rows == 0 and o.flat_bin0 == 0  # last fields: the struct sizes agree
    assert sgr.workspace_bytes(1000, 5000) > 4 * 4 * 1000  # Y, 2 thread lists, slots
    # invalid arguments are rejected before touching the device
    st = sgr._lib.Stats()
    assert lib.sgr_color(None, 10, 0, None, ctypes.byref(st)) == -1
    assert lib.sgr_color_ex(None, -1, 0, None, None, None, None, 0) == -1
    # batch entry point: count < 0, null arrays, a bad graph in the batch; count 0 is a no-op
    assert lib.sgr_color_host_batch(None, None, None, None, None, -1, None, None) == -1
    assert lib.sgr_color_host_batch(None, None, None, None, None, 1, None, None) == -1
    assert lib.sgr_color_host_batch(None, None, None, None, None, 0, None, None) == 0
    VP, I64 = ctypes.c_void_p, ctypes.c_int64
    one = np.zeros(2, np.int64)
    bad_n = lib.sgr_color_host_batch((VP * 1)(one.ctypes.data), (VP * 1)(None), (I64 * 1)(-1),
                                     (I64 * 1)(0), (VP * 1)(None), 1, None, None)
    assert bad_n == -1
    no_ci = lib.sgr_color_host_batch((VP * 1)(one.ctypes.data), (VP * 1)(None), (I64 * 1)(1),
                                     (I64 * 1)(3), (VP * 1)(one.ctypes.data), 1, None, None)
    assert no_ci == -1  # nnz > 0 with a null col_idx


def test_partition_balances_nnz():
    import paper_conf_ipps_licqfsty16_b200 as sgr
    from paper_conf_ipps_licqfsty16_b200 import gen
    g = gen.config(1)
    for P in (1, 2, 4, 8):
        r = sgr.partition(g.row_ptr, P)
        assert r[0] == 0 and r[-1] == g.n and np.all(np.diff(r) >= 0)
        for p in range(1, P):
            target = -(-p * g.nnz // P)
            assert g.row_ptr[r[p]] >= target and (r[p] == 0 or g.row_ptr[r[p] - 1] < target)


def test_product_path_refuses_cpu_tensors():
    torch = pytest.importorskip("torch")
    import paper_conf_ipps_licqfsty16_b200 as sgr
    rp = torch.zeros(2, dtype=torch.int64)
    ci = torch.zeros(0, dtype=torch.int32)
    with pytest.raises(TypeError):
        sgr.color(rp, ci)
