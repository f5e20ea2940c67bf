"""Native build for the repo: nvcc (sm_100a) for the CUDA library, g++/gcc for the
generator and the CPU oracle. Invoked by ``__graft_entry__.build()`` and ``make``.

Artefacts (git-ignored, but shipped to the GPU box by gpurun):
  paper_conf_ipps_licqfsty16_b200/lib/libsgr.so      CUDA path (C ABI: include/sgr.h)
  paper_conf_ipps_licqfsty16_b200/lib/libsgr_gen.so  input generators (include/sgr_gen.h)
  oracle/liboracle.so                                CPU oracle (test infrastructure only)
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys
import sysconfig
from pathlib import Path

PKG = Path(__file__).resolve().parent
ROOT = PKG.parent
LIB = PKG / "lib"
CSRC = PKG / "csrc"
INCLUDE = ROOT / "include"

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_dirs():
    """NCCL headers/lib: link against the libnccl.so.2 torch loads (pip nvidia-nccl)."""
    for sp in [sysconfig.get_paths()["purelib"]] + sys.path:
        d = Path(sp) / "nvidia" / "nccl"
        if (d / "include" / "nccl.h").exists() and (d / "lib" / "libnccl.so.2").exists():
            return d / "include", d / "lib"
    return None, None


def _run(cmd, cwd=None):
    print("+", " ".join(str(c) for c in cmd), flush=True)
    subprocess.run([str(c) for c in cmd], check=True, cwd=cwd)


def _newer(out: Path, srcs) -> bool:
    if not out.exists():
        return False
    t = out.stat().st_mtime
    return all(Path(s).stat().st_mtime <= t for s in srcs)


def build_gen(force=False):
    LIB.mkdir(exist_ok=True)
    out = LIB / "libsgr_gen.so"
    srcs = [PKG / "gen" / "sgr_gen.cpp", INCLUDE / "sgr_gen.h"]
    if not force and _newer(out, srcs):
        return out
    _run(["g++", "-O3", "-std=c++17", "-fPIC", "-shared", "-fopenmp", "-Wall",
          "-o", out, srcs[0]])
    return out


def build_oracle(force=False):
    odir = ROOT / "oracle"
    out = odir / "liboracle.so"
    srcs = [odir / "sgr_oracle.c", odir / "sgr_oracle.h"]
    if not all(s.exists() for s in srcs):
        return None
    if not force and _newer(out, srcs):
        return out
    _run(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-fopenmp", "-Wall", "-Wextra",
          "-o", out, srcs[0]])
    return out


def build_cuda(force=False, out=None, extra=(), tag="obj"):
    """libsgr.so; `out`/`extra` build an alternative (tools/variants.py experiments)."""
    LIB.mkdir(exist_ok=True)
    out = Path(out) if out else LIB / "libsgr.so"
    cu = sorted(CSRC.glob("*.cu"))
    if not cu:
        return None
    deps = cu + sorted(CSRC.glob("*.cuh")) + sorted(CSRC.glob("*.h")) + [INCLUDE / "sgr.h"]
    if not force and _newer(out, deps):
        return out
    nccl_inc, nccl_lib = _nccl_dirs()
    flags = ["-O3", "-std=c++17", "-lineinfo", *ARCH, "-Xcompiler", "-fPIC,-Wall",
             "-Xptxas", "-v", "--expt-relaxed-constexpr", "-I", INCLUDE, "-I", CSRC, *extra]
    link = ["-shared", "-lcudart"]
    if nccl_inc is not None:
        flags += ["-DSGR_HAVE_NCCL=1", "-I", nccl_inc]
        link += ["-L", nccl_lib, "-l:libnccl.so.2", f"-Xlinker=-rpath,{nccl_lib}"]
    objs = []
    bdir = LIB / tag
    bdir.mkdir(exist_ok=True)
    for src in cu:
        obj = bdir / (src.stem + ".o")
        _run([NVCC, *flags, "-c", "-o", obj, src])
        objs.append(obj)
    _run([NVCC, *ARCH, "-o", out, *objs, *link])
    shutil.rmtree(bdir, ignore_errors=True)
    return out


def build_all(force=False):
    build_gen(force)
    build_oracle(force)
    build_cuda(force)


if __name__ == "__main__":
    build_all(force="--force" in sys.argv)
