"""Small colorings through every kernel family, for compute-sanitizer (SURVEY §4 layer 5):

    compute-sanitizer --tool memcheck  --leak-check full python tools/sanitize_run.py
    compute-sanitizer --tool initcheck python tools/sanitize_run.py
    compute-sanitizer --tool synccheck python tools/sanitize_run.py
    compute-sanitizer --tool racecheck python tools/sanitize_run.py

Covers: the persistent kernel (hub build with multi-chunk rows and TMA stages, flat build
with dense and sparse passes, both bin-0 mappings of the flat build), both color widths, the host loop (k_round, k_finalize),
the graph loop, the topology-driven kernels, the step entry points, the sub-step variants
and the partitioned (multi-GPU protocol) path. Every result is checked against the oracle
so a run that "passes" the sanitizer also colored correctly.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402
from paper_conf_ipps_licqfsty16_b200 import gen  # noqa: E402


def hub_graph():
    """A few hubs of degree > 1020 (multi-chunk bin-2 rows) plus an R-MAT body."""
    g = gen.rmat(11, 8, 0.57, 0.19, 0.19, seed=5)
    n = 4096
    src = np.repeat(np.arange(3), 1500)
    dst = np.random.default_rng(0).integers(3, n, 4500)
    e = [np.stack([src, dst], 1)]
    rp, ci = g.row_ptr, g.col_idx
    u = np.repeat(np.arange(g.n), np.diff(rp))
    e.append(np.stack([u, ci], 1))
    return gen.from_edges(n, np.concatenate(e).astype(np.int64))


def check(name, got, ref):
    ok = np.array_equal(got, ref)
    print(f"{name}: {'ok' if ok else 'MISMATCH'}", flush=True)
    if not ok:
        sys.exit(1)


def main():
    graphs = {"hub": hub_graph(), "stencil": gen.stencil3d(10, 9, 8, 27),
              "er": gen.er(3000, 12000, seed=1)}
    for name, g in graphs.items():
        rp = torch.from_numpy(g.row_ptr).cuda()
        ci = torch.from_numpy(g.col_idx).cuda()
        ref = oracle.jacobi(g, 0).colors
        for bits in (16, 32):
            for mode in ("persistent", "host", "graph"):
                r = sgr.color(rp, ci, "lowid", color_bits=bits, loop_mode=mode)
                check(f"{name} color bits={bits} {mode}", r.colors.cpu().numpy(), ref)
        for mapping in (1, 2):  # flat build: 4-lane groups / thread-per-vertex instantiation
            r = sgr.color(rp, ci, "lowid", flat_bin0=mapping)
            check(f"{name} flat_bin0={mapping}", r.colors.cpu().numpy(), ref)
        r = sgr.color(rp, ci, "paper", flat_bin0=2)
        check(f"{name} flat_bin0=2 paper", r.colors.cpu().numpy(), oracle.jacobi(g, 1).colors)
        check(f"{name} topo", sgr.color_topo(rp, ci).colors.cpu().numpy(), ref)
        check(f"{name} partitioned P=3", sgr.color_partitioned(rp, ci, 3).colors.cpu().numpy(), ref)
        check(f"{name} gs K=4", sgr.color_gs(rp, ci, 4, "strided").colors.cpu().numpy(),
              oracle.gauss_seidel(g, 4, 0, 0).colors)
        rng = np.random.default_rng(1)
        snap = rng.integers(0, 9, g.n).astype(np.int32)
        wl = np.sort(rng.choice(g.n, g.n // 2, replace=False)).astype(np.int32)
        twl, tsnap = torch.from_numpy(wl).cuda(), torch.from_numpy(snap).cuda()
        check(f"{name} assign", sgr.assign(rp, ci, twl, tsnap).cpu().numpy(), oracle.assign(g, wl, snap))
        fl = sgr.detect(rp, ci, twl, tsnap)
        check(f"{name} detect", fl.cpu().numpy(), oracle.detect(g, wl, snap, 0))
        check(f"{name} compact", sgr.compact(twl, fl).cpu().numpy(), wl[oracle.detect(g, wl, snap, 0).astype(bool)])
    torch.cuda.synchronize()
    print("sanitize_run: all colorings match the oracle")


if __name__ == "__main__":
    main()
