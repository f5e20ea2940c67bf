"""Topology-driven (Algorithm 4, T-base: thread per vertex over V every iteration, host
reads `changed`) vs data-driven (Algorithm 5, this library's fused worklist path) on the
same graphs — the comparison of the paper's Fig. 6 / §IV, plus the
Table I synthetic shapes (rmat-er, rmat-g at 2^20 vertices, edge factor 10).
Both mappings must give identical colors (checked). Device time per coloring, median of 3.
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402
from paper_conf_ipps_licqfsty16_b200 import gen  # noqa: E402

GRAPHS = {
    "cfg1 rmat-s16": lambda: gen.config(1),
    "rmat-er s20 ef10 (Table I)": lambda: gen.rmat(20, 10, 0.25, 0.25, 0.25, seed=1),
    "rmat-g s20 ef10 (Table I)": lambda: gen.rmat(20, 10, 0.45, 0.15, 0.15, seed=1),
    "cfg2 stencil 104^3": lambda: gen.config(2),
    "cfg3 ER 2^24": lambda: gen.config(3),
}


def timed(fn, reps=3):
    ms = []
    res = None
    for _ in range(reps):
        res = fn()
        ms.append(res.stats["elapsed_ms"])
    return statistics.median(ms), res


rows = []
for name, mk in GRAPHS.items():
    g = mk()
    rp = torch.from_numpy(g.row_ptr).cuda()
    ci = torch.from_numpy(g.col_idx).cuda()
    sgr.color(rp, ci)
    d_ms, d = timed(lambda: sgr.color(rp, ci))
    t_ms, t = timed(lambda: sgr.color_topo(rp, ci), reps=1 if g.nnz > 1e8 else 3)
    same = bool(torch.equal(d.colors, t.colors)) and d.stats["rounds"] == t.stats["rounds"]
    row = {"graph": name, "n": g.n, "nnz": g.nnz, "rounds": d.stats["rounds"],
           "colors": d.stats["num_colors"], "data_driven_ms": d_ms, "topology_driven_ms": t_ms,
           "speedup_D_over_T": t_ms / d_ms, "data_GTEPS": g.nnz / d_ms / 1e6,
           "topo_GTEPS": g.nnz / t_ms / 1e6, "identical": same}
    rows.append(row)
    print(json.dumps(row), flush=True)
    del rp, ci
    torch.cuda.empty_cache()
