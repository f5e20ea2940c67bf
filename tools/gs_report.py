"""§8(f) item 4 report: the sub-step variants (sgr_color_gs) on cfg3 / cfg4 — rounds, A,
colors vs Algorithm 1 and device time — next to the Jacobi path (sgr_color).

    python tools/gs_report.py [--configs 3 4] [--out profiles/r02_gs_variants.jsonl]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import oracle  # noqa: E402  (Algorithm 1 colors only: the quality reference)
import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402
from paper_conf_ipps_licqfsty16_b200 import gen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--configs", type=int, nargs="+", default=[3, 4])
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--out", default=None)
args = ap.parse_args()
out = open(args.out, "w") if args.out else None
for cfg in args.configs:
    g = gen.config(cfg)
    a1 = int(oracle.alg1(g).max())
    rp = torch.from_numpy(g.row_ptr).cuda()
    ci = torch.from_numpy(g.col_idx).cuda()
    runs = [("jacobi (sgr_color)", None, None)] + [(f"K={K} {p}", K, p) for K in (4, 16, 64)
                                                   for p in ("strided", "blocked")] + \
        [("inplace (paper-faithful, nondeterministic)", 1, "inplace")]
    for name, K, p in runs:
        ms = []
        for _ in range(args.reps + 1):
            res = sgr.color(rp, ci) if K is None else sgr.color_gs(rp, ci, K, p)
            ms.append(res.stats["elapsed_ms"])
        st = res.stats
        rec = {"config": gen.CONFIG_NAMES[cfg], "variant": name, "ms": statistics.median(ms[1:]),
               "gteps": g.nnz / statistics.median(ms[1:]) / 1e6, "rounds": st["rounds"],
               "A_scanned_per_nnz": st["edges_scanned"] / g.nnz, "colors": st["num_colors"],
               "alg1_colors": a1, "colors_vs_alg1": st["num_colors"] / a1}
        print(json.dumps(rec), flush=True)
        if out:
            out.write(json.dumps(rec) + "\n")
