"""Per-round rates: host loop with CUDA events per round pass, joined with the round trace."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402
from paper_conf_ipps_licqfsty16_b200 import gen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=4)
ap.add_argument("--tiebreak", default="lowid")
ap.add_argument("--every", type=int, default=10)
args = ap.parse_args()
g = gen.config(args.config)
rp = torch.from_numpy(g.row_ptr).cuda()
ci = torch.from_numpy(g.col_idx).cuda()
sgr.color(rp, ci, args.tiebreak)
res = sgr.color(rp, ci, args.tiebreak, trace=True, profile=True, loop_mode="host", rounds_per_batch=1)
ms = res.extra["round_ms"]  # pass k = 2.. (one per round pass, incl. trailing no-op passes)
R = res.stats["rounds"]
sizes, edges = res.round_sizes, res.round_edges
print(f"rounds {R} total {res.stats['elapsed_ms']:.2f} ms, round kernels {res.stats['kernel_ms']}")
print(" k     |W_k|    entries      us   Gent/s")
tot_us = 0
for k in range(2, R + 1):
    us = ms[k - 2] * 1e3
    tot_us += us
    if k < 12 or k % args.every == 0 or k > R - 3:
        print(f"{k:3d} {sizes[k-1]:9d} {edges[k-1]:11d} {us:8.1f} {edges[k-1]/max(us,1e-3)/1e3:7.1f}")
cum = np.cumsum(ms[: R - 1])
half = int(np.searchsorted(cum, cum[-1] / 2)) + 2
print(f"sum of round passes {tot_us/1e3:.2f} ms; half the time is spent by round {half}")
