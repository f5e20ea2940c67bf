"""Per-round device time in the persistent kernel (%globaltimer stamps written by the loop
control at the end of every pass), joined with the round trace."""
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
ns = torch.zeros(g.n + 2, dtype=torch.int64, device="cuda")
res = sgr.color(rp, ci, args.tiebreak, trace=True, round_ns=ns, loop_mode="persistent")
R = res.stats["rounds"]
t = ns[:R].cpu().numpy()
us = np.diff(t) / 1e3  # pass k = 2..R
sizes, edges = res.round_sizes, res.round_edges
print(f"rounds {R} elapsed {res.stats['elapsed_ms']:.2f} ms; passes {us.sum()/1e3:.2f} ms")
print(" k     |W_k|    entries      us   Gent/s")
for k in range(2, R + 1):
    u = us[k - 2]
    if k < 12 or k % args.every == 0 or k > R - 3:
        print(f"{k:3d} {sizes[k-1]:9d} {edges[k-1]:11d} {u:8.1f} {edges[k-1]/max(u,1e-3)/1e3:7.1f}")
cum = np.cumsum(us)
for lo, hi in [(2, 11), (12, 30), (31, 60), (61, 100), (101, 150), (151, 200), (201, R)]:
    sel = slice(lo - 2, min(hi, R) - 1)
    print(f"rounds {lo:3d}-{min(hi, R):3d}: {us[sel].sum()/1e3:7.2f} ms, entries {np.sum(edges[lo-1:min(hi, R)])/1e6:9.1f} M")
np.save("/tmp/round_us.npy", us)
small = us[np.asarray(sizes[1:R]) < 1000]
print(f"passes with |W| < 1000: {len(small)}, {small.sum()/1e3:.2f} ms, median {np.median(small) if len(small) else 0:.1f} us")
