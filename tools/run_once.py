"""Color one BASELINE config once on cuda:0 (for ncu launch lists / captures)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402
from paper_conf_ipps_licqfsty16_b200 import gen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=4)
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--tiebreak", default="lowid")
ap.add_argument("--loop-mode", default="host")
args = ap.parse_args()
g = gen.config(args.config)
rp = torch.from_numpy(g.row_ptr).cuda()
ci = torch.from_numpy(g.col_idx).cuda()
for _ in range(args.reps):
    res = sgr.color(rp, ci, args.tiebreak, loop_mode=args.loop_mode)
print({k: res.stats[k] for k in ("rounds", "num_colors", "elapsed_ms", "launches")})
