"""Early-round cost by bin configuration (host loop, per-round events)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402
from paper_conf_ipps_licqfsty16_b200 import gen  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 4
g = gen.config(cfg)
rp = torch.from_numpy(g.row_ptr).cuda()
ci = torch.from_numpy(g.col_idx).cuda()
for name, kw in [("default", {}), ("all-bin2", dict(bin_small_max=1, bin_med_max=1)),
                 ("no-bin1", dict(bin_med_max=32)), ("i32", dict(color_bits=32)),
                 ("persistent", dict(loop_mode="persistent"))]:
    lm = kw.pop("loop_mode", "host")
    sgr.color(rp, ci, **kw, loop_mode=lm)
    res = sgr.color(rp, ci, trace=True, profile=True, loop_mode=lm, rounds_per_batch=1, **kw)
    ms = res.extra["round_ms"]
    R = res.stats["rounds"]
    early = ms[:10].sum()
    print(f"{name:10s} total {res.stats['elapsed_ms']:7.2f} ms  rounds2-11 {early:6.2f} ms  "
          f"rest {ms[10:R-1].sum():6.2f} ms  k2 {ms[0]:.3f}  entries_read {res.stats['entries_read']/g.nnz:.2f} nnz "
          f"bin_vertices {res.stats['bin_vertices']} grid {res.stats['grid_blocks']}")
