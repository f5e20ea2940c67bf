import sys, os
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_licqfsty16_b200 as sgr
from paper_conf_ipps_licqfsty16_b200 import gen
g = gen.config(2)
rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
for kw in [dict(), dict(profile=True), dict(block_size=256), dict(loop_mode="auto"), dict(trace=True), dict(profile=True, block_size=256, loop_mode="auto")]:
    for _ in range(2):
        r = sgr.color(rp, ci, "lowid", **kw)
    print(kw, round(r.stats["elapsed_ms"], 2), r.stats["bin_vertices"], r.stats.get("launches"))
