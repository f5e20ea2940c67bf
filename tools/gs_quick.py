import sys, os, statistics
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_licqfsty16_b200 as sgr
from paper_conf_ipps_licqfsty16_b200 import gen
g = gen.config(4)
rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
for K, p in [(16, "blocked"), (4, "blocked")]:
    ms = []
    for _ in range(3):
        r = sgr.color_gs(rp, ci, K, p)
        ms.append(r.stats["elapsed_ms"])
    print(os.environ.get("SGR_LIBPATH", "default"), K, p, round(statistics.median(ms), 1), r.stats["rounds"], flush=True)
