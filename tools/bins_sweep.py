"""Sweep the degree-bin boundaries (opts.bin_small_max / bin_med_max) on one config; every
coloring is compared bit-exactly with the default boundaries' colors."""
import os
import sys
import statistics

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402
from paper_conf_ipps_licqfsty16_b200 import gen  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 4
g = gen.config(cfg)
rp = torch.from_numpy(g.row_ptr).cuda()
ci = torch.from_numpy(g.col_idx).cuda()
ref = sgr.color(rp, ci).colors.clone()
for sm, mm in [(0, 0), (32, 128), (32, 192), (32, 96), (16, 256), (24, 256), (16, 128)]:
    ms = []
    for _ in range(4):
        r = sgr.color(rp, ci, bin_small_max=sm, bin_med_max=mm)
        ms.append(r.stats["elapsed_ms"])
    same = bool(torch.equal(r.colors, ref))
    print(f"cfg{cfg} small_max={sm} med_max={mm}: {statistics.median(ms[1:]):.2f} ms  same={same}  "
          f"entries/nnz={r.stats['entries_read'] / g.nnz:.2f}", flush=True)
