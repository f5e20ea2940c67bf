"""Where the warps spend their time: SM cycles per bin, summed over warps and rounds."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402
from paper_conf_ipps_licqfsty16_b200 import gen  # noqa: E402

for cfg in [int(c) for c in sys.argv[1:]] or [4]:
    g = gen.config(cfg)
    rp = torch.from_numpy(g.row_ptr).cuda()
    ci = torch.from_numpy(g.col_idx).cuda()
    sgr.color(rp, ci)
    r = sgr.color(rp, ci).stats
    cyc = r["bin_warp_cycles"]
    tot = sum(cyc.values())
    print(f"cfg{cfg}: {r['elapsed_ms']:.2f} ms, warps {r['grid_blocks'] * 8}, "
          + ", ".join(f"{k} {100 * v / tot:.1f}% ({v / (r['grid_blocks'] * 8) / 1.9e6:.2f} ms/warp)"
                      for k, v in cyc.items())
          + f" | vertices {r['bin_vertices']} entries_read {r['entries_read']} edges {r['bin_edges']}")
