"""A/B of the hub build's register budget vs warps per SM (experiment): each (library, block
size) pair colors cfg4 in its own process; bit-exact against the default build's colors.

    python tools/occupancy_ab.py lib:block [lib:block ...]   (lib 'default' = libsgr.so)
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import json, statistics, sys
sys.path.insert(0, %(root)r)
import numpy as np, torch
import paper_conf_ipps_licqfsty16_b200 as sgr
from paper_conf_ipps_licqfsty16_b200 import gen
g = gen.config(%(cfg)d)
rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
flush = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
res = sgr.color(rp, ci, block_size=%(B)d)
ms = []
for i in range(5):
    flush.fill_(i)
    res = sgr.color(rp, ci, block_size=%(B)d)
    ms.append(res.stats["elapsed_ms"])
c = res.colors.cpu().numpy()
ref = "/tmp/occ_ref_%(cfg)d.npy"
import os
if not os.path.exists(ref): np.save(ref, c)
print("RESULT " + json.dumps({"ms": statistics.median(ms), "grid": res.stats["grid_blocks"],
                              "same": bool(np.array_equal(np.load(ref), c))}))
"""
for spec in sys.argv[1:]:
    cfgs = [4]
    lib, B = spec.split(":")
    env = dict(os.environ)
    if lib != "default":
        env["SGR_LIBPATH"] = os.path.abspath(lib)
    for cfg in cfgs:
        p = subprocess.run([sys.executable, "-c", CHILD % {"root": ROOT, "B": int(B), "cfg": cfg}],
                           env=env, capture_output=True, text=True)
        line = [x for x in p.stdout.splitlines() if x.startswith("RESULT ")]
        r = json.loads(line[0][7:]) if line else {"error": p.stderr[-400:]}
        print(json.dumps({"lib": os.path.basename(lib), "block": int(B), "config": cfg, **r}), flush=True)
