"""Distributed protocol on one device: sgr_color_partitioned with the device-side exchange
(k_persistent_dist) vs the host-driven all-gather loop, against sgr_color, per config.

    python tools/dist_timing.py [--configs 4 3 2 1] [--parts 1 2 8] [--out X.jsonl]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_licqfsty16_b200 as sgr  # noqa: E402
from paper_conf_ipps_licqfsty16_b200 import gen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--configs", type=int, nargs="+", default=[4, 3, 2, 1])
ap.add_argument("--parts", type=int, nargs="+", default=[1, 2, 8])
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--out", default=None)
args = ap.parse_args()
out = open(args.out, "w") if args.out else None
flush = torch.empty(64 << 20, dtype=torch.int32, device="cuda")


def timed(fn):
    fn()
    ms = []
    for i in range(args.reps):
        flush.fill_(i)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        r = fn()
        e1.record()
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    return statistics.median(ms), r


for cfg in args.configs:
    g = gen.config(cfg)
    rp = torch.from_numpy(g.row_ptr).cuda()
    ci = torch.from_numpy(g.col_idx).cuda()
    base_ms, base = timed(lambda: sgr.color(rp, ci))
    rows = [{"config": gen.CONFIG_NAMES[cfg], "path": "sgr_color (single part)", "ms": base_ms,
             "rounds_ms": base.stats["elapsed_ms"]}]
    for P in args.parts:
        ranges = sgr.partition(g.row_ptr, P)
        for tr in ("device", "hostloop"):
            if tr == "hostloop":
                os.environ["SGR_DIST_HOSTLOOP"] = "1"
            else:
                os.environ.pop("SGR_DIST_HOSTLOOP", None)
            ms, r = timed(lambda: sgr.color_partitioned(rp, ci, P, ranges=ranges))
            # ms: the whole call (host-side split of the CSR into local rows, allocations,
            # F_1, rounds); rounds_ms: device time of the rounds (library CUDA events)
            rows.append({"config": gen.CONFIG_NAMES[cfg], "path": f"partitioned P={P} {tr}",
                         "ms": ms, "rounds_ms": r.stats["elapsed_ms"], "transport": r.stats["transport"],
                         "bit_exact_vs_sgr_color": bool(torch.equal(r.colors, base.colors)),
                         "rounds": r.stats["rounds"]})
    os.environ.pop("SGR_DIST_HOSTLOOP", None)
    for row in rows:
        print(json.dumps(row), flush=True)
        if out:
            out.write(json.dumps(row) + "\n")
    del rp, ci
    torch.cuda.empty_cache()
