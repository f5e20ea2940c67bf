"""The paper's Fig. 8 experiment on B200: coloring time vs threads per block.

    python tools/block_sweep.py [--configs 4 1 3 7] [--out profiles/r02_block_sweep.jsonl]

For each config: the data-driven fused path (sgr_color, persistent loop; hub build 64..512,
flat build 64..768 threads) and the topology-driven mapping (sgr_color_topo = T-base,
Algorithm 4, one thread per vertex; 32..1024 threads). Every coloring is checked bit-exact
against the default block size's (block size never changes the result). Device time from
the library's CUDA events (stats elapsed_ms), L2 flushed between repetitions.
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", type=int, nargs="+", default=[4, 1, 3, 7])
    ap.add_argument("--topo-configs", type=int, nargs="+", default=[1, 3, 7],
                    help="configs for the topology-driven sweep (T-base on cfg4 takes ~28 s "
                         "per coloring: a hub row is one thread's serial loop)")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    out = open(args.out, "w") if args.out else None
    flush = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
    for cfg in args.configs:
        g = gen.config(cfg)
        rp = torch.from_numpy(g.row_ptr).cuda()
        ci = torch.from_numpy(g.col_idx).cuda()
        for mapping in ("data-driven", "topology-driven"):
            if mapping == "topology-driven" and cfg not in args.topo_configs:
                continue
            fn = sgr.color if mapping == "data-driven" else sgr.color_topo
            ref = fn(rp, ci, "lowid").colors.clone()
            sizes = [64, 96, 128, 192, 256, 384, 512] if mapping == "data-driven" else \
                [32, 64, 128, 256, 512, 1024]
            for B in sizes:
                try:
                    fn(rp, ci, "lowid", block_size=B)
                except RuntimeError as e:  # e.g. a build that does not take this size
                    rec = {"config": gen.CONFIG_NAMES[cfg], "mapping": mapping, "block": B,
                           "error": str(e)[:120]}
                    print(json.dumps(rec), flush=True)
                    continue
                ms = []
                for i in range(args.reps):
                    flush.fill_(i)
                    res = fn(rp, ci, "lowid", block_size=B)
                    ms.append(res.stats["elapsed_ms"])
                same = bool(torch.equal(res.colors, ref))
                rec = {"config": gen.CONFIG_NAMES[cfg], "n": g.n, "nnz": g.nnz,
                       "mapping": mapping, "block": B, "ms": statistics.median(ms),
                       "ms_min": min(ms), "gteps": g.nnz / statistics.median(ms) / 1e6,
                       "grid": res.stats["grid_blocks"], "rounds": res.stats["rounds"],
                       "bit_exact_vs_default": same}
                print(json.dumps(rec), flush=True)
                if out:
                    out.write(json.dumps(rec) + "\n")
                    out.flush()
        del rp, ci
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
