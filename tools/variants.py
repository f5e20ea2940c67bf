"""A/B timing of alternative builds of libsgr.so (tools/build_variant.sh) on the BASELINE configs.

    python tools/variants.py --configs 2 3 4 --variants default tools/alt/x.so ...

Each variant runs in its own process (SGR_LIBPATH selects the build); every coloring is
compared bit-exactly with the default build's colors of the same config (the default build
itself is checked against the oracle by tests/test_gpu_parity.py).
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import json, os, sys, statistics
sys.path.insert(0, %(root)r)
import numpy as np, torch
import paper_conf_ipps_licqfsty16_b200 as sgr
from paper_conf_ipps_licqfsty16_b200 import gen
out = {}
for cfg in %(configs)r:
    # -1: path of 4000 vertices (4000 rounds of <= 4000 vertices: per-round loop overhead)
    g = gen.stencil2d(4000, 1, 5) if cfg == -1 else gen.config(cfg)
    rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
    colors = torch.empty(g.n, dtype=torch.int32, device="cuda")
    ws = torch.empty(sgr.workspace_bytes(g.n, g.nnz), dtype=torch.uint8, device="cuda")
    flush = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
    for _ in range(2):
        res = sgr.color(rp, ci, %(tb)r, out=colors, workspace=ws, loop_mode=%(lm)r)
    ms = []
    for i in range(%(reps)d):
        flush.fill_(i)
        res = sgr.color(rp, ci, %(tb)r, out=colors, workspace=ws, loop_mode=%(lm)r)
        ms.append(res.stats["elapsed_ms"])
    ref = "/tmp/sgr_ref_colors_c%%d_%%s.npy" %% (cfg, %(tb)r)
    c = colors.cpu().numpy()
    if %(save)r:
        np.save(ref, c); same = True
    else:
        same = bool(np.array_equal(np.load(ref), c)) if os.path.exists(ref) else None
    out[cfg] = {"ms": statistics.median(ms), "min": min(ms), "rounds": res.stats["rounds"],
                "entries_read_per_nnz": res.stats["entries_read"] / max(g.nnz, 1),
                "grid": res.stats["grid_blocks"], "same": same}
    del rp, ci, colors, ws
    torch.cuda.empty_cache()
print("RESULT " + json.dumps(out))
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", type=int, nargs="+", default=[2, 3, 4])
    ap.add_argument("--variants", nargs="+", default=["default"])
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--tiebreak", default="lowid")
    ap.add_argument("--loop-mode", default="persistent")
    args = ap.parse_args()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    for vi, v in enumerate(args.variants):
        env = dict(os.environ)
        if v != "default":
            env["SGR_LIBPATH"] = os.path.abspath(v)
        code = CHILD % {"root": ROOT, "configs": args.configs, "tb": args.tiebreak,
                        "lm": args.loop_mode, "reps": args.reps, "save": vi == 0 and v == "default"}
        p = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True)
        line = [x for x in p.stdout.splitlines() if x.startswith("RESULT ")]
        if not line:
            print(f"{v}: FAILED rc={p.returncode}\n{p.stderr[-2000:]}", flush=True)
            continue
        res = json.loads(line[0][7:])
        txt = "  ".join(f"c{c}: {r['ms']:.2f} ms (min {r['min']:.2f}, grid {r['grid']}, "
                        f"R {r['rounds']}, same={r['same']})" for c, r in res.items())
        print(f"{os.path.basename(v):28s} {txt}", flush=True)


if __name__ == "__main__":
    main()
