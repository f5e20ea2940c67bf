"""The paper's ldg ablation (D-base vs D-ldg, T-base vs T-ldg) on B200.

    python tools/build_variants.py noldg=SGR_LDG=0      # D-base / T-base build (tools/alt/)
    python tools/ldg_ablation.py [--configs 4 1 3 2 7] [--out profiles/r02_ldg_ablation.jsonl]

The default libsgr.so reads the CSR arrays R and C through the read-only data path
(__ldg, ld.global.nc: "-ldg"); the SGR_LDG=0 build uses normal loads (ld.global.ca:
"-base"). Both mappings (data-driven sgr_color, topology-driven sgr_color_topo) are timed
with each build in its own process; colors are compared bit-exactly across builds.
"""
import argparse
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
flush = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
for cfg in %(configs)r:
    g = gen.config(cfg)
    rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
    for mapping, fn in (("data-driven", sgr.color), ("topology-driven", sgr.color_topo)):
        fn(rp, ci, "lowid")
        ms = []
        for i in range(%(reps)d):
            flush.fill_(i)
            res = fn(rp, ci, "lowid")
            ms.append(res.stats["elapsed_ms"])
        h = int(np.bitwise_xor.reduce(res.colors.cpu().numpy().astype(np.uint64) *
                                      np.arange(1, g.n + 1, dtype=np.uint64)))
        print("RESULT " + json.dumps({"config": gen.CONFIG_NAMES[cfg], "mapping": mapping,
              "ms": statistics.median(ms), "ms_min": min(ms),
              "gteps": g.nnz / statistics.median(ms) / 1e6, "rounds": res.stats["rounds"],
              "colors_hash": h}), flush=True)
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", type=int, nargs="+", default=[4, 1, 3, 2, 7])
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--base-lib", default=os.path.join(ROOT, "tools", "alt", "noldg.so"))
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    rows = {}
    for name, lib in (("ldg", None), ("base", args.base_lib)):
        env = dict(os.environ)
        if lib:
            env["SGR_LIBPATH"] = os.path.abspath(lib)
        code = CHILD % {"root": ROOT, "configs": args.configs, "reps": args.reps}
        p = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True)
        for line in p.stdout.splitlines():
            if line.startswith("RESULT "):
                r = json.loads(line[7:])
                rows.setdefault((r["config"], r["mapping"]), {})[name] = r
        if p.returncode:
            print(p.stderr[-2000:], file=sys.stderr)
    out = open(args.out, "w") if args.out else None
    for (cfg, mapping), d in rows.items():
        if "ldg" not in d or "base" not in d:
            continue
        rec = {"config": cfg, "mapping": mapping,
               "scheme_ldg": ("D-ldg" if mapping == "data-driven" else "T-ldg"),
               "scheme_base": ("D-base" if mapping == "data-driven" else "T-base"),
               "ms_ldg": d["ldg"]["ms"], "ms_base": d["base"]["ms"],
               "speedup_ldg_over_base": d["base"]["ms"] / d["ldg"]["ms"],
               "bit_exact": d["ldg"]["colors_hash"] == d["base"]["colors_hash"]
               and d["ldg"]["rounds"] == d["base"]["rounds"]}
        print(json.dumps(rec), flush=True)
        if out:
            out.write(json.dumps(rec) + "\n")


if __name__ == "__main__":
    main()
