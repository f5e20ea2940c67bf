"""Condense an `ncu --metrics gpu__time_duration.sum --csv` log into the launch-list format
kept under profiles/ (id, kernel, grid, block, ns) plus per-kernel share of the total."""
import csv
import sys
from collections import defaultdict


def main(src, dst, header):
    rows = []
    with open(src) as f:
        lines = [l for l in f if l.startswith('"')]
    for r in csv.DictReader(lines):
        if r["Metric Name"] != "gpu__time_duration.sum":
            continue
        name = r["Kernel Name"].split("(sgr::")[0].split("(RoundArgs")[0].split("(")[0]
        name = r["Kernel Name"][:r["Kernel Name"].find("(")] if "(" in r["Kernel Name"] else name
        rows.append((r["ID"], name, r["Grid Size"], r["Block Size"], int(float(r["Metric Value"]))))
    tot = defaultdict(int)
    for r in rows:
        tot[r[1]] += r[4]
    all_ns = sum(tot.values())
    with open(dst, "w") as f:
        for h in header:
            f.write(f"# {h}\n")
        for k, v in sorted(tot.items(), key=lambda x: -x[1]):
            f.write(f"# share {v / all_ns:.4f}  {k}  ({v} ns total)\n")
        f.write("id,kernel,grid,block,gpu__time_duration_ns\n")
        for r in rows:
            f.write(",".join(['"%s"' % x if "," in str(x) else str(x) for x in r]) + "\n")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3:])
