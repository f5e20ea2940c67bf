"""Per-source-line stall samples and executed warp instructions from an ncu report
(`ncu -i X --page source --csv --print-source cuda,sass`)."""
import csv
import subprocess
import sys


def main(rep, top=40, kernel_filter=None):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    f = None
    fn = None
    agg = {}
    for r in rows:
        if r and r[0] == "File Path":
            f = r[1].split("/")[-1]
            continue
        if r and r[0] == "Function Name":
            fn = r[1]
            continue
        if kernel_filter and fn and kernel_filter not in fn:
            continue
        if len(r) > 8 and r[0].isdigit():
            try:
                key = (f, int(r[0]))
                s, ins = int(r[4]), int(r[7])
            except ValueError:
                continue
            a = agg.setdefault(key, [0, 0, r[1][:100]])
            a[0] += s
            a[1] += ins
    ts = sum(a[0] for a in agg.values()) or 1
    ti = sum(a[1] for a in agg.values()) or 1
    print(f"samples {ts}  warp-instructions {ti / 1e9:.2f} G")
    for k, a in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
        print(f"{100 * a[0] / ts:5.1f}% smp {100 * a[1] / ti:5.1f}% ins  {k[0]}:{k[1]}  {a[2]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40,
         sys.argv[3] if len(sys.argv) > 3 else None)
