#!/usr/bin/env python3
"""Per-CUDA-source-line executed instructions and stall samples of one
kernel launch in an ncu report (needs -lineinfo).
  python tools/ncu_lines.py rep.ncu-rep [launch-skip] [n]"""
import collections
import csv
import subprocess
import sys


def main(path, skip=0, n=35):
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "--launch-skip", str(skip), "--launch-count", "1"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    agg = collections.defaultdict(lambda: [0, 0, ""])
    fname, cur = "", None
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] in ("Function Name", "Line No"):
            continue
        try:
            ex, st = int(r[7] or 0), int(r[4] or 0)
        except (ValueError, IndexError):
            continue
        if r[0]:
            cur = (fname, r[0])
            agg[cur][2] = r[1][:100]
        if cur:
            agg[cur][0] += ex
            agg[cur][1] += st
    tot = sum(v[0] for v in agg.values()) or 1
    tst = sum(v[1] for v in agg.values()) or 1
    print(f"warp-instructions {tot:.3e}, stall samples {tst}")
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:n]:
        print(f"{100 * v[0] / tot:5.1f}% ex {100 * v[1] / tst:5.1f}% st {k[0]}:{k[1]:>4} {v[2]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 0,
         int(sys.argv[3]) if len(sys.argv) > 3 else 35)
