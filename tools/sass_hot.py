#!/usr/bin/env python3
"""Top SASS instructions of one kernel launch in an ncu report, by executed
instructions and stall samples (needs -lineinfo builds).
  python tools/sass_hot.py rep.ncu-rep <launch-skip> [n]"""
import csv
import subprocess
import sys


def main(path, skip, n=40):
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass",
                          "--launch-skip", str(skip), "--launch-count", "1"],
                         capture_output=True, text=True).stdout.splitlines()
    print(out[0][:120])
    rows = list(csv.reader(out[1:]))
    h = rows[0]
    ia, isrc, ist, iex = (h.index(x) for x in ("Address", "Source", "Warp Stall Sampling (All Samples)",
                                                "Instructions Executed"))
    data = []
    for r in rows[1:]:
        try:
            data.append((int(r[iex] or 0), int(r[ist] or 0), r[ia], r[isrc]))
        except (ValueError, IndexError):
            pass
    tot_ex = sum(d[0] for d in data)
    tot_st = sum(d[1] for d in data)
    print(f"total warp-instructions {tot_ex:.3e}, stall samples {tot_st}")
    # region summary: consecutive instructions
    for ex, st, a, s in sorted(data, key=lambda d: -d[1])[:n]:
        print(f"{a:>6} ex={ex:>11} ({100*ex/max(tot_ex,1):5.1f}%) stall={st:>7} ({100*st/max(tot_st,1):5.1f}%)  {s}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]), int(sys.argv[3]) if len(sys.argv) > 3 else 40)


def regions(path, skip, width=16):
    """Executed warp-instructions per address window (to find heavy loops)."""
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass",
                          "--launch-skip", str(skip), "--launch-count", "1"],
                         capture_output=True, text=True).stdout.splitlines()
    rows = list(csv.reader(out[1:]))
    h = rows[0]
    ia, isrc, ist, iex = (h.index(x) for x in ("Address", "Source", "Warp Stall Sampling (All Samples)",
                                                "Instructions Executed"))
    seen = set()
    data = []
    for r in rows[1:]:
        try:
            if r[ia] in seen:
                continue
            seen.add(r[ia])
            data.append((int(r[ia], 16), int(r[iex] or 0), int(r[ist] or 0), r[isrc]))
        except (ValueError, IndexError):
            pass
    data.sort()
    tot = sum(d[1] for d in data)
    for i in range(0, len(data), width):
        blk = data[i:i + width]
        ex = sum(d[1] for d in blk)
        st = sum(d[2] for d in blk)
        if ex > 0.01 * tot:
            print(f"{hex(blk[0][0])} ex={ex:.3e} ({100*ex/tot:4.1f}%) stall={st}  | " +
                  " ; ".join(d[3].strip()[:28] for d in blk[:6]))
