#!/usr/bin/env python3
"""Per-CUDA-source-line instructions executed and stall samples of one kernel
launch in an ncu report (ncu --page source --print-source sass,cuda).
  python tools/src_lines.py rep.ncu-rep <launch-skip> [n]"""
import csv
import collections
import subprocess
import sys


def main(path, skip, n=30):
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass,cuda",
                          "--launch-skip", str(skip), "--launch-count", "1"],
                         capture_output=True, text=True).stdout.splitlines()
    ex = collections.Counter()
    st = collections.Counter()
    text = {}
    fname = "?"
    hdr = None
    for r in csv.reader(out):
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < len(hdr):
            continue
        try:
            line = int(r[0])
        except ValueError:
            continue
        key = (fname, line)
        text[key] = r[1][:90]
        try:
            ex[key] += int(r[hdr.index("Instructions Executed")] or 0)
            st[key] += int(r[hdr.index("Warp Stall Sampling (All Samples)")] or 0)
        except ValueError:
            pass
    te, ts = sum(ex.values()), sum(st.values())
    print(f"total warp-instr {te:.3e}, stall samples {ts}")
    for key in sorted(ex, key=lambda k: -(ex[k] / max(te, 1) + st[k] / max(ts, 1)))[:n]:
        print(f"{key[0]}:{key[1]:<5} ex {100*ex[key]/max(te,1):5.1f}%  st {100*st[key]/max(ts,1):5.1f}%  {text[key]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]), int(sys.argv[3]) if len(sys.argv) > 3 else 30)
