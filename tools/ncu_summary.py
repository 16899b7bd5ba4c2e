#!/usr/bin/env python3
"""Summarise an ncu report: per kernel launch, the key throughput metrics."""
import csv
import subprocess
import sys

WANT = ["Duration", "DRAM Throughput", "Memory Throughput", "L2 Cache Throughput",
        "Compute (SM) Throughput", "Executed Ipc Active", "Issue Slots Busy", "Achieved Occupancy",
        "Theoretical Occupancy", "Registers Per Thread", "L1/TEX Hit Rate", "L2 Hit Rate",
        "Warp Cycles Per Issued Instruction", "Dynamic Shared Memory Per Block", "Grid Size",
        "Block Size"]


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "details", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h = rows[0]
    ki, ii, mi, vi, ui = (h.index(x) for x in ("Kernel Name", "ID", "Metric Name", "Metric Value",
                                                 "Metric Unit"))
    seen = {}
    for r in rows[1:]:
        if r[mi] in WANT:
            key = (r[ii], r[ki].split("(")[0][-40:])
            seen.setdefault(key, {})[r[mi]] = f"{r[vi]} {r[ui]}"
    for (i, k), d in seen.items():
        print(f"[{i}] {k}")
        print("    " + "; ".join(f"{m}={d[m]}" for m in WANT if m in d))
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv", "--metrics",
                          "dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,"
                          "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,"
                          "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active,"
                          "lts__t_sectors_op_write.sum,lts__t_sectors_op_read.sum"],
                         capture_output=True, text=True).stdout
    rr = list(csv.reader(raw.splitlines()))
    if len(rr) > 2:
        hh = rr[0]
        cols = [c for c in hh if c.startswith(("dram__", "smsp__inst", "sm__inst", "lts__"))]
        for r in rr[2:]:
            d = dict(zip(hh, r))
            print(d.get("ID"), d.get("Kernel Name", "")[:40], {c: d[c] for c in cols})


if __name__ == "__main__":
    main(sys.argv[1])
