#!/usr/bin/env python3
"""Write the committed profile summaries (profiles/): the per-launch device
times of one bench step (ncu launch list) aggregated per kernel, and the
key counters of the `ncu --set full` capture.

  python tools/profile_summary.py <launches.csv> <full.ncu-rep> <out-prefix>
"""
import csv
import subprocess
import sys
from collections import OrderedDict


def launches(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 5]
    h = rows[0]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    agg = OrderedDict()
    for r in rows[1:]:
        name = r[ki].split("(")[0].replace("void ", "").replace("(anonymous namespace)::", "")
        name = name.split("::")[-1]
        try:
            t = float(r[vi]) / 1e6
        except ValueError:
            continue
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += t
    return agg


def full(path):
    metrics = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
               "dram__throughput.avg.pct_of_peak_sustained_elapsed",
               "sm__throughput.avg.pct_of_peak_sustained_elapsed",
               "smsp__inst_executed.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
               "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
               "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
               "smsp__issue_active.avg.pct_of_peak_sustained_active",
               "launch__registers_per_thread", "launch__occupancy_limit_shared_mem"]
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv", "--metrics", ",".join(metrics)],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h = rows[0]
    res = []
    for r in rows[2:]:
        d = dict(zip(h, r))
        res.append((d.get("Kernel Name", "").split("(")[0].split("::")[-1], {m: d.get(m) for m in metrics}))
    return res


def main(lcsv, rep, prefix):
    agg = launches(lcsv)
    tot = sum(v[1] for k, v in agg.items() if "kernel" in k)
    with open(prefix + "_launches.md", "w") as f:
        f.write(f"# Per-kernel device time of one bench step (ncu launch list, cold-cache, serialised)\n\n")
        f.write(f"source: `{lcsv}` (`ncu --metrics gpu__time_duration.sum --clock-control none`)\n\n")
        f.write("| kernel | launches | ms | share |\n|---|---|---|---|\n")
        for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
            f.write(f"| {k} | {n} | {t:.3f} | {100 * t / max(tot, 1e-9):.1f}% |\n")
        f.write(f"| **total (our kernels)** | | {tot:.3f} | |\n")
    with open(prefix + "_ncu_full.md", "w") as f:
        f.write(f"# `ncu --set full` capture: key counters per launch\n\nsource: `{rep}`\n\n")
        for name, d in full(rep):
            f.write(f"## {name}\n\n")
            for m, v in d.items():
                f.write(f"- {m}: {v}\n")
            f.write("\n")


if __name__ == "__main__":
    main(*sys.argv[1:4])
