#!/usr/bin/env python3
"""DRAM bytes per pair of the level-II grouping stage from an ncu --set full
capture of tools/profile_run.py --c2 64 (one trial chunk: hist, scatter, fine
split and local-sort launches of level II), written to
profiles/ncu_traffic.json for bench.py's roofline.traffic.

  python tools/ncu_traffic.py gpurun_out/r2b_full_gos2m.ncu-rep gos2m <pairs of the chunk> <source tag>
"""
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GROUP_KERNELS = ("hist_kernel", "hist_bytes_kernel", "colscan_kernel", "binscan_kernel", "scatter_kernel", "scatter2_kernel",
                 "warp_local_kernel", "local_kernel", "big_kernel")


def main(rep, config, pairs, tag):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics",
                          "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr = rows[0]
    units = rows[1]
    per = {}
    tot = 0.0
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        name = d.get("Kernel Name", "")
        short = name.split("(")[0].split("::")[-1].split("<")[0].strip()
        if short not in GROUP_KERNELS:
            continue
        b = 0.0
        for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            u = units[hdr.index(m)]
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)
            b += float(d[m]) * scale
        per[short] = per.get(short, 0.0) + b
        tot += b
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    data = json.load(open(path)) if os.path.exists(path) else {}
    data.setdefault(config, {})["group2"] = {
        "bytes_per_pair": round(tot / pairs, 3),
        "per_kernel_bytes_per_pair": {k: round(v / pairs, 3) for k, v in per.items()},
        "source": f"ncu --set full, dram__bytes_read.sum + dram__bytes_write.sum of the level-II grouping "
                  f"kernels of one 64-trial chunk ({pairs} pairs), {tag}"}
    json.dump(data, open(path, "w"), indent=1)
    print(json.dumps(data[config]["group2"]))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]), sys.argv[4])
