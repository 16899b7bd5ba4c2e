#!/usr/bin/env python3
"""One small two-pass run + reports on the tiny config for compute-sanitizer
(memcheck / racecheck / synccheck): python tools/sanitize_run.py [v3]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    if len(sys.argv) > 1 and sys.argv[1] == "v3":
        os.environ["SG_GROUP"] = "v3"
    import numpy as np
    from paper_conf_ipps_wuk13_b200 import binding as B
    from synth import graphs as SG
    g = SG.make("tiny", cache=False)
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        G.run(2, 40, 101, 2, 33, 102)
        c = B.sg_get_counts(G.h)
        labels, nc = G.report(0)
        offs, verts = G.report_overlapping(0, 1)
        d = G.density(labels, 2)
        cc, ncc = G.components()
        agr = G.agreement(labels, cc)
        B.sg_get_groups(G.h, 2)
        print("ok", c["pairs1"], c["pairs2"], nc, len(offs) - 1, round(d[0], 4), ncc, agr["TP"])


if __name__ == "__main__":
    main()
