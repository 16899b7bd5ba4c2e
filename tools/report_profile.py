#!/usr/bin/env python3
"""Runs the untimed Phase III and quality calls once on a synthetic config
(for an ncu launch list of their kernels): both passes, the approach-2 report
(device union-find), approach 1 (overlapping clusters), density (Eq. 6),
pair agreement of mode 0 vs mode 1 (Eq. 2-5) and the connected components of
G.  Prints host-timed milliseconds per call.  Not part of the product path.

  python tools/report_profile.py [--config gos2m]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="gos2m")
    args = ap.parse_args()
    import torch
    from paper_conf_ipps_wuk13_b200 import binding as B
    from synth import graphs as SG
    torch.cuda.set_device(0)
    cfg = SG.CONFIGS[args.config]
    g = SG.make(args.config)
    out = {}
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        G.run(cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])

        def timed(name, f):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            r = f()
            torch.cuda.synchronize()
            out[name + "_ms"] = round((time.perf_counter() - t0) * 1e3, 3)
            return r

        l0, nc0 = timed("report_mode0", lambda: G.report(0))
        l1, _ = timed("report_mode1", lambda: G.report(1))
        offs, _ = timed("overlapping", lambda: G.report_overlapping(0))
        dens = timed("density", lambda: G.density(l0, 20))
        agr = timed("agreement", lambda: G.agreement(l0, l1))
        _, ncc = timed("components", lambda: G.components())
        out.update(clusters=nc0, overlapping=len(offs) - 1, density_ge20=dens[:2],
                   agreement_mode0_vs_mode1={k: agr[k] for k in ("PPV", "NPV", "SP", "SE")},
                   components=ncc)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
