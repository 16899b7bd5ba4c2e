#!/usr/bin/env python3
"""Profiling driver: runs the two-pass path on a named synthetic config a few
times (for ncu / quick stage timing).  Not part of the product path.

  python tools/profile_run.py --config gos2m --c1 200 --c2 200 --reps 2
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
    ap.add_argument("--s1", type=int, default=None)
    ap.add_argument("--c1", type=int, default=None)
    ap.add_argument("--s2", type=int, default=None)
    ap.add_argument("--c2", type=int, default=None)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--pass1-only", action="store_true")
    args = ap.parse_args()
    import torch
    from paper_conf_ipps_wuk13_b200 import binding as B
    from synth import graphs as SG
    torch.cuda.set_device(0)
    cfg = dict(SG.CONFIGS[args.config])
    for k in ("s1", "c1", "s2", "c2"):
        if getattr(args, k) is not None:
            cfg[k] = getattr(args, k)
    t = time.time()
    g = SG.make(args.config, cache=False)
    print(f"graph {args.config}: n={g.n} m={g.m} gen {time.time() - t:.1f}s", file=sys.stderr)
    h = B.shingle_graph_create(g.row_ptr, g.col)
    for r in range(args.reps):
        B.shingle_graph_reset(h)
        B.shingle_pass(h, cfg["s1"], cfg["c1"], cfg["seed1"])
        B.group_by_shingle(h)
        if not args.pass1_only:
            B.shingle_pass(h, cfg["s2"], cfg["c2"], cfg["seed2"])
            B.group_by_shingle(h)
        torch.cuda.synchronize()
        st = {k: round(v, 3) for k, v in B.sg_get_stage_ms(h).items() if v > 0}
        print(json.dumps({"rep": r, "stage_ms": st, "counts": B.sg_get_counts(h)}))
        free, tot = torch.cuda.mem_get_info()
        print(f"mem free {free / 1e9:.1f} / {tot / 1e9:.1f} GB", file=sys.stderr)
    B.shingle_graph_destroy(h)


if __name__ == "__main__":
    main()
