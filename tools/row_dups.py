#!/usr/bin/env python3
"""Measurement helper (not on the product path): how many pass-II rows (S1'
nodes, i.e. G_I groups with |L| >= s2) have identical member lists, and the
group-size mix of G_II for a few trials.  Identical rows give identical
pass-II shingle vectors (the twins invariant of the north_star self-checks).

  python tools/row_dups.py --config gos2m
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def mix(z):
    z = z + np.uint64(0x9E3779B97F4A7C15)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="gos2m")
    args = ap.parse_args()
    import torch
    from paper_conf_ipps_wuk13_b200 import binding as B
    from synth import graphs as SG
    torch.cuda.set_device(0)
    cfg = SG.CONFIGS[args.config]
    g = SG.make(args.config, cache=False)
    h = B.shingle_graph_create(g.row_ptr, g.col)
    B.shingle_pass(h, cfg["s1"], cfg["c1"], cfg["seed1"])
    B.group_by_shingle(h)
    out = {"config": args.config}
    with np.errstate(over="ignore"):
        hs = []
        lens = []
        for t0 in range(0, cfg["c1"], 8):
            tg, gid, offs, mem = B.sg_get_groups_range(h, 1, t0, min(cfg["c1"], t0 + 8), with_ids=False)
            sz = np.diff(offs)
            cs = np.concatenate([[np.uint64(0)], np.cumsum(mix(mem.astype(np.uint64)), dtype=np.uint64)])
            gh = mix((cs[offs[1:]] - cs[offs[:-1]]) ^ sz.astype(np.uint64))
            sel = sz >= cfg["s2"]
            hs.append(gh[sel])
            lens.append(sz[sel])
        hs = np.concatenate(hs)
        lens = np.concatenate(lens)
    u, inv, cnt = np.unique(hs, return_inverse=True, return_counts=True)
    out.update(s1p=int(len(hs)), unique_rows=int(len(u)), unique_frac=len(u) / max(1, len(hs)),
               entries2=int(lens.sum()), unique_entries2=int(np.bincount(inv, weights=lens, minlength=len(u)).dot(1.0 / cnt)) if len(u) else 0,
               mean_len=float(lens.mean()), len_hist={int(k): int(v) for k, v in zip(*np.unique(np.minimum(lens, 64), return_counts=True))},
               class_size_hist={int(k): int(v) for k, v in zip(*np.unique(np.minimum(cnt, 256), return_counts=True))})
    print(json.dumps(out), flush=True)
    B.shingle_pass(h, cfg["s2"], cfg["c2"], cfg["seed2"])
    B.group_by_shingle(h)
    tg, gid, offs, mem = B.sg_get_groups_range(h, 2, 0, 2, with_ids=False)
    sz = np.diff(offs)
    out2 = {"g2_trials": 2, "g2_groups": int(len(sz)), "g2_pairs": int(sz.sum()),
            "g2_size_hist": {int(k): int(v) for k, v in zip(*np.unique(np.minimum(sz, 64), return_counts=True))}}
    print(json.dumps(out2), flush=True)
    B.shingle_graph_destroy(h)


if __name__ == "__main__":
    main()
