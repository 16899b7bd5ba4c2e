#!/usr/bin/env python3
"""Subprocess helper of tests/test_ab_options_gpu.py: runs the two-pass path
through the library on a named synthetic config with the A/B environment the
parent set (the options are read once per process) and prints one JSON line of
SHA-256 digests of every output array (pass-I / pass-II matrices, G_I, G_II,
the S1' map)."""
import hashlib
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)


def digest(*arrays):
    h = hashlib.sha256()
    for a in arrays:
        h.update(a.tobytes(order="C"))
    return h.hexdigest()


def main():
    name, s1, c1, seed1, s2, c2, seed2 = sys.argv[1], *map(int, sys.argv[2:8])
    import torch
    from paper_conf_ipps_wuk13_b200 import binding as B
    from synth import graphs as SG
    torch.cuda.set_device(0)
    g = SG.make(name)
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        G.run(s1, c1, seed1, s2, c2, seed2)
        ids1, rows1 = B.sg_get_shingles(G.h, 1)
        ids2, rows2 = B.sg_get_shingles(G.h, 2)
        g1 = B.sg_get_groups(G.h, 1)
        g2 = B.sg_get_groups(G.h, 2)
        s1p, _ = B.sg_get_s1p(G.h)
    import numpy as np

    def grp(g):
        tg, ids, offs, mem = g
        return (np.asarray(tg, np.int64), np.asarray(ids, np.uint64), np.asarray(offs, np.int64),
                np.asarray(mem, np.uint32))
    print(json.dumps({"M1": digest(np.asarray(ids1, np.uint64), np.asarray(rows1, np.uint32)),
                      "M2": digest(np.asarray(ids2, np.uint64)), "G1": digest(*grp(g1)),
                      "G2": digest(*grp(g2)), "s1p": digest(np.asarray(s1p, np.int64))}))


if __name__ == "__main__":
    main()
