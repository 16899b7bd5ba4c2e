#!/usr/bin/env python3
"""Write tests/golden/digests_<config>.json from the CPU oracle's trial-outer
run (oracle.shingling_stream) on a seeded synthetic config: counts, per-trial
digests of every pass-I column and G_I trial, the S1' map digest, and the
G_II digests of the listed pass-II trials.  Calls only oracle/ (and synth/ for
the input graph); the GPU tests compare the library's outputs against it.

  python tools/oracle_digests.py gos2m [--keep2 0,63,64,199]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402

import digests as D  # noqa: E402
import oracle  # noqa: E402
from synth import graphs as SG  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--keep2", default="0,63,64,199")
    ap.add_argument("--keep1", default="")
    args = ap.parse_args()
    cfg = SG.CONFIGS[args.config]
    t0 = time.time()
    g = SG.make(args.config)
    tg = time.time() - t0
    keep1 = [int(x) for x in args.keep1.split(",") if x]
    keep2 = [int(x) for x in args.keep2.split(",") if x and int(x) < cfg["c2"]]
    t0 = time.time()
    st = oracle.shingling_stream(g.row_ptr, g.col, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"],
                                 cfg["seed2"], keep1=keep1, keep2=keep2)
    to = time.time() - t0
    out = dict(
        config=args.config, n=g.n, nnz=g.nnz, m=g.m,
        graph_digest=D.column(np.concatenate([g.row_ptr.astype(np.uint64), g.col.astype(np.uint64)])),
        params=dict(s1=cfg["s1"], c1=cfg["c1"], seed1=cfg["seed1"], s2=cfg["s2"], c2=cfg["c2"],
                    seed2=cfg["seed2"]),
        counts=st.counts,
        rows1_digest=D.column(st.rows1.astype(np.uint64)),
        s1p_digest=D.column(st.s1p_group.astype(np.uint64)),
        dig_M1=[int(x) for x in st.dig_M1], dig_G1=[int(x) for x in st.dig_G1],
        keep2=[int(x) for x in st.keep2], dig_G2k=[int(x) for x in st.dig_G2k],
        dig_M2k=[D.column(st.M2k[:, i]) for i in range(len(st.keep2))],
        G2k_groups=[int(st.G2k.trial_goffs[i + 1] - st.G2k.trial_goffs[i]) for i in range(len(st.keep2))],
        oracle_seconds=round(to, 1), generator_seconds=round(tg, 1),
        written_by="tools/oracle_digests.py (oracle.shingling_stream, single-threaded C)")
    path = os.path.join(ROOT, "tests", "golden", f"digests_{args.config}.json")
    with open(path, "w") as f:
        json.dump(out, f)
    print(json.dumps({k: out[k] for k in ("config", "counts", "oracle_seconds", "generator_seconds")}))


if __name__ == "__main__":
    main()
