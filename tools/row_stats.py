#!/usr/bin/env python3
"""Pass-II row-length distribution (= |L| of the first-level groups with
|L| >= s2) of a synthetic config: rows and entries per length class, and the
per-tile (8 consecutive rows) staged totals.  Diagnostics, not product."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main(config="gos2m"):
    import torch
    from paper_conf_ipps_wuk13_b200 import binding as B
    from synth import graphs as SG
    torch.cuda.set_device(0)
    cfg = SG.CONFIGS[config]
    g = SG.make(config, cache=False)
    h = B.shingle_graph_create(g.row_ptr, g.col)
    B.shingle_pass(h, cfg["s1"], cfg["c1"], cfg["seed1"])
    B.group_by_shingle(h)
    tg, _, offs, _ = B.sg_get_groups(h, 1, with_ids=False)
    L = np.diff(offs)
    L = L[L >= cfg["s2"]]
    E = L.sum()
    print(f"rows {L.size}  entries {E}  mean {L.mean():.2f}  max {L.max()}")
    edges = [2, 3, 4, 5, 9, 17, 25, 65, 257, 1025, 4097, 1 << 40]
    for lo, hi in zip(edges[:-1], edges[1:]):
        m = (L >= lo) & (L < hi)
        print(f"  len [{lo},{hi}): rows {m.sum():>10} ({100*m.mean():5.1f}%)  entries {L[m].sum():>11} ({100*L[m].sum()/E:5.1f}%)")
    pl = (L + 3) // 4 * 4
    nt = (pl.size + 7) // 8
    tot = np.add.reduceat(pl, np.arange(0, pl.size, 8))
    print(f"tiles {nt}: staged total > 1024: {(tot > 1024).sum()}  entries in them {tot[tot > 1024].sum()}")
    B.shingle_graph_destroy(h)


if __name__ == "__main__":
    main(*sys.argv[1:])
