#!/usr/bin/env python3
"""Trial sweep (BASELINE configs[4]): the gos2m graph
shingled with (s, c) in {2, 3, 5} x {50, 100, 200, 400} applied to both
passes (seeds 201 / 202), one GPU.  One JSON line per (s, c): device ms per
two-pass step (CUDA events on the library's stream, W warm-up + K timed
steps), edges/s, per-stage ms and the pass sizes.  Parity of every (s, c)
shape is covered at small size by tests/test_parity_gpu.py; this measures.

  python tools/sweep.py [--steps 3] [--warmup 1] [--s 2,3,5] [--c 50,100,200,400]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _peaks():
    hb = 6452.8
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        hb = json.load(open(p)).get("hbm_gbs", hb)
    hp = 3.2158e12
    q = os.path.join(ROOT, "profiles", "int_peak.json")
    if os.path.exists(q):
        hp = json.load(open(q))["hash_evals_per_s"]
    return hb, hp


HBM_PEAK, HASH_PEAK = _peaks()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="gos2m")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=1)
    ap.add_argument("--s", default="2,3,5")
    ap.add_argument("--c", default="50,100,200,400")
    args = ap.parse_args()
    import torch
    from paper_conf_ipps_wuk13_b200 import binding as B
    from synth import graphs as SG
    torch.cuda.set_device(0)
    cfg = SG.CONFIGS[args.config]
    g = SG.make(args.config)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    for s in (int(x) for x in args.s.split(",")):
        for c in (int(x) for x in args.c.split(",")):
            # a fresh handle (and memory pool) per point: the cached blocks of
            # another (s, c) plan would otherwise turn the next point's first
            # steps into pool releases and re-maps
            h = B.shingle_graph_create(g.row_ptr, g.col, dist={"rank": 0, "world": 1, "device": 0,
                                                               "stream": stream.cuda_stream})

            def step():
                B.shingle_graph_reset(h)
                B.shingle_pass(h, s, c, cfg["seed1"])
                B.group_by_shingle(h)
                B.shingle_pass(h, s, c, cfg["seed2"])
                B.group_by_shingle(h)
            line = {"config": args.config, "s": s, "c": c}
            try:
                for _ in range(args.warmup):
                    step()
                torch.cuda.synchronize()
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                stage = {}
                e0.record(stream)
                for _ in range(args.steps):
                    step()
                    for k, v in B.sg_get_stage_ms(h).items():
                        stage[k] = stage.get(k, 0.0) + v / args.steps
                e1.record(stream)
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1) / args.steps
                cnt = B.sg_get_counts(h)
                # rooflines as bench.py: hash stages against the measured hash
                # rate, grouping stages by SURVEY 8(d) bytes against copy bandwidth
                deg = g.degrees()
                et = {1: float(deg[deg >= s].sum()) * c, 2: float(cnt["entries2"]) * c}
                roof = {}
                for lv in (1, 2):
                    th = stage.get(f"hash{lv}", 0.0) / 1e3
                    tg = stage.get(f"group{lv}", 0.0) / 1e3
                    if th > 0:
                        roof[f"hash{lv}"] = round(et[lv] / th / HASH_PEAK, 4)
                    if tg > 0:
                        roof[f"group{lv}"] = round((32 * cnt[f"pairs{lv}"] + 8 * cnt[f"groups{lv}"]) / tg
                                                   / 1e9 / HBM_PEAK, 4)
                line.update(ms_per_step=round(ms, 3), edges_per_s=round(g.m / (ms / 1e3), 1),
                            roofline_frac=roof,
                            stage_ms={k: round(stage.get(k, 0.0), 3) for k in
                                      ("pass1", "group1", "pass2", "group2", "hash1", "hash2")},
                            counts={k: cnt[k] for k in ("n_e", "groups1", "s1p", "entries2",
                                                        "groups2", "pairs1", "pairs2",
                                                        "chunks1", "chunks2")},
                            steps=args.steps, warmup=args.warmup)
            except B.SGError as e:
                line["error"] = str(e)
            print(json.dumps(line), flush=True)
            B.shingle_graph_destroy(h)


if __name__ == "__main__":
    main()
