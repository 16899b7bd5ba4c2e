#!/usr/bin/env python3
"""Benchmark: edges/sec shingled (2 passes, device-timed, max over ranks).

One step = one pass of the whole hot path: pass I min-hash top-s
-> group I -> pass II -> group II, on the synthetic GOS-shaped 2M-vertex graph
(BASELINE.json configs[1]; s1 = s2 = 2, c1 = c2 = 200) with the CSR already
resident in HBM.  Prints ONE JSON line (rank 0).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

--impl reference times the CPU oracle (oracle/, the plain single-threaded C
program written from the paper) on a bounded row sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth import graphs as SG  # noqa: E402

METRIC = "edges/sec shingled (2 passes, device-timed, max over ranks)"
UNIT = "edges/s"


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return dict(hbm=d.get("hbm_gbs", 6650.0), sm_max_mhz=d.get("sm_max_mhz", 1965.0),
                    src="measured (MEASURED_PEAKS.json)")
    return dict(hbm=6650.0, sm_max_mhz=1965.0, src="fallback (B200_PROFILING.md)")


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, dev: int):
        self.dev = dev
        self.proc = None
        self.lines = []

    def __enter__(self):
        if os.environ.get("SG_NO_CLOCKS"):          # A/B hook: no nvidia-smi polling
            return self
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "250", "-i", str(self.dev)],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            time.sleep(0.25)
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for ln in self.proc.stdout:
            self.lines.append(ln.strip())

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.15)
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx = float(parts[2])
            except ValueError:
                continue
            for nm, v in zip(names, parts[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": mx, "reasons": [], "samples": 0}
        busy = [x for x in sm if x > 0.5 * (mx or 1965)] or sm
        return {"sm_mhz": float(np.median(busy)), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


# ---------------------------------------------------------------- workload
def workload(name: str):
    cfg = SG.CONFIGS[name]
    g = SG.make(name, cache=os.environ.get("SG_BENCH_CACHE", "0") == "1")
    return g, cfg


def oracle_sample(g, target_nnz: int):
    """Row-prefix sample: rows [0, u) keep their full adjacency lists, later
    rows are emptied (a valid CSR: the oracle accepts asymmetric rows)."""
    u = int(np.searchsorted(g.row_ptr, target_nnz))
    u = max(1, min(u, g.n))
    rp = g.row_ptr.copy()
    rp[u + 1:] = rp[u]
    col = np.ascontiguousarray(g.col[:rp[u]])
    return rp, col, u


def run_oracle(g, cfg, target_nnz):
    import oracle
    rp, col, u = oracle_sample(g, target_nnz)
    t0 = time.perf_counter()
    oracle.shingling(rp, col, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
    dt = time.perf_counter() - t0
    edges = len(col) / 2.0
    return edges / dt, dt, u, len(col)


def cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return platform.processor()


# ---------------------------------------------------------------- roofline
def int_peak(pk):
    """Integer-ALU peak for the min-hash stages: the measured rate of the
    hash's SASS mix (tools/int_peak.cu, profiles/int_peak.json) if present,
    else the issue limit 128 thread-instr/clk/SM x 148 SMs x max SM clock."""
    p = os.path.join(ROOT, "profiles", "int_peak.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hash_mix_tinstr_per_s"]), "measured (profiles/int_peak.json: " + d.get("how", "") + ")"
    return 148 * 128 * pk["sm_max_mhz"] * 1e6 / 1e12, "derived issue limit (148 SMs x 128 instr/clk x max clock)"


def roofline_table(stage_ms: dict, counts: dict, work: dict, pk: dict):
    """Algorithmic work per stage / device time.

    Grouping (a5, a8): 24 B/pair (read and write a 12-B pair once) + 8 B/pair
    run-length read of the keys + 8 B/group offsets = 32 P + 8 G bytes, over
    the whole grouping stage (all its kernels).  Min-hash (a3, a7): 7 thread
    instructions per (entry, trial) (the hash's SASS minimum + the compare).
    Per-kernel rows use the kernels' own bytes (hist 8, scatter 20, local
    16.125 B/pair)."""
    hbm = pk["hbm"]
    ipk, isrc = int_peak(pk)
    P = {1: counts["pairs1"], 2: counts["pairs2"]}
    G = {1: counts["groups1"], 2: counts["groups2"]}
    rows = {}

    def hbm_row(stage, nbytes, basis):
        t = stage_ms.get(stage, 0.0) / 1e3
        if t <= 0:
            return None
        a = nbytes / t / 1e9
        return {"bound": "hbm", "achieved": round(a, 1), "peak": hbm, "unit": "GB/s",
                "frac": round(a / hbm, 4), "ms": round(stage_ms[stage], 3), "bytes": int(nbytes),
                "basis": basis}

    def alu_row(stage, entry_trials):
        t = stage_ms.get(stage, 0.0) / 1e3
        if t <= 0:
            return None
        a = 7.0 * entry_trials / t / 1e12
        return {"bound": "alu", "achieved": round(a, 3), "peak": round(ipk, 2), "unit": "T instr/s",
                "frac": round(a / ipk, 4), "ms": round(stage_ms[stage], 3),
                "entry_trials": int(entry_trials), "basis": "7 instr per (entry, trial)", "peak_source": isrc}

    rows["hash1"] = alu_row("hash1", work["et1"])
    rows["hash2"] = alu_row("hash2", work["et2"])
    for lv in (1, 2):
        rows[f"group{lv}"] = hbm_row(f"group{lv}", 32 * P[lv] + 8 * G[lv],
                                     "SURVEY 8(d): 24 B/pair + 8 B/pair RLE read + 8 B/group")
        rows[f"hist{lv}"] = hbm_row(f"hist{lv}", 8 * P[lv], "kernel: 8 B/pair key read")
        rows[f"scatter{lv}"] = hbm_row(f"scatter{lv}", 20 * P[lv], "kernel: 8 B read + 12 B write per pair")
        rows[f"fine{lv}"] = hbm_row(f"fine{lv}", 24 * P[lv], "kernel (v1 only): 12 B read + 12 B write")
        rows[f"local{lv}"] = hbm_row(f"local{lv}", 16.125 * P[lv], "kernel: 12 B read + 4 B + 1 bit write")
    return {k: v for k, v in rows.items() if v}


def ncu_traffic(config: str, stage: str, pairs: int):
    """DRAM bytes (read + write) of a stage from the committed ncu capture of
    this build (profiles/ncu_traffic.json: bytes per pair per stage)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None, None
    d = json.load(open(p))
    e = d.get(config, {}).get(stage)
    if not e:
        return None, None
    return int(e["bytes_per_pair"] * pairs), e.get("source")


# ---------------------------------------------------------------- our arm
def bench_ours(args, rank, world, local_rank):
    import torch
    from paper_conf_ipps_wuk13_b200 import binding as B
    torch.cuda.set_device(local_rank)
    dist_on = world > 1
    if dist_on:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    g, cfg = workload(args.config)
    s1, c1, seed1, s2, c2, seed2 = (cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
    stream = torch.cuda.Stream()           # a non-default stream shared with the library
    torch.cuda.set_stream(stream)
    dinfo = {"rank": rank, "world": world, "device": local_rank, "stream": stream.cuda_stream,
             "exchange": args.exchange, "peer": args.peer}
    shard_mode = args.shard == "components" and world > 1
    if shard_mode:
        # pClust's decomposition (N3): whole connected components per rank,
        # each rank shingles its own shard with no exchange
        shard, _ = B.sg_component_shards(g.row_ptr, g.col, world)
        rp_r, col_r = B.sg_shard_csr(g.row_ptr, g.col, shard, rank)
        g = SG.Graph(rp_r, col_r, dict(g.meta, shard=rank))
        dinfo = {"rank": 0, "world": 1, "device": local_rank, "stream": stream.cuda_stream}
    m_total = g.m if not shard_mode else None
    if dist_on and not shard_mode or args.exchange:
        # one communicator for the whole run (one ncclUniqueId per communicator)
        uid = [B.nccl_unique_id() if rank == 0 else None]
        if dist_on:
            torch.distributed.broadcast_object_list(uid, src=0)
        dinfo["nccl_uid"] = uid[0]
    # pinned host copy of the input (used by the e2e leg)
    rp_pin = torch.from_numpy(g.row_ptr).pin_memory()
    col_pin = torch.from_numpy(g.col).pin_memory()
    h = B.shingle_graph_create(rp_pin.numpy(), col_pin.numpy(), dist=dinfo)

    def step():
        B.shingle_graph_reset(h)
        B.shingle_pass(h, s1, c1, seed1)
        B.group_by_shingle(h)
        B.shingle_pass(h, s2, c2, seed2)
        B.group_by_shingle(h)

    def barrier():
        if dist_on:
            torch.distributed.barrier()

    def max_over_ranks(v):
        if not dist_on:
            return v
        t = torch.tensor([v], device="cuda")
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        return float(t.item())

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    stage_sum = {}
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(local_rank) as clk:
        barrier()
        torch.cuda.synchronize()
        ev0.record(stream)
        for _ in range(args.steps):
            step()
            for k, v in B.sg_get_stage_ms(h).items():
                stage_sum[k] = stage_sum.get(k, 0.0) + v
        ev1.record(stream)
        torch.cuda.synchronize()
        barrier()
    ms = max_over_ranks(ev0.elapsed_time(ev1) / args.steps)
    counts = B.sg_get_counts(h)
    if shard_mode:
        t = torch.tensor([float(g.m)], device="cuda", dtype=torch.float64)
        torch.distributed.all_reduce(t)
        m_total = int(t.item())
    stage_ms = {k: v / args.steps for k, v in stage_sum.items()}
    # algorithmic work of the two min-hash passes: entry x trial (this rank)
    deg = g.degrees()[counts["row_lo"]:counts["row_lo"] + counts["rows"]]
    et1 = float(deg[deg >= s1].sum()) * c1
    launches = counts["launches"]              # kernels of the last step (counter reset each step)
    # Phase III on the device, outside the metric: clusters of
    # >= 20 vertices (the size the paper evaluated)
    phase3 = None
    if world == 1 and not args.no_phase3:
        lab20, ncl = B.report_dense_subgraphs(h, 0, 20, g.n)
        phase3 = {"ms": round(B.sg_get_stage_ms(h).get("report", 0.0), 3), "clusters_ge20": int(ncl),
                  "mode": "constituents (AMB-9)", "timed_in_metric": False}
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        ooffs, _ = B.report_overlapping_clusters(h, 0, 20)
        dmean, dsd, _ = B.sg_cluster_density(h, lab20, 20)
        phase3["density_ge20"] = {"mean": round(dmean, 4), "std": round(dsd, 4)}
        phase3["overlapping"] = {"ms_host": round((time.perf_counter() - t0) * 1e3, 3),
                                 "clusters_ge20": int(len(ooffs) - 1)}

    # ---- e2e: the public API with host buffers, H2D + D2H inside the region.
    # Per step: shingle_graph_load (H2D of the pinned CSR + device validation)
    # + 2 passes + 2 groupings + report_dense_subgraphs (Phase III) with the
    # labels read back (world 1; with world > 1 the report is single-rank, so
    # the counts are read back instead).
    e2e = None
    if not args.no_e2e:
        torch.cuda.synchronize()
        barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record(stream)
        d2h = 0
        for _ in range(args.steps):
            B.shingle_graph_load(h, rp_pin.numpy(), col_pin.numpy())
            B.shingle_pass(h, s1, c1, seed1)
            B.group_by_shingle(h)
            B.shingle_pass(h, s2, c2, seed2)
            B.group_by_shingle(h)
            if world == 1:
                labels, _ = B.report_dense_subgraphs(h, 0, 20, g.n)
                d2h = labels.nbytes + 8
            else:
                B.sg_get_counts(h)
                d2h = 128
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        wall = (time.perf_counter() - t0) / args.steps * 1e3
        ems = max_over_ranks(max(e0.elapsed_time(e1) / args.steps, wall))
        e2e = {"value": round(m_total / (ems / 1e3), 1), "unit": UNIT,
               "h2d_bytes_per_step": int(g.row_ptr.nbytes + g.col.nbytes) // max(world, 1),
               "d2h_bytes_per_step": int(d2h), "ms_per_step": round(ems, 3),
               "includes": ("shingle_graph_load (H2D from pinned host + device CSR validation) + 2 passes + "
                            "2 groupings + " + ("report_dense_subgraphs + labels D2H" if world == 1
                                                else "counts D2H"))}
    B.shingle_graph_destroy(h)

    if rank != 0:
        if dist_on:
            torch.distributed.destroy_process_group()
        return
    # this rank's share of the pass-II work: entries2 is global; vertex-range
    # shards carry ~1/world of every stage
    work = {"et1": et1, "et2": float(counts["entries2"]) * c2 / world}
    pk = peaks()
    rt = roofline_table(stage_ms, counts, work, pk)
    cand = [k for k in ("hash1", "hash2", "group1", "group2") if k in rt]
    dom_name = max(cand, key=lambda k: rt[k]["ms"]) if cand else None
    dom = dict(rt[dom_name]) if dom_name else None
    if dom:
        dom["kernel"] = dom_name + (" (stage: all its kernels)" if dom_name.startswith("group") else "")
        lv = dom_name[-1]
        tr, src = ncu_traffic(args.config, dom_name, counts.get(f"pairs{lv}", 0) // max(world, 1))
        dom["traffic"] = tr
        dom["traffic_source"] = src
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        v, dt, u, nnz_s = run_oracle(g, cfg, args.cpu_sample_nnz)
        cpu = {"value": round(v, 1), "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"row prefix of {args.config}: rows [0,{u}) with full adjacency ({nnz_s} entries, "
                         f"{nnz_s // 2} edges), full two-pass method, {dt:.1f} s single-threaded "
                         f"(the same sample as --impl reference)",
               "host_cpu": cpu_model(), "host_cores": os.cpu_count()}
        cpu["tiny_full"] = oracle_tiny()
    clocks = clk.summary()
    out = {
        "metric": METRIC, "value": round(m_total / (ms / 1e3), 1), "unit": UNIT,
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(ms, 3), "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u32/u64 (integer)",
        "data": "synthetic (seeded homology-like generator, synth/graphs.py)",
        "config": {"workload": f"{args.config}: n={g.n} m={g.m} (nnz={g.nnz}), s1={s1} c1={c1} s2={s2} c2={c2}",
                   "n_e": counts["n_e"], "groups1": counts["groups1"], "s1p": counts["s1p"],
                   "groups2": counts["groups2"], "pairs1": counts["pairs1"], "pairs2": counts["pairs2"],
                   "l2": "inputs larger than L2 (CSR %.0f MB; per-step intermediates tens of GB)"
                         % ((g.row_ptr.nbytes + g.col.nbytes) / 1e6),
                   "parallelism": (f"connected-component shards x{world} (no exchange)" if shard_mode
                                   else f"vertex-range shards x{world}"),
                   "exchange": bool(counts["exchange"]), "comm_world": counts["world"],
                   "exchange_transport": ("peer stores (SG_DIST_PEER)" if args.peer else "nccl send/recv")
                   if counts["exchange"] else None},
        "stage_ms": {k: round(v, 3) for k, v in stage_ms.items() if v > 0},
        "roofline": dom, "roofline_stages": rt, "peak_source": pk["src"], "phase3": phase3,
        "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches * args.steps,
        "gpu_launches_per_step": launches,
        "clocks": clocks,
    }
    print(json.dumps(out))
    if dist_on:
        torch.distributed.destroy_process_group()


def oracle_tiny():
    """The oracle on the whole tiny config (BASELINE configs[0]), 1 core."""
    import oracle
    g = SG.make("tiny", cache=False)
    c = SG.CONFIGS["tiny"]
    t0 = time.perf_counter()
    oracle.shingling(g.row_ptr, g.col, c["s1"], c["c1"], c["seed1"], c["s2"], c["c2"], c["seed2"])
    dt = time.perf_counter() - t0
    return {"value": round(g.m / dt, 1), "unit": UNIT, "seconds": round(dt, 2),
            "workload": f"tiny: n={g.n} m={g.m}, s1=s2=2, c1=c2=100 (whole config)"}


# ---------------------------------------------------------------- reference arm
def bench_reference(args, rank, world):
    if rank != 0:
        return
    g, cfg = workload(args.config)
    vals, dts = [], []
    for i in range(args.warmup + args.steps):
        v, dt, u, nnz_s = run_oracle(g, cfg, args.ref_sample_nnz)
        if i >= args.warmup:
            vals.append(v)
            dts.append(dt)
    v = float(np.median(vals))
    out = {"metric": METRIC, "value": round(v, 1), "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(float(np.median(dts)) * 1e3, 1),
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
           "dtype": "u32/u64 (integer)", "data": "synthetic (seeded homology-like generator)",
           "config": {"workload": f"{args.config} (row-prefix sample: {nnz_s} of {g.nnz} entries)"},
           "impl": "reference",
           "cpu_baseline": {"value": round(v, 1), "unit": UNIT, "cores": 1, "kind": "oracle",
                            "sample": f"row prefix of {args.config}: rows [0,{u}) with full adjacency "
                                      f"({nnz_s} entries), full two-pass method, median of {args.steps} "
                                      f"steps (the same sample as our arm's cpu_baseline)",
                            "host_cpu": cpu_model(), "host_cores": os.cpu_count(),
                            "tiny_full": oracle_tiny()},
           "e2e": {"value": round(v, 1), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out))


def spawn(args_list, n):
    """--gpus N without a torchrun environment: re-launch this script as N
    ranks (one process per GPU) with torch.distributed.run on 127.0.0.1."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + args_list
    return subprocess.call(cmd)


def bench_dry(args, rank, world):
    """--dry-run: the launch / rendezvous / max-over-ranks / JSON-line logic on
    CPU (gloo), without the CUDA library (a CPU box can check it)."""
    import torch
    import torch.distributed as dist
    if world > 1:
        dist.init_process_group("gloo")
    t0 = time.perf_counter()
    x = 0
    for _ in range(args.warmup + args.steps):
        x += sum(range(10000))
    ms = (time.perf_counter() - t0) * 1e3 / max(args.steps, 1)
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    if rank == 0:
        print(json.dumps({"metric": METRIC, "value": None, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                          "warmup": args.warmup, "ms_per_step": round(ms, 3), "dry_run": True,
                          "comm_world": world}))
    if world > 1:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="gos2m")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-phase3", action="store_true", help="skip the untimed Phase III reports")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample-nnz", type=int, default=1_500_000)
    ap.add_argument("--ref-sample-nnz", type=int, default=1_500_000)
    ap.add_argument("--peer", action="store_true",
                    help="fused exchange: the owner split stores pairs straight into the owners' receive "
                         "buffers over NVLink peer memory (SG_DIST_PEER) instead of NCCL send/recv")
    ap.add_argument("--exchange", action="store_true",
                    help="N=1: route the pairs through the NCCL exchange path anyway (a 1-rank communicator)")
    ap.add_argument("--dry-run", action="store_true", help="CPU check of the multi-rank launch logic")
    ap.add_argument("--shard", default="range", choices=["range", "components"],
                    help="N > 1: vertex ranges + owner exchange (default) or whole connected components "
                         "per rank with no exchange (pClust's decomposition)")
    args = ap.parse_args()
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        sys.exit(spawn(sys.argv[1:], args.gpus))
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.dry_run:
        bench_dry(args, rank, world)
    elif args.impl == "reference":
        bench_reference(args, rank, world)
    else:
        bench_ours(args, rank, world, local_rank)


if __name__ == "__main__":
    main()
