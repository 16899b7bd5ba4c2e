"""Host logic of the N > 1 path on CPU: two real processes over torch.distributed
(gloo, 127.0.0.1) exercise what bench.py and the library do around the
device exchange — the ncclUniqueId broadcast, the identical vertex-range
partition on every rank, and the canonical S1' index (sg_s1p_offsets) fed by
all-gathered per-trial counts.  The expected S1' order comes from the oracle
(owner(key) = floor(key * R / 2^64) gives every rank a
contiguous key range, so rank order inside a trial is canonical order)."""
import os
import socket

import numpy as np
import pytest


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    import torch.distributed as dist

    import oracle
    from paper_conf_ipps_wuk13_b200 import binding as B
    from synth import graphs as SG

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        out = {}
        # 1. ncclUniqueId broadcast (bench.py's recipe): rank 0 creates it
        uid = [B.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        got = [None] * world
        dist.all_gather_object(got, uid[0])
        out["uid_same"] = len(uid[0]) == 128 and all(g == got[0] for g in got)

        # 2. every rank computes the same row partition from the global CSR
        g = SG.make("tiny")
        b = B.sg_partition_rows(g.row_ptr, world)
        allb = [None] * world
        dist.all_gather_object(allb, b.tolist())
        out["bounds_same"] = all(x == allb[0] for x in allb)
        out["bounds"] = b.tolist()

        # 3. canonical S1' index: this rank owns the G_I groups whose key is in
        # its range; counts per trial of groups with |L| >= s2 are all-gathered
        s1, c1, s2 = 2, 24, 2
        ref = oracle.shingling(g.row_ptr, g.col, s1, c1, 5, s2, 6, 6)
        G1 = ref.G1
        sizes = np.diff(G1.offs)
        keys = np.array([oracle.mix64(int(i)) for i in G1.ids], dtype=np.uint64)
        owner = np.array([(int(k) * world) >> 64 for k in keys], np.int64)
        trial = np.searchsorted(G1.trial_goffs, np.arange(len(G1.ids)), side="right") - 1
        mine = np.flatnonzero((owner == rank) & (sizes >= s2))        # local S1' rows, (trial, key) order
        cnt = np.bincount(trial[mine], minlength=c1).astype(np.int64)
        allc = [None] * world
        dist.all_gather_object(allc, cnt.tolist())
        first, off, total = B.sg_s1p_offsets(np.array(allc, np.int64), rank)
        k = np.arange(len(mine)) + off[trial[mine]]
        out["total_ok"] = total == len(ref.s1p_group)
        out["first_ok"] = np.array_equal(first, np.concatenate([[0], np.cumsum(cnt)]))
        out["k_ok"] = bool(np.array_equal(ref.s1p_group[k], mine))
        out["k"] = k.tolist()
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_gloo_world2_host_logic():
    import torch.multiprocessing as mp

    from paper_conf_ipps_wuk13_b200 import binding as B
    try:
        B.lib()
    except ImportError:
        pytest.skip("libshingle.so not built")
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(world))
    for p in ps:
        p.join(60)
        assert p.exitcode == 0
    n = 10000
    for r in range(world):
        o = res[r]
        assert o["uid_same"] and o["bounds_same"]
        assert o["total_ok"] and o["first_ok"] and o["k_ok"], r
    b = res[0]["bounds"]
    assert b[0] == 0 and b[-1] == n and b[0] <= b[1] <= b[2]
    # the two ranks' canonical indices tile [0, |S1'|) exactly once
    ks = np.sort(np.concatenate([res[0]["k"], res[1]["k"]]))
    assert np.array_equal(ks, np.arange(len(ks)))
