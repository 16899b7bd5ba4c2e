"""Multi-rank parity on one GPU: `world` virtual ranks (one host thread each,
in-process loopback transport) run the sharded path — vertex-
range rows, owner-routed exchange before each grouping, canonical S1' index
across ranks — and the per-rank results, assembled in rank order, must equal
the single-process oracle bit for bit.  The NCCL backend runs the same code
above the transport (x_allgather_i64 / x_alltoallv)."""
import threading

import numpy as np
import pytest

import oracle
from synth import graphs as SG

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def B():
    import torch
    torch.cuda.init()
    from paper_conf_ipps_wuk13_b200 import binding
    binding.lib()
    return binding


def run_ranks(B, g, world, s1, c1, seed1, s2, c2, seed2, env_budget=None, peer=False):
    lb = B.sg_loopback_create(world)
    res, errs = [None] * world, [None] * world

    def body(r):
        h = None
        try:
            h = B.shingle_graph_create(g.row_ptr, g.col,
                                       dist={"rank": r, "world": world, "device": 0, "loopback": lb,
                                             "peer": peer})
            B.shingle_pass(h, s1, c1, seed1)
            B.group_by_shingle(h)
            B.shingle_pass(h, s2, c2, seed2)
            B.group_by_shingle(h)
            res[r] = dict(counts=B.sg_get_counts(h), M1=B.sg_get_shingles(h, 1),
                          G1=B.sg_get_groups(h, 1), s1p=B.sg_get_s1p(h),
                          M2=B.sg_get_shingles(h, 2), G2=B.sg_get_groups(h, 2))
        except Exception as e:  # noqa: BLE001 - surfaced below
            errs[r] = e
        finally:
            if h is not None:
                B.shingle_graph_destroy(h)

    ts = [threading.Thread(target=body, args=(r,)) for r in range(world)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(240)
    assert not any(t.is_alive() for t in ts), "a virtual rank hung"
    B.sg_loopback_destroy(lb)
    for e in errs:
        if e is not None:
            raise e
    return res


def assemble_groups(parts, c):
    """Concatenate per-rank groups trial by trial in rank order (ranks own
    ascending key ranges, so this is the canonical (trial, key) order)."""
    tg, ids, sizes, mem = [0], [], [], []
    goff = []   # goff[r][j] = global index of rank r's first group of trial j
    for r in range(len(parts)):
        goff.append(np.zeros(c, np.int64))
    for j in range(c):
        for r, (t, i, o, m) in enumerate(parts):
            goff[r][j] = len(ids)
            a, b = t[j], t[j + 1]
            ids.extend(i[a:b])
            sizes.extend(np.diff(o[a:b + 1]))
            mem.append(m[o[a]:o[b]])
        tg.append(len(ids))
    offs = np.concatenate([[0], np.cumsum(sizes, dtype=np.int64)]).astype(np.int64)
    mem = np.concatenate(mem) if mem else np.zeros(0, np.uint32)
    return np.array(tg, np.int64), np.array(ids, np.uint64), offs, mem, goff


def check(res, ref, c1, c2):
    world = len(res)
    # every rank agrees on the global counts
    for k in ("n_e", "groups1", "s1p", "groups2", "pairs1", "pairs2", "entries2"):
        assert len({r["counts"][k] for r in res}) == 1, k
    cnt = res[0]["counts"]
    assert cnt["n_e"] == len(ref.rows1) and cnt["s1p"] == len(ref.s1p_group)
    assert cnt["groups1"] == len(ref.G1.ids) and cnt["groups2"] == len(ref.G2.ids)
    assert cnt["pairs1"] == len(ref.G1.members) and cnt["pairs2"] == len(ref.G2.members)
    # rows: contiguous vertex ranges covering [0, n)
    lo = [r["counts"]["row_lo"] for r in res]
    assert lo[0] == 0 and all(a <= b for a, b in zip(lo, lo[1:]))
    # pass I: each rank's rows are its vertex range, in order
    ids1 = np.concatenate([r["M1"][0] for r in res])
    rows1 = np.concatenate([r["M1"][1] for r in res])
    assert np.array_equal(rows1, ref.rows1)
    assert np.array_equal(ids1, ref.M1)
    # G_I / G_II
    for lev, want, c in ((1, ref.G1, c1), (2, ref.G2, c2)):
        tg, ids, offs, mem, goff = assemble_groups([r[f"G{lev}"] for r in res], c)
        assert np.array_equal(tg, want.trial_goffs), lev
        assert np.array_equal(offs, want.offs), lev
        assert np.array_equal(mem, want.members), lev
        assert np.array_equal(ids, want.ids), lev
        if lev == 1:
            goff1 = goff
    # S1' rows: canonical index k in rowid, local G_I group in s1p
    seen = np.zeros(len(ref.s1p_group), np.int64)
    for r, part in enumerate(res):
        ids2, k = part["M2"]
        s1p, _ = part["s1p"]
        assert len(s1p) == len(k)
        assert np.all(np.diff(k.astype(np.int64)) > 0)
        assert np.array_equal(ids2, ref.M2[k])
        tgl = part["G1"][0]
        trial = np.searchsorted(tgl, s1p, side="right") - 1
        glob = goff1[r][trial] + (s1p - tgl[trial])
        assert np.array_equal(glob, ref.s1p_group[k])
        seen[k] += 1
    assert np.all(seen == 1)


@pytest.mark.timeout(600)
@pytest.mark.parametrize("world", [2, 3, 4])
def test_loopback_tiny(B, world):
    g = SG.make("tiny")
    cfg = SG.CONFIGS["tiny"]
    res = run_ranks(B, g, world, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
    ref = oracle.shingling(g.row_ptr, g.col, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"],
                           cfg["seed2"])
    check(res, ref, cfg["c1"], cfg["c2"])


@pytest.mark.timeout(600)
@pytest.mark.parametrize("world,s1,c1,s2,c2", [(2, 1, 7, 2, 5), (3, 3, 33, 3, 31), (2, 5, 20, 2, 17),
                                               (4, 2, 64, 8, 3), (5, 4, 40, 1, 64)])
def test_loopback_s_c_sweep(B, world, s1, c1, s2, c2):
    g = SG.make("tiny")
    res = run_ranks(B, g, world, s1, c1, 1000 + c1, s2, c2, 2000 + c2)
    ref = oracle.shingling(g.row_ptr, g.col, s1, c1, 1000 + c1, s2, c2, 2000 + c2)
    check(res, ref, c1, c2)


@pytest.mark.timeout(900)
def test_loopback_small_homology(B):
    g = SG.make("small")
    cfg = SG.CONFIGS["small"]
    res = run_ranks(B, g, 2, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
    ref = oracle.shingling(g.row_ptr, g.col, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"],
                           cfg["seed2"])
    check(res, ref, cfg["c1"], cfg["c2"])


@pytest.mark.timeout(600)
def test_loopback_big_bucket_and_empty_rank(B):
    """A 5,000-clique (one owner receives a >4,096 group every trial) and more
    ranks than non-trivial rows in places (some ranks own no pass-I rows)."""
    g = SG.cliques([5000, 30, 12], n=6000, seed=3)
    res = run_ranks(B, g, 3, 2, 6, 11, 2, 5, 12)
    ref = oracle.shingling(g.row_ptr, g.col, 2, 6, 11, 2, 5, 12)
    check(res, ref, 6, 5)
    # a graph with no edges: every rank has zero rows
    g = SG.Graph(np.zeros(51, np.int64), np.zeros(0, np.int32))
    res = run_ranks(B, g, 2, 2, 10, 1, 2, 10, 2)
    ref = oracle.shingling(g.row_ptr, g.col, 2, 10, 1, 2, 10, 2)
    check(res, ref, 10, 10)


@pytest.mark.timeout(600)
@pytest.mark.parametrize("world,s1,c1,s2,c2", [(2, 2, 100, 2, 100), (3, 3, 33, 3, 31),
                                               (4, 2, 64, 8, 3), (5, 4, 40, 1, 64)])
def test_loopback_fused_peer_exchange(B, world, s1, c1, s2, c2):
    """SG_DIST_PEER: the owner-partition kernel stores every
    pair straight into its owner's receive buffer (peer pointers of the other
    virtual ranks); no send buffer, no send / recv.  Same outputs as the
    oracle, element by element."""
    g = SG.make("tiny")
    res = run_ranks(B, g, world, s1, c1, 1000 + c1, s2, c2, 2000 + c2, peer=True)
    ref = oracle.shingling(g.row_ptr, g.col, s1, c1, 1000 + c1, s2, c2, 2000 + c2)
    check(res, ref, c1, c2)


@pytest.mark.timeout(900)
def test_loopback_fused_peer_small_and_chunked(B, monkeypatch):
    """The fused exchange on the homology-shaped `small` config, once with
    the planner forced into several trial chunks (the receive buffers are
    reused chunk after chunk behind the per-chunk barriers)."""
    g = SG.make("small")
    cfg = SG.CONFIGS["small"]
    args = (cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
    ref = oracle.shingling(g.row_ptr, g.col, *args)
    check(run_ranks(B, g, 2, *args, peer=True), ref, cfg["c1"], cfg["c2"])
    monkeypatch.setenv("SG_MEM_BUDGET", str(150 << 20))   # level II in several trial chunks
    res = run_ranks(B, g, 3, *args, peer=True)
    check(res, ref, cfg["c1"], cfg["c2"])
    assert any(abs(r["counts"]["chunks1"]) > 1 or abs(r["counts"]["chunks2"]) > 1 for r in res)


@pytest.mark.timeout(300)
def test_loopback_peer_failure_does_not_hang(B):
    """A rank that fails inside a collective call breaks the group: its peers
    return SG_ESTATE instead of blocking forever."""
    g = SG.make("tiny")
    lb = B.sg_loopback_create(2)
    errs = [None, None]

    def body(r):
        h = B.shingle_graph_create(g.row_ptr, g.col,
                                   dist={"rank": r, "world": 2, "device": 0, "loopback": lb})
        try:
            if r == 1:
                B.group_by_shingle(h)       # wrong order: fails before any exchange
            else:
                B.shingle_pass(h, 2, 8, 1)  # blocks in its exchange until the abort
        except B.SGError as e:
            errs[r] = e.status
        finally:
            B.shingle_graph_destroy(h)

    ts = [threading.Thread(target=body, args=(r,)) for r in range(2)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(120)
    assert not any(t.is_alive() for t in ts)
    B.sg_loopback_destroy(lb)
    assert errs[1] == B.SG_ESTATE and errs[0] == B.SG_ESTATE


def test_loopback_single_rank_calls_refuse_world_gt_1(B):
    """The report and quality calls are single-rank: with world > 1
    they fail with SG_EINVAL on every rank instead of computing a partial answer."""
    g = SG.make("tiny")
    lb = B.sg_loopback_create(2)
    codes = [[], []]

    def body(r):
        h = B.shingle_graph_create(g.row_ptr, g.col,
                                   dist={"rank": r, "world": 2, "device": 0, "loopback": lb})
        try:
            B.shingle_pass(h, 2, 8, 1)
            B.group_by_shingle(h)
            B.shingle_pass(h, 2, 8, 2)
            B.group_by_shingle(h)
            lab = np.arange(g.n, dtype=np.int32)
            for call in (lambda: B.report_dense_subgraphs(h, 0, 1, g.n),
                         lambda: B.report_overlapping_clusters(h, 0),
                         lambda: B.sg_cluster_density(h, lab),
                         lambda: B.sg_partition_agreement(h, lab, lab),
                         lambda: B.sg_connected_components(h, g.n)):
                try:
                    call()
                    codes[r].append(0)
                except B.SGError as e:
                    codes[r].append(e.status)
        finally:
            B.shingle_graph_destroy(h)

    ts = [threading.Thread(target=body, args=(r,)) for r in range(2)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(120)
    assert not any(t.is_alive() for t in ts)
    B.sg_loopback_destroy(lb)
    assert codes == [[B.SG_EINVAL] * 5, [B.SG_EINVAL] * 5]
