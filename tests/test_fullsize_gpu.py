"""Full-size parity on the bench workload (BASELINE configs[1], gos2m: 2M
vertices, 56.9M edges, s1 = s2 = 2, c1 = c2 = 200), in the launch
configuration bench.py times (one GPU, the same trial chunking).

The oracle cannot run the whole method at this size in seconds, so the checks
are (a) sampled outputs the oracle computes one by one (pass-I shingle rows),
(b) properties that hold at any size: the selected rows, the canonical order
of G_I, each sampled group's members sharing its id, the S1' filter, and the
pair / entry counts of both levels, and (c) digests written by the oracle's
trial-outer run (tools/oracle_digests.py): every pass-I column and G_I trial,
and four full pass-II columns / G_II trials.
"""
import numpy as np
import pytest

import oracle
from synth import graphs as SG

pytestmark = pytest.mark.gpu

M1 = np.uint64(0xbf58476d1ce4e5b9)
M2 = np.uint64(0x94d049bb133111eb)


def mix64_np(z):
    """splitmix64 finaliser on a uint64 array (the grouping key, AMB-19)."""
    z = z.copy()
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * M1
        z = (z ^ (z >> np.uint64(27))) * M2
        z = z ^ (z >> np.uint64(31))
    return z


@pytest.fixture(scope="module")
def run():
    import torch
    torch.cuda.init()
    from paper_conf_ipps_wuk13_b200 import binding as B
    g = SG.make("gos2m")
    cfg = SG.CONFIGS["gos2m"]
    h = B.shingle_graph_create(g.row_ptr, g.col)
    B.shingle_pass(h, cfg["s1"], cfg["c1"], cfg["seed1"])
    B.group_by_shingle(h)
    B.shingle_pass(h, cfg["s2"], cfg["c2"], cfg["seed2"])
    B.group_by_shingle(h)
    out = dict(counts=B.sg_get_counts(h), M1=B.sg_get_shingles(h, 1), G1=B.sg_get_groups(h, 1),
               s1p=B.sg_get_s1p(h), A1=B.sg_get_hash_params(h, 1, cfg["c1"]),
               rep0=B.report_dense_subgraphs(h, 0, 1, g.n), ov=B.report_overlapping_clusters(h, 0))
    # density (Eq. 6): all clusters >= 20, and a sample of 30 clusters (the
    # rest relabelled as singletons) that the oracle recounts edge by edge
    labels = out["rep0"][0]
    out["nc20"] = B.report_dense_subgraphs(h, 0, 20, g.n)[1]
    out["dens20"] = B.sg_cluster_density(h, labels, 20)
    roots, sizes = np.unique(labels, return_counts=True)
    cand = roots[(sizes >= 2) & (sizes <= 300)]
    pick = np.random.default_rng(11).choice(cand, 30, replace=False)
    lab_s = np.where(np.isin(labels, pick), labels, np.arange(g.n, dtype=np.int32)).astype(np.int32)
    out["lab_s"] = lab_s
    out["dens_s"] = B.sg_cluster_density(h, lab_s, 2)
    out["handle2"] = h            # G_II stays resident for the per-trial digest test
    out["B"] = B
    yield g, cfg, out
    B.shingle_graph_destroy(h)


def test_fullsize_rows_and_sampled_pass1_shingles(run):
    g, cfg, out = run
    ids1, rows1 = out["M1"]
    deg = np.diff(g.row_ptr)
    assert np.array_equal(rows1, np.flatnonzero(deg >= cfg["s1"]).astype(np.uint32))
    A, B = out["A1"]
    rng = np.random.default_rng(7)
    for i in rng.choice(len(rows1), 600, replace=False):
        u = int(rows1[i])
        row = g.col[g.row_ptr[u]:g.row_ptr[u + 1]]
        want = oracle.row_shingles(row, cfg["s1"], cfg["c1"], cfg["seed1"], A, B)
        assert np.array_equal(ids1[i], want), f"pass-I shingles of vertex {u}"


def test_fullsize_group1_canonical_and_sampled_members(run):
    g, cfg, out = run
    ids1, rows1 = out["M1"]
    tg, gid, offs, mem = out["G1"]
    c1 = cfg["c1"]
    n_e = len(rows1)
    assert tg[0] == 0 and tg[-1] == len(gid) and np.all(np.diff(tg) > 0)
    assert offs[-1] == len(mem) == n_e * c1
    sizes = np.diff(offs)
    assert sizes.min() >= 1
    # canonical order: per trial, keys mix64(id) strictly ascending
    key = mix64_np(gid)
    for j in range(c1):
        k = key[tg[j]:tg[j + 1]]
        assert np.all(k[1:] > k[:-1]), f"trial {j} keys not strictly ascending"
        # each trial segment holds every generator exactly once
        assert offs[tg[j + 1]] - offs[tg[j]] == n_e
    rng = np.random.default_rng(11)
    trial_of = np.searchsorted(tg, np.arange(len(gid)), side="right") - 1
    for q in rng.choice(len(gid), 2000, replace=False):
        L = mem[offs[q]:offs[q + 1]]
        assert np.all(L[1:] > L[:-1]), "members strictly ascending"
        pos = np.searchsorted(rows1, L)
        assert np.array_equal(rows1[pos], L)
        assert np.all(ids1[pos, trial_of[q]] == gid[q]), "members generate the group's shingle"


def test_fullsize_s1p_filter_and_level2_counts(run):
    g, cfg, out = run
    ids1, rows1 = out["M1"]
    tg, gid, offs, mem = out["G1"]
    c = out["counts"]
    sizes = np.diff(offs)
    sel = np.flatnonzero(sizes >= cfg["s2"])
    s1p, k0 = out["s1p"]
    assert k0 == 0 and np.array_equal(s1p, sel)
    assert c["n_e"] == len(rows1) and c["groups1"] == len(gid) and c["pairs1"] == len(mem)
    assert c["s1p"] == len(sel)
    assert c["entries2"] == int(sizes[sel].sum())
    assert c["pairs2"] == len(sel) * cfg["c2"]
    assert len(sel) <= c["groups2"] <= c["pairs2"]


def test_fullsize_overlapping_clusters(run):
    """Phase III approach 1 at full size: clusters are ascending
    vertex lists, each inside one approach-2 cluster (P:L483-488 unions a
    superset of the same constituents); sampled S1' nodes' constituents,
    recomputed one by one by the oracle, appear among the clustered vertices."""
    g, cfg, out = run
    offs, verts = out["ov"]
    labels, _ = out["rep0"]
    C = len(offs) - 1
    assert C > 0 and offs[0] == 0 and offs[-1] == len(verts)
    sizes = np.diff(offs)
    assert sizes.min() >= 1
    v = verts.astype(np.int64)
    inner = np.ones(len(v), bool)
    inner[offs[:-1]] = False
    assert np.all(v[1:][inner[1:]] > v[:-1][inner[1:]])          # ascending within a cluster
    lab = labels[v].astype(np.int64)
    assert np.array_equal(np.minimum.reduceat(lab, offs[:-1]), np.maximum.reduceat(lab, offs[:-1]))
    clustered = np.zeros(g.n, bool)
    clustered[v] = True
    tg, gid, goffs, mem = out["G1"]
    A, Bv = out["A1"]
    s1p, _ = out["s1p"]
    rng = np.random.default_rng(5)
    for k in rng.choice(len(s1p), 200, replace=False):
        gi = int(s1p[k])
        j = int(np.searchsorted(tg, gi, side="right") - 1)
        u = int(mem[goffs[gi]])
        row = g.col[g.row_ptr[u]:g.row_ptr[u + 1]]
        cons = oracle.row_constituents(row, cfg["s1"], int(A[j]), int(Bv[j]))
        assert clustered[cons].all()


def test_fullsize_density(run):
    """Eq. 6 at full size: the sampled clusters' density matches the oracle's
    edge-by-edge count (fp64, same formula); all-cluster statistics are in
    [0, 1] over exactly the clusters report_dense_subgraphs counts."""
    g, cfg, out = run
    mean, sd, nc = out["dens_s"]
    members = np.flatnonzero(out["lab_s"] != np.arange(g.n))
    keep = np.unique(out["lab_s"][members])
    sub = np.union1d(members, keep)                    # vertices of the sampled clusters
    # the oracle on the induced CSR of the sampled clusters (ids remapped)
    remap = -np.ones(g.n, np.int64)
    remap[sub] = np.arange(len(sub))
    rp = [0]
    cols = []
    for u in sub:
        row = g.col[g.row_ptr[u]:g.row_ptr[u + 1]]
        row = remap[row[remap[row] >= 0]]
        cols.append(np.sort(row))
        rp.append(rp[-1] + len(row))
    col = np.concatenate(cols).astype(np.int32)
    lab = remap[out["lab_s"][sub]]
    rm, rs, rn = oracle.cluster_density(np.asarray(rp, np.int64), col, lab, 2)
    assert nc == rn == 30
    assert abs(mean - rm) <= 1e-12 and abs(sd - rs) <= 1e-12
    mean, sd, nc = out["dens20"]
    assert nc == out["nc20"] and 0.0 < mean <= 1.0 and 0.0 <= sd <= 0.5


@pytest.mark.timeout(1800)
def test_fullsize_digests_every_pass1_trial_and_sampled_pass2_trials(run):
    """Bit-exact parity at full size (gos2m, the bench workload) against the
    oracle's trial-outer run (tests/golden/digests_gos2m.json, written by
    tools/oracle_digests.py): every pass-I column and every G_I trial by
    digest, the S1' map, and the pass-II columns and G_II trials 0, 63, 64
    and 199 (the first / last trial of the first chunk, the first of the
    second chunk, the last trial) with their G_II trials read one at a time."""
    import json
    import os

    import digests as D
    g, cfg, out = run
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "digests_gos2m.json")))
    assert gold["graph_digest"] == D.column(np.concatenate([g.row_ptr.astype(np.uint64),
                                                           g.col.astype(np.uint64)])), \
        "generator produced another graph than the one the digests were written for"
    c = out["counts"]
    for k in ("n_e", "groups1", "pairs1", "s1p", "entries2"):
        assert c[k] == gold["counts"][k], k
    ids1, rows1 = out["M1"]
    assert D.column(rows1.astype(np.uint64)) == gold["rows1_digest"]
    for j in range(cfg["c1"]):
        assert D.column(np.ascontiguousarray(ids1[:, j])) == gold["dig_M1"][j], f"pass-I column {j}"
    tg, gid, offs, mem = out["G1"]
    assert D.grouped_trials(tg, gid, offs, mem) == gold["dig_G1"]
    s1p, _ = out["s1p"]
    assert D.column(s1p.astype(np.uint64)) == gold["s1p_digest"]
    h = out["handle2"]
    B = out["B"]
    for i, t in enumerate(gold["keep2"]):
        m2, _ = B.sg_get_shingles_range(h, 2, t, t + 1)
        assert D.column(np.ascontiguousarray(m2[:, 0])) == gold["dig_M2k"][i], f"pass-II column {t}"
        tg2, gid2, offs2, mem2 = B.sg_get_groups_range(h, 2, t, t + 1)
        assert len(gid2) == gold["G2k_groups"][i]
        assert D.grouped_trial(gid2, offs2, mem2) == gold["dig_G2k"][i], f"G_II trial {t}"
