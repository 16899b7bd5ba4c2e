"""GPU parity: libshingle (sm_100a, through the C ABI) versus the CPU oracle,
element by element, bit-exact (all arithmetic is integer).  Covers pass-I
shingle matrices, G_I, the S1' map, pass-II matrices, G_II and the final
labels, across s, c, ragged tails, staging chunks, big buckets and edge cases.
"""
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


def run_both(B, g, s1, c1, seed1, s2, c2, seed2, report=True):
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        G.run(s1, c1, seed1, s2, c2, seed2)
        out = dict(
            M1=B.sg_get_shingles(G.h, 1), G1=B.sg_get_groups(G.h, 1), s1p=B.sg_get_s1p(G.h),
            M2=B.sg_get_shingles(G.h, 2), G2=B.sg_get_groups(G.h, 2), counts=B.sg_get_counts(G.h),
            A1=B.sg_get_hash_params(G.h, 1, c1), A2=B.sg_get_hash_params(G.h, 2, c2))
        if report:
            out["rep0"] = G.report(0)                        # device union-find (default)
            out["rep1"] = G.report(1, 3)
            out["rep0h"] = G.report(0 | B.SG_REPORT_HOST)    # host union-find
            out["rep1h"] = G.report(1 | B.SG_REPORT_HOST, 3)
    ref = oracle.shingling(g.row_ptr, g.col, s1, c1, seed1, s2, c2, seed2)
    return out, ref


def assert_parity(out, ref, report=True):
    ids1, rows1 = out["M1"]
    assert np.array_equal(rows1, ref.rows1)
    assert np.array_equal(ids1, ref.M1)
    assert np.array_equal(out["A1"][0], ref.A1) and np.array_equal(out["A1"][1], ref.B1)
    assert np.array_equal(out["A2"][0], ref.A2) and np.array_equal(out["A2"][1], ref.B2)
    for got, want in ((out["G1"], ref.G1), (out["G2"], ref.G2)):
        tg, ids, offs, mem = got
        assert np.array_equal(tg, want.trial_goffs)
        assert np.array_equal(offs, want.offs)
        assert np.array_equal(mem, want.members)
        assert np.array_equal(ids, want.ids)
    s1p, k0 = out["s1p"]
    assert k0 == 0 and np.array_equal(s1p, ref.s1p_group)
    ids2, rows2 = out["M2"]
    assert np.array_equal(rows2, np.arange(len(ref.s1p_group), dtype=np.uint32))
    assert np.array_equal(ids2, ref.M2)
    c = out["counts"]
    assert c["n_e"] == len(ref.rows1) and c["s1p"] == len(ref.s1p_group)
    assert c["groups1"] == len(ref.G1.ids) and c["groups2"] == len(ref.G2.ids)
    assert c["pairs1"] == len(ref.G1.members) and c["pairs2"] == len(ref.G2.members)
    if report:
        l0, n0 = out["rep0"]
        r0, m0 = ref.report(0)
        assert n0 == m0 and np.array_equal(l0, r0)
        l1, n1 = out["rep1"]
        r1, m1 = ref.report(1, 3)
        assert n1 == m1 and np.array_equal(l1, r1)
        for key, (rl, rn) in (("rep0h", (r0, m0)), ("rep1h", (r1, m1))):
            lh, nh = out[key]
            assert nh == rn and np.array_equal(lh, rl), key


def test_tiny_config_full_parity(B):
    """BASELINE configs[0]: 10K vertices, ~200K edges, 50 planted cliques, s=2, c=100."""
    g = SG.make("tiny")
    cfg = SG.CONFIGS["tiny"]
    out, ref = run_both(B, g, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
    assert_parity(out, ref)
    # the 50 planted cliques are recovered as 50 of the clusters
    assert out["rep0"][1] >= 50


@pytest.mark.parametrize("s1,c1,s2,c2", [(1, 1, 1, 1), (1, 7, 2, 5), (2, 32, 2, 33), (3, 33, 3, 31),
                                         (5, 20, 2, 17), (8, 9, 4, 40), (2, 64, 8, 3), (4, 100, 1, 64)])
def test_tiny_parity_s_c_sweep(B, s1, c1, s2, c2):
    g = SG.make("tiny")
    out, ref = run_both(B, g, s1, c1, 1000 + c1, s2, c2, 2000 + c2)
    assert_parity(out, ref)


def test_small_homology_parity(B):
    """60K vertices / 1.7M edges, same recipe as the GOS-shaped config (several
    tiles of every kernel, ragged tails, multi-chunk histograms)."""
    g = SG.make("small")
    cfg = SG.CONFIGS["small"]
    out, ref = run_both(B, g, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
    assert_parity(out, ref)


def test_hub_rows_longer_than_staging_buffer(B):
    """Rows of 5K-12K entries: longer than 2,048 entries, so pass I takes them
    with the block-per-vertex hub_kernel (staged once, < 16,384 entries)."""
    g = SG.make("hubsmall")
    assert g.degrees().max() > 4096
    cfg = SG.CONFIGS["hubsmall"]
    out, ref = run_both(B, g, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
    assert_parity(out, ref)


def test_big_bucket_path_large_clique(B):
    """A 5,000-clique: in every trial ~4,998 vertices share one shingle, a
    group of ~5K generators in one bucket."""
    g = SG.cliques([5000, 30, 12], n=6000, seed=3)
    out, ref = run_both(B, g, 2, 6, 11, 2, 5, 12)
    assert_parity(out, ref)
    assert np.diff(ref.G1.offs).max() > 4096


@pytest.mark.parametrize("cap", ["64", "1024"])
def test_oversize_buckets_take_the_global_sort(B, cap, monkeypatch):
    """SG_GROUP=v3 with SG_LOCAL_CAP shrinking the per-bucket sort's capacity
    so that coarse buckets holding big groups (the 5,000-clique) and ordinary
    ones overflow into the global-memory sort (big_kernel)."""
    monkeypatch.setenv("SG_GROUP", "v3")
    monkeypatch.setenv("SG_LOCAL_CAP", cap)
    g = SG.cliques([5000, 300, 30, 12], n=6000, seed=4)
    out, ref = run_both(B, g, 2, 7, 13, 2, 6, 14)
    assert_parity(out, ref)


def branch_graph():
    """Complete bipartite blocks K_{a,3}: the 3 right vertices of a block have
    rows of exactly a entries (pass I) and its a left vertices share every
    first-level shingle, i.e. one G_I group of a generators per trial, which
    is a pass-II row of exactly a entries.  The lengths straddle every
    min-hash branch: <= 8 (paired short rows), 24, the per-warp stage (512 /
    1,024 entries), the 2,048 hub threshold and the 16,384-entry hub stage."""
    sizes = [1, 2, 5, 8, 9, 24, 25, 511, 512, 513, 1023, 1024, 1025, 2047, 2048, 2049,
             16383, 16384, 16385, 40000]
    n = sum(sizes) + 3 * len(sizes) + 500
    rng = np.random.default_rng(9)
    perm = rng.permutation(n).astype(np.int64)
    a_list, b_list, base = [], [], 0
    for a in sizes:
        left = np.arange(base, base + a)
        right = np.arange(base + a, base + a + 3)
        a_list.append(np.repeat(left, 3))
        b_list.append(np.tile(right, a))
        base += a + 3
    # a sparse random background on the last 500 vertices
    bg = base + rng.integers(0, 500, (2, 3000))
    a_all = perm[np.concatenate(a_list + [bg[0]])]
    b_all = perm[np.concatenate(b_list + [bg[1]])]
    rp, col = SG._csr_from_pairs(n, a_all, b_all)
    return SG.Graph(rp, col, dict(name="branches", sizes=sizes))


@pytest.mark.timeout(900)
def test_minhash_branch_edges_pass1_and_pass2(B):
    """Rows of lengths 1..40,000 straddling every min-hash branch, in pass I
    (the right vertices) and pass II (the left vertices' G_I groups), with
    c1 = c2 = 40 (one 32-trial pass + an 8-trial tail pass split over
    neighbour parts)."""
    g = branch_graph()
    deg = g.degrees()
    for a in (1023, 1025, 2049, 16385, 40000):
        assert (deg == a).sum() >= 3
    out, ref = run_both(B, g, 2, 40, 21, 2, 40, 22, report=False)
    assert_parity(out, ref, report=False)
    sizes = np.diff(ref.G1.offs)[ref.s1p_group]
    for a in (1024, 1025, 2048, 2049, 16384, 16385, 40000):
        assert (sizes == a).any(), f"no pass-II row of {a} entries"


@pytest.mark.parametrize("name", ["tiny", "small"])
def test_grouping_v1_equals_v2(B, name, monkeypatch):
    """The default grouping (stable two-level partition + warp tier) and the
    alternative SG_GROUP=v3 design (unordered coarse scatter + per-bucket
    counting sort + segmented member sort, with pass-II rows in length-class
    order) give the same canonical G_I / G_II (both equal the oracle)."""
    g = SG.make(name)
    cfg = SG.CONFIGS[name]
    args = (cfg["s1"], 33, cfg["seed1"], cfg["s2"], 35, cfg["seed2"])
    out2, ref = run_both(B, g, *args, report=False)
    assert_parity(out2, ref, report=False)
    monkeypatch.setenv("SG_GROUP", "v3")
    out1, _ = run_both(B, g, *args, report=False)
    assert_parity(out1, ref, report=False)


def test_edge_cases_empty_and_degenerate(B):
    # no edges at all: no rows, empty groups
    g = SG.Graph(np.zeros(51, np.int64), np.zeros(0, np.int32))
    out, ref = run_both(B, g, 2, 10, 1, 2, 10, 2)
    assert_parity(out, ref)
    # a matching: every vertex has degree 1 < s = 2
    a = np.arange(0, 40, 2)
    g = SG.Graph(*SG._csr_from_pairs(40, a, a + 1))
    out, ref = run_both(B, g, 2, 8, 1, 2, 8, 2)
    assert_parity(out, ref)
    # s = 1 on the matching: every group has |L| = 1 < s2 = 2, so S1' is empty
    out, ref = run_both(B, g, 1, 8, 1, 2, 8, 2)
    assert_parity(out, ref)
    assert len(ref.s1p_group) == 0


def test_state_machine_and_errors(B):
    g = SG.make("tiny")
    h = B.shingle_graph_create(g.row_ptr, g.col)
    try:
        with pytest.raises(B.SGError) as e:
            B.group_by_shingle(h)
        assert e.value.status == B.SG_ESTATE
        with pytest.raises(B.SGError) as e:
            B.shingle_pass(h, 9, 10, 1)
        assert e.value.status == B.SG_EINVAL
        with pytest.raises(B.SGError) as e:
            B.shingle_pass(h, 2, 1025, 1)
        assert e.value.status == B.SG_EINVAL
        B.shingle_pass(h, 2, 10, 1)
        with pytest.raises(B.SGError) as e:
            B.shingle_pass(h, 2, 10, 1)
        assert e.value.status == B.SG_ESTATE
        with pytest.raises(B.SGError) as e:
            B.report_dense_subgraphs(h, 0, 1, g.n)
        assert e.value.status == B.SG_ESTATE
    finally:
        B.shingle_graph_destroy(h)


def test_reset_and_rerun_identical(B):
    g = SG.make("tiny")
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        G.run(2, 40, 5, 2, 30, 6)
        a = B.sg_get_groups(G.h, 2)
        G.reset()
        G.run(2, 40, 5, 2, 30, 6)
        b = B.sg_get_groups(G.h, 2)
    for x, y in zip(a, b):
        assert np.array_equal(x, y)


def test_device_pointer_input(B):
    import torch
    g = SG.make("tiny")
    rp = torch.from_numpy(g.row_ptr).cuda()
    col = torch.from_numpy(g.col).cuda()
    h = B.shingle_graph_create(rp, col)
    try:
        B.shingle_pass(h, 2, 20, 7)
        ids, rows = B.sg_get_shingles(h, 1)
    finally:
        B.shingle_graph_destroy(h)
    ref = oracle.shingling(g.row_ptr, g.col, 2, 20, 7, 2, 4, 8)
    assert np.array_equal(rows, ref.rows1) and np.array_equal(ids, ref.M1)


@pytest.mark.parametrize("budget_mb", [400, 250, 160])
def test_trial_chunking_under_memory_budget(B, budget_mb, monkeypatch):
    """A small HBM budget forces the planner to split the trials into chunks
    (eager) or to compute keys inside the grouping (deferred); grouping is per
    trial (AMB-5), so the results must not change."""
    g = SG.make("small")
    cfg = SG.CONFIGS["small"]
    monkeypatch.setenv("SG_MEM_BUDGET", str(budget_mb << 20))
    out, ref = run_both(B, g, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"],
                        report=False)
    assert_parity(out, ref, report=False)
    c = out["counts"]
    assert abs(c["chunks1"]) > 1 or abs(c["chunks2"]) > 1, c


@pytest.mark.parametrize("v3", [False, True])
@pytest.mark.parametrize("target", ["1", "4", "40", "300"])
def test_many_bins_and_tiny_buckets(B, target, v3, monkeypatch):
    """SG_GROUP_TARGET shrinks the target bucket size so that the small graph
    takes the two-level partition (coarse scatter + per-bucket scatter) used
    by the 40M-row trial segments of the GOS-shaped pass II; with SG_GROUP=v3
    the alternative design runs with up to 2^11 coarse bins and tiny
    buckets."""
    g = SG.make("small")
    cfg = SG.CONFIGS["small"]
    monkeypatch.setenv("SG_GROUP_TARGET", target)
    if v3:
        monkeypatch.setenv("SG_GROUP", "v3")
    out, ref = run_both(B, g, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"],
                        report=False)
    assert_parity(out, ref, report=False)


@pytest.mark.parametrize("target", ["2048", "3500"])
def test_cta_tier_buckets(B, target, monkeypatch):
    """Buckets of 1,025-4,096 pairs (the CTA tier, which sorts every level-II
    bucket of the 640M-edge config): atomic LSD placements, then the full
    (key, member) verification and repair, element by element against the
    oracle."""
    g = SG.make("small")
    cfg = SG.CONFIGS["small"]
    monkeypatch.setenv("SG_GROUP_TARGET", target)
    out, ref = run_both(B, g, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"],
                        report=False)
    assert_parity(out, ref, report=False)


def test_invalid_csr_rejected(B):
    g = SG.random_graph(200, 900, seed=2)
    r = int(np.argmax(np.diff(g.row_ptr) >= 2))
    a = g.row_ptr[r]
    cases = []
    bad = g.col.copy(); bad[a], bad[a + 1] = bad[a + 1], bad[a]; cases.append((g.row_ptr, bad))
    bad = g.col.copy(); bad[a + 1] = bad[a]; cases.append((g.row_ptr, bad))
    bad = g.col.copy(); bad[-1] = 200; cases.append((g.row_ptr, bad))
    bad = g.col.copy(); bad[0] = -1; cases.append((g.row_ptr, bad))
    rp = g.row_ptr.copy(); rp[-1] -= 1; cases.append((rp, g.col[:-1].copy() if False else g.col))
    for rp, col in cases:
        with pytest.raises(B.SGError) as e:
            B.shingle_graph_create(rp, col)
        assert e.value.status == B.SG_EINVAL


# ---------------------------------------------------------------- Phase III approach 1
def _ov_case(B, g, s1, c1, seed1, s2, c2, seed2, modes=(0, 1), sizes=(1, 3)):
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        G.run(s1, c1, seed1, s2, c2, seed2)
        got = {(m, ms): G.report_overlapping(m, ms) for m in modes for ms in sizes}
    ref = oracle.shingling(g.row_ptr, g.col, s1, c1, seed1, s2, c2, seed2)
    for (m, ms), (offs, verts) in got.items():
        ro, rv = oracle.report_overlapping(ref, g.row_ptr, g.col, m, ms)
        assert np.array_equal(offs, ro), (m, ms)
        assert np.array_equal(verts, rv), (m, ms)
    return got


def test_overlapping_tiny_config(B):
    """BASELINE configs[0] (10K vertices, 50 planted cliques, s=2, c=100)."""
    g = SG.make("tiny")
    cfg = SG.CONFIGS["tiny"]
    got = _ov_case(B, g, cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"],
                   sizes=(1, 20))
    assert len(got[(0, 20)][0]) - 1 >= 50


@pytest.mark.parametrize("s1,c1,s2,c2,gseed", [(1, 20, 1, 9, 31), (2, 33, 2, 40, 32),
                                             (3, 24, 2, 17, 33), (4, 40, 3, 33, 34)])
def test_overlapping_small_graphs(B, s1, c1, s2, c2, gseed):
    g = SG.Graph(*SG.homology_graph(n=3000, n_isolated=300, m_target=40000, seed=gseed,
                                    n_cliques=12, clique_lo=6, clique_hi=30, cc_max=600,
                                    fam_hi=200))
    _ov_case(B, g, s1, c1, 100 + gseed, s2, c2, 200 + gseed)


def test_overlapping_planted_cliques_and_empty(B):
    sizes = [5, 6, 8, 10, 12, 15, 20, 25, 30, 9, 7, 11]
    g = SG.cliques(sizes, n=sum(sizes) + 40, seed=17)
    got = _ov_case(B, g, 2, 100, 21, 2, 100, 22)
    assert len(got[(0, 1)][0]) - 1 == len(sizes)
    # no first-level group reaches s2 -> no S1' node, no cluster
    g3 = SG.cliques([3, 3, 3], n=20, seed=3)
    got = _ov_case(B, g3, 2, 16, 5, 2, 16, 6)
    for offs, verts in got.values():
        assert len(offs) == 1 and len(verts) == 0


def test_overlapping_errors(B):
    g = SG.cliques([6, 7], n=20, seed=4)
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        with pytest.raises(B.SGError):
            G.report_overlapping(0)          # not grouped yet
        G.run(2, 8, 1, 2, 8, 2)
        with pytest.raises(B.SGError):
            G.report_overlapping(2)          # bad mode


# ---------------------------------------------------------------- density (Eq. 6)
def test_density_tiny_and_cliques(B):
    """Device intra-cluster edge counts vs the oracle on the tiny config's
    reported clusters (both modes, min_size 2 and 20) and on planted cliques
    (density exactly 1)."""
    g = SG.make("tiny")
    cfg = SG.CONFIGS["tiny"]
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        G.run(cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
        for mode in (0, 1):
            labels, _ = G.report(mode)
            for ms in (2, 20):
                got = G.density(labels, ms)
                want = oracle.cluster_density(g.row_ptr, g.col, labels, ms)
                assert got[2] == want[2]
                assert abs(got[0] - want[0]) <= 1e-12 and abs(got[1] - want[1]) <= 1e-12
        with pytest.raises(B.SGError):
            G.density(np.full(g.n, g.n, np.int32))      # label out of range
    gc = SG.cliques([5, 8, 13], n=40, seed=6)
    with B.ShingleGraph(gc.row_ptr, gc.col) as G:
        G.run(2, 50, 1, 2, 50, 2)
        labels, nc = G.report(0)
        assert nc == 3 and G.density(labels) == (1.0, 0.0, 3)
        with pytest.raises(ValueError):                   # label array of the wrong length
            G.density(labels[:-1])
        with pytest.raises(ValueError):
            G.agreement(labels, labels[:5])
    # self-loops are not edges and one-directional entries count half (AMB-21)
    for rp, col, lab in ((np.array([0, 2, 4], np.int64), np.array([0, 1, 0, 1], np.int32), [0, 0]),
                         (np.array([0, 1, 3, 3], np.int64), np.array([1, 0, 2], np.int32), [0, 0, 0])):
        lab = np.asarray(lab, np.int32)
        with B.ShingleGraph(rp, col) as G:
            got = G.density(lab)
        want = oracle.cluster_density(rp, col, lab)
        assert got[2] == want[2] and abs(got[0] - want[0]) <= 1e-12


# ---------------------------------------------------------------- Eq. 2-5 pair counts
def test_agreement_vs_planted_families(B):
    """TP/FP/FN/TN of the reported clusters against the generator's planted
    families (the benchmark partition of Eq. 2-5), both report modes, and of
    mode 0 against mode 1 on the tiny config: exact integers vs the oracle's
    pair-by-pair count."""
    row_ptr, col, fam = SG.homology_graph(n=3000, n_isolated=300, m_target=40000, seed=41,
                                          n_cliques=12, clique_lo=6, clique_hi=30, cc_max=600,
                                          fam_hi=200, return_families=True)
    g = SG.Graph(row_ptr, col)
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        G.run(2, 60, 141, 2, 60, 241)
        for mode in (0, 1):
            labels, _ = G.report(mode)
            got = G.agreement(labels, fam)
            want = oracle.partition_agreement(labels, fam)
            assert {k: got[k] for k in ("TP", "FP", "FN", "TN")} == \
                   {k: want[k] for k in ("TP", "FP", "FN", "TN")}
            assert got["TP"] > 0
        with pytest.raises(B.SGError):
            G.agreement(np.full(g.n, -1, np.int32), fam)
    t = SG.make("tiny")
    cfg = SG.CONFIGS["tiny"]
    with B.ShingleGraph(t.row_ptr, t.col) as G:
        G.run(cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
        l0, _ = G.report(0)
        l1, _ = G.report(1)
        got = G.agreement(l0, l1)
        want = oracle.partition_agreement(l0, l1)
        assert [got[k] for k in ("TP", "FP", "FN", "TN")] == [want[k] for k in ("TP", "FP", "FN", "TN")]


# ---------------------------------------------------------------- connected components
@pytest.mark.parametrize("name", ["tiny", "small", "cliques"])
def test_components(B, name):
    if name == "tiny":
        g = SG.make("tiny")
    elif name == "small":
        g = SG.Graph(*SG.homology_graph(n=30000, n_isolated=3000, m_target=300000, seed=51,
                                        n_cliques=20, clique_lo=6, clique_hi=40, cc_max=3000,
                                        fam_hi=300))
    else:
        g = SG.cliques([5, 8, 13, 40], n=100, seed=6)
    with B.ShingleGraph(g.row_ptr, g.col) as G:
        lab, k = G.components()
    want, wk = oracle.connected_components(g.row_ptr, g.col)
    assert k == wk and np.array_equal(lab, want)


@pytest.mark.parametrize("name", ["tiny", "hubsmall"])
def test_out_of_core_entries_host_csr(B, name):
    """SG_HOST_CSR (N4): the entries stay in host memory (page-locked, mapped)
    and the kernels read them over the host link; every output, the reports,
    density and components equal the oracle / the in-HBM run."""
    g = SG.make(name)
    cfg = SG.CONFIGS[name]
    args = (cfg["s1"], 40, cfg["seed1"], cfg["s2"], 33, cfg["seed2"])
    col = np.ascontiguousarray(g.col)
    with B.ShingleGraph(g.row_ptr, col, host_csr=True) as G:
        G.run(*args)
        out = dict(
            M1=B.sg_get_shingles(G.h, 1), G1=B.sg_get_groups(G.h, 1), s1p=B.sg_get_s1p(G.h),
            M2=B.sg_get_shingles(G.h, 2), G2=B.sg_get_groups(G.h, 2), counts=B.sg_get_counts(G.h),
            A1=B.sg_get_hash_params(G.h, 1, args[1]), A2=B.sg_get_hash_params(G.h, 2, args[4]))
        out["rep0"] = G.report(0)
        out["rep1"] = G.report(1, 3)
        out["rep0h"] = G.report(0 | B.SG_REPORT_HOST)
        out["rep1h"] = G.report(1 | B.SG_REPORT_HOST, 3)
        dens = G.density(out["rep0"][0], 2)
        comp = G.components()
    ref = oracle.shingling(g.row_ptr, g.col, *args)
    assert_parity(out, ref)
    assert dens[2] == oracle.cluster_density(g.row_ptr, g.col, out["rep0"][0], 2)[2]
    assert np.array_equal(comp[0], oracle.connected_components(g.row_ptr, g.col)[0])
