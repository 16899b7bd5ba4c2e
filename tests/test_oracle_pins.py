"""Pins for the CPU oracle (-m "not gpu").  The oracle is trusted only after
these pass; each check ties it to something other than itself: published
known answers, closed forms, brute force, an N-version twin, invariants.
Self-check numbering (i)-(ix) follows SURVEY.md §8c / DESIGN.md §5.
"""
import math
import os
from collections import defaultdict

import numpy as np
import pytest

import oracle
from oracle import twin
from synth import graphs as SG

GOLD = os.path.join(os.path.dirname(__file__), "golden")
P = (1 << 31) - 1


def _gold_lines(name):
    with open(os.path.join(GOLD, name)) as f:
        return [ln.split() for ln in f if ln.strip() and not ln.startswith("#")]


# ---------------------------------------------------------------- (v) primitives
def test_splitmix64_known_answers():
    want = [int(x[0], 16) for x in _gold_lines("splitmix64_seed0.txt")]
    # the oracle's stream = mix64(state += gamma); with seed 0 the first
    # three states are gamma, 2 gamma, 3 gamma
    gamma = 0x9E3779B97F4A7C15
    got = [oracle.mix64((k * gamma) & ((1 << 64) - 1)) for k in (1, 2, 3)]
    assert got == want


def test_mix64_is_a_bijection_inverse_roundtrip():
    # closed-form inverse of the splitmix64 finaliser: the two odd multipliers
    # have inverses 0x96de1b173f119089 and 0x319642b2d24d8ec3 mod 2^64
    M = (1 << 64) - 1

    def unxs(z, s):
        x = z
        for _ in range(64 // s + 1):
            x = z ^ (x >> s)
        return x

    def inv(z):
        z = unxs(z, 31)
        z = (z * 0x319642B2D24D8EC3) & M
        z = unxs(z, 27)
        z = (z * 0x96DE1B173F119089) & M
        return unxs(z, 30)

    assert (0xBF58476D1CE4E5B9 * 0x96DE1B173F119089) & M == 1
    assert (0x94D049BB133111EB * 0x319642B2D24D8EC3) & M == 1
    rng = np.random.default_rng(7)
    for z in [0, 1, M, 1 << 63] + [int(x) for x in rng.integers(0, 1 << 63, 200, dtype=np.int64)]:
        assert inv(oracle.mix64(z)) == z


def test_hash_adversarial_vectors():
    for A, B, v, h in (map(int, r) for r in _gold_lines("m31_vectors.txt")):
        assert oracle.hash1(A, B, v) == h
        assert (A * v + B) % P == h           # big-int definition
    # the zero residue in row 1 is the closed form (P - B) * A^(P-2) mod P
    A, B = 123456789, 987654321
    assert (P - B) * pow(A, P - 2, P) % P == 773987457


def test_hash_random_vs_bigint():
    rng = np.random.default_rng(11)
    A = rng.integers(1, P, 20000)
    B = rng.integers(0, P, 20000)
    v = rng.integers(0, P, 20000)
    for a, b, x in zip(A.tolist(), B.tolist(), v.tolist()):
        assert oracle.hash1(a, b, x) == (a * x + b) % P


def test_hash_params_ranges_and_twin():
    for seed in [0, 1, 101, 2**63 + 5]:
        A, B = oracle.hash_params(seed, 500)
        assert A.min() >= 1 and A.max() <= P - 1
        assert B.max() <= P - 1
        tA, tB = twin.hash_params(seed, 500)
        assert A.tolist() == tA and B.tolist() == tB


def test_validate_rejects_bad_csr():
    g = SG.random_graph(50, 200, seed=1)
    assert oracle.validate(g.row_ptr, g.col)
    bad = g.col.copy()
    r = int(np.argmax(np.diff(g.row_ptr) >= 2))
    a = g.row_ptr[r]
    bad[a], bad[a + 1] = bad[a + 1], bad[a]          # unsorted row
    assert not oracle.validate(g.row_ptr, bad)
    bad = g.col.copy()
    bad[a + 1] = bad[a]                               # duplicate
    assert not oracle.validate(g.row_ptr, bad)
    bad = g.col.copy()
    bad[-1] = 50                                      # id >= n
    assert not oracle.validate(g.row_ptr, bad)
    rp = g.row_ptr.copy()
    rp[-1] += 1                                       # row_ptr[n] != nnz
    assert not oracle.validate(rp, g.col)


# ---------------------------------------------------------------- (i) top-s == full sort
@pytest.mark.parametrize("s", [1, 2, 3, 5])
def test_top_s_equals_bruteforce_full_sort(s):
    g = SG.make("tiny")
    c, seed = 12, 99
    A, B = oracle.hash_params(seed, c)
    deg = g.degrees()
    rows = np.nonzero(deg >= s)[0]
    rng = np.random.default_rng(s)
    rows = rows[rng.permutation(len(rows))[:800]]
    for u in rows.tolist():
        nb = g.col[g.row_ptr[u]:g.row_ptr[u + 1]].astype(np.int64)
        ids = oracle.row_shingles(nb, s, c, seed, A, B)
        hv = (A.astype(np.int64)[:, None] * nb[None, :] + B.astype(np.int64)[:, None]) % P
        hv.sort(axis=1)                                # full sort of every Gamma_j(u)
        for j in range(c):
            mins = [int(x) for x in hv[j, :s]]
            assert int(ids[j]) == twin.shingle_id(s, seed, j, mins)


def test_hash_eval_count_matches_complexity():
    # the work is one hash per (adjacency entry, trial) of every
    # eligible row in both passes: sum_{deg>=s1} deg*c1 + sum_{S1'} |L|*c2
    g = SG.make("tiny")
    s1, c1, s2, c2 = 2, 10, 2, 7
    res = oracle.shingling(g.row_ptr, g.col, s1, c1, 3, s2, c2, 4)
    d = g.degrees()
    want1 = int(d[d >= s1].sum()) * c1
    sizes = np.diff(res.G1.offs)
    want2 = int(sizes[sizes >= s2].sum()) * c2
    assert res.hash_evals == want1 + want2


# ---------------------------------------------------------------- (ii) twins
def test_identical_neighbourhoods_identical_shingles():
    rng = np.random.default_rng(3)
    n = 400
    adj = [set() for _ in range(n)]
    for _ in range(3000):
        a, b = rng.integers(0, n, 2)
        if a != b:
            adj[a].add(int(b)); adj[b].add(int(a))
    # make 300 and 301 twins: same neighbourhood, not adjacent to each other
    adj[300].discard(301); adj[301].discard(300)
    for v in list(adj[301]):
        adj[v].discard(301)
    for v in adj[300]:
        adj[v].add(301)
    adj[301] = set(adj[300])
    g = SG.from_adj([sorted(x) for x in adj])
    res = oracle.shingling(g.row_ptr, g.col, 2, 64, 5, 2, 16, 6)
    r = {int(u): i for i, u in enumerate(res.rows1)}
    assert np.array_equal(res.M1[r[300]], res.M1[r[301]])
    # and both are members of exactly the same first-level groups
    for j in range(64):
        lo, hi = res.G1.trial_goffs[j], res.G1.trial_goffs[j + 1]
        for gi in range(lo, hi):
            mem = res.G1.members[res.G1.offs[gi]:res.G1.offs[gi + 1]]
            assert (300 in mem) == (301 in mem)


# ---------------------------------------------------------------- (iii) planted cliques
@pytest.mark.parametrize("mode", [0, 1])
def test_planted_cliques_one_cluster_each(mode):
    sizes = [5, 6, 8, 10, 12, 15, 20, 25, 30, 9, 7, 11]
    g = SG.cliques(sizes, n=sum(sizes) + 40, seed=17)     # + 40 isolated vertices
    res = oracle.shingling(g.row_ptr, g.col, 2, 100, 21, 2, 100, 22)
    labels, nc = res.report(mode=mode)
    assert nc == len(sizes)
    # each clique is one CC of G: compare the label partition with the CCs
    deg = g.degrees()
    comp = _components(g)
    for v in range(g.n):
        if deg[v] == 0:
            assert labels[v] == v
    by_label = defaultdict(set)
    by_comp = defaultdict(set)
    for v in range(g.n):
        by_label[labels[v]].add(v)
        by_comp[comp[v]].add(v)
    assert sorted(map(sorted, by_label.values())) == sorted(map(sorted, by_comp.values()))


def _components(g):
    n = g.n
    lab = -np.ones(n, np.int64)
    for s in range(n):
        if lab[s] >= 0:
            continue
        lab[s] = s
        st = [s]
        while st:
            x = st.pop()
            for y in g.col[g.row_ptr[x]:g.row_ptr[x + 1]]:
                if lab[y] < 0:
                    lab[y] = s
                    st.append(int(y))
    return lab


# ---------------------------------------------------------------- (iv) min-wise rate
def _binom_two_sided_tail(k, n, p):
    """Exact two-sided binomial tail probability P(|X - np| >= |k - np|)."""
    mean = n * p
    d = abs(k - mean)
    logs = [math.lgamma(n + 1) - math.lgamma(i + 1) - math.lgamma(n - i + 1)
            + (i * math.log(p) if i else 0.0) + ((n - i) * math.log1p(-p) if n - i else 0.0)
            for i in range(n + 1)]
    return min(1.0, sum(math.exp(l) for i, l in enumerate(logs) if abs(i - mean) >= d - 1e-9))


@pytest.mark.parametrize("s,inter,union", [(1, 10, 40), (2, 30, 60), (2, 12, 30), (3, 40, 60)])
def test_minwise_collision_rate_matches_closed_form(s, inter, union):
    # [4] via P:L437-439: Pr[top-s(A) = top-s(B)] = C(|A n B|, s) / C(|A u B|, s)
    # (= Jaccard, Eq. 1, for s = 1).  Ids must be scattered.
    rng = np.random.default_rng(1000 + s * 100 + inter)
    ids = rng.choice(1_000_000, union, replace=False).astype(np.uint32)
    half = (union - inter) // 2
    Aset = np.sort(ids[: inter + half])
    Bset = np.sort(np.concatenate([ids[:inter], ids[inter + half:]]))
    T = 10_000
    sa = oracle.row_shingles(Aset, s, T, 4242)
    sb = oracle.row_shingles(Bset, s, T, 4242)
    hits = int((sa == sb).sum())
    p = math.comb(inter, s) / math.comb(len(np.union1d(Aset, Bset)), s)
    assert T * p >= 20
    assert _binom_two_sided_tail(hits, T, p) >= 1e-6, (hits, T * p)


# ---------------------------------------------------------------- (vi) ids and grouping
def test_s_le_2_ids_roundtrip_through_A_inverse():
    g = SG.make("tiny")
    for s in (1, 2):
        res = oracle.shingling(g.row_ptr, g.col, s, 8, 31, 2, 4, 32)
        for r in range(0, len(res.rows1), 97):
            u = int(res.rows1[r])
            nb = g.col[g.row_ptr[u]:g.row_ptr[u + 1]]
            for j in range(8):
                idv = int(res.M1[r, j])
                hs = [idv] if s == 1 else [idv >> 31, idv & P]
                A, B = int(res.A1[j]), int(res.B1[j])
                Ainv = pow(A, P - 2, P)
                verts = sorted((h - B) * Ainv % P for h in hs)
                want = sorted(oracle.row_constituents(nb, s, A, B).tolist())
                assert verts == want
                assert all(v in set(nb.tolist()) for v in verts)


def test_exact_tuple_grouping_equals_id_grouping_s3():
    g = SG.make("tiny")
    s, c, seed = 3, 10, 77
    res = oracle.shingling(g.row_ptr, g.col, s, c, seed, 2, 3, 78)
    A, B = res.A1, res.B1
    for j in range(c):
        tup = defaultdict(list)
        for r, u in enumerate(res.rows1.tolist()):
            nb = g.col[g.row_ptr[u]:g.row_ptr[u + 1]].astype(np.int64)
            hv = np.sort((int(A[j]) * nb + int(B[j])) % P)[:s]
            tup[tuple(hv.tolist())].append(u)
        lo, hi = res.G1.trial_goffs[j], res.G1.trial_goffs[j + 1]
        groups = sorted(res.G1.members[res.G1.offs[k]:res.G1.offs[k + 1]].tolist() for k in range(lo, hi))
        assert groups == sorted(sorted(v) for v in tup.values())


def test_group_invariants():
    g = SG.make("tiny")
    res = oracle.shingling(g.row_ptr, g.col, 2, 20, 1, 2, 20, 2)
    for G, nrows, c in ((res.G1, len(res.rows1), 20), (res.G2, len(res.s1p_group), 20)):
        assert G.offs[-1] == nrows * c                # sum |L| = rows * c
        for j in range(c):
            lo, hi = G.trial_goffs[j], G.trial_goffs[j + 1]
            keys = [oracle.mix64(int(x)) for x in G.ids[lo:hi]]
            assert keys == sorted(keys) and len(set(keys)) == len(keys)
            assert G.offs[hi] - G.offs[lo] == nrows
        for k in range(len(G.ids)):
            m = G.members[G.offs[k]:G.offs[k + 1]]
            assert len(m) >= 1 and np.all(np.diff(m.astype(np.int64)) > 0)


# ---------------------------------------------------------------- (vii) CC-locality
def test_cc_locality():
    g = SG.make("tiny")
    comp = _components(g)
    roots = np.unique(comp[g.degrees() > 0])
    part = np.isin(comp, roots[::2])            # half of the components
    runs = []
    for keep in (part, ~part):
        rp = np.zeros(g.n + 1, np.int64)
        d = np.where(keep, g.degrees(), 0)
        rp[1:] = np.cumsum(d)
        col = np.concatenate([g.col[g.row_ptr[u]:g.row_ptr[u + 1]] for u in range(g.n) if keep[u]])
        runs.append(oracle.shingling(rp, col, 2, 30, 9, 2, 30, 10))
    full = oracle.shingling(g.row_ptr, g.col, 2, 30, 9, 2, 30, 10)
    # pass-1 shingles of each vertex depend only on its own component
    rowmap = {int(u): i for i, u in enumerate(full.rows1)}
    for r in runs:
        for i, u in enumerate(r.rows1.tolist()):
            assert np.array_equal(r.M1[i], full.M1[rowmap[u]])
    # first-level groups of the union = union of the parts' groups (per trial)
    for j in range(30):
        def gs(res):
            lo, hi = res.G1.trial_goffs[j], res.G1.trial_goffs[j + 1]
            return {(int(res.G1.ids[k]), tuple(res.G1.members[res.G1.offs[k]:res.G1.offs[k + 1]].tolist()))
                    for k in range(lo, hi)}
        assert gs(full) == gs(runs[0]) | gs(runs[1])
    # final clusters of the union = union of the parts' clusters
    lf, _ = full.report()
    for r, keep in zip(runs, (part, ~part)):
        lr, _ = r.report()
        assert np.array_equal(lf[keep], lr[keep])


# ---------------------------------------------------------------- (viii)+(ix) N-version
@pytest.mark.parametrize("s1,c1,s2,c2,gseed", [(2, 6, 2, 5, 1), (1, 5, 1, 4, 2), (3, 6, 2, 4, 3),
                                             (2, 9, 3, 5, 4), (5, 4, 2, 6, 5)])
def test_oracle_equals_python_twin(s1, c1, s2, c2, gseed):
    # a small graph with dense pockets so that groups of size >= s2 exist
    g = SG.homology_graph(n=300, n_isolated=20, m_target=2500, seed=gseed, n_cliques=3,
                          clique_lo=6, clique_hi=12, cc_max=120, fam_hi=40)
    g = SG.Graph(*g)
    res = oracle.shingling(g.row_ptr, g.col, s1, c1, 100 + gseed, s2, c2, 200 + gseed)
    tw = twin.shingling(SG.to_adj(g), s1, c1, 100 + gseed, s2, c2, 200 + gseed)
    assert res.rows1.tolist() == tw["rows1"]
    assert res.M1.tolist() == tw["M1"]

    def flat(G, c):
        out = []
        for j in range(c):
            for k in range(G.trial_goffs[j], G.trial_goffs[j + 1]):
                out.append((j, int(G.ids[k]), G.members[G.offs[k]:G.offs[k + 1]].tolist()))
        return out

    assert flat(res.G1, c1) == tw["G1"]
    assert res.s1p_group.tolist() == tw["s1p"]
    assert res.M2.tolist() == tw["M2"]
    assert flat(res.G2, c2) == tw["G2"]
    for mode in (0, 1):
        for ms in (1, 3):
            lab, nc = res.report(mode=mode, min_size=ms)
            tl, tn = twin.report(tw, mode=mode, min_size=ms)
            assert lab.tolist() == tl and nc == tn


def test_report_labels_are_min_of_class():
    g = SG.make("tiny")
    res = oracle.shingling(g.row_ptr, g.col, 2, 30, 1, 2, 30, 2)
    lab, nc = res.report()
    classes = defaultdict(list)
    for v, l in enumerate(lab.tolist()):
        classes[l].append(v)
    assert all(min(vs) == l for l, vs in classes.items())
    assert nc == sum(1 for vs in classes.values() if len(vs) >= 2)


# ---------------------------------------------------------------- Phase III approach 1
@pytest.mark.parametrize("mode", [0, 1])
def test_overlapping_planted_cliques_exact(mode):
    """Disjoint planted cliques: approach 1 reports exactly the cliques."""
    sizes = [5, 6, 8, 10, 12, 15, 20, 25, 30, 9, 7, 11]
    g = SG.cliques(sizes, n=sum(sizes) + 40, seed=17)
    res = oracle.shingling(g.row_ptr, g.col, 2, 100, 21, 2, 100, 22)
    offs, verts = oracle.report_overlapping(res, g.row_ptr, g.col, mode)
    got = sorted(tuple(verts[offs[i]:offs[i + 1]].tolist()) for i in range(len(offs) - 1))
    deg = g.degrees()
    comp = _components(g)
    by_comp = defaultdict(list)
    for v in range(g.n):
        if deg[v] > 0:
            by_comp[comp[v]].append(v)
    assert got == sorted(tuple(sorted(x)) for x in by_comp.values())


@pytest.mark.parametrize("s1,gseed", [(1, 6), (2, 7), (2, 8)])
def test_overlapping_equals_decoded_bfs(s1, gseed):
    """Brute force: constituents decoded algebraically from the exact ids
    (v = (h - B_j) A_j^(P-2) mod P, s <= 2, AMB-4), components by a plain BFS
    over G_II groups (every group joins all its members)."""
    g = SG.Graph(*SG.homology_graph(n=300, n_isolated=20, m_target=2500, seed=gseed, n_cliques=3,
                                    clique_lo=6, clique_hi=12, cc_max=120, fam_hi=40))
    res = oracle.shingling(g.row_ptr, g.col, s1, 12, 100 + gseed, 2, 8, 200 + gseed)
    nk = len(res.s1p_group)
    assert nk > 0
    adj = defaultdict(set)
    G2 = res.G2
    for gi in range(len(G2.ids)):
        K = G2.members[G2.offs[gi]:G2.offs[gi + 1]].tolist()
        for x in K:
            adj[x].update(K)
    tg1 = res.G1.trial_goffs.tolist()

    def decode(gi):
        j = max(t for t in range(len(tg1) - 1) if tg1[t] <= gi)
        idv = int(res.G1.ids[gi])
        hs = [idv] if s1 == 1 else [idv >> 31, idv & P]
        A, B = int(res.A1[j]), int(res.B1[j])
        return {((h - B) * pow(A, P - 2, P)) % P for h in hs}

    seen = [False] * nk
    want = []
    for k0 in range(nk):
        if seen[k0]:
            continue
        seen[k0] = True
        stack, S = [k0], set()
        while stack:
            k = stack.pop()
            S |= decode(int(res.s1p_group[k]))
            for y in adj[k]:
                if not seen[y]:
                    seen[y] = True
                    stack.append(y)
        want.append(sorted(S))
    for ms in (1, 4):
        offs, verts = oracle.report_overlapping(res, g.row_ptr, g.col, 0, ms)
        got = [verts[offs[i]:offs[i + 1]].tolist() for i in range(len(offs) - 1)]
        assert got == [w for w in want if len(w) >= ms]


def test_overlapping_inside_union_find_clusters():
    """Each approach-1 cluster lies inside one approach-2 cluster (approach 2
    unions a superset of the same constituents)."""
    g = SG.Graph(*SG.homology_graph(n=300, n_isolated=20, m_target=2500, seed=9, n_cliques=3,
                                    clique_lo=6, clique_hi=12, cc_max=120, fam_hi=40))
    res = oracle.shingling(g.row_ptr, g.col, 2, 16, 109, 2, 12, 209)
    labels, _ = res.report(mode=0)
    offs, verts = oracle.report_overlapping(res, g.row_ptr, g.col, 0)
    assert len(offs) > 1
    for i in range(len(offs) - 1):
        assert len(set(labels[verts[offs[i]:offs[i + 1]]].tolist())) == 1


# ---------------------------------------------------------------- density (Eq. 6)
def test_density_closed_forms():
    """Cliques have density 1; a k-cycle has k / C(k, 2) = 2 / (k - 1); a
    star on k vertices has (k - 1) / C(k, 2) = 2 / k; singletons are skipped."""
    g = SG.cliques([5, 7, 9], n=30, seed=2)
    lab = np.arange(g.n)
    comp = _components(g)
    for v in range(g.n):
        lab[v] = comp[v]
    mean, sd, nc = oracle.cluster_density(g.row_ptr, g.col, lab)
    assert (mean, sd, nc) == (1.0, 0.0, 3)
    # cycle 0-1-...-9 and a star centred at 10 with leaves 11..15, as one CSR
    adj = {v: set() for v in range(16)}
    for i in range(10):
        adj[i].add((i + 1) % 10)
        adj[(i + 1) % 10].add(i)
    for leaf in range(11, 16):
        adj[10].add(leaf)
        adj[leaf].add(10)
    rp = np.zeros(17, np.int64)
    for v in range(16):
        rp[v + 1] = rp[v] + len(adj[v])
    col = np.concatenate([sorted(adj[v]) for v in range(16)]).astype(np.int32)
    lab = np.array([0] * 10 + [10] * 6)
    mean, sd, nc = oracle.cluster_density(rp, col, lab)
    want = [2 / 9, 2 / 6]
    assert nc == 2 and math.isclose(mean, np.mean(want)) and math.isclose(sd, np.std(want))
    # splitting the cycle in halves: each half is a path of 5 (4 edges / 10)
    lab2 = np.array([0] * 5 + [5] * 5 + [10] * 6)
    mean, _, nc = oracle.cluster_density(rp, col, lab2, min_size=6)
    assert nc == 1 and math.isclose(mean, 2 / 6)
    mean, _, nc = oracle.cluster_density(rp, col, lab2)
    assert nc == 3 and math.isclose(mean, (0.4 + 0.4 + 2 / 6) / 3)
    # a self-loop is not an edge between two vertices of the cluster (AMB-21):
    # the 2-vertex cluster {0, 1} with one edge and two self-loops has density 1
    rp3 = np.array([0, 2, 4], np.int64)
    col3 = np.array([0, 1, 0, 1], np.int32)
    mean, _, nc = oracle.cluster_density(rp3, col3, np.array([0, 0]))
    assert nc == 1 and mean == 1.0
    # a one-directional entry counts half an edge: {0, 1, 2}, entries 0->1, 1->0, 1->2
    rp4 = np.array([0, 1, 3, 3], np.int64)
    col4 = np.array([1, 0, 2], np.int32)
    mean, _, _ = oracle.cluster_density(rp4, col4, np.array([0, 0, 0]))
    assert math.isclose(mean, 1.5 / 3)


# ---------------------------------------------------------------- Eq. 2-5 pair counts
def test_agreement_closed_forms():
    """Identical partitions: FP = FN = 0, PPV = SE = 1; all-singletons test
    vs one block of n: TP = 0, FN = C(n, 2); counts always sum to C(n, 2);
    a hand-counted 5-vertex case; symmetric under swapping the roles (FP <-> FN)."""
    rng = np.random.default_rng(3)
    lab = rng.integers(0, 7, 60)
    r = oracle.partition_agreement(lab, lab)
    assert r["FP"] == r["FN"] == 0 and r["PPV"] == r["SE"] == 1.0
    n = 40
    r = oracle.partition_agreement(np.arange(n), np.zeros(n, int))
    assert r["TP"] == 0 and r["FN"] == n * (n - 1) // 2 and r["FP"] == r["TN"] == 0
    # test {0,1,2}{3,4}; benchmark {0,1}{2,3,4}: pairs 01 TP; 02,12 FP; 23,24 FN; 34 TP; rest TN (4)
    r = oracle.partition_agreement([0, 0, 0, 3, 3], [0, 0, 2, 2, 2])
    assert (r["TP"], r["FP"], r["FN"], r["TN"]) == (2, 2, 2, 4)
    a, b = rng.integers(0, 5, 50), rng.integers(0, 9, 50)
    r, q = oracle.partition_agreement(a, b), oracle.partition_agreement(b, a)
    assert (r["TP"], r["FP"], r["FN"], r["TN"]) == (q["TP"], q["FN"], q["FP"], q["TN"])
    assert r["TP"] + r["FP"] + r["FN"] + r["TN"] == 50 * 49 // 2


# ---------------------------------------------------------------- connected components
def test_components_vs_bfs():
    """scipy-based components = a plain BFS (this file's _components), on the
    homology generator's graphs and on cliques; labels are the minimum vertex."""
    for gseed in (1, 2):
        g = SG.Graph(*SG.homology_graph(n=400, n_isolated=30, m_target=2500, seed=gseed,
                                        n_cliques=3, clique_lo=6, clique_hi=12, cc_max=60,
                                        fam_hi=40))
        lab, k = oracle.connected_components(g.row_ptr, g.col)
        comp = _components(g)
        by = defaultdict(list)
        for v in range(g.n):
            by[comp[v]].append(v)
        assert k == len(by)
        for members in by.values():
            assert set(lab[members].tolist()) == {min(members)}
    # an asymmetric CSR (edge 0 -> 3 stored once) still joins 0 and 3
    lab, k = oracle.connected_components(np.array([0, 1, 1, 1, 1]), np.array([3], np.int32))
    assert lab.tolist() == [0, 1, 2, 0] and k == 3


@pytest.mark.parametrize("s1,c1,s2,c2,keep1,keep2", [
    (2, 20, 2, 17, [0, 5, 19], [0, 3, 16]),
    (3, 9, 2, 7, [8], [0, 6]),
    (1, 6, 3, 5, [], [2]),
])
def test_trial_outer_stream_equals_full_run(s1, c1, s2, c2, keep1, keep2):
    """The trial-outer streaming run (the large-config parity oracle) equals the
    full run's corresponding trials element by element, and its per-trial
    digests equal the digests of the full run's arrays (grouping is per trial,
    P:L404-407, AMB-5; loop order does not change outputs)."""
    import digests as D
    g = SG.make("tiny")
    args = (s1, c1, 101, s2, c2, 102)
    ref = oracle.shingling(g.row_ptr, g.col, *args)
    st = oracle.shingling_stream(g.row_ptr, g.col, *args, keep1=keep1, keep2=keep2)
    assert st.counts == dict(n_e=len(ref.rows1), groups1=len(ref.G1.ids), pairs1=len(ref.G1.members),
                             s1p=len(ref.s1p_group),
                             entries2=int(np.diff(ref.G1.offs)[ref.s1p_group].sum()))
    assert np.array_equal(st.rows1, ref.rows1)
    assert np.array_equal(st.s1p_group, ref.s1p_group)
    assert np.array_equal(st.M1k, ref.M1[:, st.keep1])
    assert np.array_equal(st.M2k, ref.M2[:, st.keep2])
    assert [int(x) for x in st.dig_M1] == [D.column(ref.M1[:, j]) for j in range(c1)]
    assert [int(x) for x in st.dig_G1] == D.grouped_trials(ref.G1.trial_goffs, ref.G1.ids, ref.G1.offs,
                                                           ref.G1.members)
    d2 = D.grouped_trials(ref.G2.trial_goffs, ref.G2.ids, ref.G2.offs, ref.G2.members)
    assert [int(x) for x in st.dig_G2k] == [d2[t] for t in st.keep2]
    for G, Gk, keep in ((ref.G1, st.G1k, st.keep1), (ref.G2, st.G2k, st.keep2)):
        for i, j in enumerate(keep):
            a, b = G.trial_goffs[j], G.trial_goffs[j + 1]
            a2, b2 = Gk.trial_goffs[i], Gk.trial_goffs[i + 1]
            assert np.array_equal(G.ids[a:b], Gk.ids[a2:b2])
            assert np.array_equal(np.diff(G.offs[a:b + 1]), np.diff(Gk.offs[a2:b2 + 1]))
            assert np.array_equal(G.members[G.offs[a]:G.offs[b]], Gk.members[Gk.offs[a2]:Gk.offs[b2]])


def test_digest_detects_a_moved_member():
    """The digests are position-sensitive: swapping two members, moving a group
    boundary, or changing one id changes the digest."""
    import digests as D
    ids = np.array([5, 9, 2], np.uint64)
    offs = np.array([0, 2, 3, 5], np.int64)
    mem = np.array([1, 4, 3, 0, 7], np.uint32)
    d = D.grouped_trial(ids, offs, mem)
    assert d != D.grouped_trial(ids, offs, mem[[1, 0, 2, 3, 4]])
    assert d != D.grouped_trial(ids, np.array([0, 1, 3, 5], np.int64), mem)
    assert d != D.grouped_trial(np.array([5, 9, 3], np.uint64), offs, mem)
    assert D.column(np.array([1, 2], np.uint64)) != D.column(np.array([2, 1], np.uint64))
