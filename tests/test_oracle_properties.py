"""Property tests (hypothesis, SURVEY §4 tier 6) of the CPU oracle on random
small graphs: the C oracle equals the independent pure-Python twin (big
integers, full sorts, dict grouping, BFS report) on every output, the
trial-outer run equals the full run, and the grouping invariants hold."""
import numpy as np
import pytest
from hypothesis import HealthCheck, given, settings
from hypothesis import strategies as st

import oracle
from oracle import twin
from synth import graphs as SG


@st.composite
def small_graph(draw):
    n = draw(st.integers(1, 24))
    k = draw(st.integers(0, 80))
    a = draw(st.lists(st.integers(0, n - 1), min_size=k, max_size=k))
    b = draw(st.lists(st.integers(0, n - 1), min_size=k, max_size=k))
    rp, col = SG._csr_from_pairs(n, np.asarray(a, np.int64), np.asarray(b, np.int64))
    return SG.Graph(rp, col)


params = st.tuples(st.integers(1, 3), st.integers(1, 7), st.integers(0, 2**63 - 1),
                   st.integers(1, 3), st.integers(1, 7), st.integers(0, 2**63 - 1))


def _flat(G, c):
    out = []
    for j in range(c):
        for k in range(G.trial_goffs[j], G.trial_goffs[j + 1]):
            out.append((j, int(G.ids[k]), G.members[G.offs[k]:G.offs[k + 1]].tolist()))
    return out


@settings(max_examples=60, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(small_graph(), params)
def test_oracle_equals_twin_on_random_graphs(g, p):
    s1, c1, seed1, s2, c2, seed2 = p
    res = oracle.shingling(g.row_ptr, g.col, s1, c1, seed1, s2, c2, seed2)
    tw = twin.shingling(SG.to_adj(g), s1, c1, seed1, s2, c2, seed2)
    assert res.rows1.tolist() == tw["rows1"]
    assert res.M1.tolist() == tw["M1"]
    assert _flat(res.G1, c1) == tw["G1"]
    assert res.s1p_group.tolist() == tw["s1p"]
    assert res.M2.tolist() == tw["M2"]
    assert _flat(res.G2, c2) == tw["G2"]
    for mode in (0, 1):
        lab, nc = res.report(mode=mode, min_size=1)
        tl, tn = twin.report(tw, mode=mode, min_size=1)
        assert lab.tolist() == tl and nc == tn


@settings(max_examples=60, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(small_graph(), params)
def test_grouping_invariants_and_trial_outer_run(g, p):
    s1, c1, seed1, s2, c2, seed2 = p
    res = oracle.shingling(g.row_ptr, g.col, s1, c1, seed1, s2, c2, seed2)
    n_e = len(res.rows1)
    # every pass-I row in every trial exactly once; keys strictly ascending per
    # trial; members strictly ascending per group; S1' = groups with |L| >= s2
    assert len(res.G1.members) == n_e * c1
    sizes = np.diff(res.G1.offs)
    for j in range(c1):
        a, b = res.G1.trial_goffs[j], res.G1.trial_goffs[j + 1]
        keys = [oracle.mix64(int(x)) for x in res.G1.ids[a:b]]
        assert keys == sorted(keys) and len(set(keys)) == len(keys)
        assert sorted(res.G1.members[res.G1.offs[a]:res.G1.offs[b]].tolist()) == res.rows1.tolist()
    for k in range(len(sizes)):
        L = res.G1.members[res.G1.offs[k]:res.G1.offs[k + 1]]
        assert np.all(np.diff(L.astype(np.int64)) > 0)
    assert res.s1p_group.tolist() == np.flatnonzero(sizes >= s2).tolist()
    keep1 = list(range(0, c1, 2))
    keep2 = list(range(1, c2, 2))
    stv = oracle.shingling_stream(g.row_ptr, g.col, s1, c1, seed1, s2, c2, seed2, keep1=keep1, keep2=keep2)
    assert np.array_equal(stv.rows1, res.rows1) and np.array_equal(stv.s1p_group, res.s1p_group)
    assert np.array_equal(stv.M1k, res.M1[:, stv.keep1]) and np.array_equal(stv.M2k, res.M2[:, stv.keep2])
