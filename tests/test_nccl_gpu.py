"""The NCCL transport on real hardware with one GPU: a world = 1 handle that
opts into the owner-routed exchange path (SG_DIST_EXCHANGE) builds a one-rank
NCCL communicator (ncclCommInitRank) and routes every pass's pairs through
ncclSend / ncclRecv and its counts through ncclAllGather.  The outputs must
equal the oracle bit for bit; a fresh ncclUniqueId is used per communicator,
and shingle_graph_load re-ingests a graph on the same communicator."""
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


def run_exchange(B, h, g, args):
    B.shingle_pass(h, args[0], args[1], args[2])
    B.group_by_shingle(h)
    B.shingle_pass(h, args[3], args[4], args[5])
    B.group_by_shingle(h)
    return dict(M1=B.sg_get_shingles(h, 1), G1=B.sg_get_groups(h, 1), M2=B.sg_get_shingles(h, 2),
                G2=B.sg_get_groups(h, 2), counts=B.sg_get_counts(h), labels=B.report_dense_subgraphs(h, 0, 1))


def check(out, ref):
    assert np.array_equal(out["M1"][0], ref.M1) and np.array_equal(out["M1"][1], ref.rows1)
    assert np.array_equal(out["M2"][0], ref.M2)
    for got, want in ((out["G1"], ref.G1), (out["G2"], ref.G2)):
        tg, ids, offs, mem = got
        assert np.array_equal(tg, want.trial_goffs) and np.array_equal(offs, want.offs)
        assert np.array_equal(mem, want.members) and np.array_equal(ids, want.ids)
    l0, n0 = out["labels"]
    r0, m0 = ref.report(0)
    assert n0 == m0 and np.array_equal(l0, r0)


@pytest.mark.timeout(600)
def test_nccl_world1_exchange_path(B):
    g = SG.make("tiny")
    args = (2, 37, 101, 2, 33, 102)
    ref = oracle.shingling(g.row_ptr, g.col, *args)
    for rep in range(2):                     # two communicators in a row, a fresh uid each
        uid = B.nccl_unique_id()
        h = B.shingle_graph_create(g.row_ptr, g.col,
                                   dist=dict(rank=0, world=1, device=0, nccl_uid=uid, exchange=True))
        try:
            out = run_exchange(B, h, g, args)
            check(out, ref)
            assert out["counts"]["world"] == 1 and out["counts"]["exchange"] == 1
            # a second graph on the same handle and communicator
            g2 = SG.cliques([40, 25, 12], n=200, seed=rep)
            B.shingle_graph_load(h, g2.row_ptr, g2.col)
            ref2 = oracle.shingling(g2.row_ptr, g2.col, *args)
            check(run_exchange(B, h, g2, args), ref2)
        finally:
            B.shingle_graph_destroy(h)


@pytest.mark.timeout(600)
def test_nccl_world1_fused_peer_exchange(B):
    """SG_DIST_PEER on a one-rank NCCL communicator: the receive buffers are
    published over the communicator (ncclAllGather), the owner-partition
    kernel stores into them, the barriers are NCCL all-gathers."""
    g = SG.make("tiny")
    args = (2, 37, 101, 2, 33, 102)
    ref = oracle.shingling(g.row_ptr, g.col, *args)
    uid = B.nccl_unique_id()
    h = B.shingle_graph_create(g.row_ptr, g.col,
                               dist=dict(rank=0, world=1, device=0, nccl_uid=uid, exchange=True, peer=True))
    try:
        check(run_exchange(B, h, g, args), ref)
    finally:
        B.shingle_graph_destroy(h)


def test_load_replaces_the_graph_and_rejects_bad_csr(B):
    g = SG.make("tiny")
    args = (2, 9, 101, 2, 7, 102)
    h = B.shingle_graph_create(g.row_ptr, g.col)
    try:
        g2 = SG.random_graph(3000, 20000, seed=5)
        B.shingle_graph_load(h, g2.row_ptr, g2.col)
        out = run_exchange(B, h, g2, args)
        check(out, oracle.shingling(g2.row_ptr, g2.col, *args))
        bad = g2.col.copy()
        bad[1], bad[0] = bad[0], bad[1]          # row 0 no longer strictly increasing
        with pytest.raises(B.SGError) as ei:
            B.shingle_graph_load(h, g2.row_ptr, bad)
        assert ei.value.status == B.SG_EINVAL
        with pytest.raises(B.SGError) as ei:      # no graph resident after a failed load
            B.shingle_pass(h, 2, 9, 101)
        assert ei.value.status == B.SG_ESTATE
        B.shingle_graph_load(h, g.row_ptr, g.col)
        out = run_exchange(B, h, g, args)
        check(out, oracle.shingling(g.row_ptr, g.col, *args))
    finally:
        B.shingle_graph_destroy(h)
