"""Component sharding (pClust's decomposition P:L162-169):
whole connected components per shard, the shard's CSR over all vertex ids,
and the merge of per-shard labels.  The CPU tests check the host functions
of libshingle and, with the ORACLE on each shard, that the merged labels equal
the whole-graph labels (CC-locality); the GPU test runs the library per shard."""
import numpy as np
import pytest

import oracle
from synth import graphs as SG


@pytest.fixture(scope="module")
def B():
    from paper_conf_ipps_wuk13_b200 import binding
    binding.lib()
    return binding


def _graph():
    g = SG.make("tiny")
    # plus a few isolated vertices and a separate clique block
    return g


def test_components_stay_whole_and_balanced(B):
    g = _graph()
    for world in (1, 2, 3, 7):
        shard, load = B.sg_component_shards(g.row_ptr, g.col, world)
        assert shard.min() >= 0 and shard.max() < world
        src = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
        assert np.array_equal(shard[src], shard[g.col]), "a component was split"
        w = np.diff(g.row_ptr) + 8
        assert load.sum() == w.sum()
        for r in range(world):
            assert load[r] == w[shard == r].sum()
        comp, _ = oracle.connected_components(g.row_ptr, g.col)
        heaviest = max(w[comp == c].sum() for c in np.unique(comp))
        assert load.max() <= w.sum() / world + heaviest


def test_shard_csr_keeps_its_rows_only(B):
    g = _graph()
    shard, _ = B.sg_component_shards(g.row_ptr, g.col, 3)
    tot = 0
    for r in range(3):
        rp, col = B.sg_shard_csr(g.row_ptr, g.col, shard, r)
        assert len(rp) == g.n + 1 and rp[-1] == len(col)
        deg = np.diff(rp)
        assert np.all(deg[shard != r] == 0)
        assert np.array_equal(deg[shard == r], np.diff(g.row_ptr)[shard == r])
        assert oracle.validate(rp, col)
        tot += len(col)
    assert tot == g.nnz


@pytest.mark.parametrize("mode", [0, 1])
def test_oracle_on_shards_merges_to_the_whole_graph(B, mode):
    """CC-locality end to end: the oracle on each shard, labels merged by
    sg_merge_shard_labels, equals the oracle on the whole graph."""
    g = _graph()
    args = (2, 24, 101, 2, 20, 102)
    want, nwant = oracle.shingling(g.row_ptr, g.col, *args).report(mode, 1)
    world = 3
    shard, _ = B.sg_component_shards(g.row_ptr, g.col, world)
    labs = []
    for r in range(world):
        rp, col = B.sg_shard_csr(g.row_ptr, g.col, shard, r)
        labs.append(oracle.shingling(rp, col, *args).report(mode, 1)[0])
    merged = B.sg_merge_shard_labels(shard, np.stack(labs))
    assert np.array_equal(merged, want)


@pytest.mark.gpu
def test_library_on_shards_merges_to_the_whole_graph(B):
    import torch
    torch.cuda.init()
    g = _graph()
    args = (2, 40, 101, 2, 33, 102)
    want, _ = oracle.shingling(g.row_ptr, g.col, *args).report(0, 1)
    world = 3
    shard, _ = B.sg_component_shards(g.row_ptr, g.col, world)
    labs = []
    h = None
    try:
        for r in range(world):
            rp, col = B.sg_shard_csr(g.row_ptr, g.col, shard, r)
            if h is None:
                h = B.shingle_graph_create(rp, col)
            else:
                B.shingle_graph_load(h, rp, col)            # one handle, one graph per shard
            B.shingle_pass(h, *args[:3])
            B.group_by_shingle(h)
            B.shingle_pass(h, *args[3:])
            B.group_by_shingle(h)
            labs.append(B.report_dense_subgraphs(h, 0, 1, g.n)[0])
    finally:
        if h is not None:
            B.shingle_graph_destroy(h)
    assert np.array_equal(B.sg_merge_shard_labels(shard, np.stack(labs)), want)
