"""C-ABI library checks that need no GPU (-m "not gpu"): it loads, exports every
symbol include/shingle.h declares, its pure-host helpers work, and without a
CUDA device it fails loudly instead of falling back to the CPU."""
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "shingle.h")


@pytest.fixture(scope="module")
def B():
    from paper_conf_ipps_wuk13_b200 import binding
    if not os.path.exists(binding.LIB_PATH):
        import __graft_entry__
        __graft_entry__.build()
    binding.lib()
    return binding


def _declared():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"^SG_API[^(]*?\b(\w+)\(", txt, re.M)))


def test_header_declares_the_four_paper_calls():
    names = _declared()
    for f in ["shingle_graph_create", "shingle_pass", "group_by_shingle", "report_dense_subgraphs"]:
        assert f in names


def test_library_exports_every_declared_symbol(B):
    import subprocess
    out = subprocess.check_output(["nm", "-D", "--defined-only", B.LIB_PATH], text=True)
    exported = {ln.split()[-1] for ln in out.splitlines() if " T " in ln}
    missing = [n for n in _declared() if n not in exported]
    assert not missing, missing
    for n in _declared():
        assert hasattr(B.lib(), n)


def test_library_is_built_for_sm100a(B):
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", B.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version(B):
    assert "sm_100a" in B.sg_version()


def test_partition_rows_balances_degree_plus_kappa(B):
    from synth import graphs as SG
    g = SG.make("tiny")
    for world in (1, 2, 3, 8):
        b = B.sg_partition_rows(g.row_ptr, world, 8)
        assert b[0] == 0 and b[-1] == g.n and np.all(np.diff(b) >= 0)
        w = g.row_ptr[b[1:]] - g.row_ptr[b[:-1]] + 8 * np.diff(b)
        tot = g.nnz + 8 * g.n
        # each cut is the first row reaching r/world of the weight
        assert w.max() <= tot / world + g.degrees().max() + 8
        for r in range(1, world):
            u = b[r]
            assert g.row_ptr[u] + 8 * u >= tot * r / world - 1e-6
            if u > 0:
                assert g.row_ptr[u - 1] + 8 * (u - 1) < tot * r / world


def test_null_handle_and_bad_args(B):
    import ctypes as C
    L = B.lib()
    assert L.shingle_pass(None, 2, 10, 1) == B.SG_EINVAL
    assert L.group_by_shingle(None) == B.SG_EINVAL
    assert L.shingle_graph_create(-1, 0, None, None, 0, None, C.byref(C.c_void_p())) == B.SG_EINVAL
    assert L.shingle_graph_create(0, 0, None, None, 0, None, None) == B.SG_EINVAL


def test_no_cpu_fallback_without_gpu(B):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    from synth import graphs as SG
    g = SG.random_graph(100, 300, seed=1)
    with pytest.raises(B.SGError) as e:
        B.shingle_graph_create(g.row_ptr, g.col)
    assert e.value.status == B.SG_ECUDA
