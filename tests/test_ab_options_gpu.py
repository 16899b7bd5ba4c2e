"""The A/B options kept in the library (each measured slower or kept for
comparison) must produce the same outputs as the oracle: one
subprocess per option (the options are read once per process), on the small
homology-shaped config with a small bucket target so the two-level partition,
the fine split, the warp tier and the CTA tier all run; outputs compared by
SHA-256 digests of every array."""
import hashlib
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
from synth import graphs as SG

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HELPER = os.path.join(ROOT, "tests", "helpers", "ab_run.py")

OPTIONS = [
    {"SG_MH_WIN": "1"},                       # windowed row-per-lane pass-II kernel
    {"SG_FBIN": "1"},                         # fine-digit bytes for the fine split
    {"SG_LOCAL_CTA_ATOMIC": "1"},             # CTA tier: atomic placements
    {"SG_LOCAL_ATOMIC": "0", "SG_SPLIT_FINE": "0"},   # match-based, key-only-verified warp tier
    {"SG_SPLIT_FINE": "2"}, {"SG_SPLIT_FINE": "3"},
    {"SG_SPLIT_COARSE": "1"}, {"SG_SPLIT_COARSE": "2"}, {"SG_SPLIT_COARSE": "3"},
    {"SG_NO_KBIN": "1"},                      # coarse histogram on the 8-B keys
    {"SG_NO_CACHE": "1"},                     # no handle-level block cache
]


def digest(*arrays):
    h = hashlib.sha256()
    for a in arrays:
        h.update(np.ascontiguousarray(a).tobytes())
    return h.hexdigest()


@pytest.fixture(scope="module")
def expected():
    g = SG.make("small")
    cfg = SG.CONFIGS["small"]
    args = (cfg["s1"], cfg["c1"], cfg["seed1"], cfg["s2"], cfg["c2"], cfg["seed2"])
    ref = oracle.shingling(g.row_ptr, g.col, *args)
    def grp(G):
        return (np.asarray(G.trial_goffs, np.int64), np.asarray(G.ids, np.uint64),
                np.asarray(G.offs, np.int64), np.asarray(G.members, np.uint32))
    want = {"M1": digest(np.asarray(ref.M1, np.uint64), np.asarray(ref.rows1, np.uint32)),
            "M2": digest(np.asarray(ref.M2, np.uint64)),
            "G1": digest(*grp(ref.G1)), "G2": digest(*grp(ref.G2)),
            "s1p": digest(np.asarray(ref.s1p_group, np.int64))}
    return args, want


@pytest.mark.timeout(900)
@pytest.mark.parametrize("target", ["300", "2500"])
@pytest.mark.parametrize("opt", OPTIONS, ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()))
def test_ab_option_matches_oracle(expected, opt, target):
    args, want = expected
    env = dict(os.environ, SG_GROUP_TARGET=target, **opt)
    out = subprocess.run([sys.executable, HELPER, "small", *map(str, args)], env=env,
                         capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    got = json.loads(out.stdout.strip().splitlines()[-1])
    assert got == want
