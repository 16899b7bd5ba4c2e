"""Order- and position-sensitive 64-bit digests of pass matrices and grouped
trials (test infrastructure; the same definition as oracle.c's trial-outer
run, restated here in numpy so GPU outputs can be digested the same way):

  column x_0..x_{N-1}:       sum_i mix64(x_i + mix64(i))                (mod 2^64)
  grouped trial (ids, members, head bits):
        sum_g mix64(id_g + mix64(2g)) + sum_p mix64((m_p | h_p << 32) + mix64(2p + 1))
"""
import numpy as np

_M1 = np.uint64(0xbf58476d1ce4e5b9)
_M2 = np.uint64(0x94d049bb133111eb)


def mix64(z):
    """splitmix64 finaliser on a uint64 array (wrapping arithmetic)."""
    z = np.asarray(z, np.uint64).copy()
    with np.errstate(over="ignore"):
        z ^= z >> np.uint64(30)
        z *= _M1
        z ^= z >> np.uint64(27)
        z *= _M2
        z ^= z >> np.uint64(31)
    return z


def _sum(x):
    with np.errstate(over="ignore"):
        return int(np.sum(x, dtype=np.uint64))


def column(x, chunk=1 << 24):
    x = np.asarray(x, np.uint64)
    tot = 0
    for a in range(0, len(x), chunk):
        i = np.arange(a, min(a + chunk, len(x)), dtype=np.uint64)
        with np.errstate(over="ignore"):
            tot += _sum(mix64(x[a:a + chunk] + mix64(i)))
    return tot % (1 << 64)


def grouped_trial(ids, offs, members, chunk=1 << 24):
    """One trial: ids[G], offs[G+1] (offs[0] may be nonzero), members[offs[0]:offs[G]]."""
    ids = np.asarray(ids, np.uint64)
    offs = np.asarray(offs, np.int64)
    G = len(ids)
    g = np.arange(G, dtype=np.uint64)
    with np.errstate(over="ignore"):
        tot = _sum(mix64(ids + mix64(np.uint64(2) * g)))
    p0, p1 = int(offs[0]), int(offs[-1])
    head = np.zeros(p1 - p0, bool)
    head[offs[:-1][offs[:-1] < p1] - p0] = True
    m = np.asarray(members[p0:p1], np.uint64) | (head.astype(np.uint64) << np.uint64(32))
    for a in range(0, len(m), chunk):
        p = np.arange(a, min(a + chunk, len(m)), dtype=np.uint64)
        with np.errstate(over="ignore"):
            tot += _sum(mix64(m[a:a + chunk] + mix64(np.uint64(2) * p + np.uint64(1))))
    return tot % (1 << 64)


def grouped_trials(trial_goffs, ids, offs, members):
    """Digest of every trial of a grouped level -> list of ints."""
    out = []
    for j in range(len(trial_goffs) - 1):
        a, b = int(trial_goffs[j]), int(trial_goffs[j + 1])
        out.append(grouped_trial(ids[a:b], offs[a:b + 1], members))
    return out
