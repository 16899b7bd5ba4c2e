"""Seeded synthetic homology-like graphs (CSR) for tests and the bench.

This module is the ONE piece both the oracle side and the CUDA side use, and
it holds none of the method's arithmetic: no hashing, no min-hash, no
grouping — only graph construction.  Recipe:

* a fraction of vertices are singletons (the 2M graph has 437,016 of
  2,000,000, i.e. 1,562,984 non-singleton vertices, Table II);
* optional planted disjoint cliques, each its own connected component
  (config 1, BASELINE.json configs[0]);
* the remaining vertices are cut into connected components with power-law
  sizes (cap = the largest CC of Table II, 10,707), each made of
  "protein families": dense random subgraphs with power-law sizes and density
  U(0.3, 0.9) (found-cluster density 0.75 +- 0.28), joined by
  sparse random intra-component "linker" edges;
* optional hubs (config 3): vertices wired to U[deg_lo, deg_hi] random
  non-hub vertices;
* vertex ids are a uniformly random permutation (required: the linear hash
  family is far from min-wise on arithmetic progressions);
* the output is simple, symmetric, rows strictly ascending: int64 row_ptr[n+1],
  int32 col[nnz], nnz = 2m (m = undirected edges, AMB-11).
"""
from __future__ import annotations

import os
from dataclasses import dataclass, field

import numpy as np

# graph cache (outside the repo so it never travels with the gpurun snapshot)
_DATA = os.environ.get("SG_DATA_DIR", "/tmp/sg_data")


@dataclass
class Graph:
    row_ptr: np.ndarray   # int64 [n+1]
    col: np.ndarray       # int32 [nnz]
    meta: dict = field(default_factory=dict)

    @property
    def n(self) -> int:
        return len(self.row_ptr) - 1

    @property
    def nnz(self) -> int:
        return len(self.col)

    @property
    def m(self) -> int:
        return self.nnz // 2

    def degrees(self) -> np.ndarray:
        return np.diff(self.row_ptr)


# --------------------------------------------------------------------------- helpers
def _powerlaw_sizes(rng, lo, hi, exponent, total, max_count=None):
    """Draw integer sizes ~ k^-exponent on [lo, hi] until they sum to `total`
    (the last one truncated).  Inverse-CDF sampling of the continuous law."""
    out = []
    acc = 0
    batch = 4096
    a = 1.0 - exponent
    while acc < total:
        u = rng.random(batch)
        if abs(a) < 1e-12:
            k = lo * (hi / lo) ** u
        else:
            k = (lo ** a + u * (hi ** a - lo ** a)) ** (1.0 / a)
        k = np.minimum(np.floor(k).astype(np.int64), hi)
        cs = np.cumsum(k) + acc
        cut = np.searchsorted(cs, total, side="left")
        if cut < batch:
            k = k[:cut + 1].copy()
            k[-1] -= cs[cut] - total
            out.append(k)
            acc = total
        else:
            out.append(k)
            acc = int(cs[-1])
    sizes = np.concatenate(out) if out else np.zeros(0, np.int64)
    return sizes[sizes > 0]


def _pairs_within(rng, base, size, draws):
    """`draws[i]` uniformly random ordered pairs inside block i = [base, base+size)."""
    draws = np.asarray(draws, np.int64)
    tot = int(draws.sum())
    if tot == 0:
        return np.zeros(0, np.int64), np.zeros(0, np.int64)
    blk = np.repeat(np.arange(len(draws)), draws)
    b0 = base[blk]
    sz = size[blk]
    a = b0 + np.floor(rng.random(tot) * sz).astype(np.int64)
    b = b0 + np.floor(rng.random(tot) * sz).astype(np.int64)
    return a, b


def _unique(x, inplace=False):
    """Sorted unique values (sort based; numpy's hash-based unique is slow here).
    inplace=True sorts the caller's array in place (no copy)."""
    if inplace:
        x.sort()
    else:
        x = np.sort(x)
    if len(x) == 0:
        return x
    keep = np.empty(len(x), bool)
    keep[0] = True
    np.not_equal(x[1:], x[:-1], out=keep[1:])
    return x[keep]


_BATCH = 1 << 25


def _codes_within(rng, base, size, draws, n):
    """Sorted unique undirected codes min*n + max of the pairs _pairs_within
    would draw (same random stream: all first endpoints, then all second
    endpoints), generated in batches so that memory stays O(draws) int32 +
    the codes (the 640M-edge config)."""
    draws = np.asarray(draws, np.int64)
    tot = int(draws.sum())
    if tot == 0:
        return np.zeros(0, np.int64)
    cum = np.cumsum(draws)
    a = np.empty(tot, np.int32 if n < 2**31 else np.int64)
    for s0 in range(0, tot, _BATCH):
        e0 = min(tot, s0 + _BATCH)
        blk = np.searchsorted(cum, np.arange(s0, e0, dtype=np.int64), side="right")
        a[s0:e0] = base[blk] + np.floor(rng.random(e0 - s0) * size[blk]).astype(np.int64)
    out = []
    for s0 in range(0, tot, _BATCH):
        e0 = min(tot, s0 + _BATCH)
        blk = np.searchsorted(cum, np.arange(s0, e0, dtype=np.int64), side="right")
        bb = base[blk] + np.floor(rng.random(e0 - s0) * size[blk]).astype(np.int64)
        aa = a[s0:e0].astype(np.int64)
        keep = aa != bb
        aa, bb = aa[keep], bb[keep]
        out.append(np.minimum(aa, bb) * n + np.maximum(aa, bb))
    del a
    codes = np.concatenate(out) if out else np.zeros(0, np.int64)
    del out
    return _unique(codes, inplace=True)


def _csr_from_unique_codes(n, codes, perm):
    """Simple symmetric CSR from sorted unique undirected codes lo*n + hi of
    slots, relabelled by the permutation perm (a bijection, so the pairs stay
    unique and loop-free): directed keys (src << 32 | dst), sorted in place."""
    m = len(codes)
    key = np.empty(2 * m, np.uint64)
    for s0 in range(0, m, _BATCH):
        e0 = min(m, s0 + _BATCH)
        lo = perm[codes[s0:e0] // n].astype(np.uint64)
        hi = perm[codes[s0:e0] % n].astype(np.uint64)
        key[s0:e0] = (lo << np.uint64(32)) | hi
        key[m + s0:m + e0] = (hi << np.uint64(32)) | lo
    key.sort()
    rows = key >> np.uint64(32)
    row_ptr = np.zeros(n + 1, np.int64)
    row_ptr[1:] = np.searchsorted(rows, np.arange(n, dtype=np.uint64), side="right")
    del rows
    col = np.ascontiguousarray(key.view(np.uint32)[0::2]).view(np.int32)
    return row_ptr, col


def _csr_from_pairs(n, a, b):
    """Simple symmetric CSR from undirected pairs (drops self-loops, duplicates)."""
    keep = a != b
    a, b = a[keep], b[keep]
    lo = np.minimum(a, b)
    hi = np.maximum(a, b)
    code = _unique(lo * n + hi)
    lo = code // n
    hi = code % n
    src = np.concatenate([lo, hi])
    dst = np.concatenate([hi, lo])
    del lo, hi, code
    key = src * n + dst
    del src, dst
    key.sort()
    counts = np.bincount(key // n, minlength=n)
    row_ptr = np.zeros(n + 1, np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    col = (key % n).astype(np.int32)
    return row_ptr, col


# --------------------------------------------------------------------------- generator
def homology_graph(n, n_isolated=0, m_target=None, seed=0,
                   n_cliques=0, clique_lo=10, clique_hi=60,
                   cc_exp=2.0, cc_lo=2, cc_max=10707,
                   fam_exp=2.0, fam_lo=4, fam_hi=600, dens_lo=0.3, dens_hi=0.9,
                   linkers=4.0, n_hubs=0, hub_lo=10001, hub_hi=20000, return_families=False):
    rng = np.random.default_rng(seed)
    perm = rng.permutation(n).astype(np.int64)          # slot -> vertex id
    ea, eb = [], []
    slot = n_isolated                                     # slots [0, n_isolated) stay isolated

    # planted cliques: each a CC of its own
    if n_cliques:
        ks = rng.integers(clique_lo, clique_hi + 1, n_cliques)
        for k in ks:
            i, j = np.triu_indices(int(k), 1)
            ea.append(slot + i.astype(np.int64))
            eb.append(slot + j.astype(np.int64))
            slot += int(k)
    rest = n - slot
    first_rest = slot

    # connected components, then families inside each component
    cc = _powerlaw_sizes(rng, cc_lo, cc_max, cc_exp, rest)
    cc_base = first_rest + np.concatenate([[0], np.cumsum(cc)[:-1]]).astype(np.int64)
    # families: one global power-law size sequence over the same slots; a
    # family that straddles a component boundary is cut there
    fs = _powerlaw_sizes(rng, fam_lo, fam_hi, fam_exp, rest)
    cuts = np.union1d(np.cumsum(fs), np.cumsum(cc))
    starts = np.concatenate([[0], cuts[:-1]])
    fam_sizes = (cuts - starts).astype(np.int64)
    fam_base = (first_rest + starts).astype(np.int64)
    dens = rng.uniform(dens_lo, dens_hi, len(fam_sizes))
    dens[fam_sizes <= 3] = 0.95        # keep tiny components connected
    npairs = fam_sizes * (fam_sizes - 1) // 2
    exp_fam_edges = float((dens * npairs).sum())
    exp_link = linkers * rest / 2.0
    if m_target is not None:
        clique_edges = sum(len(x) for x in ea)
        budget = m_target - clique_edges
        if exp_fam_edges > budget:                      # scale densities down
            dens *= budget * 0.9 / exp_fam_edges
            exp_fam_edges = float((dens * npairs).sum())
        exp_link = max(budget - exp_fam_edges, 0.0)
    # sampling with replacement: -ln(1-d) * N draws give density ~ d
    draws = np.round(-np.log1p(-np.minimum(dens, 0.95)) * npairs).astype(np.int64)
    fixed = _codes(n, np.concatenate(ea[:n_cliques]) if n_cliques else np.zeros(0, np.int64),
                   np.concatenate(eb[:n_cliques]) if n_cliques else np.zeros(0, np.int64))
    del ea, eb
    free = _codes_within(rng, fam_base, fam_sizes, draws, n)
    # linkers: random intra-component pairs, proportional to component size,
    # topped up until the undirected edge count reaches m_target (then trimmed)
    big = cc >= 3
    if m_target is None:
        m_target = len(fixed) + len(free) + int(exp_link)
    for _ in range(20):
        deficit = m_target - len(fixed) - len(free)
        if deficit <= 0 or not big.any():
            break
        ld = rng.poisson(2.0 * deficit * cc * big / max(int((cc * big).sum()), 1))
        free = _unique(np.concatenate([free, _codes_within(rng, cc_base, cc, ld, n)]), inplace=True)
    excess = len(fixed) + len(free) - m_target
    if excess > 0:
        free = np.delete(free, rng.choice(len(free), excess, replace=False))
    codes = free if len(fixed) == 0 else _unique(np.concatenate([fixed, free]), inplace=True)
    del free
    # hubs (config 3): added on top of the m_target graph
    if n_hubs:
        non_iso = np.arange(n_isolated, n, dtype=np.int64)
        hubs = rng.choice(non_iso, n_hubs, replace=False)
        is_hub = np.zeros(n, bool)
        is_hub[hubs] = True
        targets = non_iso[~is_hub[non_iso]]
        hd = rng.integers(hub_lo, hub_hi + 1, n_hubs)
        codes = _unique(np.concatenate([codes, _codes(n, np.repeat(hubs, hd),
                                                     targets[rng.integers(0, len(targets), int(hd.sum()))])]))
    row_ptr, col = _csr_from_unique_codes(n, codes, perm)
    del codes
    if not return_families:
        return row_ptr, col
    # planted partition (the "benchmark" of Eq. 2-5): cliques and families;
    # isolated vertices alone.  Label = smallest vertex id of the family.
    fam_of_slot = np.arange(n, dtype=np.int64)
    s0 = n_isolated
    for k in (ks if n_cliques else []):
        fam_of_slot[s0:s0 + int(k)] = s0
        s0 += int(k)
    for base, size in zip(fam_base, fam_sizes):
        fam_of_slot[base:base + size] = base
    fam_min = np.full(n, n, np.int64)
    np.minimum.at(fam_min, fam_of_slot, perm)
    fam = np.empty(n, np.int32)
    fam[perm] = fam_min[fam_of_slot]
    return row_ptr, col, fam


def _codes(n, a, b):
    keep = a != b
    a, b = a[keep], b[keep]
    return _unique(np.minimum(a, b) * n + np.maximum(a, b))


def stats(g: Graph) -> dict:
    d = g.degrees()
    nz = d[d > 0]
    return dict(n=g.n, m=g.m, nnz=g.nnz, non_singleton=int(len(nz)),
                deg_mean=float(nz.mean()) if len(nz) else 0.0,
                deg_std=float(nz.std()) if len(nz) else 0.0,
                deg_max=int(d.max()) if len(d) else 0)


# --------------------------------------------------------------------------- configs
# BASELINE.json "configs"; seeds from SURVEY §8d.
CONFIGS = {
    # configs[0]: 10K vertices, ~200K edges, 50 planted cliques, s1=s2=2, c1=c2=100
    "tiny": dict(gen=dict(n=10_000, n_isolated=0, m_target=200_000, n_cliques=50,
                          clique_lo=10, clique_hi=60, cc_max=2_000, fam_hi=200, linkers=6.0),
                 seed=1, s1=2, c1=100, seed1=101, s2=2, c2=100, seed2=102),
    # configs[1]: GOS-shaped 2M graph (Table II: 1,562,984 non-singleton v, 56,919,738 e)
    "gos2m": dict(gen=dict(n=2_000_000, n_isolated=437_016, m_target=56_919_738, fam_hi=3000),
                  seed=2, s1=2, c1=200, seed1=201, s2=2, c2=200, seed2=202),
    # configs[2]: config 2 + 1% hubs of degree U[10001, 20000]
    "hub2m": dict(gen=dict(n=2_000_000, n_isolated=437_016, m_target=56_919_738, fam_hi=3000,
                           n_hubs=20_000),
                  seed=3, s1=2, c1=200, seed1=301, s2=2, c2=200, seed2=302),
    # configs[3]: Pacific-Ocean-shaped 11M vertices / 640M edges (P:L71-74,
    # P:L1316-1321): the config-2 recipe scaled (same singleton share,
    # family and component size laws); s1=2, c1=200, s2=2, c2=100 (P:L843-845,
    # AMB-20)
    "pacific640m": dict(gen=dict(n=11_000_000, n_isolated=2_403_588, m_target=640_000_000, fam_hi=3000),
                        seed=4, s1=2, c1=200, seed1=401, s2=2, c2=100, seed2=402),
    # configs[4] sweep points at full size (the gos2m graph, other (s, c)):
    # the extremes checked bit-exactly by oracle digests
    "gos2m_c400": dict(gen=dict(n=2_000_000, n_isolated=437_016, m_target=56_919_738, fam_hi=3000),
                       seed=2, s1=2, c1=400, seed1=201, s2=2, c2=400, seed2=202),
    "gos2m_s5c50": dict(gen=dict(n=2_000_000, n_isolated=437_016, m_target=56_919_738, fam_hi=3000),
                        seed=2, s1=5, c1=50, seed1=201, s2=5, c2=50, seed2=202),
    # small variants for parity tests (same recipe, oracle-sized)
    "small": dict(gen=dict(n=60_000, n_isolated=13_000, m_target=1_700_000, n_cliques=20,
                           cc_max=10_707, fam_hi=600),
                  seed=5, s1=2, c1=64, seed1=501, s2=2, c2=48, seed2=502),
    "hubsmall": dict(gen=dict(n=40_000, n_isolated=8_000, m_target=600_000, n_hubs=40,
                              hub_lo=5000, hub_hi=12000, fam_hi=400),
                     seed=6, s1=2, c1=40, seed1=601, s2=2, c2=40, seed2=602),
}


def make(name: str, cache: bool = True, **overrides) -> Graph:
    cfg = CONFIGS[name]
    gen = dict(cfg["gen"])
    gen.update(overrides)
    seed = gen.pop("seed", cfg["seed"])
    tag = name + ("" if not overrides else "_" + "_".join(f"{k}{v}" for k, v in sorted(overrides.items())))
    path = os.path.join(_DATA, f"{tag}_s{seed}.npz")
    if cache and os.path.exists(path):
        z = np.load(path)
        return Graph(z["row_ptr"], z["col"], dict(name=name, seed=seed))
    row_ptr, col = homology_graph(seed=seed, **gen)
    if cache:
        os.makedirs(_DATA, exist_ok=True)
        tmp = path + ".tmp.npz"
        np.savez(tmp, row_ptr=row_ptr, col=col)
        os.replace(tmp, path)
    return Graph(row_ptr, col, dict(name=name, seed=seed))


def cliques(sizes, n=None, seed=0):
    """Disjoint cliques with randomly permuted vertex ids (self-check (iii))."""
    rng = np.random.default_rng(seed)
    tot = int(sum(sizes))
    n = tot if n is None else n
    perm = rng.permutation(n).astype(np.int64)
    ea, eb, base = [], [], 0
    for k in sizes:
        i, j = np.triu_indices(int(k), 1)
        ea.append(base + i)
        eb.append(base + j)
        base += int(k)
    a = perm[np.concatenate(ea)] if ea else np.zeros(0, np.int64)
    b = perm[np.concatenate(eb)] if eb else np.zeros(0, np.int64)
    rp, col = _csr_from_pairs(n, a, b)
    return Graph(rp, col, dict(name="cliques"))


def random_graph(n, m, seed=0):
    """Erdos-Renyi-ish simple graph with random ids (small property tests)."""
    rng = np.random.default_rng(seed)
    a = rng.integers(0, n, m)
    b = rng.integers(0, n, m)
    rp, col = _csr_from_pairs(n, a.astype(np.int64), b.astype(np.int64))
    return Graph(rp, col, dict(name="random"))


def from_adj(adj) -> Graph:
    rp = np.zeros(len(adj) + 1, np.int64)
    rp[1:] = np.cumsum([len(r) for r in adj])
    col = np.asarray([v for r in adj for v in r], np.int32)
    return Graph(rp, col)


def to_adj(g: Graph):
    return [g.col[g.row_ptr[u]:g.row_ptr[u + 1]].tolist() for u in range(g.n)]
