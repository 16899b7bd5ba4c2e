"""ORACLE TWIN — TEST INFRASTRUCTURE ONLY.  Pure Python, big integers, tiny graphs.

An N-version twin of ``oracle/oracle.c`` written independently of it: it takes
the s smallest hashed values by a FULL sort of Gamma_j(u) (the brute force
that the paper's insertion sort, must equal), groups with a dict
keyed by the exact shingle instead of a sort, and finds the components of
G_II by BFS instead of union-find.  Same definitions (AMB-1..19 in
DESIGN.md §3), different mechanics, so a slip in either shows up as a
mismatch (self-check (ix)).
"""
from __future__ import annotations

from collections import defaultdict, deque

P = (1 << 31) - 1          # AMB-1
M64 = (1 << 64) - 1
GAMMA = 0x9E3779B97F4A7C15


def mix64(z: int) -> int:
    z &= M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def splitmix_stream(seed: int):
    state = seed & M64
    while True:
        state = (state + GAMMA) & M64
        yield mix64(state)


def hash_params(seed: int, c: int):
    """A_j in [1, P-1], B_j in [0, P-1], order A0, B0, A1, B1 (AMB-2)."""
    g = splitmix_stream(seed)
    A, B = [], []
    for _ in range(c):
        A.append(1 + next(g) % (P - 1))
        B.append(next(g) % P)
    return A, B


def h(A: int, B: int, v: int) -> int:
    return (A * v + B) % P          # P:L433, exact big-int arithmetic


def shingle_id(s: int, seed: int, j: int, mins) -> int:
    """AMB-4: exact packing for s <= 2, 64-bit fold for s >= 3."""
    if s == 1:
        return mins[0]
    if s == 2:
        return (mins[0] << 31) | mins[1]
    z = mix64(seed ^ mix64(j + 1))
    for x in mins:
        z = mix64(z + x)
    return z


def top_s_fullsort(row, s, A, B):
    """Brute force: hash every neighbour, sort all, keep the first s."""
    hv = sorted((h(A, B, v), v) for v in row)
    return [x for x, _ in hv[:s]], [v for _, v in hv[:s]]


def shingle_pass(rows, s, c, seed):
    """rows: list of lists.  Returns (eligible row indices, [[id]*c per eligible row])."""
    A, B = hash_params(seed, c)
    elig, mat = [], []
    for r, row in enumerate(rows):
        if len(row) < s:
            continue
        elig.append(r)
        mat.append([shingle_id(s, seed, j, top_s_fullsort(row, s, A[j], B[j])[0]) for j in range(c)])
    return elig, mat


def group(mat, member, c):
    """Per trial (AMB-5): dict id -> members; canonical order (mix64(id), members asc)."""
    out = []   # list of (trial, id, [members])
    for j in range(c):
        d = defaultdict(list)
        for r, row in enumerate(mat):
            d[row[j]].append(member[r])
        for sid in sorted(d, key=mix64):
            out.append((j, sid, sorted(d[sid])))
    return out


def shingling(adj, s1, c1, seed1, s2, c2, seed2):
    """adj: list of sorted neighbour lists.  Returns a dict of every stage output."""
    elig, M1 = shingle_pass(adj, s1, c1, seed1)
    G1 = group(M1, elig, c1)
    s1p = [g for g, (_, _, L) in enumerate(G1) if len(L) >= s2]
    rows2 = [G1[g][2] for g in s1p]
    _, M2 = shingle_pass(rows2, s2, c2, seed2)
    G2 = group(M2, list(range(len(s1p))), c2)
    return dict(rows1=elig, M1=M1, G1=G1, s1p=s1p, M2=M2, G2=G2,
                A1=hash_params(seed1, c1), A2=hash_params(seed2, c2), adj=adj,
                s1=s1, s2=s2)


def report(res, mode=0, min_size=1):
    """Phase III approach 2: BFS components of G_II, then BFS over
    the vertex graph whose edges join each component's vertex set."""
    adj, G1, G2, s1p = res["adj"], res["G1"], res["G2"], res["s1p"]
    s1, s2 = res["s1"], res["s2"]
    A1, B1 = res["A1"]
    A2, B2 = res["A2"]
    nk = len(s1p)
    # bipartite G_II: S1' nodes k <-> S2 nodes h
    k_to_h = defaultdict(list)
    for hi, (_, _, K) in enumerate(G2):
        for k in K:
            k_to_h[k].append(hi)
    comp = [-1] * nk
    comps = []
    for k0 in range(nk):
        if comp[k0] >= 0:
            continue
        cid = len(comps)
        comp[k0] = cid
        ks, hs, dq, seen_h = [k0], [], deque([k0]), set()
        while dq:
            k = dq.popleft()
            for hi in k_to_h[k]:
                if hi in seen_h:
                    continue
                seen_h.add(hi)
                hs.append(hi)
                for k2 in G2[hi][2]:
                    if comp[k2] < 0:
                        comp[k2] = cid
                        ks.append(k2)
                        dq.append(k2)
        comps.append((ks, hs))
    n = len(adj)
    vadj = defaultdict(set)
    for ks, hs in comps:
        verts = []
        for k in ks:
            j, _, L = G1[s1p[k]]
            if mode == 0:
                verts += top_s_fullsort(adj[L[0]], s1, A1[j], B1[j])[1]
            else:
                verts += L
        if mode == 0:
            for hi in hs:
                t, _, K = G2[hi]
                row = G1[s1p[K[0]]][2]
                verts += top_s_fullsort(row, s2, A2[t], B2[t])[1]
        for a in verts[1:]:
            vadj[verts[0]].add(a)
            vadj[a].add(verts[0])
    labels = list(range(n))
    seen = [False] * n
    nclus = 0
    for v in range(n):
        if seen[v]:
            continue
        compv, dq = [v], deque([v])
        seen[v] = True
        while dq:
            x = dq.popleft()
            for y in vadj[x]:
                if not seen[y]:
                    seen[y] = True
                    compv.append(y)
                    dq.append(y)
        if len(compv) >= min_size:
            lab = min(compv)
            for x in compv:
                labels[x] = lab
        if len(compv) >= max(2, min_size):
            nclus += 1
    return labels, nclus
