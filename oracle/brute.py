"""Brute-force pairwise race enumeration, literally SURVEY.md §8(c) C1.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  O(n^2) over word-level accesses, for tiny
traces.  Independent of oracle_d.c (different algorithm, different language) and of the CUDA
path.
"""
from __future__ import annotations

R, W, AB, AG = 0, 1, 2, 3
WARP, BLOCK, GRID = 1, 2, 3
SHARED = 1 << 63


def accesses(events, block_threads, warp_size, gran_log2=2):
    """C1.1: element-level accesses (key, tid, kind, g, b, w, block, warp); an element is
    1 << gran_log2 bytes (4-byte words by default)."""
    out = []
    granule = 1 << gran_log2
    for e in events:
        addr, tid, meta = int(e["addr"]), int(e["tid"]), int(e["meta"])
        kind, size = meta & 3, 1 << ((meta >> 2) & 7)
        w, b, g = (meta >> 5) & 511, (meta >> 14) & 1023, (meta >> 24) & 255
        block, warp = tid // block_threads, (tid % block_threads) // warp_size
        word0 = (addr & ~SHARED) >> gran_log2
        for k in range(1 if size <= granule else size // granule):
            word = word0 + k
            key = (SHARED | (block << 32) | word) if addr & SHARED else word
            out.append((key, tid, kind, g, b, w, block, warp))
    return out


def concurrent(a, c):
    """C1.2."""
    _, t1, _, g1, b1, w1, blk1, wp1 = a
    _, t2, _, g2, b2, w2, blk2, wp2 = c
    if t1 == t2 or g1 != g2:
        return False
    if blk1 != blk2:
        return True
    if b1 != b2:
        return False
    return wp1 != wp2 or w1 == w2


def conflict(a, c, policy=0):
    """C1.3.  policy 1 = relaxed: a plain read never conflicts with an
    atomic (reading R2b)."""
    k1, k2 = a[2], c[2]
    if k1 == R and k2 == R:
        return False
    if policy == 1 and W not in (k1, k2) and R in (k1, k2):
        return False
    if k1 in (AB, AG) and k2 in (AB, AG):
        if k1 == AG and k2 == AG:
            return False
        return a[6] != c[6]
    return True


def level(a, c):
    if a[6] != c[6]:
        return GRID
    if a[7] != c[7]:
        return BLOCK
    return WARP


def races(events, block_threads, warp_size, policy=0, gran_log2=2):
    """Returns {key: (class, g*)} by literal enumeration of all pairs (C1.4-C1.6)."""
    acc = accesses(events, block_threads, warp_size, gran_log2)
    pairs = {}
    for i in range(len(acc)):
        for j in range(i + 1, len(acc)):
            a, c = acc[i], acc[j]
            if a[0] == c[0] and concurrent(a, c) and conflict(a, c, policy):
                # racing pair: record (g, b, level); b is shared by intra-block pairs
                pairs.setdefault(a[0], []).append((a[3], a[4], level(a, c)))
    out = {}
    for key, ps in pairs.items():
        gstar = min(p[0] for p in ps)
        in_g = [p for p in ps if p[0] == gstar]
        if any(p[2] == GRID for p in in_g):
            out[key] = (GRID, gstar)
            continue
        bstar = min(p[1] for p in in_g)
        in_b = [p for p in in_g if p[1] == bstar]
        out[key] = (BLOCK if any(p[2] == BLOCK for p in in_b) else WARP, gstar)
    return out


# ---------------------------------------------------------------------------------------------
# Cluster level (reading R16): the literal pair
# loop over C1.1'-C1.6' (see oracle_d.c).  Event encoding: addr bits 56..62 = cluster epoch c,
# shared addr bits 48..55 = DSMEM target (0 own block, r+1 = cluster rank r).
# ---------------------------------------------------------------------------------------------
CLUSTER = 4


def accesses_cluster(events, block_threads, warp_size, cluster_blocks):
    """C1.1': (key, tid, kind, g, c, b, w, cluster, block, warp) per word."""
    out = []
    for e in events:
        addr, tid, meta = int(e["addr"]), int(e["tid"]), int(e["meta"])
        kind, size = meta & 3, 1 << ((meta >> 2) & 7)
        w, b, g = (meta >> 5) & 511, (meta >> 14) & 1023, (meta >> 24) & 255
        c = (addr >> 56) & 127
        target = (addr >> 48) & 255
        block, warp = tid // block_threads, (tid % block_threads) // warp_size
        cl = block // cluster_blocks
        shared = bool(addr & SHARED)
        owner = cl * cluster_blocks + target - 1 if (shared and target) else block
        word0 = (addr & ((1 << 48) - 1)) >> 2
        for k in range(1 if size <= 4 else size // 4):
            word = word0 + k
            key = (SHARED | (owner << 32) | word) if shared else word
            out.append(dict(key=key, tid=tid, kind=kind, g=g, c=c, b=b, w=w, cl=cl, block=block, warp=warp))
    return out


def concurrent_cluster(a, d):
    """C1.2': a cluster barrier orders everything inside one cluster; __syncthreads orders a
    block; a full-warp sync a warp."""
    if a["tid"] == d["tid"] or a["g"] != d["g"]:
        return False
    if a["cl"] != d["cl"]:
        return True
    if a["c"] != d["c"]:
        return False
    if a["block"] != d["block"]:
        return True
    if a["b"] != d["b"]:
        return False
    return a["warp"] != d["warp"] or a["w"] == d["w"]


def races_cluster(events, block_threads, warp_size, cluster_blocks):
    """{key: (class, g*)} by enumeration of all pairs (C1.4'-C1.6'), strict conflict rule."""
    acc = accesses_cluster(events, block_threads, warp_size, cluster_blocks)
    pairs = {}
    for i in range(len(acc)):
        for j in range(i + 1, len(acc)):
            a, d = acc[i], acc[j]
            if a["key"] != d["key"] or not concurrent_cluster(a, d):
                continue
            if not conflict((0, 0, a["kind"], 0, 0, 0, a["block"]), (0, 0, d["kind"], 0, 0, 0, d["block"])):
                continue
            if a["cl"] != d["cl"]:
                lvl = GRID
            elif a["block"] != d["block"]:
                lvl = CLUSTER
            elif a["warp"] != d["warp"]:
                lvl = BLOCK
            else:
                lvl = WARP
            pairs.setdefault(a["key"], []).append((a["g"], a["c"], a["b"], lvl))
    out = {}
    for key, ps in pairs.items():
        gstar = min(p[0] for p in ps)
        in_g = [p for p in ps if p[0] == gstar]
        if any(p[3] == GRID for p in in_g):
            out[key] = (GRID, gstar)
            continue
        cstar = min(p[1] for p in in_g)
        in_c = [p for p in in_g if p[1] == cstar]
        if any(p[3] == CLUSTER for p in in_c):
            out[key] = (CLUSTER, gstar)
            continue
        bstar = min(p[2] for p in in_c)
        in_b = [p for p in in_c if p[2] == bstar]
        out[key] = (BLOCK if any(p[3] == BLOCK for p in in_b) else WARP, gstar)
    return out


# ---------------------------------------------------------------------------------------------
# Partial-mask __syncwarp(mask) ("a bounded history of sub-warp
# synchronizations (essentially a warp-level vector clock)"; reading R20).  The pair
# loop of C1 with same-warp concurrency decided by textbook vector clocks: every lane holds a
# vector V (V[i] = the latest sync number of lane i it knows of); a sync of mask M joins the
# vectors of its lanes and stamps V[i] = s for i in M; e1 (lane i, after sync w1) happens
# before e2 (lane j, after sync w2) iff V_j after w2 has V[i] > w1.  Unlisted numbers are
# full-mask syncs.  (oracle_d.c decides the same relation by forward knowledge propagation.)
# ---------------------------------------------------------------------------------------------


def warp_vector_clocks(listed: dict, smax: int, lanes: int) -> dict:
    """{s: V after sync s} for s = 1..smax; listed = {s: mask} of one warp in one (g, b)."""
    cur = [[0] * lanes for _ in range(lanes)]
    out = {}
    for s in range(1, smax + 1):
        m = listed.get(s, (1 << lanes) - 1)
        members = [l for l in range(lanes) if (m >> l) & 1]
        j = [max(cur[l][i] for l in members) for i in range(lanes)]
        for i in members:
            j[i] = s
        for l in members:
            cur[l] = list(j)
        out[s] = j
    return out


def races_masked(events, syncs, block_threads, warp_size, policy=0):
    """{key: (class, g*)} with C1.2'' same-warp concurrency (4-byte words)."""
    acc = accesses(events, block_threads, warp_size)
    wpb = -(-block_threads // warp_size)
    fam = {}
    for s in (syncs if syncs is not None else []):
        meta = int(s["meta"])
        fam.setdefault((meta >> 24 & 255, meta >> 14 & 1023, int(s["warp"])), {})[meta >> 5 & 511] = int(s["mask"])
    clocks = {}

    def vc(a):
        key = (a[3], a[4], a[6] * wpb + a[7])
        if key not in fam or a[5] == 0:
            return None
        if key not in clocks:
            smax = max(max(fam[key]), max(x[5] for x in acc if (x[3], x[4], x[6] * wpb + x[7]) == key))
            clocks[key] = warp_vector_clocks(fam[key], smax, warp_size)
        return clocks[key][a[5]]

    def lane(a):
        return (a[1] % block_threads) % warp_size

    def conc(a, c):
        family = (a[3], a[4], a[6] * wpb + a[7])
        same = a[1] != c[1] and family == (c[3], c[4], c[6] * wpb + c[7])
        if not same or family not in fam:
            return concurrent(a, c)
        x, y = (a, c) if a[5] <= c[5] else (c, a)
        return x[5] == y[5] or vc(y)[lane(x)] <= x[5]

    pairs = {}
    for i in range(len(acc)):
        for j in range(i + 1, len(acc)):
            a, c = acc[i], acc[j]
            if a[0] == c[0] and conflict(a, c, policy) and conc(a, c):
                pairs.setdefault(a[0], []).append((a[3], a[4], level(a, c)))
    out = {}
    for key, ps in pairs.items():
        gstar = min(p[0] for p in ps)
        in_g = [p for p in ps if p[0] == gstar]
        if any(p[2] == GRID for p in in_g):
            out[key] = (GRID, gstar)
            continue
        bstar = min(p[1] for p in in_g)
        in_b = [p for p in in_g if p[1] == bstar]
        out[key] = (BLOCK if any(p[2] == BLOCK for p in in_b) else WARP, gstar)
    return out
