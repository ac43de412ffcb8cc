"""The tree of the paper's Fig. 2 (§III), hand-built (test fixture).

Fig. 2 walks PSB over a root A with children B and C; B's children D, E, F hold
the leaves H I J / K L M / N O, and C's subtree holds G, R, S. Its narrative:
(1) pass 1 finds a leaf close to the query and an initial pruning distance;
(2) the second traversal fetches the leftmost child B of A (both B and C are
within the pruning distance); (3) then D; H is pruned; (4) I is scanned and the
kNN set changes; (5) its siblings J and K are scanned; K changes nothing, so
(6) E, K's parent, is fetched and L is pruned; (7) M is scanned, (8) then its
sibling N; N changes nothing, so (9) PSB moves to N's parent F, which has no
child within the pruning distance, and (10) up to B, to A, and on to C, whose
leaves G, R and S are visited.

This repo's trees are packed with a fanout of at least 32, so the figure is
embedded in a fanout-32, 1-D tree with the same shape where it matters:
  leaves 0..29 ("H", pruned), 30 = I, 31 = J under D (level-1 node 0);
  32 = K, 33..62 ("L", pruned), 63 = M under E (node 1);
  64 = N, 65..95 ("O", pruned) under F (node 2);
  leaves 96..1023 ("far") under level-1 nodes 3..31 (the rest of B);
  1024 = G, 1025 = R, 1026 = S (the last leaf) under node 32 ("P"), C's only child.
Every leaf but the last holds 32 points, so the count-aware bound applies.
The query is x = 0, k = 1. C's points sit at +-60, +-70, +-80, so C's box holds
the query and pass 1 descends into C (ClosestLeaf = G, the box with the
smallest MAXDIST among those at MINDIST 0) and scans G, R, S; the true nearest
neighbour (x = 1 in M) is found in pass 2, along the Fig. 2 path; G, R, S are
visited again at the end but not rescanned (R25).
"""
import numpy as np

F = 32
L = 1027
QUERY = np.array([0.0], np.float32)

# leaf -> (name, interval or explicit values)
_NAMED = {30: "I", 31: "J", 32: "K", 63: "M", 64: "N", 1024: "G", 1025: "R", 1026: "S"}
_NODES = {(3, 0): "A", (2, 0): "B", (2, 1): "C", (1, 0): "D", (1, 1): "E", (1, 2): "F", (1, 32): "P"}


def _leaf_values(j):
    if j <= 29:
        return np.linspace(50, 60, F)                # H: far from the query, pruned at D
    if j == 30:
        return np.linspace(2.4, 2.5, F)              # I
    if j == 31:
        return np.linspace(2.0, 2.5, F)              # J: better than I
    if j == 32:
        return np.linspace(5.0, 6.0, F)              # K: no change
    if j <= 62:
        return np.linspace(70, 80, F)                # L: pruned at E
    if j == 63:
        return np.linspace(1.0, 1.5, F)              # M: the nearest neighbour (x = 1)
    if j == 64:
        return np.linspace(3.0, 3.5, F)              # N: no change
    if j <= 95:
        return np.linspace(90, 100, F)               # O: pruned at F
    if j <= 1023:
        return np.linspace(200, 300, F)              # far
    v = {1024: 60.0, 1025: 70.0, 1026: 80.0}[j]      # G, R, S: +-v
    if j == 1026:
        return np.array([-v, v])
    return np.array([-v, v] * (F // 2))


def _build():
    pts = np.full((L, 1, F), np.inf, np.float32)
    ids = np.full((L, F), -1, np.int32)
    nid = 0
    for j in range(L):
        v = _leaf_values(j).astype(np.float32)
        pts[j, 0, :len(v)] = v
        ids[j, :len(v)] = np.arange(nid, nid + len(v))
        nid += len(v)
    nlev = [L]
    while nlev[-1] > 1:
        nlev.append(-(-nlev[-1] // F))
    H = len(nlev) - 1
    nodes = {}
    lo_prev = np.where(ids >= 0, pts[:, 0, :], np.inf).min(1)      # per leaf
    hi_prev = np.where(ids >= 0, pts[:, 0, :], -np.inf).max(1)
    for lvl in range(1, H + 1):
        cnt = nlev[lvl]
        blk = np.empty((cnt, 1, 2, F), np.float32)
        blk[:, 0, 0, :] = np.inf
        blk[:, 0, 1, :] = -np.inf
        for g in range(nlev[lvl - 1]):
            blk[g // F, 0, 0, g % F] = lo_prev[g]
            blk[g // F, 0, 1, g % F] = hi_prev[g]
        nodes[lvl] = blk
        lo_prev = blk[:, 0, 0, :].min(1)
        hi_prev = blk[:, 0, 1, :].max(1)
    return pts, ids, nodes, nlev, nid


_PTS, _IDS, _NODES_ARR, _NLEV, _N = _build()


def points() -> np.ndarray:
    """The points in id order ([n, 1])."""
    out = np.empty((_N, 1), np.float32)
    m = _IDS >= 0
    out[_IDS[m], 0] = _PTS[:, 0, :][m]
    return out


def blob_dict() -> dict:
    return {"d": 1, "fanout": F, "leaves": L, "levels": len(_NLEV) - 1, "nlev": np.array(_NLEV, np.int64),
            "pts": _PTS, "ids": _IDS, "nodes": _NODES_ARR, "n": _N}


def raw_blob() -> np.ndarray:
    import paper_conf_icpp_namkn16_b200 as psb
    return psb.make_blob(_PTS, _IDS, _NODES_ARR, _N)


def _name(lvl, node):
    if lvl == 0:
        if node in _NAMED:
            return _NAMED[node]
        return "H" if node < 30 else "L" if node < 63 else "O" if node < 96 else "far"
    return _NODES.get((lvl, node), f"n{lvl}.{node}")


def named(steps):
    """[(level, node, flags)] -> [(name, flags)]"""
    return [(_name(lvl, node), fl) for lvl, node, fl in steps]


P1, CH, SK, FE = 1, 2, 4, 8
EXPECTED_WALK = [
    # (1) pass 1: descend to ClosestLeaf G through C (its box holds the query),
    # then the other leaves of G's parent in MINDIST order
    ("A", P1 | FE), ("C", P1 | FE), ("P", P1 | FE), ("G", P1 | CH), ("R", P1), ("S", P1),
    # (2) A again (path cache), leftmost child B; (3) D; H pruned
    ("A", 0), ("B", FE), ("D", FE),
    # (4) I changes the kNN set; (5) its siblings J (changes) and K (no change)
    ("I", CH), ("J", CH), ("K", 0),
    # (6) K's parent E; L pruned; (7) M changes; (8) sibling N, no change
    ("E", FE), ("M", CH), ("N", 0),
    # (9) N's parent F: nothing within the pruning distance; (10) up to B, A, on to C
    ("F", FE), ("B", 0), ("A", 0), ("C", FE), ("P", FE),
    # C's leaves G, R, S: visited, already scanned in pass 1 (R25)
    ("G", SK), ("P", 0), ("R", SK), ("P", 0), ("S", SK),
]
