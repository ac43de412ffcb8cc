"""A small CPU model of the PSB traversal (test utility, NOT the oracle).

It walks Alg. 1 (§III, with DESIGN.md §2's readings R3-R12 and
R25) over an exported index blob, step by step, and records the same trace
psb_knn_trace records on the GPU: (level, node, flags) per step. It exists to pin
the *order* of the kernel's traversal (scan right while the kNN list changes,
backtrack through parent links otherwise, Fig. 2), which the result
parity tests cannot see. Its own results are checked against the oracle in
tests/test_trace_model.py before it is used to check the GPU.

Arithmetic is numpy float32 element by element (one rounding per operation, no
FMA), in the fixed dimension order of the kernels.
"""
from __future__ import annotations

import numpy as np

PASS1, CHANGED, SKIPPED, FETCHED = 1, 2, 4, 8
PAD_KEY = (0x7F800000 << 32) | 0xFFFFFFFF
F32 = np.float32


def _bits(x) -> int:
    return int(np.asarray(x, dtype=np.float32).view(np.uint32))


def _key(dist, pid) -> int:
    return (_bits(dist) << 32) | (int(pid) & 0xFFFFFFFF)


class Tree:
    """Exported index (paper_conf_icpp_namkn16_b200._parse_blob dict)."""

    def __init__(self, blob: dict):
        self.d, self.F, self.L, self.H = blob["d"], blob["fanout"], blob["leaves"], blob["levels"]
        self.nlev = [int(x) for x in blob["nlev"]]
        self.pts, self.ids, self.nodes = blob["pts"], blob["ids"], blob["nodes"]
        self.n = int((self.ids >= 0).sum())
        self.logf = self.F.bit_length() - 1
        self.span = []
        s = 1
        for _ in range(self.H + 2):
            self.span.append(s if s < self.L else self.L)
            if s < self.L:
                s *= self.F
        # irregular: a leaf other than the last holds fewer than F points
        cnt = (self.ids >= 0).sum(1)
        self.irregular = bool((cnt[:-1] < self.F).any())

    def node_bounds(self, lvl: int, node: int, q):
        """MINDIST, MAXDIST of the query to the F children of (lvl, node) (S4)."""
        blk = self.nodes[lvl][node]                       # [d, 2, F]
        md = np.zeros(self.F, F32)
        Md = np.zeros(self.F, F32)
        for j in range(self.d):
            a = (blk[j, 0] - q[j]).astype(F32)
            c = (blk[j, 1] - q[j]).astype(F32)
            m = np.maximum(np.maximum(a, -c), F32(0))
            x = np.maximum(np.abs(a), np.abs(c))
            mm, xx = (m * m).astype(F32), (x * x).astype(F32)
            md = mm if j == 0 else (md + mm).astype(F32)
            Md = xx if j == 0 else (Md + xx).astype(F32)
        return md, Md

    def leaf_dists(self, j: int, q):
        blk = self.pts[j]                                 # [d, F]
        s = np.zeros(self.F, F32)
        for c in range(self.d):
            t = (blk[c] - q[c]).astype(F32)
            tt = (t * t).astype(F32)
            s = tt if c == 0 else (s + tt).astype(F32)
        return s

    def max_leaf(self, lvl: int, node: int) -> int:
        return min((node + 1) * self.span[lvl], self.L) - 1


def psb(tree: Tree, q, k: int, use_cache: bool = True, kth_rule: bool = False):
    """Alg. 1 as the kernel runs it. Returns (ids, dists, steps)."""
    q = np.asarray(q, F32)
    T, F, L, H = tree, tree.F, tree.L, tree.H
    keys: list[int] = []                                  # sorted, <= k
    steps = []

    def thr() -> int:
        return keys[k - 1] if len(keys) >= k else PAD_KEY

    def kth_dist():
        return np.uint32(thr() >> 32).view(F32)

    # per-launch child limit of the count-aware bound (R3)
    kcnt_lim = [0] * (H + 1)
    for lvl in range(1, H + 1):
        lastc = T.nlev[lvl - 1] - 1
        last_ok = T.n - lastc * T.span[lvl - 1] * F >= k
        kcnt_lim[lvl] = lastc if last_ok else lastc - 1
    count_aware = k <= F and not kth_rule and not T.irregular

    cache = {}
    pd = F32(np.inf)

    def internal(lvl, node):
        nonlocal pd
        if use_cache and cache.get(lvl, (None,))[0] == node:
            return cache[lvl][1], False
        md, Md = T.node_bounds(lvl, node, q)
        if count_aware:
            lim = kcnt_lim[lvl] - node * F
            sel = Md[: max(0, min(F, lim + 1))]
            if sel.size:
                pd = min(pd, F32(sel.min()))
        else:
            if (Md < pd).sum() >= k:
                pd = F32(np.sort(Md)[k - 1])
        cache[lvl] = (node, md)
        return md, True

    def scan(j):
        nonlocal keys
        dist = T.leaf_dists(j, q)
        t0 = thr()
        td = np.uint32(t0 >> 32).view(F32)
        cand = [_key(dist[s], T.ids[j, s]) for s in range(F) if dist[s] <= td]
        below = [c for c in cand if c < t0]
        if below:
            keys = sorted(keys + below)[:k]
        return bool(below)

    pass1 = True
    lvl, node = H, 0
    visited = -1
    p1node, p1md, p1taken = -1, None, set()
    while True:
        if lvl > 0:
            md, fetched = internal(lvl, node)
            steps.append((lvl, node, (PASS1 if pass1 else 0) | (FETCHED if fetched else 0)))
            base = node * F
            c = F
            if pass1:
                c_hi = T.nlev[lvl - 1] - base
                _, Md = T.node_bounds(lvl, node, q)
                best = None
                for cc in range(min(F, c_hi)):
                    key = (_bits(md[cc]), _bits(Md[cc]), cc)
                    if best is None or key < best:
                        best = key
                c = best[2]
            else:
                c_end = min(F, T.nlev[lvl - 1] - base)
                c_min = ((visited + 1) >> ((lvl - 1) * T.logf)) - base if visited + 1 < L else F
                for cc in range(max(c_min, 0), c_end):
                    if md[cc] <= pd:
                        c = cc
                        break
            if c < F:
                node = base + c
                lvl -= 1
                if lvl == 0 and pass1:
                    p1node, p1md, p1taken = base >> T.logf, md.copy(), set()
            else:
                if lvl == H:
                    break
                visited = T.max_leaf(lvl, node)
                node //= F
                lvl += 1
        else:
            j = node
            pre = (not pass1) and (j >> T.logf) == p1node and (j & (F - 1)) in p1taken
            changed = False if pre else scan(j)
            steps.append((0, j, (PASS1 if pass1 else 0) | (CHANGED if changed else 0) | (SKIPPED if pre else 0)))
            pd = min(pd, kth_dist())
            if pass1:
                b1 = j & ~(F - 1)
                p1taken.add(j - b1)
                best = None
                for cc in range(F):
                    if cc in p1taken or b1 + cc >= L:
                        continue
                    key = (_bits(p1md[cc]), cc)
                    if best is None or key < best:
                        best = key
                if best is not None and np.uint32(best[0]).view(F32) <= pd:
                    node = b1 + best[1]
                    continue
                pass1 = False
                lvl, node = H, 0
                continue
            visited = j
            if j == L - 1:
                break
            if changed:
                node = j + 1
            else:
                node, lvl = j // F, 1
    out = keys + [PAD_KEY] * (k - len(keys))
    ids = np.array([(x & 0xFFFFFFFF) for x in out], np.uint32).view(np.int32)
    dists = np.array([x >> 32 for x in out], np.uint32).view(F32)
    return ids, dists, steps


def leaf_mindists(tree: Tree, q) -> np.ndarray:
    """MINDIST of the query to every leaf's box (level-1 child boxes), fp32."""
    q = np.asarray(q, F32)
    out = np.empty(tree.L, F32)
    for i in range(tree.nlev[1]):
        md, _ = tree.node_bounds(1, i, q)
        hi = min(tree.F, tree.L - i * tree.F)
        out[i * tree.F:i * tree.F + hi] = md[:hi]
    return out
