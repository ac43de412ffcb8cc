"""CPU oracle for exact kNN — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference``) may import this package. The product path
(``paper_conf_icpp_namkn16_b200``) never imports it, and this package never
imports the product: the two share nothing but ``workloads`` (input generators).

The arithmetic lives in ``oracle/oracle.c`` (plain C, binary32 round-to-nearest,
``-ffp-contract=off``), compiled by ``build()`` (called from
``__graft_entry__.build()``). See its header for the definition it implements
(PSB is exact kNN) and the passages each function
follows. Pins: ``tests/test_oracle_pins.py``. Parity is pinned for every
function here (no "parity unpinned" entries).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fexcess-precision=standard",
          "-fopenmp", "-fPIC", "-shared", "-Wall", "-Wextra"]

_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so (building the checker is not using it)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        f32p = ctypes.POINTER(ctypes.c_float)
        i32p = ctypes.POINTER(ctypes.c_int32)
        i64 = ctypes.c_int64
        L.oracle_dist.restype = ctypes.c_float
        L.oracle_dist.argtypes = [f32p, f32p, ctypes.c_int]
        L.oracle_mindist.restype = ctypes.c_float
        L.oracle_mindist.argtypes = [f32p, f32p, f32p, ctypes.c_int]
        L.oracle_maxdist.restype = ctypes.c_float
        L.oracle_maxdist.argtypes = [f32p, f32p, f32p, ctypes.c_int]
        L.oracle_knn_bruteforce.restype = ctypes.c_int
        L.oracle_knn_bruteforce.argtypes = [f32p, i64, ctypes.c_int, f32p, i64, ctypes.c_int,
                                            i32p, f32p, ctypes.c_int]
        L.oracle_tree_build.restype = ctypes.c_void_p
        L.oracle_tree_build.argtypes = [f32p, i64, ctypes.c_int, ctypes.c_int]
        L.oracle_tree_free.restype = None
        L.oracle_tree_free.argtypes = [ctypes.c_void_p]
        L.oracle_tree_nodes.restype = i64
        L.oracle_tree_nodes.argtypes = [ctypes.c_void_p]
        L.oracle_tree_node.restype = ctypes.c_int
        L.oracle_tree_node.argtypes = [ctypes.c_void_p, i64, f32p, f32p,
                                       ctypes.POINTER(i64), ctypes.POINTER(i64),
                                       ctypes.POINTER(i64), ctypes.POINTER(i64)]
        L.oracle_tree_perm.restype = ctypes.c_int
        L.oracle_tree_perm.argtypes = [ctypes.c_void_p, i32p]
        L.oracle_knn_bnb.restype = ctypes.c_int
        L.oracle_knn_bnb.argtypes = [ctypes.c_void_p, f32p, i64, ctypes.c_int, i32p, f32p,
                                     ctypes.c_int]
        L.oracle_max_threads.restype = ctypes.c_int
        L.oracle_max_threads.argtypes = []
        _lib = L
    return _lib


def _f32(a):
    a = np.ascontiguousarray(a, dtype=np.float32)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_float))


def max_threads() -> int:
    return int(lib().oracle_max_threads())


def dist(q, p) -> np.float32:
    """dist(q,p) of SURVEY.md §8(c): squared Euclidean, fixed order, binary32 RN."""
    q, qp = _f32(q)
    p, pp = _f32(p)
    assert q.shape == p.shape and q.ndim == 1
    return np.float32(lib().oracle_dist(qp, pp, q.shape[0]))


def mindist(q, lo, hi) -> np.float32:
    q, qp = _f32(q)
    lo, lp = _f32(lo)
    hi, hp = _f32(hi)
    return np.float32(lib().oracle_mindist(qp, lp, hp, q.shape[0]))


def maxdist(q, lo, hi) -> np.float32:
    q, qp = _f32(q)
    lo, lp = _f32(lo)
    hi, hp = _f32(hi)
    return np.float32(lib().oracle_maxdist(qp, lp, hp, q.shape[0]))


def _outs(nq, k):
    ids = np.empty((nq, k), dtype=np.int32)
    dists = np.empty((nq, k), dtype=np.float32)
    return ids, dists, ids.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), \
        dists.ctypes.data_as(ctypes.POINTER(ctypes.c_float))


def knn_bruteforce(points, queries, k: int, threads: int = 0):
    """Exact kNN by definition: (ids int32 [q,k], dists float32 [q,k]), (-1,+inf) pads."""
    pts, pp = _f32(points)
    qs, qp = _f32(queries)
    n, d = pts.shape
    nq = qs.shape[0]
    assert qs.shape[1] == d
    ids, dists, ip, dp = _outs(nq, k)
    rc = lib().oracle_knn_bruteforce(pp, n, d, qp, nq, k, ip, dp, threads)
    if rc != 0:
        raise RuntimeError(f"oracle_knn_bruteforce failed ({rc})")
    return ids, dists


class Tree:
    """The oracle's own top-down median-split box tree (leaf <= leaf_size points)."""

    def __init__(self, points, leaf_size: int = 16):
        self.pts, pp = _f32(points)        # kept alive: the C tree points into it
        self.n, self.d = self.pts.shape
        self._h = lib().oracle_tree_build(pp, self.n, self.d, leaf_size)
        if not self._h:
            raise MemoryError("oracle_tree_build failed")

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        if h and _lib is not None:
            _lib.oracle_tree_free(h)

    def nodes(self):
        """[(lo, hi, a, b, left, right)] for invariant tests; perm = ids in tree order."""
        L = lib()
        i64 = ctypes.c_int64
        out = []
        lo = np.empty(self.d, np.float32)
        hi = np.empty(self.d, np.float32)
        a, b, l, r = i64(), i64(), i64(), i64()
        for i in range(L.oracle_tree_nodes(self._h)):
            L.oracle_tree_node(self._h, i, _f32(lo)[1], _f32(hi)[1], ctypes.byref(a),
                               ctypes.byref(b), ctypes.byref(l), ctypes.byref(r))
            out.append((lo.copy(), hi.copy(), a.value, b.value, l.value, r.value))
        return out

    def perm(self):
        out = np.empty(self.n, np.int32)
        lib().oracle_tree_perm(self._h, out.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)))
        return out

    def knn(self, queries, k: int, threads: int = 0):
        qs, qp = _f32(queries)
        assert qs.shape[1] == self.d
        ids, dists, ip, dp = _outs(qs.shape[0], k)
        rc = lib().oracle_knn_bnb(self._h, qp, qs.shape[0], k, ip, dp, threads)
        if rc != 0:
            raise RuntimeError(f"oracle_knn_bnb failed ({rc})")
        return ids, dists


def knn_bnb(points, queries, k: int, threads: int = 0, leaf_size: int = 16):
    return Tree(points, leaf_size).knn(queries, k, threads)
