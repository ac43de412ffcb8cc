"""Pins for the CPU oracle (oracle/): checks it against things OTHER than itself.

Each test names what fixes the expected value: a hand-worked case
(tests/golden/hand_cases.json), a closed form (Gauss circle counts), exact
integer arithmetic, the binary32 error bound of the distance, a textbook special
case (1-D two-pointer merge), or the second, independent oracle route (brute
force vs recursive branch-and-bound over a different tree).
A plausible mistake in the oracle — a dropped term, a wrong sign or index, a
transposed operand, an off-by-one in the best-k list, a wrong tie-break, a
strict/non-strict pruning slip — fails at least one of these.
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "hand_cases.json")))


def _f(v):
    return np.float32(np.inf) if v == "inf" else np.float32(v)


@pytest.mark.parametrize("case", GOLD["cases"], ids=lambda c: c["name"][:40])
@pytest.mark.parametrize("route", ["brute", "bnb"])
def test_hand_cases(case, route):
    P = np.array(case["points"], np.float32)
    Q = np.array([case["query"]], np.float32)
    k = case["k"]
    fn = oracle.knn_bruteforce if route == "brute" else (lambda p, q, k: oracle.knn_bnb(p, q, k, leaf_size=2))
    ids, dists = fn(P, Q, k)
    assert ids[0].tolist() == case["ids"]
    assert dists[0].tolist() == [float(_f(v)) for v in case["dists"]]


def test_fma_sensitive_distance():
    """Round-to-nearest per operation, not fused (SURVEY.md §8(c) FMA pin)."""
    c = GOLD["fma_case"]
    q = np.array([float.fromhex(v) for v in c["query"]], np.float32)
    p = np.array([float.fromhex(v) for v in c["point"]], np.float32)
    got = int(oracle.dist(q, p).view(np.uint32))
    assert got == int(c["rn_bits"], 16)
    assert got != int(c["fma_bits"], 16)
    # and through the kNN routes
    ids, d = oracle.knn_bruteforce(p[None], q[None], 1)
    assert int(d.view(np.uint32)[0, 0]) == int(c["rn_bits"], 16)


def test_lattice_closed_form():
    """Interior integer query on a 2-D integer lattice: kNN radii follow the Gauss
    circle counts; inside a shell the tie-break takes the smallest row-major ids."""
    m = 11
    P = np.array([(x, y) for x in range(m) for y in range(m)], np.float32)  # id = x*m + y
    q = np.array([[5, 5]], np.float32)
    lat = GOLD["lattice_2d"]
    for R, cnt in zip(lat["R"], lat["count"]):
        for fn in (oracle.knn_bruteforce, oracle.knn_bnb):
            ids, d = fn(P, q, cnt)
            assert d[0, -1] == R                      # k-th distance is exactly R
            assert (d[0] <= R).all()
            ids2, d2 = fn(P, q, cnt + 1)
            assert d2[0, -1] > R                      # the (count+1)-th lies outside
    # shell R=5 has 8 points; k = 13 + 3 takes the 3 smallest ids of that shell
    shell5 = sorted(x * m + y for x in range(m) for y in range(m) if (x - 5) ** 2 + (y - 5) ** 2 == 5)
    for fn in (oracle.knn_bruteforce, oracle.knn_bnb):
        ids, d = fn(P, q, 16)
        assert ids[0, 13:].tolist() == shell5[:3]
        assert d[0, 13:].tolist() == [5.0, 5.0, 5.0]


@pytest.mark.parametrize("d", [1, 2, 3, 5, 8, 16])
def test_exact_integer_distances(d):
    """Integer coordinates: every distance is an integer < 2^24, so binary32 is
    exact and the result must equal exact integer kNN computed with Python ints."""
    rng = np.random.default_rng(100 + d)
    n, nq, k = 300, 20, 17
    lim = int((2 ** 24 / d) ** 0.5 / 2) - 1
    lim = min(lim, 60)
    P = rng.integers(-lim, lim + 1, size=(n, d))
    Q = rng.integers(-lim, lim + 1, size=(nq, d))
    ids, dists = oracle.knn_bruteforce(P.astype(np.float32), Q.astype(np.float32), k)
    ids2, dists2 = oracle.knn_bnb(P.astype(np.float32), Q.astype(np.float32), k)
    for i in range(nq):
        exact = sorted((sum((int(P[p, j]) - int(Q[i, j])) ** 2 for j in range(d)), p) for p in range(n))[:k]
        assert ids[i].tolist() == [p for _, p in exact]
        assert dists[i].tolist() == [float(v) for v, _ in exact]
        assert ids2[i].tolist() == ids[i].tolist()
        assert dists2[i].tolist() == dists[i].tolist()


def test_distance_within_binary32_error_bound():
    """|fl(dist) - dist| <= gamma_{d+1} * dist (recursive summation of d rounded
    squares of rounded differences; Higham Thm 3.1 / Lemma 3.1 with u = 2^-24)."""
    rng = np.random.default_rng(7)
    u = Fraction(1, 2 ** 24)
    for d in (1, 2, 3, 8, 16, 64):
        for _ in range(200):
            q = rng.normal(size=d).astype(np.float32) * np.float32(rng.choice([1e-3, 1, 1e3]))
            p = rng.normal(size=d).astype(np.float32) * np.float32(rng.choice([1e-3, 1, 1e3]))
            exact = sum((Fraction(float(a)) - Fraction(float(b))) ** 2 for a, b in zip(p, q))
            got = Fraction(float(oracle.dist(q, p)))
            n_ops = d + 2
            gamma = n_ops * u / (1 - n_ops * u)
            assert abs(got - exact) <= gamma * exact


def test_distance_symmetric_and_sign():
    """(p-q)^2 == (q-p)^2 bit for bit (fl(-x) = -fl(x)); a sign slip breaks it."""
    rng = np.random.default_rng(3)
    for _ in range(500):
        d = int(rng.integers(1, 20))
        a = rng.normal(size=d).astype(np.float32) * 100
        b = rng.normal(size=d).astype(np.float32) * 100
        assert oracle.dist(a, b).view(np.uint32) == oracle.dist(b, a).view(np.uint32)
        assert oracle.dist(a, a) == 0


def test_one_dimensional_two_pointer():
    """d = 1 (the O(log n) 1-D case, §I): expand two pointers
    outward from the query's position in the sorted array, merging by (dist, id)."""
    rng = np.random.default_rng(11)
    for trial in range(30):
        n = int(rng.integers(1, 400))
        x = rng.integers(-50, 50, size=n).astype(np.float32) * np.float32(0.37)
        q = np.float32(rng.normal() * 10)
        k = int(rng.integers(1, n + 4))
        order = sorted(range(n), key=lambda i: (x[i], i))
        # first index with x >= q
        pos = next((t for t, i in enumerate(order) if x[i] >= q), n)
        lo, hi = pos - 1, pos
        out = []
        dd = lambda i: float(np.float32(np.float32(x[i] - q) * np.float32(x[i] - q)))
        while len(out) < min(k, n):
            # candidates on each side: the nearest equal-coordinate run, smallest id first
            cands = []
            if lo >= 0:
                cands.append((dd(order[lo]), order[lo], "lo"))
            if hi < n:
                cands.append((dd(order[hi]), order[hi], "hi"))
            # within an equal-distance group, ids may interleave between sides and
            # inside a run: gather the whole group, then sort by id
            best = min(c[0] for c in cands)
            group = []
            while lo >= 0 and dd(order[lo]) == best:
                group.append(order[lo]); lo -= 1
            while hi < n and dd(order[hi]) == best:
                group.append(order[hi]); hi += 1
            out.extend((best, i) for i in sorted(group))
        out = out[:k]
        ids, d = oracle.knn_bruteforce(x[:, None], np.array([[q]], np.float32), k)
        exp_ids = [i for _, i in out] + [-1] * (k - len(out))
        exp_d = [v for v, _ in out] + [float("inf")] * (k - len(out))
        assert ids[0].tolist() == exp_ids, trial
        assert d[0].tolist() == exp_d, trial


def _lattice(m, d):
    g = np.stack(np.meshgrid(*[np.arange(m)] * d, indexing="ij"), -1).reshape(-1, d)
    return g.astype(np.float32)


@pytest.mark.parametrize("d", [1, 2, 3, 8, 16])
@pytest.mark.parametrize("kind", ["uniform", "lattice", "dups"])
def test_bruteforce_equals_bnb(d, kind):
    """Two independent routes (definition vs recursive B&B over the oracle's own
    tree) agree bit for bit — including on massive-tie inputs."""
    rng = np.random.default_rng(d * 10 + ["uniform", "lattice", "dups"].index(kind))
    if kind == "uniform":
        P = rng.random((3000 if d <= 3 else 2000, d), dtype=np.float32)
        Q = rng.random((40, d), dtype=np.float32)
    elif kind == "lattice":
        m = {1: 500, 2: 40, 3: 12, 8: 3, 16: 2}[d]
        P = _lattice(m, d)
        if len(P) > 10_000:
            P = P[:10_000]
        Q = rng.integers(0, m, size=(40, d)).astype(np.float32)
    else:
        base = rng.integers(0, 4, size=(60, d)).astype(np.float32)
        P = base[rng.integers(0, 60, size=2500)]
        Q = rng.integers(0, 4, size=(40, d)).astype(np.float32)
    n = len(P)
    for k in (1, 8, 32, 64, n, n + 5):
        for leaf in (1, 16):
            a = oracle.knn_bruteforce(P, Q, k)
            b = oracle.knn_bnb(P, Q, k, leaf_size=leaf)
            assert np.array_equal(a[0], b[0]), (k, leaf)
            assert np.array_equal(a[1].view(np.uint32), b[1].view(np.uint32)), (k, leaf)


def _np_dists(P, q):
    """Independent numpy binary32 evaluation, fixed dimension order (elementwise
    ops are single-rounded; numpy never contracts to FMA)."""
    s = np.zeros(len(P), np.float32)
    for j in range(P.shape[1]):
        t = P[:, j] - q[j]
        s = s + t * t
    return s


@pytest.mark.parametrize("seed", range(5))
def test_result_invariants(seed):
    """north_star invariants: rows ascending by (dist, id); every returned
    distance <= every non-returned one (ties: returned ids smaller); ids distinct."""
    rng = np.random.default_rng(seed)
    d = int(rng.choice([2, 3, 8]))
    P = (rng.normal(size=(4000, d)) * 50).astype(np.float32)
    Q = (rng.normal(size=(25, d)) * 50).astype(np.float32)
    k = int(rng.choice([1, 7, 32, 100]))
    ids, dists = oracle.knn_bruteforce(P, Q, k)
    for i in range(len(Q)):
        keys = list(zip(dists[i].tolist(), ids[i].tolist()))
        assert keys == sorted(keys)
        assert len(set(ids[i].tolist())) == k
        all_d = _np_dists(P, Q[i])
        assert np.array_equal(all_d[ids[i]].view(np.uint32), dists[i].view(np.uint32))
        rest = np.setdiff1d(np.arange(len(P)), ids[i])
        kth, kid = dists[i, -1], ids[i, -1]
        assert (all_d[rest] >= kth).all()
        assert all(r > kid for r in rest[all_d[rest] == kth])


def test_special_cases():
    rng = np.random.default_rng(5)
    # all points identical -> ids 0..k-1
    P = np.tile(np.float32([[1.5, -2.0, 3.25]]), (50, 1))
    ids, d = oracle.knn_bruteforce(P, np.float32([[0, 0, 0]]), 10)
    assert ids[0].tolist() == list(range(10))
    assert (d[0] == np.float32(1.5 * 1.5 + 4.0 + 3.25 * 3.25)).all()
    # k = n is the full (dist, id) order
    P = rng.integers(0, 5, size=(200, 2)).astype(np.float32)
    q = np.float32([[2, 2]])
    ids, d = oracle.knn_bruteforce(P, q, 200)
    exp = sorted(range(200), key=lambda i: (int((P[i, 0] - 2) ** 2 + (P[i, 1] - 2) ** 2), i))
    assert ids[0].tolist() == exp
    # empty query batch
    ids, d = oracle.knn_bruteforce(P, np.zeros((0, 2), np.float32), 3)
    assert ids.shape == (0, 3)


def test_mindist_maxdist_bracket_point_distances():
    """App. C lemma, checked on the oracle's bound functions: for every point p in
    a box B (exact min/max), MINDIST(q,B) <= dist(q,p) <= MAXDIST(q,B) in the
    computed binary32 arithmetic; MINDIST is 0 for q inside B."""
    rng = np.random.default_rng(9)
    for trial in range(300):
        d = int(rng.integers(1, 9))
        pts = (rng.normal(size=(int(rng.integers(1, 20)), d)) * rng.choice([1e-2, 1, 1e3])).astype(np.float32)
        lo, hi = pts.min(0), pts.max(0)
        for _ in range(5):
            q = (rng.normal(size=d) * rng.choice([1e-2, 1, 1e3])).astype(np.float32)
            mn, mx = oracle.mindist(q, lo, hi), oracle.maxdist(q, lo, hi)
            for p in pts:
                dd = oracle.dist(q, p)
                assert mn <= dd <= mx
        inside = pts[0]
        assert oracle.mindist(inside, lo, hi) == 0
    # hand value: box [0,1]x[0,1], q=(3,-2): MINDIST = 2^2+2^2 = 8, MAXDIST = 3^2+3^2 = 18
    assert oracle.mindist([3, -2], [0, 0], [1, 1]) == 8
    assert oracle.maxdist([3, -2], [0, 0], [1, 1]) == 18


def test_oracle_tree_invariants():
    rng = np.random.default_rng(2)
    P = (rng.normal(size=(3000, 3)) * 10).astype(np.float32)
    t = oracle.Tree(P, leaf_size=16)
    perm = t.perm()
    assert sorted(perm.tolist()) == list(range(3000))
    nodes = t.nodes()
    for lo, hi, a, b, l, r in nodes:
        sub = P[perm[a:b]]
        assert np.array_equal(lo, sub.min(0)) and np.array_equal(hi, sub.max(0))
        if l < 0:
            assert b - a <= 16
        else:
            assert nodes[l][2] == a and nodes[r][3] == b and nodes[l][3] == nodes[r][2]
