"""Input generators (workloads/): deterministic, exact, shaped like the paper's data."""
import numpy as np

import workloads as W


def test_u24_exact_and_deterministic():
    a = W.u24(123, 0, 1000)
    b = W.u24(123, 0, 1000)
    assert np.array_equal(a, b)
    assert (a >= 0).all() and (a < 1).all()
    assert np.array_equal(a.astype(np.float32).astype(np.float64), a)   # exact binary32
    assert np.array_equal(W.u24(123, 500, 10), a[500:510])              # counter-based


def test_uniform_shape_and_chunking():
    p = W.gen_uniform(1000, 3, 7)
    assert p.shape == (1000, 3) and p.dtype == np.float32
    assert np.array_equal(p.ravel(), W.u24(7, 0, 3000).astype(np.float32))


def test_clustered_centres_shared_with_queries():
    c = W.config("C2")
    p = c.points(n=20_000)
    q = c.queries(q=500)
    cen = W.cluster_centres(3, c.points_seed)
    # every query is within a few sigma of some data centre (queries land in the data)
    dq = ((q[:, None, :].astype(np.float64) - cen[None]) ** 2).sum(-1).min(1) ** 0.5
    assert np.median(dq) < 4 * c.sigma
    # points of cluster 0 (first block) sit around centre 0
    per = -(-20_000 // 100)
    assert np.abs(p[:per].mean(0) - cen[0]).max() < 50


def test_configs_match_baseline():
    import json, os
    bj = json.load(open(os.path.join(os.path.dirname(__file__), "..", "BASELINE.json")))
    assert len(bj["configs"]) == 5
    assert W.CONFIGS["C1"].n == 10_000 and W.CONFIGS["C1"].k == 8 and W.CONFIGS["C1"].fanout == 32
    assert W.CONFIGS["C2"].n == 1_000_000 and W.CONFIGS["C2"].k == 32 and W.CONFIGS["C2"].fanout == 64
    assert W.CONFIGS["C3"].q == 100_000 and W.CONFIGS["C3"].d == 8
    assert W.CONFIGS["C5"].n == 512_000_000


def test_slabs_are_rows_of_the_full_set():
    """Data-sharded ranks generate their own slab: it must equal the same rows of
    the full set (counter-based generator)."""
    full = W.gen_uniform(10_000, 3, 9)
    assert np.array_equal(W.gen_uniform(2_500, 3, 9, row0=5_000), full[5_000:7_500])
    c = W.config("C2", n=20_000)
    allp = c.points()
    assert np.array_equal(c.points(n=4_000, row0=12_000), allp[12_000:16_000])
