"""CPU pins of the PSB trace model (tests/psb_model.py) before it is used to
check the GPU's traversal order (tests/test_gpu_trace.py).

The model's results must equal the oracle's brute force bit for bit, and its
walk must have the properties Alg. 1 and DESIGN.md §2 give
it: pass-2 leaf visits in strictly increasing leaf order (left-to-right scan,
P:L510-515), no leaf scanned twice, every leaf whose MINDIST <= d_k scanned
(exactness), pass-1 leaves all children of one node."""
import numpy as np
import pytest

import oracle
import psb_model as M
import workloads as W


def _psb():
    import paper_conf_icpp_namkn16_b200 as psb
    return psb


def _trees():
    rng = np.random.default_rng(7)
    lat = np.stack(np.meshgrid(np.arange(40), np.arange(40), indexing="ij"), -1).reshape(-1, 2).astype(np.float32)
    return {
        "C1": (W.config("C1").points(), W.config("C1").queries(60), 32),
        "clustered3d": (W.config("C2").points(n=20_000), W.config("C2").queries(40), 64),
        "uniform8d": (rng.random((6000, 8), dtype=np.float32), rng.random((25, 8), dtype=np.float32), 32),
        "lattice": (lat, np.array([[3, 3], [20, 21], [39, 0], [10.5, 10.5]], np.float32), 32),
    }


def check_walk(tree, q, k, steps, dists):
    """Trace properties every PSB walk must have (shared with the GPU tests)."""
    leaves = [(node, fl) for lvl, node, fl in steps if lvl == 0]
    p1 = [n for n, fl in leaves if fl & M.PASS1]
    p2 = [n for n, fl in leaves if not fl & M.PASS1]
    assert p1, "pass 1 scans at least ClosestLeaf"
    assert len({n // tree.F for n in p1}) == 1, "pass-1 leaves are children of one node"
    assert all(a < b for a, b in zip(p2, p2[1:])), "pass-2 leaves strictly increasing"
    scanned = p1 + [n for n, fl in leaves if not fl & M.PASS1 and not fl & M.SKIPPED]
    assert len(scanned) == len(set(scanned)), "no leaf scanned twice"
    skipped = {n for n, fl in leaves if fl & M.SKIPPED}
    assert skipped <= set(p1), "only pass-1 leaves are skipped"
    dk = dists[k - 1]
    need = np.nonzero(M.leaf_mindists(tree, q) <= dk)[0]
    assert set(need.tolist()) <= set(scanned), "every leaf with MINDIST <= d_k is scanned"


@pytest.mark.parametrize("name", ["C1", "clustered3d", "uniform8d", "lattice"])
@pytest.mark.parametrize("k", [1, 8, 33])
def test_model_equals_oracle_and_walk_invariants(name, k):
    psb = _psb()
    pts, qs, F = _trees()[name]
    tree = M.Tree(psb.psb_build_host_blob(pts, F))
    exp_i, exp_d = oracle.knn_bruteforce(pts, qs, k)
    for r, q in enumerate(qs):
        ids, d, steps = M.psb(tree, q, k)
        assert np.array_equal(ids, exp_i[r]) and np.array_equal(d.view(np.uint32), exp_d[r].view(np.uint32)), r
        check_walk(tree, q, k, steps, d)


def test_model_kth_rule_and_nocache_same_results():
    psb = _psb()
    pts, qs, F = _trees()["clustered3d"]
    tree = M.Tree(psb.psb_build_host_blob(pts, F))
    for q in qs[:15]:
        a = M.psb(tree, q, 16)
        b = M.psb(tree, q, 16, kth_rule=True)
        c = M.psb(tree, q, 16, use_cache=False)
        assert np.array_equal(a[0], b[0]) and np.array_equal(a[0], c[0])
        # without the path cache every internal visit is a fetch; the walk is the same
        assert [s[:2] for s in a[2]] == [s[:2] for s in c[2]]
        assert all(fl & M.FETCHED for lvl, _, fl in c[2] if lvl > 0)


def test_fig2_tree_model_walk():
    """The Fig. 2 narrative on the hand-built tree of
    tests/fig2.py, in the model: see that module for the expected walk."""
    import fig2
    tree = M.Tree(fig2.blob_dict())
    ids, d, steps = M.psb(tree, fig2.QUERY, 1)
    exp_i, exp_d = oracle.knn_bruteforce(fig2.points(), fig2.QUERY[None, :], 1)
    assert ids[0] == exp_i[0, 0] and d[0] == exp_d[0, 0]
    assert fig2.named(steps) == fig2.EXPECTED_WALK
