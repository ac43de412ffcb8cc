"""The GPU's traversal ORDER, not just its answer (psb_knn_trace, include/psb.h).

Result parity (test_gpu_parity.py) cannot tell PSB from any other exact
traversal. These tests pin Alg. 1 (§III; Fig. 2):
  - the GPU trace equals, step for step and flag for flag, the CPU walk of
    tests/psb_model.py (itself pinned against the oracle in test_trace_model.py)
    on the Fig. 2 tree and on packed trees of the configs' shapes;
  - on whole batches: pass-2 leaves strictly increasing, no leaf scanned twice,
    every leaf with MINDIST <= d_k scanned;
  - the compile-time-d kernels (the ones bench.py times) and the runtime-d
    kernels walk identically (same traces, same counters)."""
import numpy as np
import pytest

import oracle
import psb_model as M
import workloads as W

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _psb():
    import paper_conf_icpp_namkn16_b200 as psb
    return psb


def _gpu_steps(tr, tl, r):
    psb = _psb()
    return psb.trace_steps(tr[r], int(tl[r]))


def test_fig2_tree_gpu_walk_equals_narrative():
    """Fig. 2's narrative on the hand-built tree (tests/fig2.py), imported with
    psb_index_import: the GPU walks A C P G R S | A B D I J K E M N F B A C P G P R P S."""
    import fig2
    psb = _psb()
    idx = psb.psb_index_import(fig2.raw_blob())
    qd = torch.from_numpy(fig2.QUERY[None, :]).cuda()
    for variant in (0, psb.PSB_VAR_GENERIC_D):
        ids, d, st, tr, tl = psb.psb_knn_trace(idx, qd, 1, cap=256, variant=variant)
        torch.cuda.synchronize()
        steps = _gpu_steps(tr.cpu().numpy(), tl.cpu().numpy(), 0)
        assert fig2.named(steps) == fig2.EXPECTED_WALK
        exp = oracle.knn_bruteforce(fig2.points(), fig2.QUERY[None, :], 1)
        assert ids.cpu().numpy()[0, 0] == exp[0][0, 0]
    idx.free()


def test_import_round_trip_and_validation():
    psb = _psb()
    cfg = W.config("C2")
    pts = cfg.points(n=50_000)
    qs = cfg.queries(500)
    a = psb.psb_build(pts, 64)
    blob = psb.psb_index_export_raw(a)
    b = psb.psb_index_import(blob)
    assert b.info() == a.info()
    qd = torch.from_numpy(qs).cuda()
    r1, r2 = psb.psb_knn(a, qd, 32), psb.psb_knn(b, qd, 32)
    assert torch.equal(r1[0], r2[0]) and torch.equal(r1[1], r2[1])
    # a box that does not contain its leaf is rejected (exactness would break)
    bad = psb._parse_blob(blob.copy())
    bad["nodes"][1][0, 0, 0, 0] += 1.0                      # lo of dim 0, child 0 moved inward
    raw = psb.make_blob(bad["pts"], bad["ids"], bad["nodes"], bad["n"])
    with pytest.raises(psb.PSBError):
        psb.psb_index_import(raw)
    with pytest.raises(psb.PSBError):
        psb.psb_index_import(blob[:-4])
    a.free()
    b.free()


CASES = [  # name, n, query count compared with the model, k, variant
    ("C1", None, 100, 8, 0),
    ("C2", 200_000, 60, 32, 0),
    ("C3", 400_000, 12, 16, 0),
    ("C4", 300_000, 3, 64, 0),
    ("C2", 100_000, 30, 100, 0),                 # k > fanout: the k-th MAXDIST rule
    ("C2", 100_000, 30, 16, 1),                  # PSB_VAR_NOCACHE
]


@pytest.mark.parametrize("name,n,nq,k,variant", CASES)
def test_gpu_trace_equals_model(name, n, nq, k, variant):
    psb = _psb()
    cfg = W.config(name)
    pts = cfg.points(n=n) if n else cfg.points()
    qs = cfg.queries(nq)
    idx = psb.psb_build(pts, cfg.fanout)
    tree = M.Tree(psb.psb_index_export(idx))
    qd = torch.from_numpy(qs).cuda()
    ids, d, st, tr, tl = psb.psb_knn_trace(idx, qd, k, cap=8192, variant=variant)
    torch.cuda.synchronize()
    tr, tl = tr.cpu().numpy(), tl.cpu().numpy()
    ids, d = ids.cpu().numpy(), d.cpu().numpy()
    for r in range(nq):
        mi, md, steps = M.psb(tree, qs[r], k, use_cache=not (variant & 1))
        assert tl[r] <= 8192
        assert _gpu_steps(tr, tl, r) == steps, f"{name} query {r}: walk differs from the model"
        assert np.array_equal(ids[r], mi) and np.array_equal(d[r].view(np.uint32), md.view(np.uint32))
    idx.free()


def _walk_invariants(tree_F, tr, tl, ids_k_d, leaf_md_fn=None):
    """Vectorisable checks on whole batches (no model): see module docstring."""
    for r in range(len(tl)):
        steps = _gpu_steps(tr, tl, r)
        leaves = [(node, fl) for lvl, node, fl in steps if lvl == 0]
        p1 = [n for n, fl in leaves if fl & M.PASS1]
        p2 = [n for n, fl in leaves if not fl & M.PASS1]
        assert p1 and len({n // tree_F for n in p1}) == 1
        assert all(a < b for a, b in zip(p2, p2[1:])), f"query {r}: pass-2 leaves not increasing"
        scanned = p1 + [n for n, fl in leaves if not fl & M.PASS1 and not fl & M.SKIPPED]
        assert len(scanned) == len(set(scanned)), f"query {r}: a leaf scanned twice"
        if leaf_md_fn is not None:
            need = np.nonzero(leaf_md_fn(r) <= ids_k_d[r])[0]
            assert set(need.tolist()) <= set(scanned), f"query {r}: a leaf with MINDIST <= d_k was not scanned"


def test_c2_full_batch_walk_invariants():
    """All 10^4 C2 queries at full size (the bench launch): every walk has the
    PSB properties; on 300 of them, every leaf with MINDIST <= d_k was scanned."""
    psb = _psb()
    cfg = W.config("C2")
    pts = cfg.points()
    qs = cfg.queries()
    idx = psb.psb_build(pts, cfg.fanout)
    qd = torch.from_numpy(qs).cuda()
    ids, d, st, tr, tl = psb.psb_knn_trace(idx, qd, cfg.k, cap=2048)
    torch.cuda.synchronize()
    tr, tl, d = tr.cpu().numpy(), tl.cpu().numpy(), d.cpu().numpy()
    assert (tl <= 2048).all()
    # the counters agree with the trace: leaf scans = scanned leaf steps
    stn = st.cpu().numpy()
    scans = [sum(1 for lvl, _, fl in _gpu_steps(tr, tl, r) if lvl == 0 and not fl & M.SKIPPED) for r in range(200)]
    assert np.array_equal(stn[:200, 1], scans)
    _walk_invariants(cfg.fanout, tr, tl, d[:, -1])
    tree = M.Tree(psb.psb_index_export(idx))
    sub = np.arange(0, len(qs), len(qs) // 300)
    _walk_invariants(cfg.fanout, tr[sub], tl[sub], d[sub, -1], lambda r: M.leaf_mindists(tree, qs[sub[r]]))
    idx.free()


@pytest.mark.parametrize("name,nq", [("C2", 10_000), ("C3", 3000), ("C4", 300), ("C5", 3000)])
def test_specialised_and_generic_kernels_walk_identically(name, nq):
    """The compile-time-d kernel (timed by bench.py; its counters give the
    roofline's algorithmic bytes) and the runtime-d kernel take the same steps
    for every query: traces and counters equal, rows equal."""
    psb = _psb()
    cfg = W.config(name)
    pts = cfg.points(n=64_000_000 // 8) if name == "C5" else cfg.points()
    qs = cfg.queries(nq)
    idx = psb.psb_build(pts, cfg.fanout)
    qd = torch.from_numpy(qs).cuda()
    a = psb.psb_knn_trace(idx, qd, cfg.k, cap=4096)
    b = psb.psb_knn_trace(idx, qd, cfg.k, cap=4096, variant=psb.PSB_VAR_GENERIC_D)
    torch.cuda.synchronize()
    for x, y in zip(a[:2], b[:2]):
        assert torch.equal(x, y)
    assert torch.equal(a[2][:, :6], b[2][:, :6])            # counters (not the timestamps)
    assert torch.equal(a[4], b[4])
    m = min(4096, int(a[4].max()))
    assert torch.equal(a[3][:, :m], b[3][:, :m])
    idx.free()
