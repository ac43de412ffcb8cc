"""GPU parity: libpsb.so (through its C ABI via the thin binding) vs the CPU oracle.

Bar (north_star): bit-exact ids AND bit-exact binary32 squared
distances for every query compared. Small configs compare every query; the
full BASELINE.json sizes compare every query against the oracle's B&B (itself
pinned to the oracle's brute force) or a stated sample against brute force.
"""
import numpy as np
import pytest

import oracle
import workloads as W

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ALGOS = ("psb", "bnb", "brute")


def _psb():
    import paper_conf_icpp_namkn16_b200 as psb
    return psb


def run(idx, qs, k, algo="psb", variant=0):
    psb = _psb()
    a = {"psb": psb.PSB_ALGO_PSB, "bnb": psb.PSB_ALGO_BNB, "brute": psb.PSB_ALGO_BRUTE}[algo]
    qd = torch.from_numpy(np.ascontiguousarray(qs, np.float32)).cuda()
    ids, d = psb.psb_knn_ex(idx, qd, k, algo=a, variant=variant)
    torch.cuda.synchronize()
    return ids.cpu().numpy(), d.cpu().numpy()


def assert_same(got, exp, what=""):
    gi, gd = got
    ei, ed = exp
    bad = np.nonzero((gi != ei).any(1) | (gd.view(np.uint32) != ed.view(np.uint32)).any(1))[0]
    if len(bad):
        r = bad[0]
        raise AssertionError(f"{what}: {len(bad)} rows differ; first row {r}:\n gpu ids {gi[r][:12]}\n"
                             f" exp ids {ei[r][:12]}\n gpu d {gd[r][:6]}\n exp d {ed[r][:6]}")


@pytest.fixture(scope="module")
def c1():
    cfg = W.config("C1")
    pts, qs = cfg.points(), cfg.queries()
    idx = _psb().psb_build(pts, cfg.fanout)
    exp = oracle.knn_bruteforce(pts, qs, cfg.k)
    yield cfg, pts, qs, idx, exp
    idx.free()


@pytest.mark.parametrize("algo", ALGOS)
def test_c1_all_queries(c1, algo):
    cfg, pts, qs, idx, exp = c1
    assert_same(run(idx, qs, cfg.k, algo), exp, f"C1 {algo}")


@pytest.mark.parametrize("variant", [1, 2, 3, 16, 32, 64, 65, 66, 128, 129, 192, 256, 304])
@pytest.mark.parametrize("algo", ["psb", "bnb"])
def test_c1_variants(c1, algo, variant):
    cfg, pts, qs, idx, exp = c1
    assert_same(run(idx, qs, cfg.k, algo, variant), exp, f"C1 {algo} var{variant}")


@pytest.mark.parametrize("k", [1, 2, 31, 32, 33, 64, 65, 100, 128])
def test_c1_k_sweep(c1, k):
    cfg, pts, qs, idx, _ = c1
    exp = oracle.knn_bruteforce(pts, qs, k)
    for algo in ALGOS:
        assert_same(run(idx, qs, k, algo), exp, f"C1 k={k} {algo}")


@pytest.fixture(scope="module")
def c2():
    cfg = W.config("C2")
    pts, qs = cfg.points(), cfg.queries()
    idx = _psb().psb_build(pts, cfg.fanout)
    tree = oracle.Tree(pts)
    exp = tree.knn(qs, cfg.k)
    yield cfg, pts, qs, idx, exp
    idx.free()


def test_c2_oracle_routes_agree_on_sample(c2):
    cfg, pts, qs, idx, exp = c2
    s = np.arange(0, cfg.q, 97)
    bf = oracle.knn_bruteforce(pts, qs[s], cfg.k)
    assert_same(bf, (exp[0][s], exp[1][s]), "oracle brute vs oracle bnb")


@pytest.mark.parametrize("algo", ALGOS)
def test_c2_full_all_queries(c2, algo):
    """BASELINE.json configs[1]: 3-D clustered n=1M F=64 q=10^4 k=32, every query,
    in the launch configuration bench.py times."""
    cfg, pts, qs, idx, exp = c2
    assert_same(run(idx, qs, cfg.k, algo), exp, f"C2 {algo}")


def test_c2_nocache_and_batches(c2):
    cfg, pts, qs, idx, exp = c2
    sl = slice(0, 3000)
    assert_same(run(idx, qs[sl], cfg.k, "psb", 1), (exp[0][sl], exp[1][sl]), "C2 psb nocache")
    # pass 1 with the index-only ClosestLeaf tie-break, and with the L1 prefetches
    assert_same(run(idx, qs[sl], cfg.k, "psb", 64), (exp[0][sl], exp[1][sl]), "C2 psb index tie")
    assert_same(run(idx, qs[sl], cfg.k, "psb", 16 | 32), (exp[0][sl], exp[1][sl]), "C2 psb prefetch")
    # the paper's k-th smallest MAXDIST bound instead of the count-aware one
    assert_same(run(idx, qs[sl], cfg.k, "psb", 128), (exp[0][sl], exp[1][sl]), "C2 psb k-th MAXDIST")
    assert_same(run(idx, qs[sl], cfg.k, "bnb", 128), (exp[0][sl], exp[1][sl]), "C2 bnb k-th MAXDIST")
    # batching/order independence: single queries and a reversed batch
    for i in (0, 17, 4999):
        assert_same(run(idx, qs[i:i + 1], cfg.k), (exp[0][i:i + 1], exp[1][i:i + 1]), "C2 single")
    r = run(idx, qs[::-1][:2000], cfg.k)
    assert_same(r, (exp[0][::-1][:2000], exp[1][::-1][:2000]), "C2 reversed")


@pytest.mark.parametrize("algo", ["psb", "bnb"])
def test_c2_query_order_independent(c2, algo):
    """Batch scheduling (closest-leaf order, default for >= 1024 queries) and input
    order return the same rows, both equal to the oracle; also a ragged batch just
    above the reorder threshold and one with duplicated queries."""
    psb = _psb()
    cfg, pts, qs, idx, exp = c2
    sl = slice(0, 5000)
    assert_same(run(idx, qs[sl], cfg.k, algo, psb.PSB_VAR_INPUT_ORDER), (exp[0][sl], exp[1][sl]), "input order")
    lo = psb.PSB_VAR_LEAF_ORDER
    assert_same(run(idx, qs[sl], cfg.k, algo, lo), (exp[0][sl], exp[1][sl]), "leaf order")
    assert_same(run(idx, qs[sl], cfg.k, algo, lo | 1), (exp[0][sl], exp[1][sl]), "leaf order, no cache")
    sel = np.r_[np.arange(1025), np.arange(7)]          # 1032 queries, 7 repeated
    assert_same(run(idx, qs[sel], cfg.k, algo, lo), (exp[0][sel], exp[1][sel]), "ragged + duplicates")
    assert_same(run(idx, qs[:3], cfg.k, algo, lo), (exp[0][:3], exp[1][:3]), "tiny batch")


def test_query_order_generic_d_and_sphere():
    """The reorder pre-pass on the runtime-d kernels (d=5) and on sphere nodes."""
    psb = _psb()
    rng = np.random.default_rng(7)
    pts = rng.random((60000, 5), dtype=np.float32)
    qs = rng.random((1500, 5), dtype=np.float32)
    exp = oracle.knn_bruteforce(pts, qs, 10)
    for flags in (0, psb.PSB_NODE_SPHERE):
        idx = psb.psb_build_ex(pts, 64, packing=flags)
        for algo in ("psb", "bnb"):
            assert_same(run(idx, qs, 10, algo, psb.PSB_VAR_LEAF_ORDER), exp, f"d=5 flags={flags} {algo}")
        idx.free()


def test_c3_full_batch_sampled():
    """configs[2]: 8-D uniform n=4M F=128 k=16, the bench's default workload, in the
    launch configuration bench.py times (all 10^5 queries in one launch: closest-leaf
    order, persistent grid); 2,000 rows spread over the batch against the oracle's
    B&B, 40 against its brute force."""
    cfg = W.config("C3")
    pts = cfg.points()
    qs = cfg.queries()
    idx = _psb().psb_build(pts, cfg.fanout)
    sub = np.arange(0, len(qs), len(qs) // 2000)
    exp = oracle.Tree(pts).knn(qs[sub], cfg.k)
    for algo in ("psb", "bnb"):
        gi, gd = run(idx, qs, cfg.k, algo)
        assert_same((gi[sub], gd[sub]), exp, f"C3 {algo} (full batch)")
    gi, gd = run(idx, qs[:2000], cfg.k, "brute")
    assert_same((gi[sub[sub < 2000]], gd[sub[sub < 2000]]), (exp[0][: (sub < 2000).sum()], exp[1][: (sub < 2000).sum()]),
                "C3 brute")
    bf = oracle.knn_bruteforce(pts, qs[sub[:40]], cfg.k)
    gi, gd = run(idx, qs, cfg.k)
    assert_same((gi[sub[:40]], gd[sub[:40]]), bf, "C3 psb vs oracle brute")
    idx.free()


def test_c4_full_batch_all_rows():
    """configs[3]: 16-D clustered n=16M F=128 k=64, in the launch configuration
    bench.py times: all 10^4 queries in one launch, in closest-leaf order; every row
    against the oracle's B&B (PSB and B&B; brute force on 200 queries)."""
    cfg = W.config("C4")
    pts = cfg.points()
    qs = cfg.queries()
    idx = _psb().psb_build(pts, cfg.fanout)
    exp = oracle.Tree(pts).knn(qs, cfg.k)
    for algo in ("psb", "bnb"):
        assert_same(run(idx, qs, cfg.k, algo), exp, f"C4 {algo} (full batch)")
    assert_same(run(idx, qs[:200], cfg.k, "brute"), (exp[0][:200], exp[1][:200]), "C4 brute")
    # the batch split into interleaved-node parts (auto: 2-8 parts per query)
    si, sd = _psb().psb_knn_split(idx, torch.from_numpy(qs).cuda(), cfg.k, parts=0)
    torch.cuda.synchronize()
    assert_same((si.cpu().numpy(), sd.cpu().numpy()), exp, "C4 psb split (full batch)")
    idx.free()


def test_c5_slab_full_batch_sampled():
    """configs[4], one GPU's share of the data-sharded C5: slab 0 of 8 (64M 3-D
    uniform points, ids 0..64M-1), F=128, k=32, in the launch configuration bench.py
    times (all 10^6 queries in one launch); 2,000 rows spread over the batch against
    the oracle's B&B over the same slab."""
    cfg = W.config("C5")
    n = cfg.n // 8
    pts = cfg.points(n=n, row0=0)
    qs = cfg.queries()
    idx = _psb().psb_build_ex(pts, cfg.fanout, id_base=0)
    sub = np.arange(0, len(qs), len(qs) // 2000)
    exp = oracle.Tree(pts).knn(qs[sub], cfg.k)
    for algo in ("psb", "bnb"):
        gi, gd = run(idx, qs, cfg.k, algo)
        assert_same((gi[sub], gd[sub]), exp, f"C5 slab {algo} (full batch)")
    idx.free()


@pytest.mark.parametrize("d,n", [(2, 9_000_000), (4, 4_000_000)])
def test_hilbert_batch_order_low_d(d, n):
    """Large batches at d <= 4 are ordered by the queries' Hilbert key (knn_order.cu):
    leaves above 64 MiB and >= 1,024 queries, so the d = 2 (16 bits per axis) and
    d = 4 (8 bits) key paths run; rows equal to the oracle, and to the closest-leaf
    order (PSB_VAR_LEAF_ORDER) and the input order, for PSB and B&B."""
    psb = _psb()
    pts = W.gen_uniform(n, d, 0xB0 + d)
    qs = W.gen_uniform(4000, d, 0xB1 + d)
    qs[:50] = qs[:50] * 3.0 - 1.0                     # some queries outside the data's box
    idx = psb.psb_build(pts, 64)
    sub = np.arange(0, 4000, 20)
    exp = oracle.knn_bruteforce(pts, qs[sub], 16)
    for algo in ("psb", "bnb"):
        got = run(idx, qs, 16, algo)
        assert_same((got[0][sub], got[1][sub]), exp, f"d={d} {algo} Hilbert order")
        for var in (psb.PSB_VAR_LEAF_ORDER, psb.PSB_VAR_INPUT_ORDER):
            other = run(idx, qs, 16, algo, var)
            assert np.array_equal(other[0], got[0]) and np.array_equal(other[1].view(np.uint32), got[1].view(np.uint32))
    idx.free()


def test_ctx_paper_shape_all_rows():
    """SURVEY §8(d) "ctx": the paper's experiment shape (64-D clustered, n=10^6,
    F=128, 240 queries, k=32; runtime-d kernels), every row of PSB, PSB latency
    mode, B&B and brute force against the oracle's brute force."""
    psb = _psb()
    cfg = W.config("CTX")
    pts, qs = cfg.points(), cfg.queries()
    idx = psb.psb_build(pts, cfg.fanout)
    exp = oracle.knn_bruteforce(pts, qs, cfg.k)
    for algo in ("psb", "bnb", "brute"):
        assert_same(run(idx, qs, cfg.k, algo), exp, f"CTX {algo}")
    si, sd = psb.psb_knn_split(idx, torch.from_numpy(qs).cuda(), cfg.k, parts=0)
    torch.cuda.synchronize()
    assert_same((si.cpu().numpy(), sd.cpu().numpy()), exp, "CTX psb split (auto)")
    idx.free()


@pytest.mark.parametrize("case", [
    dict(n=1, d=2, F=32, k=4), dict(n=31, d=3, F=32, k=40), dict(n=33, d=3, F=32, k=33),
    dict(n=1000, d=1, F=32, k=10), dict(n=5000, d=5, F=64, k=20), dict(n=3000, d=64, F=32, k=9),
    dict(n=20000, d=4, F=256, k=50), dict(n=20000, d=3, F=512, k=128), dict(n=70000, d=2, F=32, k=7),
    dict(n=4097, d=16, F=128, k=64), dict(n=1500, d=7, F=128, k=1)])
def test_edge_shapes(case):
    rng = np.random.default_rng(case["n"] * 7 + case["d"])
    pts = (rng.normal(size=(case["n"], case["d"])) * 30).astype(np.float32)
    qs = (rng.normal(size=(64, case["d"])) * 35).astype(np.float32)
    idx = _psb().psb_build(pts, case["F"])
    exp = oracle.knn_bruteforce(pts, qs, case["k"])
    for algo in ALGOS:
        assert_same(run(idx, qs, case["k"], algo), exp, f"{case} {algo}")
    idx.free()


@pytest.mark.parametrize("kind", ["lattice", "dups", "identical"])
def test_tie_heavy(kind):
    rng = np.random.default_rng(4)
    if kind == "lattice":
        g = np.stack(np.meshgrid(np.arange(60), np.arange(60), indexing="ij"), -1).reshape(-1, 2)
        pts = g.astype(np.float32)
        qs = rng.integers(0, 60, size=(100, 2)).astype(np.float32)
    elif kind == "dups":
        base = rng.integers(0, 5, size=(40, 3)).astype(np.float32)
        pts = base[rng.integers(0, 40, size=5000)]
        qs = rng.integers(0, 5, size=(100, 3)).astype(np.float32)
    else:
        pts = np.ones((3000, 3), np.float32)
        qs = rng.normal(size=(50, 3)).astype(np.float32)
    idx = _psb().psb_build(pts, 32)
    for k in (1, 13, 64, 128):
        exp = oracle.knn_bruteforce(pts, qs, k)
        for algo in ALGOS:
            assert_same(run(idx, qs, k, algo), exp, f"{kind} k={k} {algo}")
    idx.free()


@pytest.mark.parametrize("sphere", [False, True])
def test_fma_case_on_gpu(sphere):
    import json, os
    psb = _psb()
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "hand_cases.json")))["fma_case"]
    p = np.array([[float.fromhex(v) for v in g["point"]]] * 40, np.float32)
    q = np.array([[float.fromhex(v) for v in g["query"]]], np.float32)
    idx = psb.psb_build_ex(p, 32, packing=psb.PSB_NODE_SPHERE if sphere else 0)
    for algo in (ALGOS if not sphere else ("psb", "bnb")):
        ids, d = run(idx, q, 1, algo)
        assert int(d.view(np.uint32)[0, 0]) == int(g["rn_bits"], 16)
    idx.free()


def test_hand_cases_on_gpu():
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "hand_cases.json")))
    for c in g["cases"]:
        P = np.array(c["points"], np.float32)
        idx = _psb().psb_build(P, 32)
        for algo in ALGOS:
            ids, d = run(idx, np.array([c["query"]], np.float32), c["k"], algo)
            assert ids[0].tolist() == c["ids"], (c["name"], algo)
            assert d[0].tolist() == [float("inf") if v == "inf" else float(v) for v in c["dists"]]
        idx.free()


def test_packing_and_fanout_invariance():
    cfg = W.config("C2")
    pts = cfg.points(n=200_000)
    qs = cfg.queries(q=500)
    exp = oracle.knn_bruteforce(pts, qs, 32)
    psb = _psb()
    for F in (32, 64, 128, 256):
        for pack in (psb.PSB_PACK_HILBERT, psb.PSB_PACK_STR):
            idx = psb.psb_build_ex(pts, F, packing=pack)
            assert_same(run(idx, qs, 32), exp, f"F={F} pack={pack}")
            idx.free()


def test_export_matches_host_blob():
    psb = _psb()
    pts = W.gen_uniform(5000, 3, 12)
    idx = psb.psb_build_ex(pts, 64, id_base=5)
    a = psb.psb_index_export(idx)
    b = psb.psb_build_host_blob(pts, 64, id_base=5)
    assert np.array_equal(a["pts"], b["pts"]) and np.array_equal(a["ids"], b["ids"])
    for lv in a["nodes"]:
        assert np.array_equal(a["nodes"][lv], b["nodes"][lv])
    # device input for psb_build_ex gives the same index
    idx2 = psb.psb_build_ex(torch.from_numpy(pts).cuda(), 64, id_base=5)
    c = psb.psb_index_export(idx2)
    assert np.array_equal(a["pts"], c["pts"]) and np.array_equal(a["ids"], c["ids"])
    idx.free()
    idx2.free()


def test_data_sharded_merge_equals_unsharded():
    """Data-sharded mode on one GPU: P sub-trees over slabs (global ids via
    id_base), local kNN on each, psb_merge_topk -> identical to unsharded/oracle."""
    psb = _psb()
    cfg = W.config("C2")
    pts = cfg.points(n=300_000)
    qs = cfg.queries(q=2000)
    exp = oracle.Tree(pts).knn(qs, 32)
    qd = torch.from_numpy(qs).cuda()
    for P in (2, 3, 8):
        bounds = [len(pts) * r // P for r in range(P + 1)]
        ids = torch.empty((P, len(qs), 32), dtype=torch.int32, device="cuda")
        ds = torch.empty((P, len(qs), 32), dtype=torch.float32, device="cuda")
        for r in range(P):
            sub = psb.psb_build_ex(pts[bounds[r]:bounds[r + 1]], 64, id_base=bounds[r])
            psb.psb_knn(sub, qd, 32, out=(ids[r], ds[r]))
            torch.cuda.synchronize()
            sub.free()
        mi, md = psb.psb_merge_topk(ids, ds, 32)
        torch.cuda.synchronize()
        assert_same((mi.cpu().numpy(), md.cpu().numpy()), exp, f"sharded P={P}")


def test_error_codes_on_gpu():
    psb = _psb()
    pts = W.gen_uniform(100, 2, 1)
    idx = psb.psb_build(pts, 32)
    qd = torch.zeros((4, 2), device="cuda")
    with pytest.raises(psb.PSBError) as e:
        psb.psb_knn(idx, qd, 0)
    assert e.value.code == psb.PSB_EINVAL
    with pytest.raises(psb.PSBError) as e:
        psb.psb_knn(idx, qd, psb.PSB_KMAX + 1)
    assert e.value.code == psb.PSB_EUNSUPPORTED
    # q = 0 is a no-op
    ids, d = psb.psb_knn(idx, torch.zeros((0, 2), device="cuda"), 5)
    assert ids.shape == (0, 5)
    with pytest.raises(psb.PSBError):
        psb.psb_build(np.full((10, 2), np.inf, np.float32), 32)
    idx.free()


def test_pinned_queries_read_in_place(c2):
    """Pinned host queries are read by the kernels in place (zero-copy, include/psb.h),
    also through an interior pointer of a larger pinned tensor, and also by the
    closest-leaf pre-pass of a reordered batch; split mode and brute force stage them.
    Every route returns the oracle's rows into pinned and device outputs."""
    psb = _psb()
    cfg, pts, qs, idx, exp = c2
    big = torch.from_numpy(qs[:3000].copy()).pin_memory()
    sl = slice(517, 2517)                        # interior pointer, 2,000 queries
    hq = big[sl]
    e = (exp[0][sl], exp[1][sl])
    hi = torch.empty((2000, cfg.k), dtype=torch.int32, pin_memory=True)
    hd = torch.empty((2000, cfg.k), dtype=torch.float32, pin_memory=True)
    di = torch.empty((2000, cfg.k), dtype=torch.int32, device="cuda")
    dd = torch.empty((2000, cfg.k), dtype=torch.float32, device="cuda")
    calls = {
        "psb": lambda o: psb.psb_knn(idx, hq, cfg.k, out=o),
        "psb leaf order": lambda o: psb.psb_knn_ex(idx, hq, cfg.k, variant=psb.PSB_VAR_LEAF_ORDER, out=o),
        "bnb": lambda o: psb.psb_knn_branch_and_bound(idx, hq, cfg.k, out=o),
        "split 4": lambda o: psb.psb_knn_split(idx, hq, cfg.k, parts=4, out=o),
        "brute": lambda o: psb.psb_knn_bruteforce(idx, hq, cfg.k, out=o),
    }
    for name, call in calls.items():
        for o in ((hi, hd), (di, dd)):
            o[0].fill_(-7)
            ids, d = call(o)
            torch.cuda.synchronize()
            assert_same((ids.cpu().numpy(), d.cpu().numpy()), e, f"pinned queries, {name}, out on {o[0].device}")
    # a batch above the zero-copy limit (16,384 queries): staged with one copy
    big2 = torch.from_numpy(np.concatenate([qs, qs])).pin_memory()
    ids, d = psb.psb_knn(idx, big2, cfg.k)
    torch.cuda.synchronize()
    assert_same((ids.numpy(), d.numpy()), (np.concatenate([exp[0], exp[0]]), np.concatenate([exp[1], exp[1]])),
                "pinned queries above the zero-copy limit")
    # one query at a time (the latency path): interior pointers of one row
    for r in (0, 1, 999):
        ids, d = psb.psb_knn(idx, hq[r:r + 1], cfg.k, out=(hi[:1], hd[:1]))
        assert np.array_equal(ids.numpy()[0], e[0][r]) and np.array_equal(d.numpy()[0].view(np.uint32),
                                                                          e[1][r].view(np.uint32))


def test_host_buffers_and_stats(c2):
    """Host (pinned and pageable) buffers through the C ABI give identical rows;
    the instrumented entry point changes nothing and its counters are sane."""
    psb = _psb()
    cfg, pts, qs, idx, exp = c2
    sl = slice(0, 2000)
    e = (exp[0][sl], exp[1][sl])
    hq = torch.from_numpy(qs[sl].copy()).pin_memory()
    ids, d = psb.psb_knn(idx, hq, cfg.k)
    torch.cuda.synchronize()
    assert not ids.is_cuda
    assert_same((ids.numpy(), d.numpy()), e, "pinned host buffers")
    ids, d = psb.psb_knn(idx, torch.from_numpy(qs[sl].copy()), cfg.k,
                         out=(torch.empty((2000, cfg.k), dtype=torch.int32),
                              torch.empty((2000, cfg.k), dtype=torch.float32)))
    torch.cuda.synchronize()
    assert_same((ids.numpy(), d.numpy()), e, "pageable host buffers")
    qd = torch.from_numpy(qs[sl].copy()).cuda()
    for algo in (psb.PSB_ALGO_PSB, psb.PSB_ALGO_BNB):
        got = []
        for var in (0, 1):
            i, dd, st = psb.psb_knn_stats(idx, qd, cfg.k, algo=algo, variant=var)
            torch.cuda.synchronize()
            assert_same((i.cpu().numpy(), dd.cpu().numpy()), e, f"stats algo={algo} var={var}")
            st = st.cpu().numpy()
            assert (st[:, 7] >= st[:, 6]).all() and (st[:, 6] > 0).all()   # service-time stamps
            st = st[:, :6]
            assert (st[:, 1] >= 1).all()                 # every query scans a leaf
            assert (st[:, 0] >= idx.levels).all()        # and fetches at least one root-to-leaf path
            got.append(st)
        i2, _, st2 = psb.psb_knn_stats(idx, qd, cfg.k, algo=algo)
        torch.cuda.synchronize()
        assert np.array_equal(st2.cpu().numpy()[:, :6], got[0])          # deterministic
        _, _, st3 = psb.psb_knn_stats(idx, qd, cfg.k, algo=algo, variant=psb.PSB_VAR_LEAF_ORDER)
        torch.cuda.synchronize()
        assert np.array_equal(st3.cpu().numpy()[:, :6], got[0])          # same traversal in any query order
        assert (got[1][:, 3] == 0).all()                           # no cache -> no hits
        assert np.array_equal(got[0][:, 0] + got[0][:, 3], got[1][:, 0])  # same visits, cache or not
        assert np.array_equal(got[0][:, 1], got[1][:, 1])          # same leaves scanned
        assert (got[0][:, 4] <= got[0][:, 1]).all() and (got[0][:, 5] >= got[0][:, 4]).all()


@pytest.mark.parametrize("case", [
    dict(n=200_000, d=3, F=64, dist="clustered"), dict(n=1, d=2, F=32, dist="uniform"),
    dict(n=5_001, d=1, F=32, dist="uniform"), dict(n=3_000, d=64, F=512, dist="uniform"),
    dict(n=100_003, d=16, F=128, dist="clustered"), dict(n=70_000, d=8, F=256, dist="uniform"),
    dict(n=20_000, d=5, F=32, dist="dups")])
def test_gpu_bulk_load_matches_host_loader(case):
    """NEXT-1: the GPU loader (Hilbert keys, CUB radix sort, permutation, MBR
    levels) builds the same index as the host loader, for host and device input."""
    psb = _psb()
    n, d, F = case["n"], case["d"], case["F"]
    if case["dist"] == "uniform":
        pts = W.gen_uniform(n, d, 77)
    elif case["dist"] == "clustered":
        pts = W.gen_clustered(n, d, 78)
    else:
        base = np.random.default_rng(1).integers(0, 6, size=(50, d)).astype(np.float32)
        pts = base[np.random.default_rng(2).integers(0, 50, size=n)]
    ref = psb.psb_build_host_blob(pts, F, id_base=11)
    for src in (pts, torch.from_numpy(pts).cuda()):
        idx = psb.psb_build_ex(src, F, id_base=11)
        got = psb.psb_index_export(idx)
        idx.free()
        assert np.array_equal(got["ids"], ref["ids"])
        assert np.array_equal(got["pts"], ref["pts"])
        for lv in ref["nodes"]:
            assert np.array_equal(got["nodes"][lv], ref["nodes"][lv]), lv
    host = psb.psb_build_ex(pts, F, id_base=11, packing=psb.PSB_BUILD_HOST)
    assert np.array_equal(psb.psb_index_export(host)["ids"], ref["ids"])
    host.free()


@pytest.mark.parametrize("nq,parts", [(1, 0), (1, 7), (3, 64), (64, 0), (1000, 2), (200, 1),
                                      (5000, 2), (8000, 5), (9000, 8)])
def test_split_latency_mode(c2, nq, parts):
    """psb_knn_split (each query over `parts` warps, shared pruning distance,
    filtered merge) returns exactly psb_knn's rows, in both ownership modes:
    contiguous leaf ranges (few tasks) and interleaved level-1 nodes (the last
    three cases fill the GPU with (query, part) tasks)."""
    psb = _psb()
    cfg, pts, qs, idx, exp = c2
    sl = slice(100, 100 + nq)
    ids, d = psb.psb_knn_split(idx, torch.from_numpy(qs[sl].copy()).cuda(), cfg.k, parts=parts)
    torch.cuda.synchronize()
    assert_same((ids.cpu().numpy(), d.cpu().numpy()), (exp[0][sl], exp[1][sl]), f"split nq={nq} parts={parts}")


@pytest.mark.parametrize("case", [dict(n=5, d=3, F=32, k=8, parts=4), dict(n=40_000, d=16, F=128, k=100, parts=0),
                                  dict(n=30_000, d=5, F=64, k=1, parts=13), dict(n=9_000, d=2, F=32, k=64, parts=300)])
def test_split_edges(case):
    psb = _psb()
    rng = np.random.default_rng(case["n"])
    pts = (rng.normal(size=(case["n"], case["d"])) * 10).astype(np.float32)
    qs = (rng.normal(size=(5, case["d"])) * 12).astype(np.float32)
    idx = psb.psb_build(pts, case["F"])
    ids, d = psb.psb_knn_split(idx, torch.from_numpy(qs).cuda(), case["k"], parts=case["parts"])
    torch.cuda.synchronize()
    assert_same((ids.cpu().numpy(), d.cpu().numpy()), oracle.knn_bruteforce(pts, qs, case["k"]), str(case))
    idx.free()


@pytest.mark.parametrize("cfgname,nsub,nq", [("C1", None, 100), ("C2", 300_000, 2000), ("C3", 500_000, 300),
                                             ("C4", 400_000, 100)])
def test_sphere_index_parity(cfgname, nsub, nq):
    """NEXT-2 SS-tree variant: sphere nodes (parallel Ritter, conservative radii,
    directed-rounding bounds) give exactly the oracle's rows with PSB, B&B and
    the latency mode."""
    psb = _psb()
    cfg = W.config(cfgname) if nsub is None else W.config(cfgname, n=nsub)
    pts, qs = cfg.points(), cfg.queries(q=nq)
    idx = psb.psb_build_ex(pts, cfg.fanout, packing=psb.PSB_NODE_SPHERE)
    exp = oracle.Tree(pts).knn(qs, cfg.k)
    for algo in ("psb", "bnb"):
        for var in (0, 1):
            assert_same(run(idx, qs, cfg.k, algo, var), exp, f"sphere {cfgname} {algo} var{var}")
    ids, d = psb.psb_knn_split(idx, torch.from_numpy(qs[:8].copy()).cuda(), cfg.k, parts=32)
    torch.cuda.synchronize()
    assert_same((ids.cpu().numpy(), d.cpu().numpy()), (exp[0][:8], exp[1][:8]), "sphere split")
    idx.free()


@pytest.mark.parametrize("case", [dict(n=1, d=2, F=32), dict(n=5_000, d=1, F=32), dict(n=20_000, d=64, F=64),
                                  dict(n=33_333, d=7, F=256), dict(n=10_000, d=3, F=32, dups=True)])
def test_sphere_containment_and_parity(case):
    """Every point lies inside its leaf's sphere and every child sphere inside its
    parent's, checked in float64 on the exported index; and results are exact."""
    psb = _psb()
    rng = np.random.default_rng(case["n"] + case["d"])
    if case.get("dups"):
        pts = rng.integers(0, 4, size=(case["n"], case["d"])).astype(np.float32)
    else:
        pts = (rng.normal(size=(case["n"], case["d"])) * 20).astype(np.float32)
    idx = psb.psb_build_ex(pts, case["F"], packing=psb.PSB_NODE_SPHERE)
    ex = psb.psb_index_export(idx)
    assert ex["sphere"]
    F, d, L = ex["fanout"], ex["d"], ex["leaves"]
    lv1 = ex["nodes"][1]
    for j in range(L):
        c = lv1[j // F, :d, j % F].astype(np.float64)
        r = float(lv1[j // F, d, j % F])
        cnt = min(F, ex["n"] - j * F)
        P = ex["pts"][j, :, :cnt].T.astype(np.float64)
        assert (np.sqrt(((P - c) ** 2).sum(1)) <= r).all()
    for lv in range(2, ex["levels"] + 1):
        below, cur = ex["nodes"][lv - 1], ex["nodes"][lv]
        for g in range(below.shape[0]):
            pc = cur[g // F, :d, g % F].astype(np.float64)
            pr = float(cur[g // F, d, g % F])
            cnt = min(F, ex["nlev"][lv - 2] - g * F)
            cc = below[g, :d, :cnt].T.astype(np.float64)
            cr = below[g, d, :cnt].astype(np.float64)
            assert (np.sqrt(((cc - pc) ** 2).sum(1)) + cr <= pr * (1 + 1e-6) + 1e-6).all()
    qs = (rng.normal(size=(40, case["d"])) * 25).astype(np.float32)
    for k in (1, 17, 64):
        exp = oracle.knn_bruteforce(pts, qs, k)
        for algo in ("psb", "bnb"):
            assert_same(run(idx, qs, k, algo), exp, f"{case} k={k} {algo}")
    idx.free()


@pytest.mark.parametrize("k", [129, 200, 512, 1000, 2048])
def test_large_k(c2, k):
    """NEXT-3: k > 128 (shared-memory kNN list, in-place merge insertion) for
    PSB, B&B, brute force (with its chunk merge) and the split entry point."""
    psb = _psb()
    cfg, pts, qs, idx, _ = c2
    sub = qs[:40]
    exp = oracle.Tree(pts).knn(sub, k)
    for algo in ALGOS:
        assert_same(run(idx, sub, k, algo), exp, f"k={k} {algo}")
    ids, d = psb.psb_knn_split(idx, torch.from_numpy(sub[:4].copy()).cuda(), k)
    torch.cuda.synchronize()
    assert_same((ids.cpu().numpy(), d.cpu().numpy()), (exp[0][:4], exp[1][:4]), f"k={k} split")


def test_large_k_small_n_and_merge():
    psb = _psb()
    rng = np.random.default_rng(8)
    pts = rng.integers(0, 7, size=(700, 3)).astype(np.float32)    # ties everywhere, k > n
    qs = rng.integers(0, 7, size=(20, 3)).astype(np.float32)
    idx = psb.psb_build(pts, 32)
    exp = oracle.knn_bruteforce(pts, qs, 1000)
    for algo in ALGOS:
        assert_same(run(idx, qs, 1000, algo), exp, f"k>n {algo}")
    # data-sharded merge with large k
    b = [0, 250, 700]
    ids = torch.empty((2, 20, 300), dtype=torch.int32, device="cuda")
    ds = torch.empty((2, 20, 300), dtype=torch.float32, device="cuda")
    for r in range(2):
        sub = psb.psb_build_ex(pts[b[r]:b[r + 1]], 32, id_base=b[r])
        psb.psb_knn(sub, torch.from_numpy(qs).cuda(), 300, out=(ids[r], ds[r]))
        torch.cuda.synchronize()
        sub.free()
    mi, md = psb.psb_merge_topk(ids, ds, 300)
    torch.cuda.synchronize()
    e = oracle.knn_bruteforce(pts, qs, 300)
    assert_same((mi.cpu().numpy(), md.cpu().numpy()), e, "merge k=300")
    idx.free()


@pytest.mark.parametrize("sphere", [False, True])
def test_kmeans_packing_parity(sphere):
    """NEXT-4 k-means packing (k = #leaves, Lloyd steps via the library's own exact
    1-NN): a valid packing (every point exactly once) and exact results."""
    psb = _psb()
    cfg = W.config("C2", n=200_000)
    pts, qs = cfg.points(), cfg.queries(q=1000)
    flags = psb.PSB_PACK_KMEANS | (psb.PSB_NODE_SPHERE if sphere else 0)
    idx = psb.psb_build_ex(pts, cfg.fanout, packing=flags)
    ex = psb.psb_index_export(idx)
    ids = ex["ids"].reshape(-1)
    assert sorted(ids[ids >= 0].tolist()) == list(range(len(pts)))
    exp = oracle.Tree(pts).knn(qs, cfg.k)
    for algo in ("psb", "bnb"):
        assert_same(run(idx, qs, cfg.k, algo), exp, f"kmeans sphere={sphere} {algo}")
    # deterministic
    idx2 = psb.psb_build_ex(pts, cfg.fanout, packing=flags)
    assert np.array_equal(psb.psb_index_export(idx2)["ids"], ex["ids"])
    idx.free()
    idx2.free()
