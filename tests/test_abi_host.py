"""CPU tests of libpsb.so: it loads, exports every symbol include/psb.h declares,
validates arguments without touching a GPU, and its host bulk loader produces the
layout DESIGN.md §4 specifies (checked here with independent numpy code and the
oracle's MINDIST/MAXDIST, not with the library's own arithmetic)."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "psb.h")).read()
    declared = set(re.findall(r"\b(psb_[a-z0-9_]+)\s*\(", hdr))
    assert declared == set(psb.EXPORTS)
    assert all(psb.symbols_exported().values())
    assert "sm_100a" in psb.psb_version()


def test_so_contains_sm100a_cubin():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", psb.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_argument_errors_without_gpu():
    L = psb._lib
    # null index / bad k are rejected before any CUDA call
    assert L.psb_knn(None, None, 1, 8, None, None, None) == psb.PSB_EINVAL
    assert "NULL" in psb.psb_last_error()
    assert L.psb_knn_ex(None, None, 1, 8, None, None, None, 0, 0) == psb.PSB_EINVAL
    assert L.psb_merge_topk(None, None, 0, 1, 8, None, None, None) == psb.PSB_EINVAL
    assert L.psb_merge_topk(None, None, 2, 1, psb.PSB_KMAX + 1, None, None, None) == psb.PSB_EUNSUPPORTED
    assert L.psb_merge_topk(None, None, 2, 1, 200, None, None, None) == psb.PSB_EINVAL   # NULL buffers
    assert L.psb_index_info(None, None, None, None, None, None, None) == psb.PSB_EINVAL
    out = ctypes.c_void_p()
    assert L.psb_build_ex(None, 10, 2, 32, 0, 0, ctypes.byref(out)) == psb.PSB_EINVAL
    L.psb_free(None)  # no-op


@pytest.mark.parametrize("bad", [
    dict(fanout=48), dict(fanout=16), dict(d=0), dict(d=65), dict(n=0), dict(id_base=-1),
    dict(id_base=2 ** 31 - 5), dict(flags=7), dict(nan=True)])
def test_host_build_validation(bad):
    n, d = bad.get("n", 100), bad.get("d", 3)
    pts = np.random.default_rng(0).random((max(n, 1), max(d, 1)), dtype=np.float32)
    if bad.get("nan"):
        pts[5, 0] = np.nan
    used = ctypes.c_int64()
    rc = psb._lib.psb_build_host_blob(pts.ctypes.data, n, d, bad.get("fanout", 32), bad.get("id_base", 0),
                                      bad.get("flags", 0), None, 0, ctypes.byref(used))
    assert rc == psb.PSB_EINVAL, psb.psb_last_error()
    assert psb.psb_last_error()


def _check_layout(pts, F, id_base, blob):
    n, d = pts.shape
    L = -(-n // F)
    assert blob["leaves"] == L and blob["fanout"] == F and blob["d"] == d and blob["n"] == n
    # level sizes: closed form, root is one node, at least one internal level
    nlev = [L]
    while True:
        nlev.append(-(-nlev[-1] // F))
        if nlev[-1] == 1:
            break
    assert blob["levels"] == len(nlev) - 1
    assert blob["nlev"].tolist() == nlev
    ids = blob["ids"]
    flat = ids.reshape(-1)
    real = flat[:n]
    assert (flat[n:] == -1).all()                      # pads only at the tail of the last leaf
    assert sorted((real - id_base).tolist()) == list(range(n))
    P = blob["pts"]                                     # [L][d][F]
    coords = P.transpose(0, 2, 1).reshape(-1, d)
    assert np.array_equal(coords[:n], pts[real - id_base])
    assert np.isinf(coords[n:]).all() and (coords[n:] > 0).all()
    # level-1 blocks: exact min/max of each leaf's real points; empty slots (+inf, -inf)
    boxes = []   # per level: (lo [N][d], hi [N][d]) of the nodes at that level
    lo0 = np.full((L, d), np.inf, np.float32)
    hi0 = np.full((L, d), -np.inf, np.float32)
    for j in range(L):
        cnt = min(F, n - j * F)
        lo0[j] = P[j, :, :cnt].min(1)
        hi0[j] = P[j, :, :cnt].max(1)
    boxes.append((lo0, hi0))
    for lv in range(1, blob["levels"] + 1):
        blk = blob["nodes"][lv]                         # [N][d][2][F]
        clo, chi = boxes[lv - 1]
        Nb = clo.shape[0]
        for i in range(blk.shape[0]):
            for c in range(F):
                g = i * F + c
                if g < Nb:
                    assert np.array_equal(blk[i, :, 0, c], clo[g]) and np.array_equal(blk[i, :, 1, c], chi[g])
                else:
                    assert np.isposinf(blk[i, :, 0, c]).all() and np.isneginf(blk[i, :, 1, c]).all()
        lo = np.stack([blk[i, :, 0, :].min(1) for i in range(blk.shape[0])])
        hi = np.stack([blk[i, :, 1, :].max(1) for i in range(blk.shape[0])])
        boxes.append((lo, hi))
    return boxes


@pytest.mark.parametrize("n,d,F,packing", [
    (10_000, 2, 32, psb.PSB_PACK_HILBERT), (10_000, 2, 32, psb.PSB_PACK_STR),
    (5_000, 3, 64, psb.PSB_PACK_HILBERT), (3_001, 8, 128, psb.PSB_PACK_HILBERT),
    (1, 4, 32, psb.PSB_PACK_HILBERT), (33, 1, 32, psb.PSB_PACK_STR), (40_000, 5, 32, psb.PSB_PACK_HILBERT),
    (2_000, 16, 256, psb.PSB_PACK_STR), (700, 64, 512, psb.PSB_PACK_HILBERT)])
def test_host_layout_invariants(n, d, F, packing):
    pts = (np.random.default_rng(n + d).normal(size=(n, d)) * 10).astype(np.float32)
    blob = psb.psb_build_host_blob(pts, F, id_base=17, packing=packing)
    _check_layout(pts, F, 17, blob)


def test_hilbert_packing_is_local():
    """Hilbert-packed leaves are far tighter than packing in input order (the
    reason the paper sorts by a space-filling curve, §IV-A)."""
    pts = W.gen_uniform(20_000, 2, 99)
    blob = psb.psb_build_host_blob(pts, 32)
    P = blob["pts"][:-1]
    ext = (P.max(2) - P.min(2)).prod(1).mean()
    rnd = pts[: (len(pts) // 32) * 32].reshape(-1, 32, 2)
    ext_rnd = (rnd.max(1) - rnd.min(1)).prod(1).mean()
    assert ext < ext_rnd / 50


def test_bounds_bracket_points_on_built_tree():
    """App. C lemma on the packed tree: for every point p under node N,
    MINDIST(q, N) <= dist(q, p) <= MAXDIST(q, N), and MINDIST(parent) <=
    MINDIST(child) — evaluated with the oracle's bound functions."""
    pts = W.config("C2").points(n=4_000)
    qs = W.config("C2").queries(q=6)
    F = 64
    blob = psb.psb_build_host_blob(pts, F)
    L = blob["leaves"]
    lvl1 = blob["nodes"][1]
    for q in qs:
        for j in range(L):
            blk = lvl1[j // F]
            lo, hi = blk[:, 0, j % F], blk[:, 1, j % F]
            mn, mx = oracle.mindist(q, lo, hi), oracle.maxdist(q, lo, hi)
            for s in range(F):
                if blob["ids"][j, s] < 0:
                    continue
                dd = oracle.dist(q, blob["pts"][j, :, s])
                assert mn <= dd <= mx
            # root block box of the subtree containing leaf j
            top = blob["nodes"][blob["levels"]][0]
            c = j // F ** (blob["levels"] - 1)
            assert oracle.mindist(q, top[:, 0, c], top[:, 1, c]) <= mn


def test_pack_modes_and_id_base_only_change_layout():
    pts = W.gen_uniform(3000, 3, 5)
    a = psb.psb_build_host_blob(pts, 32, id_base=0)
    b = psb.psb_build_host_blob(pts, 32, id_base=1000)
    assert np.array_equal(a["pts"], b["pts"])
    assert np.array_equal(a["ids"][a["ids"] >= 0] + 1000, b["ids"][b["ids"] >= 0])
    s = psb.psb_build_host_blob(pts, 32, packing=psb.PSB_PACK_STR)
    assert sorted(s["ids"][s["ids"] >= 0].tolist()) == list(range(3000))


def test_sass_has_no_fused_multiply_add(tmp_path):
    """Bit-exactness guard: no contracted FFMA/FFMA2 in libpsb.so's sm_100a SASS
    (the distance and the bounds are sub, mul, add each rounded once, R14).
    ptxas contracts mul.f32x2 -> add.f32x2 into FFMA2 even with --fmad=false,
    so this check is what keeps the packed path honest. The one FFMA2 form
    allowed is the square x*x + (-0 pair from constant memory), which rounds
    exactly like the multiply (psb_device.cuh f2_sq): both multiplicands the
    same register, the addend a uniform register (loaded from the constant
    bank; a running sum is per-thread and can never be uniform)."""
    import subprocess
    from concurrent.futures import ThreadPoolExecutor
    subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-xelf", "all", psb.LIB_PATH], cwd=tmp_path,
                   check=True, capture_output=True)
    cubins = sorted(p for p in os.listdir(tmp_path) if p.endswith(".cubin"))
    assert cubins and all("sm_100a" in c for c in cubins), cubins
    # the query path (knn_*): distances, bounds, merges. The bulk loader's only
    # DFMAs are inside the correctly rounded __ddiv_rn routine (Newton steps).
    cubins = [c for c in cubins if c.startswith("knn_")]
    assert len(cubins) >= 11, cubins

    src_cache = {}
    # kernels whose output is only a processing order (never a distance, bound or
    # result row): the Hilbert key of a query for the batch order (knn_order.cu)
    # divides in double, whose library routine refines with DFMA
    ORDER_ONLY = ("hilbert_query_keys",)

    def src_line(path, n):
        if path not in src_cache:
            try:
                src_cache[path] = open(path).read().splitlines()
            except OSError:
                src_cache[path] = []
        lines = src_cache[path]
        return lines[n - 1] if 0 < n <= len(lines) else ""

    def scan(c):
        """Per kernel: FFMA/DFMA lines. The one other FFMA allowed is inside a
        directed-rounding square root of the sphere bounds (R24): __fsqrt_rd /
        __fsqrt_ru are correctly rounded library sequences (MUFU.RSQ + FFMA
        Newton steps, or CUDA's sqrt_r[du] slow-path subroutine). With
        -lineinfo, nvdisasm -g attributes every instruction to a source line;
        an FFMA passes only if that line calls __fsqrt_r* or it sits in the
        slow-path subroutine. So the sphere kernels' leaf distances and bounds
        are checked like every other kernel's (no whole-kernel exemption)."""
        out = subprocess.run(["/usr/local/cuda/bin/nvdisasm", "-g", str(tmp_path / c)], capture_output=True,
                             text=True).stdout
        fused, fn = [], "?"
        square = re.compile(r"\bFFMA2 R\d+, (R\d+)(?:\.reuse)?\.F32x2\.HI_LO, \1(?:\.reuse)?\.F32x2\.HI_LO, "
                            r"(U?R\d+)(?:\.reuse)?\.F32x2\.HI_LO ;")
        dest = re.compile(r"^\s*/\*[0-9a-f]+\*/\s+(?:@!?U?P\w+\s+)?([A-Z0-9_.]+)\s+(U?R)(\d+)\b")
        copy = re.compile(r"\b(?:IMAD\.U32|IMAD\.MOV\.U32) (U?R\d+), RZ, RZ, (U?R\d+) ;|\bU?MOV (U?R\d+), (U?R\d+) ;")
        cur_src, in_sqrt_sub = "", False
        n_sqrt = 0
        nz = set()   # registers holding a half of the -0 pair of c_neg_zero2 (program order)
        for l in out.splitlines():
            m = re.match(r"\s*\.text\.(\S+):", l)
            if m:
                fn, nz, cur_src, in_sqrt_sub = m.group(1), set(), "", False
                continue
            m = re.match(r"\s*//## File \"([^\"]+)\", line (\d+)", l)
            if m:
                cur_src = src_line(m.group(1), int(m.group(2)))
                continue
            m = re.match(r"^(\S+):\s*$", l)
            if m:   # a label: CUDA's internal subroutines start with $__internal_
                if m.group(1).startswith("$__internal_"):
                    in_sqrt_sub = bool(re.search(r"sqrt_r[du]_f32_slowpath", m.group(1)))
                continue
            if re.search(r"\bFFMA2?\b|\bDFMA\b", l) and not any(x in fn for x in ORDER_ONLY):
                # allowed: a square whose addend is the -0 pair read from the
                # constant bank (possibly copied between registers)
                sq = square.search(l)
                ok = False
                if sq:
                    p_, i_ = re.match(r"(U?R)(\d+)", sq.group(2)).groups()
                    ok = sq.group(2) in nz and "%s%d" % (p_, int(i_) + 1) in nz
                if not ok and re.search(r"\bFFMA\b", l) and (in_sqrt_sub or "__fsqrt_r" in cur_src):
                    ok, n_sqrt = True, n_sqrt + 1
                if not ok:
                    fused.append((fn, l.strip()))
            d = dest.match(l)
            if d:
                r = int(d.group(3))
                n = 4 if ".128" in d.group(1) else 2 if re.search(r"\.64|\.WIDE|F32x2|^[A-Z]+2 ", d.group(1) + " " + l) else 1
                regs = ["%s%d" % (d.group(2), r + i) for i in range(n)]
                if re.search(r"\bLDCU?\.64 U?R\d+, c\[0x3\]\[U?RZ\]", l):
                    src_nz = True
                else:
                    cm = copy.search(l)
                    src_nz = bool(cm) and (cm.group(2) or cm.group(4)) in nz
                nz.difference_update(regs)
                if src_nz:
                    nz.update(regs)
        return c, ("FADD" in out or "FMUL" in out), fused, n_sqrt

    with ThreadPoolExecutor(max_workers=os.cpu_count() or 4) as ex:
        res = list(ex.map(scan, cubins))
    assert any(r[1] for r in res)
    assert any(r[3] for r in res), "no sphere-bound sqrt FFMA seen: the line attribution broke"
    bad = {c: f[:3] for c, _, f, _ in res if f}
    assert not bad, bad
