"""Pins of the CPU oracle against things other than itself (CPU only).

Each test names the passage or mathematical fact it pins. A plausible
mistake in the oracle (a dropped term, a transposed operand, a wrong index,
non-fused arithmetic, <= instead of <) fails at least one of them.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
import seeded_inputs as si
from oracle import footprint as fp
from oracle import lru
from oracle import b200_rule

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ------------------------------------------------------------------ generator
@pytest.mark.parametrize("mode", [si.MODE_UNIFORM, si.MODE_DYADIC])
def test_generator_c_matches_numpy(mode):
    n = 1 << 20
    a = si.values(11, n, offset=123, mode=mode)
    b = oracle.fill(11, n, offset=123, mode=mode)
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))


def test_generator_high_index_bits():
    # indices above 2^32 use the hi word (no aliasing of idx and idx + 2^32)
    a = si.values(3, 64, offset=(1 << 32) + 5)
    b = si.values(3, 64, offset=5)
    c = oracle.fill(3, 64, offset=(1 << 32) + 5)
    assert not np.array_equal(a, b)
    assert np.array_equal(a, c)


def test_generator_ranges():
    u = si.values(1, 1 << 16)
    d = si.values(1, 1 << 16, mode=si.MODE_DYADIC)
    assert u.min() >= 0 and u.max() < 1 and abs(float(u.mean()) - 0.5) < 0.01
    assert set(np.unique(d * 16).astype(int)) <= set(range(16))


# ------------------------------------------------------------------ loop nests
def _rel(a, b):
    a, b = np.asarray(a, np.float64), np.asarray(b, np.float64)
    return float(np.max(np.abs(a - b) / np.maximum(np.abs(b), 1e-30)))


def test_atax_vs_numpy_textbook():
    m, n = 300, 257                                  # rectangular, ragged
    A = si.matrix(1, m, n)
    x = si.values(101, n)
    tmp, y = oracle.atax(A, x)
    tmp_ref = A.astype(np.float64) @ x.astype(np.float64)
    y_ref = A.astype(np.float64).T @ tmp_ref
    # sequential fp32 sum of positive terms: |err| <= n*u*sum (u = 2^-24)
    assert _rel(tmp, tmp_ref) < n * 2.0 ** -24
    assert _rel(y, y_ref) < (m + n) * 2.0 ** -24
    tmp64, y64 = oracle.atax(A, x, mode=oracle.SEQ_F64)
    assert _rel(tmp64, tmp_ref) <= 2.0 ** -24 and _rel(y64, y_ref) <= 2.0 ** -24


def test_atax_transpose_is_pinned():
    # y must be A^T tmp, not A tmp: non-square, non-symmetric
    A = si.matrix(2, 64, 48)
    x = si.values(3, 48)
    tmp, y = oracle.atax(A, x)
    assert y.shape == (48,) and tmp.shape == (64,)
    assert _rel(y, A.T.astype(np.float64) @ (A.astype(np.float64) @ x)) < 1e-5


def test_seq_fmaf_is_fused():
    # row [1, a], x = [-r, b] with r = fl(a*b): fused gives a*b - r (the
    # rounding error of a*b, nonzero); unfused would give exactly 0.
    a = np.float32(1.1)
    b = np.float32(1.3)
    r = np.float32(a * b)
    exact = float(a) * float(b) - float(r)
    assert exact != 0.0
    A = np.array([[1.0, a]], np.float32)
    x = np.array([-r, b], np.float32)
    tmp, _ = oracle.atax(A, x)
    assert float(tmp[0]) == np.float32(exact)


@pytest.mark.parametrize("n", [64, 129, 256])
def test_dyadic_inputs_are_exact_everywhere(n):
    # exact-dyadic inputs: every partial sum is exact, so fp32 sequential ==
    # fp64 == numpy in any order (SURVEY 8(c) c1 mode 3)
    D = si.MODE_DYADIC
    A = si.matrix(5, n, n, mode=D)
    B = si.matrix(6, n, n, mode=D)
    x = si.values(7, n, mode=D)
    r = si.values(8, n, mode=D)
    A64, B64, x64, r64 = (v.astype(np.float64) for v in (A, B, x, r))
    q, s = oracle.bicg(A, x, r)
    assert np.array_equal(q, (A64 @ x64).astype(np.float32))
    assert np.array_equal(s, (r64 @ A64).astype(np.float32))
    y, tmp = oracle.gesummv(A, B, x, 1.5, 1.25)
    assert np.array_equal(tmp, (A64 @ x64).astype(np.float32))
    assert np.array_equal(y, (1.5 * (A64 @ x64) + 1.25 * (B64 @ x64)).astype(np.float32))


def test_bicg_vs_numpy():
    nx, ny = 200, 333
    A = si.matrix(2, nx, ny)
    p, r = si.values(102, ny), si.values(202, nx)
    q, s = oracle.bicg(A, p, r)
    A64 = A.astype(np.float64)
    assert _rel(q, A64 @ p) < ny * 2.0 ** -24
    assert _rel(s, r.astype(np.float64) @ A64) < nx * 2.0 ** -24


def test_mvt_vs_numpy_and_inout():
    n = 190
    a = si.matrix(3, n, n)
    y1, y2, x1, x2 = (si.values(103 + 100 * k, n) for k in range(4))
    o1, o2 = oracle.mvt(a, y1, y2, x1, x2)
    a64 = a.astype(np.float64)
    assert _rel(o1, x1 + a64 @ y1) < n * 2.0 ** -24
    assert _rel(o2, x2 + a64.T @ y2) < n * 2.0 ** -24
    # A = 0 leaves x1, x2 unchanged (in/out, not overwrite)
    z1, z2 = oracle.mvt(np.zeros_like(a), y1, y2, x1, x2)
    assert np.array_equal(z1, x1) and np.array_equal(z2, x2)


def test_gesummv_vs_numpy_and_special_cases():
    n = 150
    A, B = si.matrix(5, n, n), si.matrix(105, n, n)
    x = si.values(205, n)
    y, tmp = oracle.gesummv(A, B, x, 1.5, 1.2)
    A64, B64 = A.astype(np.float64), B.astype(np.float64)
    assert _rel(tmp, A64 @ x) < n * 2.0 ** -24
    assert _rel(y, 1.5 * (A64 @ x) + 1.2 * (B64 @ x)) < 2 * n * 2.0 ** -24
    # beta = 0 -> y = alpha * A x exactly as rounded alpha * tmp
    y0, tmp0 = oracle.gesummv(A, B, x, 1.5, 0.0)
    assert np.array_equal(y0, (np.float32(1.5) * tmp0).astype(np.float32))
    # alpha = 0 -> y = beta * B x
    ya, _ = oracle.gesummv(A, B, x, 0.0, 1.2)
    assert _rel(ya, 1.2 * (B64 @ x)) < n * 2.0 ** -24


def test_rows3_vs_numpy_and_special_cases():
    """The three-stream row loop (DESIGN R29): numpy float64 within 3n u; with
    B = C = 0 it is BICG's q = A p bit for bit (the same fmaf chain, then +0
    twice); on exact-dyadic inputs it equals numpy exactly; swapping the
    order of A and C (a wrong stream) changes the rounding."""
    m, n = 90, 170
    A, B, C = si.matrix(5, m, n), si.matrix(105, m, n), si.matrix(305, m, n)
    x = si.values(205, n)
    y = oracle.rows3(A, B, C, x)
    ref = (A.astype(np.float64) @ x + B.astype(np.float64) @ x) + C.astype(np.float64) @ x
    assert _rel(y, ref) < 3 * n * 2.0 ** -24
    assert _rel(oracle.rows3(A, B, C, x, mode=oracle.SEQ_F64), ref) < 2.0 ** -23
    z = np.zeros_like(A)
    q, _ = oracle.bicg(A, x, np.zeros(m, np.float32))
    assert np.array_equal(oracle.rows3(A, z, z, x), q)
    D = si.MODE_DYADIC
    Ad, Bd, Cd, xd = si.matrix(6, m, n, D), si.matrix(7, m, n, D), si.matrix(8, m, n, D), si.values(9, n, mode=D)
    want = (Ad.astype(np.float64) @ xd + Bd.astype(np.float64) @ xd) + Cd.astype(np.float64) @ xd
    assert np.array_equal(oracle.rows3(Ad, Bd, Cd, xd), want.astype(np.float32))
    assert not np.array_equal(oracle.rows3(C, B, A, x), y)


def test_syrk_vs_numpy_and_symmetry():
    n, m = 70, 45
    A = si.matrix(6, n, m)
    C = si.matrix(106, n, n)
    out = oracle.syrk(A, C, 1.5, 1.2)
    ref = 1.2 * C.astype(np.float64) + 1.5 * (A.astype(np.float64) @ A.astype(np.float64).T)
    assert _rel(out, ref) < 2 * m * 2.0 ** -24
    # full square: with alpha = 1 (alpha*a_ik exact) and beta = 0 the result is
    # exactly symmetric; with alpha = 1.5 it is not (alpha*a_ik is rounded first)
    s = oracle.syrk(A, C, 1.0, 0.0)
    assert np.array_equal(s, s.T)
    # alpha = 0 -> beta * C, exactly
    b = oracle.syrk(A, C, 0.0, 1.2)
    assert np.array_equal(b, (C * np.float32(1.2)).astype(np.float32))


def test_syrk_rows_equals_full_rows():
    A, C = si.matrix(6, 50, 33), si.matrix(106, 50, 50)
    full = oracle.syrk(A, C, 1.5, 1.2)
    rows = np.array([0, 7, 49])
    assert np.array_equal(oracle.syrk_rows(A, C, 1.5, 1.2, rows), full[rows])


def test_syr2k_vs_numpy_and_special_cases():
    n, m = 60, 37
    A, B, C = si.matrix(8, n, m), si.matrix(108, n, m), si.matrix(208, n, n)
    out = oracle.syr2k(A, B, C, 1.5, 1.2)
    A64, B64 = A.astype(np.float64), B.astype(np.float64)
    ref = 1.2 * C.astype(np.float64) + 1.5 * (A64 @ B64.T + B64 @ A64.T)
    assert _rel(out, ref) < 4 * m * 2.0 ** -24
    # swapping A and B gives the same matrix mathematically (A B^T + B A^T)
    assert _rel(oracle.syr2k(B, A, C, 1.5, 1.2), ref) < 4 * m * 2.0 ** -24      # symmetric in (A, B) mathematically
    # B = 0 -> beta * C exactly (every s is 0); alpha = 0 likewise
    assert np.array_equal(oracle.syr2k(A, np.zeros_like(B), C, 1.5, 1.2), (C * np.float32(1.2)).astype(np.float32))
    # exact dyadic inputs: bit-equal to float64 (alpha = 1.5, beta = 1.25 dyadic)
    D = si.MODE_DYADIC
    Ad, Bd, Cd = si.matrix(9, n, m, D), si.matrix(109, n, m, D), si.matrix(209, n, n, D)
    refd = 1.25 * Cd.astype(np.float64) + 1.5 * (Ad.astype(np.float64) @ Bd.T.astype(np.float64)
                                                 + Bd.astype(np.float64) @ Ad.T.astype(np.float64))
    assert np.array_equal(oracle.syr2k(Ad, Bd, Cd, 1.5, 1.25), refd.astype(np.float32))
    rows = np.array([0, 17, 59])
    assert np.array_equal(oracle.syr2k_rows(A, B, C, 1.5, 1.2, rows), out[rows])


def test_kmeans_vs_bruteforce_argmin():
    npts, nf, k = 1000, 34, 5
    ld = npts + 3                                         # misaligned leading dimension
    feat = si.values(4, nf * ld)
    F = feat.reshape(nf, ld)[:, :npts].T.astype(np.float64)   # points x features
    clusters = F[:k].astype(np.float32)                     # centres = first k points
    memb, margin = oracle.kmeans_assign(feat, ld, npts, nf, clusters, mode=oracle.SEQ_F64)
    d = ((F[:, None, :] - clusters[None, :, :].astype(np.float64)) ** 2).sum(-1)
    ref = d.argmin(1)
    clear = margin > 1e-4
    assert clear.mean() > 0.95
    assert np.array_equal(memb[clear], ref[clear])
    assert np.array_equal(memb[:k], np.arange(k))         # each centre is its own point


def test_kmeans_distance_is_fused_per_feature():
    # R16: d = fmaf(diff, diff, d) per feature, f ascending (one rounding per
    # feature). With the point at the origin and the centres (a, b) and (b, a)
    # the exact distances are equal; one rounding per feature makes (b, a)
    # strictly nearer for these a, b, while a mul-then-add order rounds both to
    # the same value (a tie: centre 0). Expected value from exact rationals
    # rounded once (oracle.kmeans.round_f32, pinned on its own).
    from fractions import Fraction
    from oracle.kmeans import round_f32
    a, b = np.float32(0.7971469759941101), np.float32(0.13876742124557495)

    def fused(c):
        d = np.float32(0)
        for ci in c:
            df = np.float32(np.float32(0) - ci)
            d = round_f32(Fraction(float(df)) ** 2 + Fraction(float(d)))
        return d
    assert fused([b, a]) < fused([a, b])
    assert np.float32(a * a) + np.float32(b * b) == np.float32(b * b) + np.float32(a * a)   # unfused: a tie
    memb, _ = oracle.kmeans_assign(np.zeros(2, np.float32), 1, 1, 2, np.array([[a, b], [b, a]], np.float32))
    assert memb.tolist() == [1]


def test_kmeans_ties_lowest_index():
    nf, k, npts = 4, 3, 8
    feat = np.zeros(nf * npts, np.float32)
    clusters = np.zeros((k, nf), np.float32)              # three identical centres
    memb, _ = oracle.kmeans_assign(feat, npts, npts, nf, clusters)
    assert np.all(memb == 0)


def test_atax_hashed_matches_materialised():
    m, n = 96, 80
    A = si.matrix(7, m, n)
    x = si.values(107, n)
    tmp, y = oracle.atax(A, x)
    cols = np.array([0, 5, 79])
    t2, yc = oracle.atax_hashed(7, 0, x, m, n, cols)
    assert np.array_equal(tmp, t2) and np.array_equal(y[cols], yc)


# ------------------------------------------------------------------ footprint model
def _paper_loop(refs, grid, block=256, force=-1, trip=40960):
    rs = [fp.Ref(c_gid=(ct, 0, 0), c_iter=(ci,), array_id=k) for k, (ct, ci) in enumerate(refs)]
    return fp.Loop(refs=rs, trips=(trip,), block=(block, 1, 1), grid=(grid, 1, 1),
                   mode=fp.MODE_PAPER, force_carveout_kb=force)


def test_worked_coefficients_and_locality():
    # tmp[i] (C_tid 1, C_i 0), A[i*NX+j] (C_tid NX, C_i 1), B[j] (0, 1);
    # A and B have intra-thread locality (C_i*4 B < 128 B), P:221 strictness.
    hw = fp.titan_v()
    loop = _paper_loop([(1, 0), (40960, 1), (0, 1)], grid=320)
    assert [fp.req_warp_paper(r, loop, hw) for r in loop.refs] == [1, 32, 1]
    ref = fp.Ref(c_gid=(1, 0, 0), c_iter=(32, 31))        # 31*4 < 128: consecutive reuse
    assert fp._window(ref, (4, 10), 128) == (True, None)
    ref1 = fp.Ref(c_gid=(1, 0, 0), c_iter=(31, 32))       # 32*4 = 128 B: not at the inner level (strict <)
    assert fp._window(ref1, (3, 5), 128)[1] == [(0, k) for k in range(5)]   # ... but across the outer
    ref2 = fp.Ref(c_gid=(1, 0, 0), c_iter=(32, 32))       # no reuse at any level
    assert fp._window(ref2, (3, 5), 128) == (True, None)


def test_req_warp_examples_p235():
    # inter-thread distance 0 -> 1 line; distance 8 (32 B) -> 8 lines
    hw = fp.titan_v()
    loop = _paper_loop([(0, 1), (8, 1)], grid=80)
    assert [fp.req_warp_paper(r, loop, hw) for r in loop.refs] == [1, 8]


def test_fig5_tb_cap_arithmetic():
    # Fig 5: 48 KB of shared memory per TB in a 96 KB carveout -> 2 TBs
    hw = fp.titan_v()
    loop = _paper_loop([(1, 0)], grid=320)
    loop.smem = 48 * 1024
    W, T, carve, l1d = fp.occupancy(loop, hw)
    assert (W, T, carve, l1d) == (8, 2, 96, 32 * 1024)


def test_table3_paper_mode_rows():
    g = json.load(open(os.path.join(GOLDEN, "table3_paper_mode.json")))
    hw = fp.titan_v()
    for c in g["cases"]:
        for key, force in (("catt_max", -1), ("catt_32kb", 96)):
            res = fp.analyse(_paper_loop(c["refs"], c["grid"], c["block"], force), hw)
            assert (res["base_warps"], res["base_ctas"]) == tuple(c["baseline"]), c["name"]
            assert (res["active_warps"], res["active_ctas"]) == tuple(c[key]), (c["name"], key, res)


def test_gsmv_requires_coalesced_refs():
    # SURVEY 0 finding 1 / reading R3: without the coalesced references GSMV at
    # max L1D would not be throttled, contradicting Table 3's (4,2).
    hw = fp.titan_v()
    res = fp.analyse(_paper_loop([(40960, 1), (40960, 1)], grid=160), hw)
    assert (res["active_warps"], res["active_ctas"]) == (8, 2)


def test_give_up_rule():
    # P:244 / P:395 (CORR): if even (1 warp, 1 TB) does not fit, keep the baseline
    hw = fp.titan_v()
    refs = [(40960, 0)] * 40                                # 40 x 32 lines per warp, no reuse
    res = fp.analyse(_paper_loop(refs, grid=80, force=96), hw)
    assert res["flags"] == fp.FIT_UNRESOLVABLE
    assert (res["active_warps"], res["active_ctas"]) == (res["base_warps"], res["base_ctas"])


def test_cta_level_after_warp_level():
    # Eq 9 order: warp level first, then TBs with 1 warp
    hw = fp.titan_v()
    refs = [(40960, 1)] * 3                                  # 96 lines per warp
    res = fp.analyse(_paper_loop(refs, grid=320, force=96), hw)  # L1D 256 lines, T = 4
    assert (res["active_warps"], res["active_ctas"], res["flags"]) == (1, 2, fp.FIT_CTA)


def test_union_equals_closed_form_on_aligned_1d():
    # brute-force enumeration reduces to Eq 7's closed form for 128 B-aligned
    # 1-D warps with no lines shared between references
    hw = fp.titan_v()
    for ct in (1, 2, 3, 8, 31, 32, 33, 1000):
        loop = _paper_loop([(ct, 1)], grid=80)
        loop.mode = fp.MODE_UNION
        m = fp.Model(loop, hw)
        assert m.lines_per_warp_iter == min(32, ct)


# ------------------------------------------------------------------ LRU pins
def _hw_small(l1d_lines):
    """A tiny fake GPU so contention shows up at small sizes (2 SMs)."""
    carve = [0, 8, 16, 32]
    return dict(num_sms=2, max_warps_sm=16, max_ctas_sm=4, regs_sm=65536, reg_alloc_unit=256,
                warp_size=32, smem_alloc_unit=128, reserved_smem_cta=0, line_bytes=128,
                carveout_kb=carve, l1d_bytes=[n * 128 for n in l1d_lines])


def _row_loop(M, N, cta, nblocks_x, vec=1, nmat=1):
    refs = []
    for k in range(nmat):
        refs.append(fp.Ref(c_gid=(N // vec, 0, 0), c_iter=(1,), elem_bytes=4 * vec, array_id=10 + k))
        refs.append(fp.Ref(c_gid=(0, 0, 0), c_iter=(1,), elem_bytes=4 * vec, array_id=1))
    return fp.Loop(refs=refs, trips=(N // vec,), block=(cta, 1, 1), grid=(nblocks_x, 1, 1), extent=(M, 0, 0))


def _col_loop(M, N, cta):
    refs = [fp.Ref(c_gid=(1, 0, 0), c_iter=(N,), array_id=10), fp.Ref(c_gid=(0, 0, 0), c_iter=(1,), array_id=1)]
    return fp.Loop(refs=refs, trips=(M,), block=(cta, 1, 1), grid=((N + cta - 1) // cta, 1, 1), extent=(N, 0, 0))


def _kmeans_loop(npts, nf, k, ld, cta):
    refs = [fp.Ref(c_gid=(1, 0, 0), c_iter=(0, ld), array_id=10)]
    return fp.Loop(refs=refs, trips=(k, nf), block=(cta, 1, 1), grid=((npts + cta - 1) // cta, 1, 1),
                   extent=(npts, 0, 0))


def _syrk_loop(N, Mk):
    refs = [fp.Ref(c_gid=(0, Mk, 0), c_iter=(1,), array_id=10), fp.Ref(c_gid=(Mk, 0, 0), c_iter=(1,), array_id=10)]
    return fp.Loop(refs=refs, trips=(Mk,), block=(32, 8, 1), grid=(N // 32, N // 8, 1), extent=(N, N, 0))


LRU_CASES = [
    # (name, loop, kernel, l1d lines table for carveouts 0/8/16/32)
    ("row256", _row_loop(256, 64, 256, 1), lru.RowKernel(256, 64, 256), [400, 257, 256, 64]),
    ("row_vec", _row_loop(256, 64, 256, 1, vec=4), lru.RowKernel(256, 64, 256, vec=4), [300, 200, 100, 40]),
    ("row_ragged", _row_loop(200, 96, 128, 2), lru.RowKernel(200, 96, 128), [300, 100, 60, 20]),
    ("row_multi_cta", _row_loop(1024, 64, 128, 8), lru.RowKernel(1024, 64, 128), [600, 300, 120, 40]),
    ("gesummv", _row_loop(256, 64, 256, 1, nmat=2), lru.RowKernel(256, 64, 256, matrices=("A", "B")), [600, 400, 200, 70]),
    ("col", _col_loop(64, 512, 256), lru.ColKernel(64, 512, 256), [64, 16, 9, 4]),
    ("kmeans", _kmeans_loop(2048, 6, 3, 2048, 128), lru.KmeansKernel(2048, 6, 3, 2048, 128), [200, 100, 40, 8]),
    ("kmeans_misaligned", _kmeans_loop(2040, 6, 3, 2044, 128), lru.KmeansKernel(2040, 6, 3, 2044, 128), [200, 100, 40, 8]),
    ("syrk", _syrk_loop(64, 40), lru.SyrkKernel(64, 40), [200, 80, 50, 20]),
    ("syrk128", _syrk_loop(128, 64), lru.SyrkKernel(128, 64), [200, 64, 40, 30]),
]


@pytest.mark.parametrize("name,loop,kern,table", LRU_CASES, ids=[c[0] for c in LRU_CASES])
def test_union_decision_matches_lru(name, loop, kern, table):
    hw = _hw_small(table)
    for carve in hw["carveout_kb"]:
        loop.force_carveout_kb = carve
        res = fp.analyse(loop, hw)
        W, T = res["base_warps"], res["base_ctas"]
        cap = res["l1d_bytes"] // 128
        a, m, how = lru.decide_by_lru(kern, W, T, cap, hw["num_sms"])
        assert (res["active_warps"], res["active_ctas"]) == (a, m), (name, carve, res, how)
        # and the analyser's own claim: zero intra-thread capacity misses at its pick
        blocks = lru.sm0_blocks(kern, hw["num_sms"], T)
        st = lru.simulate(kern, blocks, res["active_warps"], res["active_ctas"], cap)
        if res["flags"] != fp.FIT_UNRESOLVABLE:
            assert st["intra_thread_capacity_misses"] == 0


def test_lru_trace_lines_match_descriptor():
    # brute-force per-warp line counts from the traces equal the analyser's
    # lines_per_warp_iter / reuse_span
    hw = _hw_small([400, 300, 200, 100])
    for loop, kern, per_iter_events in [
        (_row_loop(256, 64, 256, 1), lru.RowKernel(256, 64, 256), 2),
        (_kmeans_loop(2040, 6, 3, 2044, 128), lru.KmeansKernel(2040, 6, 3, 2044, 128), 1),
        (_syrk_loop(64, 40), lru.SyrkKernel(64, 40), 2),
    ]:
        m = fp.Model(loop, hw)
        ev = kern.events(0, 0)
        assert m.lines_per_warp_iter == sum(len({ln for ln, _ in e}) for e in ev[:per_iter_events])
        if isinstance(kern, lru.KmeansKernel):
            assert m.reuse_span == len({ln for e in ev[: kern.nf] for ln, _ in e})


def test_paper_arithmetic_consistency():
    # P:7: 42.96% over baseline, 31.19% for BFTT -> 8.97% over BFTT
    assert abs(1.4296 / 1.3119 - 1.0897) < 1e-4
    assert math.isclose(1.8923 / 1.6817, 1.125, abs_tol=2e-3)   # P:405 (32 KB L1D)


def test_union_decision_matches_lru_random():
    """Seeded random 1-D configurations (ragged sizes, rows that do not start
    on a line boundary, float4 rows, tiny caches): the union-mode decision is
    the LRU decision. 2-D SYRK is pinned on line-aligned rows only (DESIGN.md
    'Known limits of the union model')."""
    import random
    rnd = random.Random(20191)
    for _ in range(40):
        kind = rnd.choice(["row", "rowv", "col", "km", "ges"])
        if kind in ("row", "rowv", "ges"):
            cta = rnd.choice([32, 64, 96, 128, 256])
            M = rnd.randint(1, 400)
            N = rnd.choice([4, 8, 12, 20, 36, 40, 64, 100])
            vec = 4 if kind == "rowv" else 1
            nm = 2 if kind == "ges" else 1
            loop = _row_loop(M, N, cta, (M + cta - 1) // cta, vec=vec, nmat=nm)
            kern = lru.RowKernel(M, N, cta, vec=vec, matrices=("A", "B")[:nm])
        elif kind == "col":
            cta = rnd.choice([32, 64, 128])
            M, N = rnd.randint(1, 30), rnd.randint(1, 500)
            loop, kern = _col_loop(M, N, cta), lru.ColKernel(M, N, cta)
        else:
            cta = rnd.choice([32, 64, 128])
            npts = rnd.randint(1, 700)
            ld = npts + rnd.randint(0, 40)
            nf, k = rnd.randint(1, 8), rnd.randint(1, 4)
            loop, kern = _kmeans_loop(npts, nf, k, ld, cta), lru.KmeansKernel(npts, nf, k, ld, cta)
        full = fp.analyse(loop, _hw_small([1 << 20] * 4))["footprint_lines_full"]
        caps = sorted({max(1, full - 1), full, rnd.randint(1, full + 5)})
        hw = _hw_small(caps + [caps[-1]] * (4 - len(caps)))
        for carve in hw["carveout_kb"][: len(caps)]:
            loop.force_carveout_kb = carve
            res = fp.analyse(loop, hw)
            cap = res["l1d_bytes"] // 128
            got = lru.decide_by_lru(kern, res["base_warps"], res["base_ctas"], cap, hw["num_sms"])
            assert (res["active_warps"], res["active_ctas"]) == got[:2], (kind, vars(kern), cap, res, got)


def test_no_locality_no_throttle():
    # contention is measured only for loops where locality presents;
    # a one-iteration loop re-touches nothing, whatever its footprint
    hw = _hw_small([4, 4, 4, 4])
    res = fp.analyse(_row_loop(256, 4, 256, 1, vec=4), hw)
    assert res["flags"] == fp.FIT_NONE_NEEDED and res["active_warps"] == 8


def test_locality_strict_at_one_line_model_level():
    # Eq 6 / P:221 strictness at the decision level: a divergent row reference
    # whose iteration stride is exactly one line (32 floats = 128 B) re-touches
    # nothing, so the loop is never throttled; 31 floats re-touch the line and
    # the same loop (footprint far above the L1D) is throttled
    hw = fp.titan_v()
    one_line = fp.analyse(_paper_loop([(40960, 32)], grid=640), hw)
    assert not fp.has_locality(fp.Ref(c_gid=(40960, 0, 0), c_iter=(32,)), (40960,), 128)
    assert one_line["flags"] == fp.FIT_NONE_NEEDED and one_line["active_warps"] == one_line["base_warps"]
    below = fp.analyse(_paper_loop([(40960, 31)], grid=640), hw)
    assert fp.has_locality(fp.Ref(c_gid=(40960, 0, 0), c_iter=(31,)), (40960,), 128)
    assert below["active_warps"] < below["base_warps"]


@pytest.mark.parametrize("e", [1, 2, 4, 8, 16])
@pytest.mark.parametrize("c", [1, 2, 3, 5, 7])
def test_req_warp_equals_brute_force_line_count(c, e):
    # Eq 7 against brute force: the distinct 128-B lines that the 32
    # lanes' addresses (lane * c * e bytes from a line-aligned base) fall in.
    # 1-, 2- and 8-byte elements make 32*c*e/128 fractional, where Eq 7's
    # ceiling matters (a floor would give 0 lines for c = 1, e = 2).
    hw = fp.titan_v()
    loop = _paper_loop([(c, 1)], grid=80)
    loop.refs[0].elem_bytes = e
    want = len({(lane * c * e) // 128 for lane in range(32)})
    assert fp.req_warp_paper(loop.refs[0], loop, hw) == want


def test_req_warp_printed_form_overcounts_a_partial_stride():
    # Eq 7 as printed counts 32 whole strides: c = 33 one-byte elements span
    # 31*33 + 1 = 1024 B (8 lines) but ceil(32*33/128) = 9 (R2 takes the printed
    # form in paper mode; union mode enumerates the lanes' lines instead)
    hw = fp.titan_v()
    for c, e, printed, lines in ((33, 1, 9, 8), (33, 2, 17, 16)):
        loop = _paper_loop([(c, 1)], grid=80)
        loop.refs[0].elem_bytes = e
        assert fp.req_warp_paper(loop.refs[0], loop, hw) == printed == math.ceil(32 * c * e / 128)
        assert len({(lane * c * e) // 128 for lane in range(32)}) == lines


@pytest.mark.parametrize("regs,want", [(32, 8), (40, 6), (64, 4), (128, 2), (255, 1)])
def test_b200_register_limit_closed_form(regs, want):
    # Eq 2 on B200 (DESIGN Eq 1-3 reading): 64 K registers per SM in 4
    # sub-partitions of 16 K, allocated per warp in units of 256 registers.
    # A 256-thread CTA (8 warps) with r registers per thread: a warp takes
    # roundup(32 r, 256) registers, a sub-partition holds 16384 // that many
    # warps, the SM 4x as many; T = those warps // 8 (other limits: 64 warps
    # -> 8 CTAs, 32 CTA slots, 148 x 64 CTAs in the grid, no shared memory).
    #   r = 32: 1024 -> 16 warps/SP -> 64 -> T 8;  r = 40: 1280 -> 12 -> 48 -> 6
    #   r = 64: 2048 -> 8 -> 32 -> 4;  r = 128: 4096 -> 4 -> 16 -> 2
    #   r = 255: 8160 -> 8192 -> 2 -> 8 -> 1
    hw = b200_rule.b200_hw()
    loop = fp.Loop(refs=[fp.Ref(c_gid=(1, 0, 0), c_iter=(1,))], trips=(4,), block=(256, 1, 1),
                   grid=(148 * 64, 1, 1), regs=regs, mode=fp.MODE_UNION, force_carveout_kb=-1)
    W, T, _, _ = fp.occupancy(loop, hw)
    assert (W, T) == (8, want)


def test_gemm_pins():
    """PolyBench gemm (CI negative control)."""
    rng = np.random.default_rng(11)
    A = rng.random((37, 23), dtype=np.float32)
    B = rng.random((23, 19), dtype=np.float32)          # non-square: a transposed operand fails
    C = rng.random((37, 19), dtype=np.float32)
    got = oracle.gemm(A, B, C, 1.5, 1.2)
    ref = 1.2 * C.astype(np.float64) + 1.5 * (A.astype(np.float64) @ B.astype(np.float64))
    assert np.max(np.abs(got - ref) / np.abs(ref)) < 4 * 23 * 2.0 ** -24
    assert np.array_equal(oracle.gemm(A, B, C, 0.0, 1.25), (C * np.float32(1.25)).astype(np.float32))
    # the same evaluation order as SYRK: gemm(A, A^T) is syrk(A) bit for bit
    S = rng.random((29, 17), dtype=np.float32)
    Cs = rng.random((29, 29), dtype=np.float32)
    assert np.array_equal(oracle.gemm(S, np.ascontiguousarray(S.T), Cs, 1.5, 1.2), oracle.syrk(S, Cs, 1.5, 1.2))
    # exact-dyadic inputs: every partial sum exact -> equal to numpy exactly
    Ad = (rng.integers(0, 16, (40, 31)) / 16).astype(np.float32)
    Bd = (rng.integers(0, 16, (31, 12)) / 16).astype(np.float32)
    Cd = (rng.integers(0, 16, (40, 12)) / 16).astype(np.float32)
    want = (np.float64(1.25) * Cd + 1.5 * (Ad.astype(np.float64) @ Bd)).astype(np.float32)
    assert np.array_equal(oracle.gemm(Ad, Bd, Cd, 1.5, 1.25), want)


def test_corr_pins():
    """PolyBench correlation: Pearson correlation of the columns."""
    rng = np.random.default_rng(12)
    n, m = 300, 9
    data = (rng.standard_normal((n, m)) * rng.uniform(0.5, 3, m) + rng.uniform(-2, 2, m)).astype(np.float32)
    data[:, 3] += 0.7 * data[:, 1]                        # a correlated pair
    sym, mean, std, centred = oracle.corr(data)
    ref = np.corrcoef(data.astype(np.float64).T)
    assert np.max(np.abs(sym - ref)) < 2e-5
    assert np.array_equal(sym, sym.T) and np.all(np.diag(sym) == 1.0)
    assert np.allclose(mean, data.astype(np.float64).mean(0), rtol=1e-5, atol=1e-6)
    assert np.allclose(std, data.astype(np.float64).std(0), rtol=1e-5)
    assert np.allclose(centred, (data - data.mean(0)) / (np.sqrt(n) * data.std(0)), rtol=1e-4, atol=1e-6)
    # affine invariance of the definition
    sym2, _, _, _ = oracle.corr(data * 2.0 + 3.0)
    assert np.max(np.abs(sym2 - sym)) < 2e-5
    # a constant column: std <= eps -> 1, so its correlations are ~0, not NaN
    data[:, 5] = 0.25
    sym3, _, std3, _ = oracle.corr(data)
    assert std3[5] == 1.0 and np.all(np.isfinite(sym3))
    assert np.max(np.abs(np.delete(sym3[5], 5))) < 1e-6
    # the fp64 mode is the textbook value
    sym64, _, _, _ = oracle.corr(data[:, :5], mode=oracle.SEQ_F64)
    assert np.max(np.abs(sym64 - np.corrcoef(data[:, :5].astype(np.float64).T))) < 1e-6


def test_mutation_harness_still_applies():
    # tools/oracle_mutants.py (DESIGN 3, "Do the pins have teeth?") types each
    # mistake into a copy of oracle/ by text replacement: every mutant's text
    # must still occur exactly once, or an oracle edit silently retired it
    import importlib.util
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    spec = importlib.util.spec_from_file_location("oracle_mutants", os.path.join(root, "tools", "oracle_mutants.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    assert len(m.MUTANTS) >= 40
    for name, (fn, old, new, count, what) in m.MUTANTS.items():
        src = open(os.path.join(root, "oracle", fn)).read()
        assert src.count(old) == 1, name
        assert (old == new) == (name == "control_unchanged"), name
