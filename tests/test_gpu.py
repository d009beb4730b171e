"""GPU parity tests: the CUDA path (through the C ABI) against the CPU oracle.

Bars:
  - LITERAL / VEC4 / STAGED variants and SYRK STAGED keep the sequential
    per-output order: bit-exact to the oracle's seq-fmaf mode;
  - COOP variants reorder the sums: max relative error <= 1e-5 against the
    fp64 oracle (BASELINE north_star), and bit-exact on exact-dyadic inputs;
  - KMEANS membership: bit-exact (decided in fp32 in the same order);
  - throttles never change results; the residency probe shows them enforced.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
import paper_conf_icpp_kimhlsh19_b200 as catt
import seeded_inputs as si

pytestmark = pytest.mark.gpu
DYADIC = si.MODE_DYADIC
TOL = 1e-5


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def relerr(got, ref):
    got, ref = np.asarray(got, np.float64), np.asarray(ref, np.float64)
    return float(np.max(np.abs(got - ref) / np.maximum(np.abs(ref), 1e-30))) if got.size else 0.0


def bits_equal(a, b):
    return np.array_equal(np.asarray(a, np.float32).view(np.uint32), np.asarray(b, np.float32).view(np.uint32))


EXACT = ["literal", "vec4", "staged"]
ROW_SHAPES = [(257, 36), (64, 1024), (1000, 132), (33, 4)]      # ragged rows/cols, several tiles and warps
COL_SHAPES = [(36, 257), (1024, 64), (131, 1000), (4, 33)]


# ------------------------------------------------------------------ generator
@pytest.mark.parametrize("mode", [0, 1])
def test_fill_hash_matches_generator(mode):
    n = 1 << 20
    t = torch.empty(n, device="cuda")
    catt.fill_hash(t, 17, offset=(1 << 32) - 1000, mode=mode)
    want = si.values(17, n, offset=(1 << 32) - 1000, mode=mode)
    assert bits_equal(host(t), want)


# ------------------------------------------------------------------ ATAX / BICG / MVT / GESUMMV
def _vec_ok(variant, n):
    return not (variant in ("vec4", "staged") and n % 4)


@pytest.mark.parametrize("variant", EXACT)
@pytest.mark.parametrize("m,n", ROW_SHAPES)
def test_atax_exact(variant, m, n):
    A, x = si.matrix(1, m, n), si.values(101, n)
    tmp_o, y_o = oracle.atax(A, x)
    t = catt.Throttle(variant=variant)
    if not _vec_ok(variant, n):
        with pytest.raises(catt.CattError):
            catt.atax(dev(A), dev(x), k1=t)
        return
    tmp, y = catt.atax(dev(A), dev(x), k1=t, k2=catt.Throttle(variant=variant))
    assert bits_equal(host(tmp), tmp_o) and bits_equal(host(y), y_o)


@pytest.mark.parametrize("variant", EXACT + ["coop"])
@pytest.mark.parametrize("m,n", COL_SHAPES)
def test_bicg(variant, m, n):
    A, p, r = si.matrix(2, m, n), si.values(102, n), si.values(202, m)
    q_o, s_o = oracle.bicg(A, p, r)
    q64, s64 = oracle.bicg(A, p, r, mode=oracle.SEQ_F64)
    col_var = variant
    if not _vec_ok(variant, n):
        with pytest.raises(catt.CattError):
            catt.bicg(dev(A), dev(p), dev(r), k1=catt.Throttle(variant=col_var), k2=catt.Throttle(variant=variant))
        return
    q, s = catt.bicg(dev(A), dev(p), dev(r), k1=catt.Throttle(variant=col_var), k2=catt.Throttle(variant=variant))
    q, s = host(q), host(s)
    if variant == "coop":
        assert relerr(q, q64) <= TOL and relerr(s, s64) <= TOL
    else:
        assert bits_equal(q, q_o) and bits_equal(s, s_o)


@pytest.mark.parametrize("variant", EXACT + ["coop"])
@pytest.mark.parametrize("n", [1, 36, 257, 1024])
def test_mvt(variant, n):
    a = si.matrix(3, n, n)
    y1, y2, x1, x2 = (si.values(103 + 100 * k, n) for k in range(4))
    o1, o2 = oracle.mvt(a, y1, y2, x1, x2)
    e1, e2 = oracle.mvt(a, y1, y2, x1, x2, mode=oracle.SEQ_F64)
    col_var = variant
    X1, X2 = dev(x1), dev(x2)
    if not _vec_ok(variant, n):
        with pytest.raises(catt.CattError):
            catt.mvt(dev(a), dev(y1), dev(y2), X1, X2, k1=catt.Throttle(variant=variant))
        return
    catt.mvt(dev(a), dev(y1), dev(y2), X1, X2, k1=catt.Throttle(variant=variant), k2=catt.Throttle(variant=col_var))
    if variant == "coop":
        assert relerr(host(X1), e1) <= TOL and relerr(host(X2), e2) <= TOL
    else:
        assert bits_equal(host(X1), o1) and bits_equal(host(X2), o2)


@pytest.mark.parametrize("variant", EXACT + ["coop"])
@pytest.mark.parametrize("n", [36, 130, 1024])
def test_gesummv(variant, n):
    A, B, x = si.matrix(5, n, n), si.matrix(105, n, n), si.values(205, n)
    y_o, t_o = oracle.gesummv(A, B, x, 1.5, 1.2)
    y64, t64 = oracle.gesummv(A, B, x, 1.5, 1.2, mode=oracle.SEQ_F64)
    if not _vec_ok(variant, n):
        return
    y, tmp = catt.gesummv(dev(A), dev(B), dev(x), 1.5, 1.2, t=catt.Throttle(variant=variant))
    if variant == "coop":
        assert relerr(host(y), y64) <= TOL and relerr(host(tmp), t64) <= TOL
    else:
        assert bits_equal(host(y), y_o) and bits_equal(host(tmp), t_o)


@pytest.mark.parametrize("m,n,t", [(130, 70, catt.Throttle()), (1000, 96, catt.Throttle(active_warps=2)),
                                   (700, 257, catt.Throttle(cta_threads=384, active_warps=3, carveout_kb=228)),
                                   (148 * 256 * 2 + 5, 64, catt.Throttle(active_ctas=1))])
def test_rows3_literal_bit_exact(m, n, t):
    """The three-stream row loop (CATT_ROWS_SUM3, DESIGN R29) through catt_rows,
    throttled or not: bit-exact to the oracle's fmaf chains."""
    A, BC, x = si.matrix(5, m, n), si.matrix(105, 2 * m, n), si.values(205, n)
    y_o = oracle.rows3(A, BC[:m], BC[m:], x)
    y = torch.empty(m, device="cuda")
    catt.rows(dev(A), dev(x), y, catt.ROWS_SUM3, B=dev(BC), t=t)
    assert bits_equal(host(y), y_o)
    with pytest.raises(catt.CattError):                   # literal only
        catt.rows(dev(A), dev(x), y, catt.ROWS_SUM3, B=dev(BC), t=catt.Throttle(variant="coop"))
    with pytest.raises(catt.CattError):                   # B must hold both matrices
        catt.rows(dev(A), dev(x), y, catt.ROWS_SUM3, B=dev(BC[:m]), t=t)


@pytest.mark.parametrize("n", [64, 1024])
def test_coop_bit_exact_on_dyadic_inputs(n):
    A, p, r = (si.matrix(9, n, n, DYADIC), si.values(19, n, mode=DYADIC), si.values(29, n, mode=DYADIC))
    q_o, s_o = oracle.bicg(A, p, r)
    q, s = catt.bicg(dev(A), dev(p), dev(r), k1=catt.Throttle(variant="coop"), k2=catt.Throttle(variant="coop"))
    assert bits_equal(host(q), q_o) and bits_equal(host(s), s_o)


def test_empty_and_degenerate_shapes():
    # n = 0 columns: tmp is the empty sum 0, y is empty; m = 0 rows: y = 0
    A = torch.empty((5, 0), device="cuda")
    tmp, y = catt.atax(A, torch.empty(0, device="cuda"))
    assert np.all(host(tmp) == 0) and y.numel() == 0
    A = torch.empty((0, 7), device="cuda")
    tmp, y = catt.atax(A, torch.ones(7, device="cuda"))
    assert tmp.numel() == 0 and np.all(host(y) == 0)
    A = dev(si.matrix(4, 1, 1))
    tmp, y = catt.atax(A, dev(np.array([2.0], np.float32)))
    a = float(host(A)[0, 0])
    assert float(host(tmp)[0]) == np.float32(a * 2) and float(host(y)[0]) == np.float32(np.float32(a * 2) * a)


def test_invalid_arguments_raise():
    A, x = dev(si.matrix(1, 64, 64)), dev(si.values(2, 64))
    with pytest.raises(catt.CattError):
        catt.atax(A, x, k1=catt.Throttle(active_warps=9))                   # > warps per CTA
    with pytest.raises(catt.CattError):
        catt.atax(A, x, k1=catt.Throttle(carveout_kb=50))                   # not an option
    with pytest.raises(catt.CattError):
        catt.atax(A, x, k1=catt.Throttle(cta_threads=100))                  # not a warp multiple
    with pytest.raises(catt.CattError):
        catt.atax(A, x, k1=catt.Throttle(variant="staged", active_warps=1, cta_threads=64))
    with pytest.raises(catt.CattError):
        catt.atax(A.cpu(), x)                                                 # host tensor


# ------------------------------------------------------------------ throttles never change results
THROTTLES = [
    catt.Throttle(active_warps=1),
    catt.Throttle(active_warps=3),
    catt.Throttle(active_warps=4, gate=catt.GATE_BARRIER),
    catt.Throttle(active_warps=2, active_ctas=2),
    catt.Throttle(active_warps=1, active_ctas=1, carveout_kb=228),
    catt.Throttle(active_ctas=3, cap=catt.CAP_SMEM_PAD, carveout_kb=64),
    catt.Throttle(cta_threads=1024, active_warps=5, carveout_kb=196),
    catt.Throttle(cta_threads=64, active_warps=1, variant="vec4"),
]


@pytest.mark.parametrize("t", THROTTLES, ids=repr)
def test_throttled_results_identical(t):
    m, n = 3000, 68
    A, x = si.matrix(1, m, n), si.values(101, n)
    tmp_o, y_o = oracle.atax(A, x)
    tmp, y = catt.atax(dev(A), dev(x), k1=t, k2=t.copy(variant=catt.VAR_LITERAL))
    assert bits_equal(host(tmp), tmp_o) and bits_equal(host(y), y_o)


# ------------------------------------------------------------------ SYRK
@pytest.mark.parametrize("variant", ["literal", "staged"])
@pytest.mark.parametrize("n,m", [(64, 40), (130, 37), (256, 256)])
def test_syrk_exact(variant, n, m):
    A, C = si.matrix(6, n, m), si.matrix(106, n, n)
    C_o = oracle.syrk(A, C, 1.5, 1.2)
    Cd = dev(C)
    catt.syrk(dev(A), Cd, 1.5, 1.2, t=catt.Throttle(variant=variant))
    assert bits_equal(host(Cd), C_o)


@pytest.mark.parametrize("n,m,t", [(1601, 37, catt.Throttle(variant="staged")),
                                   (1537, 129, catt.Throttle(variant="staged", active_ctas=1)),
                                   (1664, 16, catt.Throttle(variant="staged"))])
def test_syrk_staged_large_tiles(n, m, t):
    """The two-CTA-per-SM tile kernel (T2: >= 148 tiles of 128 x 128) with a
    ragged edge (n % 128 != 0), a ragged last k stage (m % 16 != 0), one
    exact stage, and under a CTA cap."""
    A, C = si.matrix(6, n, m), si.matrix(106, n, n)
    C_o = oracle.syrk(A, C, 1.5, 1.2)
    Cd = dev(C)
    catt.syrk(dev(A), Cd, 1.5, 1.2, t=t)
    assert bits_equal(host(Cd), C_o)


@pytest.mark.parametrize("n,m", [(1001, 33), (1800, 21)])
def test_syrk_syr2k_mixed_tile_ragged(n, m):
    """The mixed 56-row T2 tile (warps 0-3: 8 rows, 4-7: 6 rows; chosen at
    these sizes by t2_use_mix): the last CTA of a strip holds 49 (n = 1001:
    seven warps active, the seventh partly; SYR2K, SYRK takes the 64 x 64
    small tile there) or 8 rows (n = 1800: one warp), with a ragged last k
    stage. SYRK and SYR2K bit-exact."""
    A, B, C = si.matrix(6, n, m), si.matrix(8, n, m), si.matrix(106, n, n)
    Cd = dev(C)
    catt.syrk(dev(A), Cd, 1.5, 1.2, t=catt.Throttle(variant="staged"))
    assert bits_equal(host(Cd), oracle.syrk(A, C, 1.5, 1.2))
    Cd = dev(C)
    catt.syr2k(dev(A), dev(B), Cd, 1.5, 1.2, t=catt.Throttle(variant="staged"))
    assert bits_equal(host(Cd), oracle.syr2k(A, B, C, 1.5, 1.2))


def test_t2_geometry_sweep_bit_exact():
    """Sizes around the switch between the mixed 56-row tile and the uniform
    64-row tile (one wave vs several, t2_use_mix) and ragged k: SYRK and SYR2K
    through T2 at each, bit-exact (the geometry never changes an element's
    k order)."""
    for n, m in [(1537, 9), (1999, 17), (2047, 5), (2101, 16), (2304, 3), (2561, 11)]:
        A, B, C = si.matrix(6, n, m), si.matrix(8, n, m), si.matrix(106, n, n)
        Cd = dev(C)
        catt.syrk(dev(A), Cd, 1.5, 1.2, t=catt.Throttle(variant="staged"))
        assert bits_equal(host(Cd), oracle.syrk(A, C, 1.5, 1.2)), n
        if n < 2200:
            Cd = dev(C)
            catt.syr2k(dev(A), dev(B), Cd, 1.5, 1.2, t=catt.Throttle(variant="staged"))
            assert bits_equal(host(Cd), oracle.syr2k(A, B, C, 1.5, 1.2)), n


@pytest.mark.parametrize("alpha,beta", [(1.0, 0.5), (1.5, 0.0), (-0.75, 1.0)])
def test_syrk_syr2k_staged_alpha_beta_forms(alpha, beta):
    """T2 with alpha == 1 (one k-major copy serves both operands), beta == 0
    and a negative alpha, SYRK and SYR2K, ragged n and m: bit-exact."""
    n, m = 1601, 37
    A, B, C = si.matrix(6, n, m), si.matrix(8, n, m), si.matrix(106, n, n)
    Cd = dev(C)
    catt.syrk(dev(A), Cd, alpha, beta, t=catt.Throttle(variant="staged"))
    assert bits_equal(host(Cd), oracle.syrk(A, C, alpha, beta))
    n2 = 300
    C2 = si.matrix(208, n2, n2)
    Cd = dev(C2)
    catt.syr2k(dev(A[:n2]), dev(B[:n2]), Cd, alpha, beta, t=catt.Throttle(variant="staged"))
    assert bits_equal(host(Cd), oracle.syr2k(A[:n2], B[:n2], C2, alpha, beta))


def test_syrk_throttled():
    A, C = si.matrix(6, 96, 64), si.matrix(106, 96, 96)
    C_o = oracle.syrk(A, C, 1.5, 1.2)
    for t in (catt.Throttle(active_warps=2), catt.Throttle(active_warps=1, active_ctas=2),
              catt.Throttle(cta_threads=512, active_warps=4, gate=catt.GATE_BARRIER)):
        Cd = dev(C)
        catt.syrk(dev(A), Cd, 1.5, 1.2, t=t)
        assert bits_equal(host(Cd), C_o)


# ------------------------------------------------------------------ SYR2K
@pytest.mark.parametrize("variant", ["literal", "staged"])
@pytest.mark.parametrize("n,m", [(64, 40), (130, 37), (257, 8), (256, 256), (1, 3)])
def test_syr2k_exact(variant, n, m):
    A, B, C = si.matrix(8, n, m), si.matrix(108, n, m), si.matrix(208, n, n)
    C_o = oracle.syr2k(A, B, C, 1.5, 1.2)
    Cd = dev(C)
    catt.syr2k(dev(A), dev(B), Cd, 1.5, 1.2, t=catt.Throttle(variant=variant))
    assert bits_equal(host(Cd), C_o)


def test_syr2k_empty_inner_and_throttled():
    n = 96
    C = si.matrix(208, n, n)
    Cd = dev(C)
    z = torch.empty(n, 0, device="cuda")
    catt.syr2k(z, z, Cd, 1.5, 1.25)
    assert bits_equal(host(Cd), (C * np.float32(1.25)).astype(np.float32))
    A, B = si.matrix(8, n, 64), si.matrix(108, n, 64)
    C_o = oracle.syr2k(A, B, C, 1.5, 1.2)
    for t in (catt.Throttle(active_warps=2), catt.Throttle(active_warps=4, active_ctas=2),
              catt.Throttle(cta_threads=512, active_warps=4, gate=catt.GATE_BARRIER),
              catt.Throttle(variant="staged", active_ctas=1)):
        Cd = dev(C)
        catt.syr2k(dev(A), dev(B), Cd, 1.5, 1.2, t=t)
        assert bits_equal(host(Cd), C_o)


def test_syr2k_2048_sampled_rows():
    """Table 2 P:77 size, both variants, rows spanning tile edges."""
    n = m = 2048
    A = torch.empty(n * m, device="cuda")
    B = torch.empty(n * m, device="cuda")
    C = torch.empty(n * n, device="cuda")
    catt.fill_hash(A, si.SEED_SYR2K)
    catt.fill_hash(B, si.sub_seed(si.SEED_SYR2K, 1))
    catt.fill_hash(C, si.sub_seed(si.SEED_SYR2K, 2))
    Ah = oracle.fill(si.SEED_SYR2K, n * m).reshape(n, m)
    Bh = oracle.fill(si.sub_seed(si.SEED_SYR2K, 1), n * m).reshape(n, m)
    Ch = oracle.fill(si.sub_seed(si.SEED_SYR2K, 2), n * n).reshape(n, n)
    rows = np.array([0, 7, 127, 128, 1111, 2047])
    want = oracle.syr2k_rows(Ah, Bh, Ch, 1.5, 1.2, rows)
    for v in ("literal", "staged"):
        Cd = C.clone().view(n, n)
        catt.syr2k(A.view(n, m), B.view(n, m), Cd, 1.5, 1.2, t=catt.Throttle(variant=v))
        assert bits_equal(host(Cd)[rows], want), v


def test_bypass_rows_equal_literal():
    """BYPASS is the literal loop with L2-only loads: bit-identical results."""
    m, n = 777, 301
    A, B = si.matrix(2, m, n), si.matrix(3, m, n)
    x, y0 = si.values(4, n), si.values(5, m)
    for mode in (catt.ROWS_STORE, catt.ROWS_ACCUM, catt.ROWS_GESUMMV):
        outs = []
        for v in ("literal", "bypass"):
            y, tmp = dev(y0), torch.empty(m, device="cuda")
            catt.rows(dev(A), dev(x), y, mode, B=dev(B), tmp=tmp, alpha=1.5, beta=1.2, t=catt.Throttle(variant=v))
            outs.append((host(y), host(tmp)))
        assert bits_equal(outs[0][0], outs[1][0])
        if mode == catt.ROWS_GESUMMV:
            assert bits_equal(outs[0][1], outs[1][1])
    t, r = catt.plan(catt.problem(catt.K_BICG_2, m=4096, n=4096), catt.Throttle(variant="bypass", carveout_kb=228),
                     catt.paper_rule(catt.hw_query()))
    assert r["flags"] == catt.FIT_NONE_NEEDED            # nothing of the divergent rows in L1


# ------------------------------------------------------------------ GEMM (CI control)
@pytest.mark.parametrize("variant", ["literal", "staged"])
@pytest.mark.parametrize("ni,nj,nk", [(64, 64, 64), (130, 70, 37), (257, 129, 8), (1, 3, 2), (512, 512, 512),
                                      (100, 130, 1), (2048, 1200, 64)])   # the last: 128 x 128 tiles
def test_gemm_exact(variant, ni, nj, nk):
    A, B, C = si.matrix(21, ni, nk), si.matrix(22, nk, nj), si.matrix(23, ni, nj)
    C_o = oracle.gemm(A, B, C, 1.5, 1.2)
    Cd = dev(C)
    catt.gemm(dev(A), dev(B), Cd, 1.5, 1.2, t=catt.Throttle(variant=variant))
    assert bits_equal(host(Cd), C_o)


def test_gemm_throttled_and_empty():
    A, B, C = si.matrix(21, 96, 40), si.matrix(22, 40, 70), si.matrix(23, 96, 70)
    C_o = oracle.gemm(A, B, C, 1.5, 1.2)
    for t in (catt.Throttle(active_warps=2), catt.Throttle(active_warps=4, active_ctas=1),
              catt.Throttle(cta_threads=512, active_warps=4, gate=catt.GATE_BARRIER)):
        Cd = dev(C)
        catt.gemm(dev(A), dev(B), Cd, 1.5, 1.2, t=t)
        assert bits_equal(host(Cd), C_o)
    Cd = dev(C)
    z1, z2 = torch.empty(96, 0, device="cuda"), torch.empty(0, 70, device="cuda")
    catt.gemm(z1, z2, Cd, 1.5, 1.25)
    assert bits_equal(host(Cd), (C * np.float32(1.25)).astype(np.float32))


# ------------------------------------------------------------------ CORR (give-up case)
@pytest.mark.parametrize("variant", ["literal", "staged"])
@pytest.mark.parametrize("n,m", [(300, 70), (128, 257), (33, 5), (1000, 129)])
def test_corr_exact(variant, n, m):
    data = si.matrix(24, n, m)
    data[:, 2] = 0.5                                  # a constant column: the eps branch
    sym_o, mean_o, std_o, d_o = oracle.corr(data)
    D = dev(data)
    sym, mean, std = catt.corr(D, t=catt.Throttle(variant=variant))
    assert bits_equal(host(D), d_o) and bits_equal(host(mean), mean_o) and bits_equal(host(std), std_o)
    assert bits_equal(host(sym), sym_o)


@pytest.mark.parametrize("n,m", [(37, 1604), (20, 1601), (300, 1664)])
def test_corr_staged_direct_and_transposed_forms(n, m):
    """STAGED CORR at sizes where the tiled SYRK is T2: m % 4 == 0 takes the
    direct form (column-strip statistics in place, T2 straight from the
    centred data; 1604 leaves a ragged 4-column strip), m = 1601 the
    transposed form. Bit-exact to the oracle, a constant column included."""
    data = si.matrix(24, n, m)
    data[:, 5] = 0.25
    sym_o, mean_o, std_o, d_o = oracle.corr(data)
    D = dev(data)
    sym, mean, std = catt.corr(D, t=catt.Throttle(variant="staged"))
    assert bits_equal(host(D), d_o) and bits_equal(host(mean), mean_o) and bits_equal(host(std), std_o)
    assert bits_equal(host(sym), sym_o)


def test_corr_2048_full_size():
    """Table 2 P:81 size (2K x 2K), both variants, and a throttled literal run."""
    n = m = 2048
    data = oracle.fill(si.SEED_CORR, n * m).reshape(n, m)
    sym_o, mean_o, std_o, _ = oracle.corr(data)
    for t in (catt.Throttle(variant="staged"), catt.Throttle(), catt.Throttle(active_warps=4)):
        D = torch.empty(n * m, device="cuda")
        catt.fill_hash(D, si.SEED_CORR)
        sym, mean, std = catt.corr(D.view(n, m), t=t)
        assert bits_equal(host(sym), sym_o) and bits_equal(host(mean), mean_o), t


# ------------------------------------------------------------------ KMEANS
@pytest.mark.parametrize("variant", ["literal", "regs", "staged", "coop"])
def test_kmeans_distance_fused_per_feature(variant):
    """R16 on the device: the crafted case of the oracle pin
    tests/test_oracle.py::test_kmeans_distance_is_fused_per_feature (equal
    exact distances, one rounding per feature makes centre 1 nearer; an
    unfused order would tie and pick centre 0). Every point at the origin."""
    a, b = np.float32(0.7971469759941101), np.float32(0.13876742124557495)
    npts, nf = 64, 2
    feat = np.zeros(nf * npts, np.float32)
    cl = np.array([[a, b], [b, a]], np.float32)
    memb_o, _ = oracle.kmeans_assign(feat, npts, npts, nf, cl)
    assert np.all(memb_o == 1)
    memb = catt.kmeans_assign(dev(feat), npts, npts, nf, dev(cl), t=catt.Throttle(variant=variant))
    assert np.array_equal(host(memb), memb_o)


@pytest.mark.parametrize("variant", ["literal", "regs", "staged", "coop"])
@pytest.mark.parametrize("npts,nf,k,pad", [(1000, 34, 5, 4), (4099, 34, 5, 29), (257, 7, 3, 3), (300, 50, 12, 4),
                                           (70000, 34, 5, 4), (1, 3, 1, 3), (131, 34, 8, 1), (130, 9, 2, 2)])
def test_kmeans_exact(variant, npts, nf, k, pad):
    ld = npts + pad
    if variant in ("staged", "coop") and ld % 4:
        ld += 4 - ld % 4                                 # TMA rows / 16-byte loads need a 16-byte stride
    if variant == "coop" and k > 8:
        with pytest.raises(catt.CattError):
            catt.kmeans_assign(dev(si.values(4, nf * ld)), ld, npts, nf, dev(np.zeros((k, nf), np.float32)),
                               t=catt.Throttle(variant="coop"))
        return
    feat = si.values(4, nf * ld)
    clusters = feat.reshape(nf, ld)[:, :k].T.copy()          # centres = first k points
    memb_o, _ = oracle.kmeans_assign(feat, ld, npts, nf, clusters)
    ts = [catt.Throttle(variant=variant)]
    if variant not in ("staged", "coop"):                # staged / coop have no L1 reuse to throttle
        ts.append(catt.Throttle(variant=variant, active_warps=2, active_ctas=3))
    for t in ts:
        memb = catt.kmeans_assign(dev(feat), ld, npts, nf, dev(clusters), t=t)
        assert np.array_equal(host(memb), memb_o)


# ------------------------------------------------------------------ full BASELINE sizes
def test_bicg_mvt_4096_full():
    n = 4096
    A = torch.empty(n * n, device="cuda")
    catt.fill_hash(A, si.SEED_BICG)
    Ah = oracle.fill(si.SEED_BICG, n * n).reshape(n, n)
    p, r = si.values(si.sub_seed(si.SEED_BICG, 1), n), si.values(si.sub_seed(si.SEED_BICG, 2), n)
    q_o, s_o = oracle.bicg(Ah, p, r)
    q64, s64 = oracle.bicg(Ah, p, r, mode=oracle.SEQ_F64)
    A = A.view(n, n)
    for v in ("literal", "vec4", "staged", "coop"):
        q, s = catt.bicg(A, dev(p), dev(r), k1=catt.Throttle(variant=v), k2=catt.Throttle(variant=v))
        q, s = host(q), host(s)
        if v == "coop":
            assert relerr(q, q64) <= TOL and relerr(s, s64) <= TOL
        else:
            assert bits_equal(q, q_o) and bits_equal(s, s_o)


def test_kmeans_rodinia_shape_full():
    npts, nf, k = 494020, 34, 5
    for ld in (494020, 494048):
        feat = torch.empty(nf * ld, device="cuda")
        catt.fill_hash(feat, si.SEED_KMEANS)
        fh = oracle.fill(si.SEED_KMEANS, nf * ld)
        clusters = fh.reshape(nf, ld)[:, :k].T.copy()
        memb_o, _ = oracle.kmeans_assign(fh, ld, npts, nf, clusters)
        hw = catt.hw_query()
        t, r = catt.plan(catt.problem(catt.K_KMEANS, m=npts, n=nf, k=k, ld=ld), catt.Throttle(), hw)
        # the bench's launch: STAGED planned by CATT (Eq 4 -> the 228 KB carveout, 2 CTAs per SM)
        tb, _ = catt.plan(catt.problem(catt.K_KMEANS, m=npts, n=nf, k=k, ld=ld),
                          catt.Throttle(cta_threads=256, variant="staged"), hw)
        assert tb.carveout_kb == 228
        for tt in (catt.Throttle(), t, catt.Throttle(variant="regs"), catt.Throttle(variant="staged"),
                   catt.Throttle(variant="coop"), tb):
            memb = catt.kmeans_assign(feat, ld, npts, nf, dev(clusters), t=tt)
            assert np.array_equal(host(memb), memb_o)


def test_gesummv_8192_full():
    n = 8192
    A, B = torch.empty(n * n, device="cuda"), torch.empty(n * n, device="cuda")
    catt.fill_hash(A, si.SEED_GESUMMV)
    catt.fill_hash(B, si.sub_seed(si.SEED_GESUMMV, 1))
    x = si.values(si.sub_seed(si.SEED_GESUMMV, 2), n)
    Ah = oracle.fill(si.SEED_GESUMMV, n * n).reshape(n, n)
    Bh = oracle.fill(si.sub_seed(si.SEED_GESUMMV, 1), n * n).reshape(n, n)
    y_o, t_o = oracle.gesummv(Ah, Bh, x, 1.5, 1.2)
    y64, _ = oracle.gesummv(Ah, Bh, x, 1.5, 1.2, mode=oracle.SEQ_F64)
    for v in ("literal", "staged", "coop"):
        y, tmp = catt.gesummv(A.view(n, n), B.view(n, n), dev(x), 1.5, 1.2, t=catt.Throttle(variant=v))
        if v == "coop":
            assert relerr(host(y), y64) <= TOL
        else:
            assert bits_equal(host(y), y_o) and bits_equal(host(tmp), t_o)


def test_syrk_2048_sampled_rows():
    n = m = 2048
    A = torch.empty(n * m, device="cuda")
    C = torch.empty(n * n, device="cuda")
    catt.fill_hash(A, si.SEED_SYRK)
    catt.fill_hash(C, si.sub_seed(si.SEED_SYRK, 1))
    Ah = oracle.fill(si.SEED_SYRK, n * m).reshape(n, m)
    Ch = oracle.fill(si.sub_seed(si.SEED_SYRK, 1), n * n).reshape(n, n)
    rows = np.array([0, 1, 127, 128, 1000, 2047])
    want = oracle.syrk_rows(Ah, Ch, 1.5, 1.2, rows)
    for v in ("literal", "staged"):
        Cd = C.clone().view(n, n)
        catt.syrk(A.view(n, m), Cd, 1.5, 1.2, t=catt.Throttle(variant=v))
        assert bits_equal(host(Cd)[rows], want), v


def test_atax_65536x16384_sampled():
    m, n = 65536, 16384
    A = torch.empty(m * n, device="cuda")
    catt.fill_hash(A, si.SEED_ATAX_SHARDED)
    x = si.values(si.sub_seed(si.SEED_ATAX_SHARDED, 1), n)
    cols = np.array([0, 1, 31, 32, 4097, 16383])
    tmp_o, y_o = oracle.atax_hashed(si.SEED_ATAX_SHARDED, 0, x, m, n, cols)
    tmp, y = catt.atax(A.view(m, n), dev(x), k1=catt.Throttle(variant="staged"), k2=catt.Throttle(variant="staged"))
    assert bits_equal(host(tmp), tmp_o) and bits_equal(host(y)[cols], y_o)
    tmp, y = catt.atax(A.view(m, n), dev(x), k1=catt.Throttle(variant="coop"), k2=catt.Throttle(variant="coop"))
    t64, y64 = oracle.atax_hashed(si.SEED_ATAX_SHARDED, 0, x, m, n, cols, mode=oracle.SEQ_F64)
    assert relerr(host(tmp), t64) <= TOL and relerr(host(y)[cols], y64) <= TOL


# ------------------------------------------------------------------ throttle enforcement (residency probe)
def _max_overlap(ivs):
    ev = sorted([(a, 1) for a, b in ivs] + [(b, -1) for a, b in ivs])   # ends before starts at equal stamps
    cur = best = 0
    for _, d in ev:
        cur += d
        best = max(best, cur)
    return best


def _concurrency(rec, W):
    """rec: [ncta*W, 3] (smid, t0, t1) per warp around the loop. Returns the
    most warps of one CTA inside the loop at once, the most CTAs of one SM
    with a warp inside the loop at once, and the most warps of one SM inside
    the loop at once."""
    rec = rec.reshape(-1, W, 3)
    valid = rec[:, :, 2] > 0
    max_w = max(_max_overlap([(rec[c, w, 1], rec[c, w, 2]) for w in range(W) if valid[c, w]])
                for c in range(rec.shape[0]))
    cta_iv, warp_iv = {}, {}
    for c in range(rec.shape[0]):
        if not valid[c].any():
            continue
        sm = int(rec[c, valid[c], 0][0])
        cta_iv.setdefault(sm, []).append((rec[c, valid[c], 1].min(), rec[c, valid[c], 2].max()))
        warp_iv.setdefault(sm, []).extend((rec[c, w, 1], rec[c, w, 2]) for w in range(W) if valid[c, w])
    max_c = max(_max_overlap(v) for v in cta_iv.values())
    max_ws = max(_max_overlap(v) for v in warp_iv.values())
    return max_w, max_c, max_ws


def _steady_warps(rec, W):
    """The number of warps of one SM inside the loop that holds for the most
    time, summed over SMs (the time-weighted mode of the per-SM step
    function). A warp slot is released when its warp exits, so a new CTA can
    start while the last warps of two older ones still run: the maximum then
    briefly exceeds a*T by one CTA's a; the steady state is a*T exactly."""
    rec = rec.reshape(-1, 3)
    rec = rec[rec[:, 2] > 0]
    dur = {}
    for sm in np.unique(rec[:, 0]):
        r = rec[rec[:, 0] == sm]
        ev = sorted([(int(a), 1) for a in r[:, 1]] + [(int(b), -1) for b in r[:, 2]], key=lambda e: (e[0], e[1]))
        cur, last = 0, None
        for t, d in ev:
            if last is not None and t > last and cur > 0:
                dur[cur] = dur.get(cur, 0) + (t - last)
            cur += d
            last = t
    return max(dur, key=dur.get)


@pytest.mark.parametrize("t,want", [
    (catt.Throttle(carveout_kb=16), (8, 0, 64)),
    (catt.Throttle(active_warps=2, carveout_kb=16), (2, 0, 16)),
    (catt.Throttle(active_warps=4, gate=catt.GATE_BARRIER, carveout_kb=16), (4, 0, 32)),
    (catt.Throttle(active_warps=1, active_ctas=3, carveout_kb=16), (1, 3, 3)),
    (catt.Throttle(active_ctas=2, cap=catt.CAP_SMEM_PAD, carveout_kb=64), (8, 2, 16)),
], ids=repr)
def test_residency_probe_enforces_throttle(t, want):
    """a6 (Fig 4/5) and a1 (Eq 1-4): the measured concurrency equals the
    throttle -- warps per CTA inside the loop (a), CTAs per SM inside the loop
    under a CTA cap (m), and warps per SM inside the loop (a * T, or a * m).
    Full TLP co-schedules W * T = 8 * 8 = 64 warps per SM at the carveout Eq 4
    picks (16 KB for 8 CTAs of 1 KB reserved + 16 B). Without a cap the
    number of CTAs with a warp in the loop can exceed T (a warp's slot is
    freed when the warp exits, so the next CTA starts while the last warps of
    the previous one still run), so T is checked through the warps per SM.
    A forced small carveout does not cap CTAs: the driver takes a larger
    shared-memory configuration when that fits more CTAs (8 KB forced: 12 CTAs
    measured), which is why the library's CTA cap is the per-SM counter."""
    # long rows so CTAs overlap in time; 148 SMs x 8 CTAs x 256 rows x 2 waves
    m, n = 148 * 8 * 256 * 2, 512
    prob = catt.problem(catt.K_ATAX_1, m=m, n=n)
    _, r = catt.plan(prob, catt.Throttle(carveout_kb=t.carveout_kb), catt.hw_query())
    _, r0 = catt.plan(prob, catt.Throttle(), catt.hw_query())
    assert r0["carveout_kb"] == 16 and (r0["base_warps"], r0["base_ctas"]) == (8, 8)   # Eq 4's own pick
    A = torch.empty(m * n, device="cuda")
    catt.fill_hash(A, 1)
    x = torch.ones(n, device="cuda")
    ncta = m // 256
    probe = torch.zeros(ncta * 8 * 3, dtype=torch.int64, device="cuda")
    tt = t.copy(probe=probe.data_ptr())
    catt.atax(A.view(m, n), x, k1=tt)
    rec = host(probe).astype(np.int64)
    mw, mc, mws = _concurrency(rec, 8)
    assert mw == want[0]                                   # the warp slots: used and never exceeded
    if want[1]:
        assert mc == want[1]                               # the CTA cap: used and never exceeded
        assert mws == want[2]                              # a * m warps per SM in the loop, never more
    else:
        assert _steady_warps(rec, 8) == want[2]            # a * T warps per SM in the loop in steady state
        assert want[2] <= mws <= want[2] + want[0]         # + one CTA's a at a hand-over (slots freed per warp)


P_ = catt.problem
OCC_CASES = [   # (problem, launch, extra dynamic smem): register-, smem-, warp- and CTA-slot-limited launches
    (P_(catt.K_ATAX_1, m=1 << 22, n=256), catt.Throttle(), 0),                              # 8 warps: #TB_HW
    (P_(catt.K_ATAX_1, m=1 << 22, n=256), catt.Throttle(cta_threads=384), 0),               # 12 warps: 64 // 12
    (P_(catt.K_ATAX_1, m=1 << 22, n=256), catt.Throttle(cta_threads=1024), 0),
    (P_(catt.K_ATAX_1, m=1 << 22, n=256), catt.Throttle(cta_threads=32), 0),                # 32-CTA slot limit
    (P_(catt.K_ATAX_1, m=1 << 22, n=4096), catt.Throttle(variant="staged"), 0),              # row_tma: >= 128 regs + ring
    (P_(catt.K_ATAX_1, m=1 << 22, n=4096), catt.Throttle(variant="staged", cta_threads=64), 0),
    (P_(catt.K_GESUMMV, n=1 << 20), catt.Throttle(variant="staged"), 0),
    (P_(catt.K_ATAX_2, m=4096, n=1 << 22), catt.Throttle(variant="staged"), 0),
    (P_(catt.K_SYRK, n=16384, k=2048), catt.Throttle(variant="staged"), 0),                 # tiled: 128+ regs
    (P_(catt.K_SYR2K, n=16384, k=2048), catt.Throttle(variant="staged"), 0),
    (P_(catt.K_GEMM, m=16384, n=16384, k=512), catt.Throttle(variant="staged"), 0),
    (P_(catt.K_KMEANS, m=494020 * 8, n=34, k=5, ld=494020 * 8), catt.Throttle(variant="staged"), 0),   # ~106 KB ring
    (P_(catt.K_KMEANS, m=494020 * 8, n=34, k=5, ld=494020 * 8), catt.Throttle(), 0),
    (P_(catt.K_KMEANS_T, m=494020 * 8, n=34, ld=494020 * 8), catt.Throttle(variant="coop"), 0),
    (P_(catt.K_ATAX_1, m=1 << 22, n=256), catt.Throttle(), 100 * 1024),                     # Fig 5 pads: 2, 3, 5 CTAs
    (P_(catt.K_ATAX_1, m=1 << 22, n=256), catt.Throttle(), 70 * 1024),
    (P_(catt.K_ATAX_1, m=1 << 22, n=256), catt.Throttle(), 40 * 1024),
]


@pytest.mark.parametrize("prob,launch,pad", OCC_CASES, ids=[f"{c[0].loop}-{c[1]!r}-{c[2]}" for c in OCC_CASES])
def test_occupancy_model_matches_cuda_occupancy_api(prob, launch, pad):
    """a1 pin (Eq 1-3, the B200 arm of reading R9): the analyser's
    #TB_SM from the kernel's real registers and shared memory equals what the
    CUDA runtime computes for the same kernel, CTA size and dynamic shared
    memory at the largest carveout (Eq 1 divides the maximum shared memory);
    the grids are large enough that ceil(grid / #SM) does not bind."""
    hw = catt.hw_query()
    assert hw.num_sms == 148
    api, dyn = catt.kernel_occupancy(prob, launch, pad)
    d, keep = catt.kernel_desc(prob, launch)
    regs, ssm = catt.kernel_attrs(prob, launch)
    assert d.regs_per_thread == regs
    assert d.smem_per_cta + pad == ssm + dyn
    d.smem_per_cta += pad
    r = catt.footprint(d, hw)
    grid = d.grid[0] * d.grid[1] * d.grid[2]
    # persistent kernels size their grid to the occupancy: there the grid bound
    # (R8) equals it; everywhere else the grid is large enough not to bind
    want = min(api, -(-grid // 148))
    assert r["base_ctas"] == want, dict(api=api, regs=regs, smem=ssm, dyn=dyn, threads=d.block[0] * d.block[1],
                                        grid=grid, model=r["base_ctas"])


# ------------------------------------------------------------------ FUSED (both loops in one pass)
FUSED_SHAPES = [(33, 4), (300, 64), (1000, 132), (257, 4096), (700, 8192), (130, 16384)]   # NW = 8, 16, 32


@pytest.mark.parametrize("m,n", FUSED_SHAPES)
def test_fused_bicg_mvt_atax(m, n):
    A, p, r = si.matrix(2, m, n), si.values(102, n), si.values(202, m)
    q64, s64 = oracle.bicg(A, p, r, mode=oracle.SEQ_F64)
    q, s = catt.bicg(dev(A), dev(p), dev(r), k1=catt.Throttle(variant="fused"))
    assert relerr(host(q), q64) <= TOL and relerr(host(s), s64) <= TOL
    # dyadic: every partial sum exact -> bit-exact to the sequential oracle
    D = si.MODE_DYADIC
    Ad, pd, rd = si.matrix(3, m, n, D), si.values(4, n, mode=D), si.values(5, m, mode=D)
    qo, so = oracle.bicg(Ad, pd, rd)
    q, s = catt.bicg(dev(Ad), dev(pd), dev(rd), k1=catt.Throttle(variant="fused"))
    assert bits_equal(host(q), qo) and bits_equal(host(s), so)
    # ATAX (dependent: y uses the finished tmp)
    x = si.values(101, n)
    t64, y64 = oracle.atax(A, x, mode=oracle.SEQ_F64)
    tmp, y = catt.atax(dev(A), dev(x), k1=catt.Throttle(variant="fused"))
    assert relerr(host(tmp), t64) <= TOL and relerr(host(y), y64) <= TOL


@pytest.mark.parametrize("n", [64, 1024, 4096])
def test_fused_mvt_inout(n):
    a = si.matrix(3, n, n)
    y1, y2, x1, x2 = (si.values(103 + 100 * k, n) for k in range(4))
    e1, e2 = oracle.mvt(a, y1, y2, x1, x2, mode=oracle.SEQ_F64)
    X1, X2 = dev(x1), dev(x2)
    catt.mvt(dev(a), dev(y1), dev(y2), X1, X2, k1=catt.Throttle(variant="fused"))
    assert relerr(host(X1), e1) <= TOL and relerr(host(X2), e2) <= TOL


def test_dual_flags_and_errors():
    m, n = 500, 256
    A, xr, xc = si.matrix(7, m, n), si.values(8, n), si.values(9, m)
    yr0, yc0 = si.values(10, m), si.values(11, n)
    YR, YC = dev(yr0), dev(yc0)
    catt.dual(dev(A), dev(xr), YR, YC, xc=dev(xc), row_accumulate=True, col_accumulate=False)
    _, s64 = oracle.bicg(A, xr, xc, mode=oracle.SEQ_F64)
    assert relerr(host(YC), s64) <= TOL
    q64 = yr0.astype(np.float64) + A.astype(np.float64) @ xr.astype(np.float64)
    assert relerr(host(YR), q64) <= TOL
    with pytest.raises(catt.CattError):
        catt.dual(dev(A), dev(xr), YR, YC, xc=dev(xc), t=catt.Throttle(active_warps=2))     # nothing to throttle
    with pytest.raises(catt.CattError):
        catt.dual(dev(A), dev(xr), YR, YC, row_accumulate=True, dependent=True)


def test_fused_atax_65536x16384_sampled():
    m, n = 65536, 16384
    A = torch.empty(m * n, device="cuda")
    catt.fill_hash(A, si.SEED_ATAX_SHARDED)
    x = si.values(si.sub_seed(si.SEED_ATAX_SHARDED, 1), n)
    cols = np.array([0, 1, 31, 32, 4097, 16383])
    t64, y64 = oracle.atax_hashed(si.SEED_ATAX_SHARDED, 0, x, m, n, cols, mode=oracle.SEQ_F64)
    tmp, y = catt.atax(A.view(m, n), dev(x), k1=catt.Throttle(variant="fused"))
    assert relerr(host(tmp), t64) <= TOL and relerr(host(y)[cols], y64) <= TOL


@pytest.mark.parametrize("shapes", [[(1000, 132), (300, 132)], [(4096, 4096), (4096, 4096)], [(33, 64), (5000, 64), (7, 64)]])
def test_dual_group_bicg_and_mvt_in_one_launch(shapes):
    """BICG and MVT problems (same n) in one grouped fused launch."""
    probs, want = [], []
    for k, (m, n) in enumerate(shapes):
        A = si.matrix(20 + k, m, n, si.MODE_DYADIC)
        xr, xc = si.values(30 + k, n, mode=si.MODE_DYADIC), si.values(40 + k, m, mode=si.MODE_DYADIC)
        yr0, yc0 = si.values(50 + k, m, mode=si.MODE_DYADIC), si.values(60 + k, n, mode=si.MODE_DYADIC)
        acc = k % 2 == 1                                   # odd problems: MVT-style in/out
        YR, YC = dev(yr0), dev(yc0)
        probs.append(dict(A=dev(A), xr=dev(xr), xc=dev(xc), yr=YR, yc=YC, row_accumulate=acc, col_accumulate=acc))
        q, s = oracle.bicg(A, xr, xc)                         # dyadic: exact, any order
        if acc:
            q = (yr0.astype(np.float64) + q).astype(np.float32)
            s = (yc0.astype(np.float64) + s).astype(np.float32)
        want.append((YR, YC, q, s))
    catt.dual_group(probs)
    for YR, YC, q, s in want:
        assert bits_equal(host(YR), q) and bits_equal(host(YC), s)


def _dual_case(shapes, seed0):
    probs, want = [], []
    for k, (m, n) in enumerate(shapes):
        A = si.matrix(seed0 + k, m, n, si.MODE_DYADIC)
        xr, xc = si.values(seed0 + 10 + k, n, mode=si.MODE_DYADIC), si.values(seed0 + 20 + k, m, mode=si.MODE_DYADIC)
        yr0, yc0 = si.values(seed0 + 30 + k, m, mode=si.MODE_DYADIC), si.values(seed0 + 40 + k, n, mode=si.MODE_DYADIC)
        acc = k % 2 == 1
        YR, YC = dev(yr0), dev(yc0)
        probs.append(dict(A=dev(A), xr=dev(xr), xc=dev(xc), yr=YR, yc=YC, row_accumulate=acc, col_accumulate=acc))
        q, s = oracle.bicg(A, xr, xc)
        if acc:
            q = (yr0.astype(np.float64) + q).astype(np.float32)
            s = (yc0.astype(np.float64) + s).astype(np.float32)
        want.append((YR, YC, yr0, yc0, q, s))
    return probs, want


@pytest.mark.parametrize("barrier", ["0", "1", "2"])
def test_dual_group_barrier_modes_repeated(barrier, monkeypatch):
    """Every grid-barrier form of the single-read fused kernel (0: fenced
    count/generation, 1: ordered atomics, 2: per-problem monotonic arrival
    counters with host-tracked targets, the default) over repeated launches
    whose groups change shape (so the per-problem CTA counts, and with them
    the arrival targets, change between launches): bit-exact every time."""
    monkeypatch.setenv("CATT_FUSED_BARRIER", barrier)
    cases = [_dual_case([(4096, 4096), (4096, 4096)], 300), _dual_case([(33, 64), (5000, 64), (7, 64)], 400),
             _dual_case([(1000, 132), (300, 132)], 500)]
    for rep in range(7):
        probs, want = cases[rep % 3]
        for p, (YR, YC, yr0, yc0, _, _) in zip(probs, want):
            YR.copy_(dev(yr0))
            YC.copy_(dev(yc0))
        catt.dual_group(probs)
        for YR, YC, _, _, q, s in want:
            assert bits_equal(host(YR), q) and bits_equal(host(YC), s), (barrier, rep)


def test_dual_group_default_launch_uniform_vs_f64_oracle():
    """The bench's default configs[1] launch as it runs there: BICG and MVT
    4096^2 in one grouped single-read launch, on uniform (inexact) inputs,
    every output element within 1e-5 of the fp64 sequential oracle (the
    dyadic tests above pin the order; this pins the arithmetic on the
    distribution the bench uses)."""
    n = 4096
    Ab, Am = si.matrix(si.SEED_BICG, n, n), si.matrix(si.SEED_MVT, n, n)
    p, r = si.values(102, n), si.values(202, n)
    y1, y2, x1, x2 = (si.values(s, n) for s in (103, 203, 104, 204))
    q, s_ = torch.zeros(n, device="cuda"), torch.zeros(n, device="cuda")
    X1, X2 = dev(x1), dev(x2)
    catt.dual_group([dict(A=dev(Ab), xr=dev(p), xc=dev(r), yr=q, yc=s_),
                     dict(A=dev(Am), xr=dev(y1), xc=dev(y2), yr=X1, yc=X2, row_accumulate=True, col_accumulate=True)])
    q64, s64 = oracle.bicg(Ab, p, r, mode=oracle.SEQ_F64)
    x1_64, x2_64 = oracle.mvt(Am, y1, y2, x1, x2, mode=oracle.SEQ_F64)
    assert relerr(host(q), q64) <= TOL and relerr(host(s_), s64) <= TOL
    assert relerr(host(X1), x1_64) <= TOL and relerr(host(X2), x2_64) <= TOL


def test_dual_group_uniform_same_bits_every_barrier(monkeypatch):
    """The barrier form changes only when the partials are read, never the
    order they are added in: uniform (inexact) inputs give the same bits."""
    n = 2048
    A, B = dev(si.matrix(71, n, n)), dev(si.matrix(72, n, n))
    v = [dev(si.values(80 + i, n)) for i in range(8)]
    outs = []
    for barrier in ("0", "1", "2"):
        monkeypatch.setenv("CATT_FUSED_BARRIER", barrier)
        yr1, yc1, yr2, yc2 = (torch.zeros(n, device="cuda") for _ in range(4))
        catt.dual_group([dict(A=A, xr=v[0], xc=v[1], yr=yr1, yc=yc1), dict(A=B, xr=v[2], xc=v[3], yr=yr2, yc=yc2)])
        outs.append([host(t) for t in (yr1, yc1, yr2, yc2)])
    for o in outs[1:]:
        for a_, b_ in zip(outs[0], o):
            assert bits_equal(a_, b_)


def test_dual_group_graph_capture_replays():
    """A captured grouped launch falls back to the self-resetting barrier (the
    arrival targets of the default form are host-tracked and would go stale
    in a replay): three replays with new inputs are bit-exact."""
    probs, want = _dual_case([(4096, 4096), (4096, 4096)], 600)
    catt.dual_group(probs)                      # grows the workspace outside the capture
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        catt.dual_group(probs)
    for rep in range(3):
        for p, (YR, YC, yr0, yc0, _, _) in zip(probs, want):
            YR.copy_(dev(yr0))
            YC.copy_(dev(yc0))
        g.replay()
        torch.cuda.synchronize()
        for YR, YC, _, _, q, s in want:
            assert bits_equal(host(YR), q) and bits_equal(host(YC), s), rep
    catt.dual_group(probs)                      # the default form after a capture still agrees
    for p, (YR, YC, yr0, yc0, _, _) in zip(probs, want):
        YR.copy_(dev(yr0))
        YC.copy_(dev(yc0))
    catt.dual_group(probs)
    for YR, YC, _, _, q, s in want:
        assert bits_equal(host(YR), q) and bits_equal(host(YC), s)


# ------------------------------------------------------------------ SM partition (green context)
@pytest.mark.parametrize("min_sms", [8, 16])
def test_sm_partition_confines_ctas_and_keeps_results(min_sms):
    """catt_sm_partition_create: launches on the partition's stream run on at
    most `sms` distinct SMs (residency probe %smid), plan with num_sms = sms
    gives the multi-CTA-per-SM base of Eq 3 (SURVEY 8(d) [3]: GESUMMV's 32
    CTAs at 4 / 2 per SM), a CTA cap is enforced there, and results are the
    literal loop's (bit-exact to seq-fmaf)."""
    with catt.SmPartition(min_sms) as part:
        assert min_sms <= part.sms < 148
        hw = part.hw(catt.hw_query())
        assert hw.num_sms == part.sms
        n = 8192
        t, r = catt.plan(catt.problem(catt.K_GESUMMV, n=n), catt.Throttle(cta_threads=256, carveout_kb=8,
                                                                          variant="literal"), hw)
        assert r["base_ctas"] == min(8, -(-32 // part.sms))
        m, nn = 64 * 256, 256                                   # 64 CTAs of 256 rows
        A = torch.empty(m * nn, device="cuda")
        catt.fill_hash(A, 1)
        x = torch.ones(nn, device="cuda")
        probe = torch.zeros((m // 256) * 8 * 3, dtype=torch.int64, device="cuda")
        with torch.cuda.stream(part.stream):
            tmp, y = catt.atax(A.view(m, nn), x, k1=catt.Throttle(active_ctas=2, probe=probe.data_ptr()))
        part.stream.synchronize()
        rec = host(probe).astype(np.int64).reshape(-1, 3)
        sms = set(int(s) for s in rec[rec[:, 2] > 0, 0])
        assert 1 <= len(sms) <= part.sms
        mw, mc, mws = _concurrency(rec, 8)
        assert mc == 2 and mws <= 16
        Ah = oracle.fill(1, m * nn).reshape(m, nn)
        tmp_o, y_o = oracle.atax(Ah, np.ones(nn, dtype=np.float32))
        assert bits_equal(host(tmp), tmp_o) and bits_equal(host(y), y_o)


def test_sm_partition_errors():
    with pytest.raises(catt.CattError):
        catt.SmPartition(0)
    with pytest.raises(catt.CattError):
        catt.SmPartition(10_000)


# ------------------------------------------------------------------ ATAX in one kernel, a throttle per loop
@pytest.mark.parametrize("m,n,k1,k2", [
    (1000, 700, catt.Throttle(), catt.Throttle()),
    (4096, 260, catt.Throttle(cta_threads=1024, active_warps=8, carveout_kb=196), catt.Throttle()),
    (513, 2049, catt.Throttle(cta_threads=256, active_warps=2, carveout_kb=228), catt.Throttle(active_warps=8)),
    (3000, 3000, catt.Throttle(cta_threads=256, active_warps=4, active_ctas=1, carveout_kb=228),
     catt.Throttle(active_warps=1, active_ctas=1)),
    (777, 1500, catt.Throttle(cta_threads=512, active_warps=4, gate=catt.GATE_BARRIER), catt.Throttle(active_warps=2)),
], ids=repr)
def test_atax_onekernel_per_loop_throttles_exact(m, n, k1, k2):
    """Both literal loops in one cooperative kernel, each under its own warp
    gate, the CTA cap for the whole kernel: bit-exact
    to the sequential oracle whatever the throttles."""
    A, x = si.matrix(1, m, n), si.values(101, n)
    tmp_o, y_o = oracle.atax(A, x)
    tmp, y = catt.atax_onekernel(dev(A), dev(x), k1=k1, k2=k2)
    assert bits_equal(host(tmp), tmp_o) and bits_equal(host(y), y_o)


def test_atax_onekernel_rejects_a_second_launch_shape():
    A, x = dev(si.matrix(1, 64, 64)), dev(si.values(101, 64))
    with pytest.raises(catt.CattError):                      # loop 2 cannot change the CTA size
        catt.atax_onekernel(A, x, k1=catt.Throttle(cta_threads=256), k2=catt.Throttle(cta_threads=512))
    with pytest.raises(catt.CattError):                      # nor the kernel's CTA cap
        catt.atax_onekernel(A, x, k1=catt.Throttle(active_ctas=2), k2=catt.Throttle(active_ctas=1))
    with pytest.raises(catt.CattError):                      # LITERAL only
        catt.atax_onekernel(A, x, k1=catt.Throttle(variant="coop"))
