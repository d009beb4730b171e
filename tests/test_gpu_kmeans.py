"""GPU parity of the KMEANS full iteration against
oracle/kmeans.py: transpose (bit-exact copy), assignment + exact centroid sums
+ rounding (bit-exact), the device loop (bit-exact memberships, centres and
iteration count), partition invariance of the sums, and the inexact flag."""
import numpy as np
import pytest
import torch

import oracle
from oracle import kmeans as okm
import seeded_inputs as si
import paper_conf_icpp_kimhlsh19_b200 as catt

pytestmark = pytest.mark.gpu


def dev(a, dtype=None):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def feat_fm(seed, npts, nf, ld, mode=si.MODE_UNIFORM):
    """feature-major features with zero padding columns"""
    v = si.values(seed, nf * ld, mode=mode).reshape(nf, ld)
    v[:, npts:] = 0
    return v.ravel()


def first_k(feat, ld, nf, k):
    return np.stack([feat[f * ld:f * ld + k] for f in range(nf)], axis=1).astype(np.float32)


@pytest.mark.parametrize("variant", ["literal", "coop"])
@pytest.mark.parametrize("npts,nf,pad", [(1, 1, 0), (257, 7, 0), (1000, 34, 4), (70001, 34, 29), (300, 64, 3)])
def test_transpose_exact(variant, npts, nf, pad):
    ld = npts + pad
    pm = si.values(31, npts * nf)
    out = torch.full((nf * ld,), -7.0, device="cuda")
    catt.kmeans_transpose(dev(pm), npts, nf, out, ld, t=catt.Throttle(variant=variant))
    want = okm.transpose(pm, npts, nf, ld)
    got = host(out).reshape(nf, ld)
    assert np.array_equal(got[:, :npts], want.reshape(nf, ld)[:, :npts])
    assert np.all(got[:, npts:] == -7.0)                      # padding columns untouched


def test_transpose_throttled_literal():
    npts, nf = 5000, 34
    pm = si.values(32, npts * nf)
    want = okm.transpose(pm, npts, nf, npts)
    for t in (catt.Throttle(active_warps=2), catt.Throttle(active_warps=1, active_ctas=2),
              catt.Throttle(cta_threads=512, active_warps=4, gate=catt.GATE_BARRIER)):
        out = torch.empty(nf * npts, device="cuda")
        catt.kmeans_transpose(dev(pm), npts, nf, out, npts, t=t)
        assert np.array_equal(host(out), want)


@pytest.mark.parametrize("npts,nf,k,pad", [(1000, 34, 5, 4), (4099, 34, 5, 29), (257, 7, 3, 3), (300, 50, 12, 4),
                                           (70000, 34, 5, 0), (2000, 64, 16, 1), (513, 1, 1, 0)])
def test_one_iteration_exact(npts, nf, k, pad):
    ld = npts + pad
    feat = feat_fm(33, npts, nf, ld)
    cl0 = first_k(feat, ld, nf, k)
    memb_o, _ = oracle.kmeans_assign(feat, ld, npts, nf, cl0)
    cl_o, cnt_o = okm.update(feat, ld, npts, nf, memb_o, cl0)
    F, C = dev(feat), dev(cl0)
    memb = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
    acc = torch.zeros(catt.kmeans_acc_words(k, nf), dtype=torch.int64, device="cuda")
    stats = torch.zeros(3, dtype=torch.int64, device="cuda")
    catt.kmeans_accumulate(F, ld, npts, nf, C, memb, acc)
    a = host(acc)
    K4 = 4 * k * nf
    assert np.array_equal(a[K4:K4 + k], cnt_o) and a[K4 + k] == npts and a[K4 + k + 1] == 0
    catt.kmeans_finalize(acc, C, stats)
    assert np.array_equal(host(memb), memb_o)
    assert np.array_equal(host(C), cl_o)
    assert host(stats).tolist() == [npts, 0, npts] and not host(acc).any()    # zeroed for the next pass


def test_sums_are_partition_invariant():
    """Two accumulate calls over halves of the points = one call over all."""
    npts, nf, k = 10000, 34, 5
    feat = feat_fm(34, npts, nf, npts)
    cl0 = first_k(feat, npts, nf, k)
    F = dev(feat)
    h = 4321
    Fa = dev(np.concatenate([feat[f * npts:f * npts + h] for f in range(nf)]))
    Fb = dev(np.concatenate([feat[f * npts + h:(f + 1) * npts] for f in range(nf)]))
    W = catt.kmeans_acc_words(k, nf)
    acc1 = torch.zeros(W, dtype=torch.int64, device="cuda")
    acc2 = torch.zeros(W, dtype=torch.int64, device="cuda")
    m1 = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
    m2 = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
    catt.kmeans_accumulate(F, npts, npts, nf, dev(cl0), m1, acc1)
    catt.kmeans_accumulate(Fa, h, h, nf, dev(cl0), m2[:h], acc2)
    catt.kmeans_accumulate(Fb, npts - h, npts - h, nf, dev(cl0), m2[h:], acc2)
    a1, a2 = host(acc1), host(acc2)
    K4 = 4 * k * nf
    # limbs may differ (carries land in different chunks); the sums they encode may not
    def sums(a):
        return [sum(int(a[q * 4 + l]) << (32 * l) for l in range(4)) for q in range(k * nf)]
    assert sums(a1) == sums(a2) and np.array_equal(a1[K4:], a2[K4:])
    assert np.array_equal(host(m1), host(m2))


@pytest.mark.parametrize("npts,nf,k,max_iter", [(2000, 4, 3, 20), (20000, 34, 5, 12), (3001, 9, 16, 6)])
def test_kmeans_loop_exact(npts, nf, k, max_iter):
    ld = npts + 3
    feat = feat_fm(35, npts, nf, ld)
    cl0 = first_k(feat, ld, nf, k)
    cl_o, memb_o, it_o, deltas = okm.kmeans(feat, ld, npts, nf, cl0, max_iter=max_iter)
    C = dev(cl0)
    memb, it = catt.kmeans(dev(feat), ld, npts, nf, C, max_iter=max_iter)
    assert it == it_o, (it, it_o, deltas)
    assert np.array_equal(host(memb), memb_o)
    assert np.array_equal(host(C), cl_o)


def test_kmeans_loop_converges_on_blobs():
    rng = np.random.default_rng(6)
    npts, nf, k = 5000, 8, 4
    centres = (np.arange(k)[:, None] * 10.0 + rng.random((k, nf))).astype(np.float32)
    labels = rng.integers(0, k, npts)
    labels[:k] = np.arange(k)
    pts = (centres[labels] + (rng.random((npts, nf)) - 0.5) * 0.5).astype(np.float32)
    feat = np.ascontiguousarray(pts.T).ravel()
    C = dev(pts[:k].copy())
    memb, it = catt.kmeans(dev(feat), npts, npts, nf, C, max_iter=50)
    m = host(memb)
    assert np.array_equal(m, labels) and it <= 3
    cl_o, _ = okm.update(feat, npts, npts, nf, m, pts[:k])
    assert np.array_equal(host(C), cl_o)


def test_inexact_values_are_flagged():
    npts, nf, k = 600, 3, 2
    feat = feat_fm(36, npts, nf, npts)
    feat[5] = 3.0e9                      # >= 2^31
    feat[npts + 7] = 2.0 ** -70          # bits below 2^-64
    cl0 = first_k(feat, npts, nf, k)
    acc = torch.zeros(catt.kmeans_acc_words(k, nf), dtype=torch.int64, device="cuda")
    memb = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
    catt.kmeans_accumulate(dev(feat), npts, npts, nf, dev(cl0), memb, acc)
    assert host(acc)[4 * k * nf + k + 1] == 2
    with pytest.raises(catt.CattError, match="inexact"):
        catt.kmeans(dev(feat), npts, npts, nf, dev(cl0), max_iter=2)


def test_negative_and_wide_range_values_exact():
    """Signed values with |x| in [2^-41, 2^30) (the exact domain: ulp >= 2^-64,
    |x| < 2^31): still exact (two's complement limbs)."""
    rng = np.random.default_rng(7)
    npts, nf, k = 4000, 5, 3
    e = rng.integers(-41, 30, nf * npts)
    sign = np.where(rng.random(nf * npts) < 0.5, -1.0, 1.0)
    feat = (sign * (1.0 + rng.random(nf * npts)) * 2.0 ** e).astype(np.float32)
    cl0 = first_k(feat, npts, nf, k)
    memb_o, _ = oracle.kmeans_assign(feat, npts, npts, nf, cl0)
    cl_o, _ = okm.update(feat, npts, npts, nf, memb_o, cl0)
    C = dev(cl0)
    acc = torch.zeros(catt.kmeans_acc_words(k, nf), dtype=torch.int64, device="cuda")
    memb = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
    catt.kmeans_accumulate(dev(feat), npts, npts, nf, C, memb, acc)
    assert host(acc)[4 * k * nf + k + 1] == 0
    catt.kmeans_finalize(acc, C)
    assert np.array_equal(host(memb), memb_o) and np.array_equal(host(C), cl_o)


def test_full_size_iteration_exact():
    """BASELINE configs[2] shape (494020 x 34, k = 5): one assignment + update,
    then the transpose of the point-major copy, all bit-exact."""
    npts, nf, k = 494020, 34, 5
    ld = npts
    F = torch.empty(nf * ld, device="cuda")
    catt.fill_hash(F, si.SEED_KMEANS)
    feat = oracle.fill(si.SEED_KMEANS, nf * ld)
    cl0 = first_k(feat, ld, nf, k)
    memb_o, _ = oracle.kmeans_assign(feat, ld, npts, nf, cl0)
    cl_o, cnt_o = okm.update(feat, ld, npts, nf, memb_o, cl0)
    C = dev(cl0)
    acc = torch.zeros(catt.kmeans_acc_words(k, nf), dtype=torch.int64, device="cuda")
    memb = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
    catt.kmeans_accumulate(F, ld, npts, nf, C, memb, acc)
    catt.kmeans_finalize(acc, C)
    assert np.array_equal(host(memb), memb_o) and np.array_equal(host(C), cl_o)
    pm = torch.from_numpy(np.ascontiguousarray(feat.reshape(nf, ld).T)).cuda().reshape(-1)
    for v in ("coop", "literal"):
        out = torch.empty(nf * ld, device="cuda")
        catt.kmeans_transpose(pm, npts, nf, out, ld, t=catt.Throttle(variant=v))
        assert torch.equal(out, F), v


def test_invalid_arguments():
    acc = torch.zeros(catt.kmeans_acc_words(3, 4), dtype=torch.int64, device="cuda")
    feat = torch.zeros(4 * 10, device="cuda")
    memb = torch.zeros(10, dtype=torch.int32, device="cuda")
    with pytest.raises(catt.CattError):
        catt.kmeans_accumulate(feat, 5, 10, 4, torch.zeros(3, 4, device="cuda"), memb, acc)      # ld < npoints
    with pytest.raises(catt.CattError):
        catt.kmeans_accumulate(torch.zeros(65 * 10, device="cuda"), 10, 10, 65, torch.zeros(3, 65, device="cuda"),
                               memb, acc)                                                        # nf > 64
    with pytest.raises(catt.CattError):
        catt.kmeans_transpose(feat, 10, 4, feat, 5, t=catt.Throttle(variant="coop"))             # ld < npoints


@pytest.mark.parametrize("npts,nf,k,pad", [(1000, 34, 5, 4), (70001, 34, 5, 29), (300, 50, 12, 4), (257, 7, 3, 3)])
def test_step_equals_accumulate_then_finalize(npts, nf, k, pad):
    """catt_kmeans_step (one launch, last-CTA finalize) is bit-identical to
    catt_kmeans_accumulate + catt_kmeans_finalize, over two iterations (the
    second checks that the step left acc zeroed and its counter reset)."""
    ld = npts + pad + (-(npts + pad)) % 4
    feat = si.values(4, nf * ld)
    cl0 = feat.reshape(nf, ld)[:, :k].T.copy()
    F = dev(feat)
    runs = []
    for fused in (False, True):
        C = dev(cl0)
        memb = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
        acc = torch.zeros(catt.kmeans_acc_words(k, nf), dtype=torch.int64, device="cuda")
        stats = torch.zeros(3, dtype=torch.int64, device="cuda")
        out = []
        for _ in range(2):
            if fused:
                catt.kmeans_step(F, ld, npts, nf, C, memb, acc, stats)
            else:
                catt.kmeans_accumulate(F, ld, npts, nf, C, memb, acc)
                catt.kmeans_finalize(acc, C, stats)
            torch.cuda.synchronize()
            out.append((host(C).copy(), host(memb).copy(), host(stats).copy(), host(acc).copy()))
        runs.append(out)
    for (c0, m0, s0, a0), (c1, m1, s1, a1) in zip(*runs):
        assert np.array_equal(c0.view(np.uint32), c1.view(np.uint32))
        assert np.array_equal(m0, m1) and np.array_equal(s0, s1) and np.array_equal(a0, a1)
        assert not a1.any()
