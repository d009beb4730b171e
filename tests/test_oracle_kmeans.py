"""Pins for oracle/kmeans.py against things other than itself:
math.fsum (correctly rounded double sums), numpy's double -> float32 rounding,
closed forms on dyadic data, brute-force loops, and separated-blob k-means
whose answer is known by construction."""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle
from oracle import kmeans as km
import seeded_inputs as si


def test_transpose_matches_explicit_loop():
    rng = np.random.default_rng(1)
    for npts, nf, pad in [(1, 1, 0), (7, 3, 1), (33, 34, 5)]:
        pm = rng.random(npts * nf, dtype=np.float32)
        ld = npts + pad
        out = km.transpose(pm, npts, nf, ld)
        want = np.zeros(nf * ld, np.float32)
        for p in range(npts):
            for f in range(nf):
                want[f * ld + p] = pm[p * nf + f]
        assert np.array_equal(out, want)


def test_exact_sum_against_fsum_and_cancellation():
    rng = np.random.default_rng(2)
    for n in (1, 2, 17, 1000):
        v = (rng.standard_normal(n) * 10.0 ** rng.integers(-30, 30, n)).astype(np.float32)
        assert float(km.exact_sum(v)) == math.fsum(v.astype(np.float64))
    tiny = np.float32(2.0 ** -149)
    assert km.exact_sum(np.array([3e38, tiny, -3e38], np.float32)) == Fraction(2) ** -149
    assert km.exact_sum(np.array([], np.float32)) == 0


def test_round_f32_against_numpy_double_rounding():
    rng = np.random.default_rng(3)
    xs = np.concatenate([rng.standard_normal(2000) * 10.0 ** rng.integers(-45, 39, 2000),
                         [1.0 + 2.0 ** -24, 1.0 + 3 * 2.0 ** -24, 2.0 ** -149 * 0.5, 2.0 ** -149 * 1.5,
                          3.4028235e38, 3.4028236e38, 1e39, -1e39, 2.0 ** -126, 0.0]])
    for x in xs:
        with np.errstate(over="ignore"):
            want = np.float32(x)               # IEEE round-to-nearest-even of a double (exact input)
        got = km.round_f32(Fraction(float(x)))
        assert (np.isinf(want) and np.isinf(got) and np.sign(want) == np.sign(got)) or got == want, x
        if want != 0:
            assert np.signbit(got) == np.signbit(want)


def test_round_f32_is_single_rounding():
    # 1 + 2^-24 + 2^-60 is above the midpoint between 1 and 1 + 2^-23: it rounds up.
    # Going through a double first lands exactly on the midpoint and then rounds to 1.0.
    q = 1 + Fraction(2) ** -24 + Fraction(2) ** -60
    assert km.round_f32(q) == np.float32(1 + 2.0 ** -23)
    assert np.float32(float(q)) == np.float32(1.0)


def test_update_closed_form_dyadic_and_invariants():
    npts, nf, k = 4096, 5, 4
    ld = npts + 3
    feat = si.values(40, nf * ld, mode=si.MODE_DYADIC)                # multiples of 1/16 in [0, 1)
    memb = (np.arange(npts) % k).astype(np.int32)               # 1024 points each: a power of two
    memb[:8] = 3                                                # 1030 points for centre 3 (not a power of 2)
    old = np.full((k, nf), 7.0, np.float32)
    new, counts = km.update(feat, ld, npts, nf, memb, old)
    F = feat.reshape(nf, ld)[:, :npts].astype(np.float64)
    for c in range(k):
        sel = memb == c
        assert counts[c] == sel.sum()
        for f in range(nf):
            s = F[f, sel].sum()                                 # exact in float64 (dyadic, < 2^53)
            assert new[c, f] == np.float32(s / sel.sum()) or c == 3   # power-of-two count: one rounding
            assert abs(float(new[c, f]) - s / sel.sum()) <= 2.0 ** -24 * abs(s / sel.sum())
    # order invariance: permuting points (features and membership together) changes nothing
    perm = np.random.default_rng(4).permutation(npts)
    feat_p = np.zeros_like(feat)
    for f in range(nf):
        feat_p[f * ld:f * ld + npts] = feat[f * ld:f * ld + npts][perm]
    new_p, _ = km.update(feat_p, ld, npts, nf, memb[perm], old)
    assert np.array_equal(new, new_p)
    # a centre with no points keeps its old value
    memb2 = np.where(memb == 2, 1, memb).astype(np.int32)
    new2, counts2 = km.update(feat, ld, npts, nf, memb2, old)
    assert counts2[2] == 0 and np.array_equal(new2[2], old[2])


def test_update_random_against_fsum():
    rng = np.random.default_rng(5)
    npts, nf, k = 3000, 3, 3
    feat = rng.standard_normal(nf * npts).astype(np.float32)
    memb = rng.integers(0, k, npts).astype(np.int32)
    new, counts = km.update(feat, npts, npts, nf, memb, np.zeros((k, nf), np.float32))
    F = feat.reshape(nf, npts).astype(np.float64)
    for c in range(k):
        for f in range(nf):
            mean = math.fsum(F[f, memb == c]) / counts[c]
            assert abs(float(new[c, f]) - mean) <= 2.0 ** -24 * abs(mean) * 1.0001


def _blobs(npts, nf, k, seed):
    """k well separated blobs (centres 10 apart, spread < 0.5), feature-major."""
    rng = np.random.default_rng(seed)
    centres = (np.arange(k)[:, None] * 10.0 + rng.random((k, nf))).astype(np.float32)
    labels = rng.integers(0, k, npts)
    labels[:k] = np.arange(k)[::-1]                 # the first k points (the initial centres) span all blobs
    pts = (centres[labels] + (rng.random((npts, nf)) - 0.5) * 0.5).astype(np.float32)
    ld = npts + 1
    feat = np.zeros(nf * ld, np.float32)
    for f in range(nf):
        feat[f * ld:f * ld + npts] = pts[:, f]
    return feat, ld, labels.astype(np.int32), pts


def test_kmeans_loop_on_separated_blobs():
    npts, nf, k = 2000, 4, 3
    feat, ld, labels, pts = _blobs(npts, nf, k, 6)
    init = pts[:k].copy()                           # R14: the first k points
    cl, memb, iters, deltas = km.kmeans(feat, ld, npts, nf, init, max_iter=20)
    order = memb[:k]                                # centre c started at point c
    assert sorted(order.tolist()) == list(range(k))
    # the same partition as the construction, and the centres are its means
    for c in range(k):
        assert len(set(labels[memb == c].tolist())) == 1
    want, _ = km.update(feat, ld, npts, nf, memb, init)
    assert np.array_equal(cl, want)
    assert deltas[0] == npts and deltas[-1] == 0 and iters == len(deltas) <= 3
    # max_iter bounds the loop
    _, _, it1, d1 = km.kmeans(feat, ld, npts, nf, init, max_iter=1)
    assert it1 == 1 and d1 == [npts]
