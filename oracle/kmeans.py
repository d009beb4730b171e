"""KMEANS full iteration, oracle side — TEST INFRASTRUCTURE ONLY (see
oracle/__init__.py for who may import it).

SURVEY 8(f) f2: the steps around the assignment step of Rodinia kmeans, the KM
workload of the paper (Table 2; Table 3 P:338-339 lists its two loops):

  transpose(feat_pm)          KM's other kernel: point-major feat_pm[p*nf + f]
                              -> feature-major feat[f*ld + p]
  assign                      oracle.kmeans_assign (loops.c, reading R16)
  update(feat, memb, old)     centre[c][f] = the mean of feature f over the
                              points assigned to c, rounded once to the nearest
                              fp32 (ties to even); a centre without points
                              keeps its old value (reading R21)
  kmeans(...)                 the loop: assign, count the changed memberships
                              (delta), update; stop after the first iteration
                              with delta <= max_changes, or after max_iter
                              (reading R21; Rodinia's loop [ext])

The mean is the plain definition: an exact sum, then one rounding. The exact
sum is computed by writing each fp32 as an integer mantissa times a power of
two (numpy frexp), summing the integer mantissas of equal exponent in int64
(exact), and combining the per-exponent sums as Python integers/fractions.
The rounding is round-to-nearest-even on the exact rational, written out.
"""
from __future__ import annotations

from fractions import Fraction

import numpy as np


def transpose(feat_pm, npoints, nf, ld):
    """feat[f*ld + p] = feat_pm[p*nf + f]; padding columns p >= npoints are 0."""
    src = np.asarray(feat_pm, np.float32).reshape(npoints, nf)
    out = np.zeros(nf * ld, np.float32)
    for f in range(nf):
        out[f * ld:f * ld + npoints] = src[:, f]
    return out


def exact_sum(values) -> Fraction:
    """The exact (unrounded) sum of fp32 values, as a Fraction."""
    v = np.asarray(values, np.float32).astype(np.float64)      # exact widening
    if v.size == 0:
        return Fraction(0)
    m, e = np.frexp(v)                                         # v = m * 2**e, 0.5 <= |m| < 1
    mi = np.rint(m * 2.0 ** 24).astype(np.int64)               # exact: fp32 has 24 significant bits
    total = Fraction(0)
    for ex in np.unique(e):
        s = int(mi[e == ex].sum())                             # |s| < 2**24 * n: exact in int64
        total += Fraction(s) * Fraction(2) ** (int(ex) - 24)
    return total


def round_f32(q: Fraction) -> np.float32:
    """Round a rational to the nearest fp32, ties to even (IEEE 754 default)."""
    if q == 0:
        return np.float32(0.0)
    sign = -1 if q < 0 else 1
    q = abs(q)
    e = q.numerator.bit_length() - q.denominator.bit_length()  # 2**e <= q < 2**(e+2)
    if Fraction(2) ** e > q:
        e -= 1
    if Fraction(2) ** (e + 1) <= q:
        e += 1
    ulp_exp = max(e - 23, -149)                                # subnormals: fixed ulp 2**-149
    scaled = q / Fraction(2) ** ulp_exp
    n = scaled.numerator // scaled.denominator
    rem = scaled - n
    if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and n % 2 == 1):
        n += 1
    if ulp_exp + n.bit_length() > 128:                         # beyond FLT_MAX
        return np.float32(sign * np.inf)
    return np.float32(sign * float(Fraction(n) * Fraction(2) ** ulp_exp))


def update(feat, ld, npoints, nf, memb, old_clusters):
    """New centres (k x nf fp32) and per-centre counts from a membership."""
    feat = np.asarray(feat, np.float32).ravel()
    memb = np.asarray(memb)
    old = np.asarray(old_clusters, np.float32)
    k = old.shape[0]
    new = old.copy()
    counts = np.zeros(k, np.int64)
    for c in range(k):
        members = np.nonzero(memb[:npoints] == c)[0]
        counts[c] = len(members)
        if len(members) == 0:
            continue                                           # empty centre keeps its value (R21)
        for f in range(nf):
            new[c, f] = round_f32(exact_sum(feat[f * ld + members]) / len(members))
    return new, counts


def kmeans(feat, ld, npoints, nf, init_clusters, max_iter, max_changes=0):
    """Rodinia's loop order. Returns (clusters, membership, iterations, deltas)."""
    from . import kmeans_assign
    clusters = np.asarray(init_clusters, np.float32).copy()
    memb = np.full(npoints, -1, np.int32)
    deltas = []
    for it in range(max_iter):
        new_memb, _ = kmeans_assign(feat, ld, npoints, nf, clusters)
        delta = int(np.count_nonzero(new_memb != memb))
        memb = new_memb
        clusters, _ = update(feat, ld, npoints, nf, memb, clusters)
        deltas.append(delta)
        if delta <= max_changes:
            break
    return clusters, memb, len(deltas), deltas
