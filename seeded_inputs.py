"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no loop nest, no footprint
formula): only the counter-based generator that both sides draw inputs from,
and the workload recipes (shapes, seeds) of BASELINE.json's configs.

Generator:
    key(seed, hi) = fmix32(seed * 0x9E3779B9 + hi * 0x632BE5AB + 0x7F4A7C15)
    h(seed, idx)  = fmix32((lo32(idx) * 0x85EBCA77) ^ key(seed, hi32(idx)))
    uniform : (h >> 8) * 2^-24          in [0, 1), exact in fp32
    dyadic  : (h & 15) / 16             in {0, 1/16, ..., 15/16}, exact in fp32
fmix32 is the MurmurHash3 finaliser. The CUDA library implements the same
generator in device code (catt_fill_hash) and oracle/loops.c implements it in
C; tests check all three agree bit for bit.

Positive values avoid cancellation, so relative error is well conditioned;
the dyadic mode makes every partial sum of the hot-path loops exact in fp32
(SURVEY.md 8(c) c1 mode 3), so any summation order is bit-identical.
"""
from __future__ import annotations

import numpy as np

MODE_UNIFORM = 0
MODE_DYADIC = 1

_M32 = np.uint64(0xFFFFFFFF)


def _fmix32(h: np.ndarray) -> np.ndarray:
    h = h.astype(np.uint32, copy=True)
    h ^= h >> np.uint32(16)
    h *= np.uint32(0x85EBCA6B)
    h ^= h >> np.uint32(13)
    h *= np.uint32(0xC2B2AE35)
    h ^= h >> np.uint32(16)
    return h


def hash_u32(seed: int, idx: np.ndarray) -> np.ndarray:
    """h(seed, idx) for an array of non-negative 64-bit indices."""
    idx = np.asarray(idx, dtype=np.uint64)
    lo = (idx & _M32).astype(np.uint32)
    hi = (idx >> np.uint64(32)).astype(np.uint32)
    with np.errstate(over="ignore"):
        key = _fmix32(np.uint32(seed & 0xFFFFFFFF) * np.uint32(0x9E3779B9)
                      + hi * np.uint32(0x632BE5AB) + np.uint32(0x7F4A7C15))
        return _fmix32((lo * np.uint32(0x85EBCA77)) ^ key)


def values(seed: int, n: int, offset: int = 0, mode: int = MODE_UNIFORM) -> np.ndarray:
    """float32 values for flat indices offset .. offset+n-1."""
    h = hash_u32(seed, np.arange(offset, offset + n, dtype=np.uint64))
    if mode == MODE_UNIFORM:
        return ((h >> np.uint32(8)).astype(np.float32) * np.float32(2.0 ** -24))
    if mode == MODE_DYADIC:
        return (h & np.uint32(15)).astype(np.float32) * np.float32(1.0 / 16.0)
    raise ValueError(f"unknown mode {mode}")


def matrix(seed: int, rows: int, cols: int, mode: int = MODE_UNIFORM, row0: int = 0) -> np.ndarray:
    """Row-major rows x cols block of the global matrix whose flat index is
    (row0 + r) * cols + c; row shards of one matrix therefore agree for any G."""
    return values(seed, rows * cols, offset=row0 * cols, mode=mode).reshape(rows, cols)


# Seeds per workload; each array of a workload gets seed + 100*k.
SEED_ATAX, SEED_BICG, SEED_MVT, SEED_KMEANS, SEED_GESUMMV, SEED_SYRK, SEED_ATAX_SHARDED, SEED_SYR2K = 1, 2, 3, 4, 5, 6, 7, 8
SEED_CORR, SEED_GEMM = 9, 10


def sub_seed(seed: int, k: int) -> int:
    return seed + 100 * k


# BASELINE.json configs: shapes only.
CONFIGS = {
    "atax256": dict(kernel="atax", m=256, n=256),
    "bicg4096": dict(kernel="bicg", m=4096, n=4096),
    "mvt4096": dict(kernel="mvt", n=4096),
    "kmeans": dict(kernel="kmeans", npoints=494020, nfeatures=34, k=5, ld=494020),
    "kmeans_padded": dict(kernel="kmeans", npoints=494020, nfeatures=34, k=5, ld=494048),
    "gesummv8192": dict(kernel="gesummv", n=8192, alpha=1.5, beta=1.2),
    "syrk2048": dict(kernel="syrk", n=2048, m=2048, alpha=1.5, beta=1.2),
    "atax_sharded": dict(kernel="atax", m=65536, n=16384),
}
