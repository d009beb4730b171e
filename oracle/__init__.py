"""CPU ORACLE for the CATT hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline and
`--impl reference` legs may import, call, link or execute anything under
oracle/. The product package (paper_conf_icpp_kimhlsh19_b200) never imports
it, and this package never imports the product package: the two share no code.

  oracle/loops.c      plain C loop nests (seq-fmaf and seq-f64 modes) and the
                      counter-based generator; built into oracle/liborc.so
  oracle/footprint.py Eq 1-9 in the paper's order (paper and union modes)
  oracle/lru.py       kernel address traces + LRU L1D simulator

Parity status of each function is recorded in DESIGN.md "Oracle pins".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "loops.c")
LIB = os.path.join(HERE, "liborc.so")

SEQ_FMAF = 0
SEQ_F64 = 1

_lib = None


def build(force: bool = False) -> str:
    """Compile oracle/loops.c with gcc (no fast-math, no implicit contraction)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        cmd = ["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-shared", "-fPIC",
               SRC, "-o", LIB + ".tmp", "-lm"]
        subprocess.run(cmd, check=True)
        os.replace(LIB + ".tmp", LIB)
    return LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        f32p = ctypes.POINTER(ctypes.c_float)
        i64, i32, u32 = ctypes.c_int64, ctypes.c_int32, ctypes.c_uint32
        L.orc_fill.argtypes = [u32, ctypes.c_uint64, i64, ctypes.c_int, f32p]
        L.orc_atax.argtypes = [ctypes.c_int, f32p, f32p, f32p, f32p, i64, i64]
        L.orc_bicg.argtypes = [ctypes.c_int, f32p, f32p, f32p, f32p, f32p, i64, i64]
        L.orc_mvt.argtypes = [ctypes.c_int, f32p, f32p, f32p, f32p, f32p, i64]
        L.orc_gesummv.argtypes = [ctypes.c_int, f32p, f32p, f32p, f32p, f32p, i64, ctypes.c_float, ctypes.c_float]
        L.orc_rows3.argtypes = [ctypes.c_int, f32p, f32p, f32p, f32p, f32p, i64, i64]
        L.orc_syrk.argtypes = [ctypes.c_int, f32p, f32p, i64, i64, ctypes.c_float, ctypes.c_float]
        L.orc_syrk_rows.argtypes = [ctypes.c_int, f32p, f32p, i64, i64, ctypes.c_float, ctypes.c_float,
                                    ctypes.POINTER(ctypes.c_int64), i64, f32p]
        L.orc_gemm.argtypes = [ctypes.c_int, f32p, f32p, f32p, i64, i64, i64, ctypes.c_float, ctypes.c_float]
        L.orc_corr.argtypes = [ctypes.c_int, f32p, i64, i64, f32p, f32p, f32p]
        L.orc_syr2k.argtypes = [ctypes.c_int, f32p, f32p, f32p, i64, i64, ctypes.c_float, ctypes.c_float]
        L.orc_syr2k_rows.argtypes = [ctypes.c_int, f32p, f32p, f32p, i64, i64, ctypes.c_float, ctypes.c_float,
                                     ctypes.POINTER(ctypes.c_int64), i64, f32p]
        L.orc_kmeans_assign.argtypes = [ctypes.c_int, f32p, i64, i64, i32, f32p, i32,
                                        ctypes.POINTER(ctypes.c_int32), f32p]
        L.orc_atax_hashed.argtypes = [ctypes.c_int, u32, ctypes.c_int, f32p, i64, i64, f32p,
                                      ctypes.POINTER(ctypes.c_int64), i64, f32p]
        L.orc_num_threads.restype = ctypes.c_int
        L.orc_set_num_threads.argtypes = [ctypes.c_int]
        L.orc_set_num_threads.restype = None
        _lib = L
    return _lib


def _p(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"]
    if a.dtype == np.float32:
        return a.ctypes.data_as(ctypes.POINTER(ctypes.c_float))
    if a.dtype == np.int32:
        return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int32))
    if a.dtype == np.int64:
        return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))
    raise TypeError(a.dtype)


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def num_threads() -> int:
    return int(lib().orc_num_threads())


def set_num_threads(n: int):
    """OpenMP threads for the loop nests (torchrun exports OMP_NUM_THREADS=1)."""
    lib().orc_set_num_threads(int(n))


def fill(seed: int, n: int, offset: int = 0, mode: int = 0) -> np.ndarray:
    out = np.empty(n, np.float32)
    lib().orc_fill(seed & 0xFFFFFFFF, offset, n, mode, _p(out))
    return out


def atax(A, x, mode=SEQ_FMAF):
    A, x = _f32(A), _f32(x)
    m, n = A.shape
    tmp, y = np.empty(m, np.float32), np.empty(n, np.float32)
    lib().orc_atax(mode, _p(A), _p(x), _p(tmp), _p(y), m, n)
    return tmp, y


def bicg(A, p, r, mode=SEQ_FMAF):
    A, p, r = _f32(A), _f32(p), _f32(r)
    nx, ny = A.shape
    q, s = np.empty(nx, np.float32), np.empty(ny, np.float32)
    lib().orc_bicg(mode, _p(A), _p(p), _p(r), _p(q), _p(s), nx, ny)
    return q, s


def mvt(a, y1, y2, x1, x2, mode=SEQ_FMAF):
    a, y1, y2 = _f32(a), _f32(y1), _f32(y2)
    x1, x2 = _f32(x1).copy(), _f32(x2).copy()
    lib().orc_mvt(mode, _p(a), _p(y1), _p(y2), _p(x1), _p(x2), a.shape[0])
    return x1, x2


def gesummv(A, B, x, alpha, beta, mode=SEQ_FMAF):
    A, B, x = _f32(A), _f32(B), _f32(x)
    n = A.shape[0]
    if A.shape != (n, n) or B.shape != (n, n) or x.shape != (n,):   # the C loop assumes square n x n
        raise ValueError(f"gesummv: A {A.shape}, B {B.shape}, x {x.shape}: need n x n, n x n, n")
    y, tmp = np.empty(n, np.float32), np.empty(n, np.float32)
    lib().orc_gesummv(mode, _p(A), _p(B), _p(x), _p(y), _p(tmp), n, alpha, beta)
    return y, tmp


def rows3(A, B, C, x, mode=SEQ_FMAF):
    """y = (A x + B x) + C x, each product an fmaf chain in j order (the
    three-stream row loop, DESIGN R29)."""
    A, B, C, x = _f32(A), _f32(B), _f32(C), _f32(x)
    m, n = A.shape
    y = np.empty(m, np.float32)
    lib().orc_rows3(mode, _p(A), _p(B), _p(C), _p(x), _p(y), m, n)
    return y


def syrk(A, C, alpha, beta, mode=SEQ_FMAF):
    A = _f32(A)
    C = _f32(C).copy()
    n, m = A.shape
    lib().orc_syrk(mode, _p(A), _p(C), n, m, alpha, beta)
    return C


def syrk_rows(A, C, alpha, beta, rows, mode=SEQ_FMAF):
    """Rows `rows` of syrk(A, C, alpha, beta) without computing the rest."""
    A, C = _f32(A), _f32(C)
    n, m = A.shape
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    out = np.empty((len(rows), n), np.float32)
    lib().orc_syrk_rows(mode, _p(A), _p(C), n, m, alpha, beta, _p(rows), len(rows), _p(out))
    return out


def syr2k(A, B, C, alpha, beta, mode=SEQ_FMAF):
    A, B = _f32(A), _f32(B)
    C = _f32(C).copy()
    n, m = A.shape
    lib().orc_syr2k(mode, _p(A), _p(B), _p(C), n, m, alpha, beta)
    return C


def syr2k_rows(A, B, C, alpha, beta, rows, mode=SEQ_FMAF):
    A, B, C = _f32(A), _f32(B), _f32(C)
    n, m = A.shape
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    out = np.empty((len(rows), n), np.float32)
    lib().orc_syr2k_rows(mode, _p(A), _p(B), _p(C), n, m, alpha, beta, _p(rows), len(rows), _p(out))
    return out


def gemm(A, B, C, alpha, beta, mode=SEQ_FMAF):
    """C := beta C + alpha A B (PolyBench gemm order); returns the new C."""
    A, B, C = _f32(A), _f32(B), _f32(C).copy()
    ni, nk = A.shape
    nj = B.shape[1]
    lib().orc_gemm(mode, _p(A), _p(B), _p(C), ni, nj, nk, alpha, beta)
    return C


def corr(data, mode=SEQ_FMAF):
    """PolyBench correlation of the columns of data (n x m).
    Returns (symmat m x m, mean, std, centred-and-scaled data)."""
    d = _f32(data).copy()
    n, m = d.shape
    mean, std = np.empty(m, np.float32), np.empty(m, np.float32)
    sym = np.empty((m, m), np.float32)
    lib().orc_corr(mode, _p(d), n, m, _p(mean), _p(std), _p(sym))
    return sym, mean, std, d


def kmeans_assign(feat, ld, npoints, nf, clusters, mode=SEQ_FMAF):
    """feat: flat feature-major array of nf*ld floats; clusters: k x nf."""
    feat, clusters = _f32(feat).ravel(), _f32(clusters)
    k = clusters.shape[0]
    memb = np.empty(npoints, np.int32)
    margin = np.empty(npoints, np.float32)
    lib().orc_kmeans_assign(mode, _p(feat), ld, npoints, nf, _p(clusters), k, _p(memb), _p(margin))
    return memb, margin


def atax_hashed(seedA, amode, x, m, n, cols, mode=SEQ_FMAF):
    x = _f32(x)
    cols = np.ascontiguousarray(cols, dtype=np.int64)
    tmp = np.empty(m, np.float32)
    ycols = np.empty(len(cols), np.float32)
    lib().orc_atax_hashed(mode, seedA & 0xFFFFFFFF, amode, _p(x), m, n, _p(tmp), _p(cols), len(cols), _p(ycols))
    return tmp, ycols
