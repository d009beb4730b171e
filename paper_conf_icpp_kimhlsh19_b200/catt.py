"""Python binding of the CATT C ABI (include/catt.h) — argument marshalling only.

Every step of the hot path runs in libcatt.so (hand-written sm_100a kernels and
the C++ footprint analyser). There is no CPU fallback: if the library is
missing or a call fails, an exception is raised. Device tensors are PyTorch
tensors (float32, contiguous, on the current CUDA device); the stream is
torch's current stream.

Names follow the C ABI without the `catt_` prefix.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Tuple

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libcatt.so")

# ------------------------------------------------------------------ constants (catt.h)
OK, EINVAL, ECUDA, EUNSUPPORTED, ENOMEM, ENODEV, EINEXACT = 0, -1, -2, -3, -4, -5, -6
MAX_LOOPS, MAX_CARVEOUTS = 4, 16
REF_IRREGULAR, REF_STORE, REF_NOT_L1 = 1, 2, 4
MODE_UNION, MODE_PAPER = 0, 1
FIT_NONE_NEEDED, FIT_WARP, FIT_CTA, FIT_UNRESOLVABLE, FIT_GUARDED = 1, 2, 4, 8, 16
VAR_LITERAL, VAR_VEC4, VAR_STAGED, VAR_COOP, VAR_REGS, VAR_FUSED, VAR_BYPASS = 0, 1, 2, 3, 4, 5, 6
ROWS_STORE, ROWS_ACCUM, ROWS_GESUMMV, ROWS_SUM3 = 0, 1, 2, 3
PEER_HANDLE_BYTES = 64
GATE_SEMAPHORE, GATE_BARRIER = 0, 1
CAP_SM_COUNTER, CAP_SMEM_PAD = 0, 1
(K_ATAX_1, K_ATAX_2, K_BICG_1, K_BICG_2, K_MVT_1, K_MVT_2, K_GESUMMV, K_SYRK, K_KMEANS, K_SYR2K,
 K_KMEANS_T, K_CORR, K_GEMM, K_ROWS3) = range(14)

VARIANTS = {"literal": VAR_LITERAL, "vec4": VAR_VEC4, "staged": VAR_STAGED, "coop": VAR_COOP, "regs": VAR_REGS,
            "fused": VAR_FUSED, "bypass": VAR_BYPASS}
FLAG_NAMES = {FIT_NONE_NEEDED: "none", FIT_WARP: "warp", FIT_CTA: "cta", FIT_UNRESOLVABLE: "unresolvable",
              FIT_NONE_NEEDED | FIT_GUARDED: "none(guard)", FIT_WARP | FIT_GUARDED: "warp(guard)",
              FIT_CTA | FIT_GUARDED: "cta(guard)"}


class CattError(RuntimeError):
    pass


# ------------------------------------------------------------------ structs
class Ref(ctypes.Structure):
    _fields_ = [("c_gid", ctypes.c_int64 * 3), ("c_iter", ctypes.c_int64 * MAX_LOOPS), ("base", ctypes.c_int64),
                ("elem_bytes", ctypes.c_int32), ("flags", ctypes.c_int32), ("array_id", ctypes.c_int32),
                ("reserved_", ctypes.c_int32)]


class LoopDesc(ctypes.Structure):
    _fields_ = [("n_refs", ctypes.c_int32), ("n_loops", ctypes.c_int32), ("refs", ctypes.POINTER(Ref)),
                ("trip", ctypes.c_int64 * MAX_LOOPS), ("block", ctypes.c_int32 * 3), ("mode", ctypes.c_int32),
                ("grid", ctypes.c_int64 * 3), ("extent", ctypes.c_int64 * 3), ("regs_per_thread", ctypes.c_int32),
                ("smem_per_cta", ctypes.c_int32), ("force_carveout_kb", ctypes.c_int32), ("reserved_", ctypes.c_int32)]


class Hw(ctypes.Structure):
    _fields_ = [("num_sms", ctypes.c_int32), ("max_warps_sm", ctypes.c_int32), ("max_ctas_sm", ctypes.c_int32),
                ("regs_sm", ctypes.c_int32), ("reg_alloc_unit", ctypes.c_int32), ("warp_size", ctypes.c_int32),
                ("smem_alloc_unit", ctypes.c_int32), ("reserved_smem_cta", ctypes.c_int32),
                ("line_bytes", ctypes.c_int32), ("n_carveouts", ctypes.c_int32),
                ("min_warps_sm", ctypes.c_int32), ("divergent_lines", ctypes.c_int32),
                ("min_retouch", ctypes.c_int32), ("min_reuse_trip", ctypes.c_int32),
                ("max_stream_pct", ctypes.c_int32), ("cta_fallback", ctypes.c_int32),
                ("stream_floor", ctypes.c_int32), ("private_streams", ctypes.c_int32),
                ("carveout_kb", ctypes.c_int32 * MAX_CARVEOUTS), ("carveout_pct", ctypes.c_int32 * MAX_CARVEOUTS),
                ("l1d_bytes", ctypes.c_int64 * MAX_CARVEOUTS)]

    def as_dict(self):
        n = self.n_carveouts
        d = {f: getattr(self, f) for f, _ in self._fields_[:18]}
        d["carveout_kb"] = list(self.carveout_kb[:n])
        d["carveout_pct"] = list(self.carveout_pct[:n])
        d["l1d_bytes"] = list(self.l1d_bytes[:n])
        return d

    @classmethod
    def from_dict(cls, d):
        h = cls()
        for f, _ in cls._fields_[:18]:
            if f in d:
                setattr(h, f, d[f])
        n = len(d["carveout_kb"])
        h.n_carveouts = n
        for i in range(n):
            h.carveout_kb[i] = d["carveout_kb"][i]
            h.carveout_pct[i] = d.get("carveout_pct", [0] * n)[i]
            h.l1d_bytes[i] = d["l1d_bytes"][i]
        return h


class FootprintResult(ctypes.Structure):
    _fields_ = [("lines_per_warp_iter", ctypes.c_int64), ("reuse_span", ctypes.c_int64),
                ("footprint_lines_full", ctypes.c_int64), ("footprint_lines", ctypes.c_int64),
                ("footprint_bytes", ctypes.c_int64), ("l1d_bytes", ctypes.c_int64),
                ("base_warps", ctypes.c_int32), ("base_ctas", ctypes.c_int32), ("active_warps", ctypes.c_int32),
                ("active_ctas", ctypes.c_int32), ("carveout_kb", ctypes.c_int32), ("flags", ctypes.c_int32)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class Throttle(ctypes.Structure):
    """catt_throttle. Zero = default launch (256 threads, LITERAL, full TLP)."""
    _fields_ = [("cta_threads", ctypes.c_int32), ("active_warps", ctypes.c_int32), ("active_ctas", ctypes.c_int32),
                ("carveout_kb", ctypes.c_int32), ("variant", ctypes.c_int32), ("gate", ctypes.c_int32),
                ("cap", ctypes.c_int32), ("reserved_", ctypes.c_int32), ("probe", ctypes.c_void_p)]

    def __init__(self, cta_threads=0, active_warps=0, active_ctas=0, carveout_kb=0, variant=VAR_LITERAL,
                 gate=GATE_SEMAPHORE, cap=CAP_SM_COUNTER, probe=None):
        if isinstance(variant, str):
            variant = VARIANTS[variant]
        super().__init__(cta_threads, active_warps, active_ctas, carveout_kb, variant, gate, cap, 0,
                         probe if probe is None else int(probe))

    def copy(self, **kw):
        d = {f: getattr(self, f) for f, _ in self._fields_ if f != "reserved_"}
        d.update(kw)
        return Throttle(**d)

    def __repr__(self):
        return (f"Throttle(cta={self.cta_threads}, warps={self.active_warps}, ctas={self.active_ctas}, "
                f"carveout={self.carveout_kb}KB, variant={self.variant}, gate={self.gate}, cap={self.cap})")


class DualProblem(ctypes.Structure):
    _fields_ = [("A", ctypes.c_void_p), ("xr", ctypes.c_void_p), ("xc", ctypes.c_void_p), ("yr", ctypes.c_void_p),
                ("yc", ctypes.c_void_p), ("m", ctypes.c_int64), ("n", ctypes.c_int64),
                ("row_accumulate", ctypes.c_int32), ("col_accumulate", ctypes.c_int32)]


class Problem(ctypes.Structure):
    _fields_ = [("loop", ctypes.c_int32), ("reserved_", ctypes.c_int32), ("m", ctypes.c_int64),
                ("n", ctypes.c_int64), ("k", ctypes.c_int64), ("ld", ctypes.c_int64)]


# ------------------------------------------------------------------ library
_lib = None


def lib():
    """Load libcatt.so (building it with nvcc if it is absent or stale)."""
    global _lib
    if _lib is None:
        from . import build as _build
        if not _build.up_to_date():
            _build.build()
        if not os.path.exists(LIB_PATH):
            raise CattError(f"libcatt.so missing at {LIB_PATH}: the CUDA extension is required (no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        P, V, i32, i64, u32, u64, f32 = (ctypes.POINTER, ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64,
                                         ctypes.c_uint32, ctypes.c_uint64, ctypes.c_float)
        T = P(Throttle)
        sig = {
            "catt_hw_query": [ctypes.c_int, P(Hw)],
            "catt_hw_b200": [P(Hw)],
            "catt_hw_titanv": [P(Hw)],
            "catt_footprint": [P(LoopDesc), P(Hw), P(FootprintResult)],
            "catt_kernel_desc": [P(Problem), T, i32, P(LoopDesc), P(Ref), i32],
            "catt_plan": [P(Problem), T, P(Hw), i32, T, P(FootprintResult)],
            "catt_atax": [V, V, V, V, i64, i64, T, T, V],
            "catt_bicg": [V, V, V, V, V, i64, i64, T, T, V],
            "catt_mvt": [V, V, V, V, V, i64, T, T, V],
            "catt_gesummv": [V, V, V, V, V, i64, f32, f32, T, V],
            "catt_syrk": [V, V, i64, i64, f32, f32, T, V],
            "catt_syr2k": [V, V, V, i64, i64, f32, f32, T, V],
            "catt_gemm": [V, V, V, i64, i64, i64, f32, f32, T, V],
            "catt_corr": [V, i64, i64, V, V, V, V, T, V],
            "catt_kmeans_assign": [V, i64, i64, i32, V, i32, V, T, V],
            "catt_kmeans_transpose": [V, V, i64, i32, i64, T, V],
            "catt_kmeans_accumulate": [V, i64, i64, i32, V, i32, V, V, V],
            "catt_kmeans_finalize": [V, i32, i32, V, V, i32, V],
            "catt_kmeans_step": [V, i64, i64, i32, V, i32, V, V, V, V],
            "catt_kmeans": [V, i64, i64, i32, V, i32, V, i32, i64, V, P(i32), V],
            "catt_rows": [V, V, V, V, V, i64, i64, f32, f32, i32, T, V],
            "catt_dual": [V, V, V, V, V, i64, i64, i32, i32, i32, T, V],
            "catt_dual_group": [P(DualProblem), i32, i32, T, V],
            "catt_cols": [V, V, V, i64, i64, i32, T, V],
            "catt_fill_hash": [V, i64, u32, u64, i32, V],
            "catt_calibrate_l1": [ctypes.c_int, i32, P(i32), i32, P(f32)],
            "catt_kernel_attrs": [P(Problem), T, P(i32), P(i32)],
            "catt_kernel_occupancy": [P(Problem), T, i64, P(i32), P(i64)],
            "catt_fused_trace": [P(u64), i32],
            "catt_peer_create": [i32, i32, i64, P(V), V],
            "catt_peer_open": [V, i32, V],
            "catt_peer_create_mapped": [i32, i32, i64, P(V), V, P(V)],
            "catt_peer_check": [V, P(i32)],
            "catt_peer_destroy": [V],
            "catt_atax_peer": [V, V, V, V, i64, i64, V, V],
            "catt_dual_group_peer": [P(DualProblem), i32, V, V],
            "catt_atax_onekernel": [V, V, V, V, i64, i64, T, T, V],
            "catt_status_str": [ctypes.c_int],
            "catt_last_cuda_error": [],
            "catt_abi_version": [],
            "catt_sm_partition_create": [ctypes.c_int, i32, P(V), P(i32)],
            "catt_sm_partition_destroy": [V],
        }
        for name, args in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = ctypes.c_int
        L.catt_status_str.restype = ctypes.c_char_p
        L.catt_kmeans_acc_words.argtypes = [i32, i32]
        L.catt_kmeans_acc_words.restype = ctypes.c_int64
        L.catt_peer_bytes.argtypes = [i32, i64]
        L.catt_peer_bytes.restype = ctypes.c_int64
        _lib = L
    return _lib


EXPORTED = ["catt_hw_query", "catt_hw_b200", "catt_hw_titanv", "catt_footprint", "catt_kernel_desc", "catt_plan",
            "catt_atax", "catt_bicg", "catt_mvt", "catt_gesummv", "catt_syrk", "catt_syr2k", "catt_gemm", "catt_corr", "catt_kmeans_assign",
            "catt_kmeans_acc_words", "catt_kmeans_transpose", "catt_kmeans_accumulate", "catt_kmeans_finalize",
            "catt_kmeans_step",
            "catt_kmeans", "catt_rows", "catt_cols", "catt_dual", "catt_dual_group", "catt_fill_hash", "catt_calibrate_l1", "catt_kernel_attrs",
            "catt_kernel_occupancy", "catt_status_str",
            "catt_last_cuda_error", "catt_abi_version", "catt_fused_trace", "catt_peer_create", "catt_peer_open",
            "catt_peer_bytes", "catt_peer_create_mapped",
            "catt_peer_check", "catt_peer_destroy", "catt_atax_peer", "catt_dual_group_peer", "catt_atax_onekernel", "catt_sm_partition_create",
            "catt_sm_partition_destroy"]


def _check(st: int, what: str):
    if st != OK:
        L = lib()
        msg = L.catt_status_str(st).decode()
        extra = f" (cudaError {L.catt_last_cuda_error()})" if st == ECUDA else ""
        raise CattError(f"{what}: {msg}{extra}")


# ------------------------------------------------------------------ hardware / analyser
def hw_b200() -> Hw:
    h = Hw()
    _check(lib().catt_hw_b200(ctypes.byref(h)), "catt_hw_b200")
    return h


def paper_rule(hw: Hw) -> Hw:
    """A copy of hw with the B200 guards off: the paper's Eq 9 rule as printed."""
    h = Hw.from_dict(hw.as_dict())
    h.min_warps_sm = 0
    h.divergent_lines = 0
    h.min_retouch = 0
    h.min_reuse_trip = 0
    h.max_stream_pct = 0
    h.cta_fallback = 0
    h.stream_floor = 0
    h.private_streams = 0
    return h


def hw_titanv() -> Hw:
    h = Hw()
    _check(lib().catt_hw_titanv(ctypes.byref(h)), "catt_hw_titanv")
    return h


def hw_query(device: int = 0) -> Hw:
    h = Hw()
    _check(lib().catt_hw_query(device, ctypes.byref(h)), "catt_hw_query")
    return h


def make_desc(refs, trips, block, grid, extent=(0, 0, 0), regs=0, smem=0, mode=MODE_UNION, force_carveout_kb=-1):
    """Build a LoopDesc from plain tuples. refs: dicts with c_gid, c_iter and
    optional base, elem_bytes, flags, array_id. Returns (desc, keepalive)."""
    arr = (Ref * max(1, len(refs)))()
    for i, r in enumerate(refs):
        g = list(r["c_gid"]) + [0] * (3 - len(r["c_gid"]))
        it = list(r["c_iter"]) + [0] * (MAX_LOOPS - len(r["c_iter"]))
        arr[i].c_gid[:] = g
        arr[i].c_iter[:] = it
        arr[i].base = r.get("base", 0)
        arr[i].elem_bytes = r.get("elem_bytes", 4)
        arr[i].flags = r.get("flags", 0)
        arr[i].array_id = r.get("array_id", 0)
    d = LoopDesc()
    d.n_refs = len(refs)
    d.n_loops = len(trips)
    d.refs = ctypes.cast(arr, ctypes.POINTER(Ref))
    d.trip[:] = list(trips) + [0] * (MAX_LOOPS - len(trips))
    d.block[:] = list(block)
    d.grid[:] = list(grid)
    d.extent[:] = list(extent)
    d.mode = mode
    d.regs_per_thread = regs
    d.smem_per_cta = smem
    d.force_carveout_kb = force_carveout_kb
    return d, arr


def footprint(desc: LoopDesc, hw: Hw) -> dict:
    r = FootprintResult()
    _check(lib().catt_footprint(ctypes.byref(desc), ctypes.byref(hw), ctypes.byref(r)), "catt_footprint")
    return r.as_dict()


def problem(loop: int, m=0, n=0, k=0, ld=0) -> Problem:
    return Problem(loop, 0, m, n, k, ld)


def kernel_desc(prob: Problem, launch: Optional[Throttle] = None, mode: int = MODE_UNION):
    refs = (Ref * 8)()
    d = LoopDesc()
    _check(lib().catt_kernel_desc(ctypes.byref(prob), ctypes.byref(launch) if launch else None, mode,
                                  ctypes.byref(d), refs, 8), "catt_kernel_desc")
    return d, refs


def plan(prob: Problem, launch: Optional[Throttle] = None, hw: Optional[Hw] = None,
         mode: int = MODE_UNION) -> Tuple[Throttle, dict]:
    """The CATT throttle for one loop (catt_plan)."""
    if hw is None:
        hw = hw_query()
    out, r = Throttle(), FootprintResult()
    _check(lib().catt_plan(ctypes.byref(prob), ctypes.byref(launch) if launch else None, ctypes.byref(hw), mode,
                           ctypes.byref(out), ctypes.byref(r)), "catt_plan")
    return out, r.as_dict()


def kernel_attrs(prob: Problem, launch: Optional[Throttle] = None) -> Tuple[int, int]:
    regs, smem = ctypes.c_int32(), ctypes.c_int32()
    _check(lib().catt_kernel_attrs(ctypes.byref(prob), ctypes.byref(launch) if launch else None,
                                   ctypes.byref(regs), ctypes.byref(smem)), "catt_kernel_attrs")
    return regs.value, smem.value


def kernel_occupancy(prob: Problem, launch: Optional[Throttle] = None, extra_dyn_smem: int = 0) -> Tuple[int, int]:
    """cudaOccupancyMaxActiveBlocksPerMultiprocessor for the loop's kernel at the
    largest carveout (catt_kernel_occupancy). Returns (CTAs per SM, dynamic bytes)."""
    n, dyn = ctypes.c_int32(), ctypes.c_int64()
    _check(lib().catt_kernel_occupancy(ctypes.byref(prob), ctypes.byref(launch) if launch else None,
                                       int(extra_dyn_smem), ctypes.byref(n), ctypes.byref(dyn)),
           "catt_kernel_occupancy")
    return n.value, dyn.value


# ------------------------------------------------------------------ device calls
def _torch():
    import torch
    return torch


def _dev(t, name, dtype=None, n=0):
    """Device pointer of t after the checks the C ABI cannot make: a contiguous
    CUDA tensor of `dtype` on the current device with at least n elements
    (the extent the entry point reads or writes; an undersized buffer would be
    read or written out of bounds)."""
    torch = _torch()
    dtype = dtype or torch.float32
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise CattError(f"{name}: expected a CUDA tensor")
    if t.dtype != dtype or not t.is_contiguous():
        raise CattError(f"{name}: expected a contiguous {dtype} tensor")
    if t.device.index != torch.cuda.current_device():
        raise CattError(f"{name}: tensor on cuda:{t.device.index}, current device is cuda:{torch.cuda.current_device()}")
    if t.numel() < n:
        raise CattError(f"{name}: {t.numel()} elements, the call needs {n}")
    return ctypes.c_void_p(t.data_ptr())


def _fm(ld, npoints, nf):
    """Elements a feature-major [nf][ld] array must hold to reach point npoints - 1 of feature nf - 1."""
    return (nf - 1) * ld + npoints if npoints > 0 and nf > 0 else 0


def _stream():
    return ctypes.c_void_p(_torch().cuda.current_stream().cuda_stream)


def _tp(t: Optional[Throttle]):
    return ctypes.byref(t) if t is not None else None


def atax(A, x, tmp=None, y=None, k1: Optional[Throttle] = None, k2: Optional[Throttle] = None):
    """tmp = A x; y = A^T tmp (catt_atax). Returns (tmp, y)."""
    torch = _torch()
    m, n = A.shape
    tmp = torch.empty(m, device=A.device) if tmp is None else tmp
    y = torch.empty(n, device=A.device) if y is None else y
    _check(lib().catt_atax(_dev(A, "A", n=m * n), _dev(x, "x", n=n), _dev(tmp, "tmp", n=m), _dev(y, "y", n=n), m, n, _tp(k1), _tp(k2),
                           _stream()), "catt_atax")
    return tmp, y


def atax_onekernel(A, x, tmp=None, y=None, k1: Optional[Throttle] = None, k2: Optional[Throttle] = None):
    """Both ATAX loops in one literal kernel, a warp throttle per loop
    (catt_atax_onekernel): k1 = the launch and loop 1's gate, k2 = loop 2's
    gate. Returns (tmp, y)."""
    torch = _torch()
    m, n = A.shape
    tmp = torch.empty(m, device=A.device) if tmp is None else tmp
    y = torch.empty(n, device=A.device) if y is None else y
    _check(lib().catt_atax_onekernel(_dev(A, "A", n=m * n), _dev(x, "x", n=n), _dev(tmp, "tmp", n=m), _dev(y, "y", n=n), m, n, _tp(k1),
                                     _tp(k2), _stream()), "catt_atax_onekernel")
    return tmp, y


def bicg(A, p, r, q=None, s=None, k1: Optional[Throttle] = None, k2: Optional[Throttle] = None):
    """s = A^T r (loop 1), q = A p (loop 2) (catt_bicg). Returns (q, s)."""
    torch = _torch()
    nx, ny = A.shape
    q = torch.empty(nx, device=A.device) if q is None else q
    s = torch.empty(ny, device=A.device) if s is None else s
    _check(lib().catt_bicg(_dev(A, "A", n=nx * ny), _dev(p, "p", n=ny), _dev(r, "r", n=nx), _dev(q, "q", n=nx), _dev(s, "s", n=ny), nx, ny,
                           _tp(k1), _tp(k2), _stream()), "catt_bicg")
    return q, s


def mvt(A, y1, y2, x1, x2, k1: Optional[Throttle] = None, k2: Optional[Throttle] = None):
    """x1 += A y1, x2 += A^T y2, in place (catt_mvt). Returns (x1, x2)."""
    n = A.shape[0]
    _check(lib().catt_mvt(_dev(A, "A", n=n * n), _dev(y1, "y1", n=n), _dev(y2, "y2", n=n), _dev(x1, "x1", n=n), _dev(x2, "x2", n=n), n,
                          _tp(k1), _tp(k2), _stream()), "catt_mvt")
    return x1, x2


def gesummv(A, B, x, alpha, beta, y=None, tmp=None, t: Optional[Throttle] = None):
    """y = alpha A x + beta B x, tmp = A x (catt_gesummv). Returns (y, tmp)."""
    torch = _torch()
    n = A.shape[0]
    y = torch.empty(n, device=A.device) if y is None else y
    tmp = torch.empty(n, device=A.device) if tmp is None else tmp
    _check(lib().catt_gesummv(_dev(A, "A", n=n * n), _dev(B, "B", n=n * n), _dev(x, "x", n=n), _dev(y, "y", n=n), _dev(tmp, "tmp", n=n), n,
                              float(alpha), float(beta), _tp(t), _stream()), "catt_gesummv")
    return y, tmp


def rows(A, x, y, mode=ROWS_STORE, B=None, tmp=None, alpha=0.0, beta=0.0, t: Optional[Throttle] = None):
    """One row loop (catt_rows): y = A x (STORE), y += A x (ACCUM), GESUMMV, or
    SUM3 (y = A x + B x + C x with B holding B and C back to back)."""
    m, n = A.shape
    nb = (2 if mode == ROWS_SUM3 else 1) * m * n
    _check(lib().catt_rows(_dev(A, "A", n=m * n), _dev(B, "B", n=nb) if B is not None else None, _dev(x, "x", n=n), _dev(y, "y", n=m),
                           _dev(tmp, "tmp", n=m) if tmp is not None else None, m, n, float(alpha), float(beta), mode,
                           _tp(t), _stream()), "catt_rows")
    return y


def cols(A, v, y, accumulate=False, t: Optional[Throttle] = None):
    """One column loop (catt_cols): y (+)= A^T v."""
    m, n = A.shape
    _check(lib().catt_cols(_dev(A, "A", n=m * n), _dev(v, "v", n=m), _dev(y, "y", n=n), m, n, int(bool(accumulate)), _tp(t),
                           _stream()), "catt_cols")
    return y


def dual(A, xr, yr, yc, xc=None, row_accumulate=False, col_accumulate=False, dependent=False,
         t: Optional[Throttle] = None):
    """Both loops in one pass over A (catt_dual): yr (+)= A xr; yc (+)= A^T (yr if dependent else xc)."""
    m, n = A.shape
    _check(lib().catt_dual(_dev(A, "A", n=m * n), _dev(xr, "xr", n=n), _dev(xc, "xc", n=m) if xc is not None else None, _dev(yr, "yr", n=m),
                           _dev(yc, "yc", n=n), m, n, int(bool(row_accumulate)), int(bool(col_accumulate)),
                           int(bool(dependent)), _tp(t), _stream()), "catt_dual")
    return yr, yc


def dual_group(problems, dependent=False, t: Optional[Throttle] = None):
    """Grouped catt_dual: problems = [dict(A=, xr=, yr=, yc=, xc=None, row_accumulate=False,
    col_accumulate=False)], same column count, one launch."""
    arr = _dual_array(problems)
    _check(lib().catt_dual_group(arr, len(problems), int(bool(dependent)), _tp(t), _stream()), "catt_dual_group")


def _dual_array(problems):
    arr = (DualProblem * len(problems))()
    for i, p in enumerate(problems):
        m, n = p["A"].shape
        arr[i] = DualProblem(_dev(p["A"], "A", n=m * n).value, _dev(p["xr"], "xr", n=n).value,
                             _dev(p["xc"], "xc", n=m).value if p.get("xc") is not None else None,
                             _dev(p["yr"], "yr", n=m).value, _dev(p["yc"], "yc", n=n).value, m, n,
                             int(bool(p.get("row_accumulate"))), int(bool(p.get("col_accumulate"))))
    return arr


def dual_group_peer(problems, peer: "Peer"):
    """Row-sharded grouped BICG / MVT step (catt_dual_group_peer): each
    problem's A is this rank's rows; the column outputs yc are summed over
    ranks inside the kernel (peer memory, rank order, then the initial value
    for col_accumulate) and are bit-identical on every rank; yr stays local.
    `peer` holds n x len(problems) columns."""
    arr = _dual_array(problems)
    _check(lib().catt_dual_group_peer(arr, len(problems), peer.ptr, _stream()), "catt_dual_group_peer")


def syrk(A, C, alpha, beta, t: Optional[Throttle] = None):
    """C = beta C + alpha A A^T in place (catt_syrk). Returns C."""
    n, m = A.shape
    _check(lib().catt_syrk(_dev(A, "A", n=n * m), _dev(C, "C", n=n * n), n, m, float(alpha), float(beta), _tp(t), _stream()),
           "catt_syrk")
    return C


def syr2k(A, B, C, alpha, beta, t: Optional[Throttle] = None):
    """C = beta C + alpha (A B^T + B A^T) in place (catt_syr2k). Returns C."""
    n, m = A.shape
    _check(lib().catt_syr2k(_dev(A, "A", n=n * m), _dev(B, "B", n=n * m), _dev(C, "C", n=n * n), n, m, float(alpha), float(beta), _tp(t),
                            _stream()), "catt_syr2k")
    return C


class Peer:
    """This rank's peer-memory all-reduce state (catt_peer_*): create, ship
    `handle` (bytes) to the other ranks, `open` theirs, then `atax_peer`."""

    def __init__(self, world, rank, n, _mapped=None):
        self.ptr = ctypes.c_void_p()
        self.world, self.rank, self.n = world, rank, n
        self.multicast = False
        if _mapped is not None:                      # Peer.mapped
            bases, mc, self._keep = _mapped
            arr = (ctypes.c_void_p * world)(*bases)
            _check(lib().catt_peer_create_mapped(world, rank, n, arr, ctypes.c_void_p(mc or None), ctypes.byref(self.ptr)),
                   "catt_peer_create_mapped")
            self.handle = None
            self.multicast = bool(mc)
            return
        buf = ctypes.create_string_buffer(PEER_HANDLE_BYTES)
        _check(lib().catt_peer_create(world, rank, n, ctypes.byref(self.ptr), buf), "catt_peer_create")
        self.handle = buf.raw

    @staticmethod
    def nbytes(world, n) -> int:
        """Bytes of one rank's peer buffer (catt_peer_bytes)."""
        return int(lib().catt_peer_bytes(world, n))

    @classmethod
    def mapped(cls, world, rank, n, bases, multicast_ptr=0, keep=None):
        """Peer state over caller-mapped memory (catt_peer_create_mapped):
        bases[r] = rank r's buffer as mapped here (symmetric memory), each
        Peer.nbytes(world, n) bytes, zero-filled; multicast_ptr = the NVLS
        multicast alias or 0. `keep` is held so the mapping outlives the peer."""
        return cls(world, rank, n, _mapped=(list(bases), multicast_ptr, keep))

    def open(self, peer_rank, handle: bytes):
        buf = ctypes.create_string_buffer(handle, PEER_HANDLE_BYTES)
        _check(lib().catt_peer_open(self.ptr, peer_rank, buf), "catt_peer_open")

    def error(self) -> int:
        """catt_peer_check's error word: 0 none, 1 a wait timed out, 2 the ranks launched different grids."""
        v = ctypes.c_int32()
        _check(lib().catt_peer_check(self.ptr, ctypes.byref(v)), "catt_peer_check")
        return v.value

    def timed_out(self) -> bool:
        return self.error() != 0

    def close(self):
        if self.ptr:
            _check(lib().catt_peer_destroy(self.ptr), "catt_peer_destroy")
            self.ptr = ctypes.c_void_p()


def atax_peer(A_g, x, peer: Peer, tmp_g=None, y=None):
    """Row-sharded ATAX step with the A^T partials all-reduced inside the fused
    kernel through peer memory (catt_atax_peer): tmp_g = A_g x, y = sum over
    ranks of A_g^T tmp_g (identical on every rank). Returns (tmp_g, y)."""
    torch = _torch()
    m, n = A_g.shape
    tmp_g = torch.empty(m, device=A_g.device) if tmp_g is None else tmp_g
    y = torch.empty(n, device=A_g.device) if y is None else y
    _check(lib().catt_atax_peer(_dev(A_g, "A", n=m * n), _dev(x, "x", n=n), _dev(tmp_g, "tmp", n=m), _dev(y, "y", n=n), m, n, peer.ptr,
                                _stream()), "catt_atax_peer")
    return tmp_g, y


def fused_trace(nctas):
    """Phase timestamps (ns) of the last traced FUSED single-read launch
    (CATT_FUSED_TRACE set at launch): array [nctas, 6] (catt_fused_trace)."""
    import numpy as np
    out = np.zeros(nctas * 6, dtype=np.uint64)
    _check(lib().catt_fused_trace(out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), nctas * 6), "catt_fused_trace")
    return out.reshape(nctas, 6)


def kmeans_assign(feat, ld, npoints, nf, clusters, membership=None, t: Optional[Throttle] = None):
    """membership[p] = argmin_c |feat[:, p] - clusters[c]|^2 (catt_kmeans_assign)."""
    torch = _torch()
    k = clusters.shape[0]
    membership = torch.empty(npoints, dtype=torch.int32, device=feat.device) if membership is None else membership
    _check(lib().catt_kmeans_assign(_dev(feat, "feat", n=_fm(ld, npoints, nf)), ld, npoints, nf,
                                    _dev(clusters, "clusters", n=k * nf), k,
                                    _dev(membership, "membership", torch.int32, npoints), _tp(t), _stream()),
           "catt_kmeans_assign")
    return membership


def gemm(A, B, C, alpha, beta, t: Optional[Throttle] = None):
    """C = beta C + alpha A B in place (catt_gemm). Returns C."""
    ni, nk = A.shape
    nj = B.shape[1]
    _check(lib().catt_gemm(_dev(A, "A", n=ni * nk), _dev(B, "B", n=nk * nj), _dev(C, "C", n=ni * nj), ni, nj, nk, float(alpha), float(beta), _tp(t),
                           _stream()), "catt_gemm")
    return C


def corr(data, mean=None, stdv=None, symmat=None, work=None, t: Optional[Throttle] = None):
    """Pearson correlation of the columns of data (n x m, centred and scaled in
    place). Returns (symmat, mean, stdv). STAGED needs a work buffer of n*m floats
    (allocated here when not given)."""
    torch = _torch()
    n, m = data.shape
    mk = lambda shape: torch.empty(shape, dtype=torch.float32, device=data.device)
    mean = mk(m) if mean is None else mean
    stdv = mk(m) if stdv is None else stdv
    symmat = mk((m, m)) if symmat is None else symmat
    staged = t is not None and t.variant == VAR_STAGED
    if staged and work is None:
        work = mk(n * m)
    wp = _dev(work, "work", n=n * m) if work is not None else None
    _check(lib().catt_corr(_dev(data, "data", n=n * m), n, m, _dev(mean, "mean", n=m), _dev(stdv, "stdv", n=m),
                           _dev(symmat, "symmat", n=m * m),
                           wp, _tp(t), _stream()), "catt_corr")
    return symmat, mean, stdv


def kmeans_acc_words(k: int, nf: int) -> int:
    """Length of the exact-sum buffer (catt_kmeans_acc_words)."""
    return int(lib().catt_kmeans_acc_words(k, nf))


def kmeans_transpose(feat_pm, npoints, nf, out, ld, t: Optional[Throttle] = None):
    """out[f*ld + p] = feat_pm[p*nf + f] (catt_kmeans_transpose). Returns out."""
    _check(lib().catt_kmeans_transpose(_dev(feat_pm, "in", n=npoints * nf), _dev(out, "out", n=_fm(ld, npoints, nf)), npoints, nf, ld, _tp(t), _stream()),
           "catt_kmeans_transpose")
    return out


def kmeans_accumulate(feat, ld, npoints, nf, clusters, membership, acc):
    """Assignment + exact centroid sums into acc (catt_kmeans_accumulate)."""
    torch = _torch()
    _check(lib().catt_kmeans_accumulate(_dev(feat, "feat", n=_fm(ld, npoints, nf)), ld, npoints, nf,
                                        _dev(clusters, "clusters", n=clusters.shape[0] * nf),
                                        clusters.shape[0], _dev(membership, "membership", torch.int32, npoints),
                                        _dev(acc, "acc", torch.int64, kmeans_acc_words(clusters.shape[0], nf)), _stream()),
           "catt_kmeans_accumulate")


def kmeans_finalize(acc, clusters, stats=None, zero_acc=True):
    """clusters := exact means from acc (catt_kmeans_finalize)."""
    torch = _torch()
    k, nf = clusters.shape
    sp = _dev(stats, "stats", torch.int64, 3) if stats is not None else None
    _check(lib().catt_kmeans_finalize(_dev(acc, "acc", torch.int64, kmeans_acc_words(k, nf)), k, nf,
                                      _dev(clusters, "clusters", n=k * nf), sp,
                                      int(bool(zero_acc)), _stream()), "catt_kmeans_finalize")
    return clusters


def kmeans_step(feat, ld, npoints, nf, clusters, membership, acc, stats=None):
    """One k-means iteration in one launch (catt_kmeans_step): accumulate, then
    the last CTA rounds the new centres into clusters and zeroes acc."""
    torch = _torch()
    k = clusters.shape[0]
    sp = _dev(stats, "stats", torch.int64, 3) if stats is not None else None
    _check(lib().catt_kmeans_step(_dev(feat, "feat", n=_fm(ld, npoints, nf)), ld, npoints, nf,
                                  _dev(clusters, "clusters", n=k * nf), k,
                                  _dev(membership, "membership", torch.int32, npoints),
                                  _dev(acc, "acc", torch.int64, kmeans_acc_words(k, nf)), sp,
                                  _stream()), "catt_kmeans_step")
    return clusters


def kmeans(feat, ld, npoints, nf, clusters, membership=None, max_iter=500, max_changes=0, ws=None):
    """The k-means loop on one GPU (catt_kmeans); clusters updated in place.
    Returns (membership, iterations)."""
    torch = _torch()
    k = clusters.shape[0]
    if membership is None:
        membership = torch.empty(npoints, dtype=torch.int32, device=feat.device)
    if ws is None:
        ws = torch.empty(kmeans_acc_words(k, nf) + 4, dtype=torch.int64, device=feat.device)
    it = ctypes.c_int32(0)
    _check(lib().catt_kmeans(_dev(feat, "feat", n=_fm(ld, npoints, nf)), ld, npoints, nf,
                             _dev(clusters, "clusters", n=k * nf), k,
                             _dev(membership, "membership", torch.int32, npoints), max_iter, max_changes,
                             _dev(ws, "ws", torch.int64, kmeans_acc_words(k, nf) + 4), ctypes.byref(it), _stream()),
           "catt_kmeans")
    return membership, it.value


def fill_hash(t, seed: int, offset: int = 0, mode: int = 0):
    """Fill a CUDA float32 tensor with the seeded_inputs generator (in device code)."""
    _check(lib().catt_fill_hash(_dev(t, "t"), t.numel(), seed & 0xFFFFFFFF, offset, mode, _stream()),
           "catt_fill_hash")
    return t


def calibrate_l1(device: int, pct: int, kb_list):
    n = len(kb_list)
    kb = (ctypes.c_int32 * n)(*kb_list)
    out = (ctypes.c_float * n)()
    _check(lib().catt_calibrate_l1(device, pct, kb, n, out), "catt_calibrate_l1")
    return list(out)


class SmPartition:
    """A stream on a partition of >= min_sms SMs (catt_sm_partition_create, a
    CUDA green context). `stream` is a torch ExternalStream: inside
    `with torch.cuda.stream(p.stream):` every catt launch runs on the
    partition. `sms` is the partition's SM count; `hw(base)` is the hardware
    table to plan with (num_sms = sms, Eq 3's ceil(grid / #SM) bound)."""

    def __init__(self, min_sms: int, device: int = 0):
        h, n = ctypes.c_void_p(), ctypes.c_int32()
        _check(lib().catt_sm_partition_create(device, min_sms, ctypes.byref(h), ctypes.byref(n)),
               "catt_sm_partition_create")
        self._h, self.sms = h, n.value
        self.stream = _torch().cuda.ExternalStream(h.value, device=_torch().device("cuda", device))

    def hw(self, base: "Hw") -> "Hw":
        h = Hw()
        ctypes.memmove(ctypes.byref(h), ctypes.byref(base), ctypes.sizeof(Hw))
        h.num_sms = self.sms
        return h

    def close(self):
        if self._h is not None:
            self.stream.synchronize()
            _check(lib().catt_sm_partition_destroy(self._h), "catt_sm_partition_destroy")
            self._h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()
