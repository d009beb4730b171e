"""CPU ORACLE — CATT footprint model and throttle search (section 4).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / reference legs may import this. It shares no code with
paper_conf_icpp_kimhlsh19_b200/ (the C++/CUDA path) and imports nothing from it.

Steps, in the paper's order and notation (DESIGN.md lists every reading R1..R17):

  a1  Eq 1-3: #TB_shm, #TB_reg, #TB_HW -> #TB_SM, plus the grid
      bound ceil(grid/#SM) (R8, needed by Table 3's ATAX baseline (8,4) under
      <<<80*4, 256>>>, P:115 + P:330).
      Eq 4: the smallest configurable shared-memory option that
      holds #TB_SM blocks; the L1D is what that option leaves.
  a2  Eq 5-6: affine index C_tid*tid + C_i*i; locality iff
      |C_i| * elem_bytes < line (R1: strict, bytes).
  a3  Eq 7: REQ_warp = 1 if C_tid = 0 else min(C_tid, 32) for
      4-byte elements, generalised to ceil(32*|C_tid|*e/line) capped at 32
      (R2). Multi-dimensional blocks whose warps span rows: "examine every
      address".
  a4  Eq 8: paper mode SIZE_req = sum over memory instructions of
      REQ_warp * (#Warps_TB * #TB_SM) (R3: all references in the loop).
      Union mode (the B200 default, R4): the exact number of distinct lines
      the co-resident warps retain, by enumerating every lane address.
  a5  Eq 9 (order P:357 + P:371): N over the divisors of
      #Warps_TB (ascending, R6) first; then TB-level, M = 1 .. #TB_SM-1 with
      one warp per TB (R7); give up (CORR) if nothing fits.
      B200 rule (union mode with hw keys min_warps_sm / divergent_lines set,
      R18, R19): no throttle unless a reused reference touches at least
      divergent_lines lines per warp request (the memory divergence of P:32);
      every (a, m) pair by active warps per SM descending, ties -> fewer CTAs
      of more warps (a per-SM cap is cheap on B200); none below min_warps_sm;
      if none at or above it fits, the most throttled one that respects it.
      R23 adds two conditions on that divergent reference: it re-touches its
      line >= min_retouch times per thread and its reuse loop runs >=
      min_reuse_trip iterations (retouches(), reuse_trip()). R24: no throttle
      when stores and loads without reuse exceed max_stream_pct % of a lane's
      bytes per iteration. R27 (hw key cta_fallback): when that fallback is
      taken and an SM holds several CTAs (T >= 2), cap whole CTAs instead --
      (W, m), the smallest m with floor <= W m <= 2 floor. R29 (hw key
      stream_floor): with T = 1 and S >= 2 such divergent reused loads, the
      floor is ceil(min_warps_sm / S). R32 (hw key private_streams): a load
      whose first request lines are the same in warp 1 as in warp 0 of CTA 0
      (shared by the CTA's warps) is neither divergent nor a stream.

Units: footprints are in cache lines; "fits" means lines*line_bytes <= L1D
bytes (throttle iff strictly larger, P:239 R5).
"""
from __future__ import annotations

import itertools
import math
from dataclasses import dataclass, field
from typing import Dict, List, Sequence, Tuple

MODE_UNION = 0
MODE_PAPER = 1

REF_IRREGULAR = 1
REF_STORE = 2
REF_NOT_L1 = 4

FIT_NONE_NEEDED = 1
FIT_WARP = 2
FIT_CTA = 4
FIT_UNRESOLVABLE = 8
FIT_GUARDED = 16

MAX_LOOPS = 4
MAX_WINDOW = 1 << 20


@dataclass
class Ref:
    """One memory instruction in the loop: index = base + sum_d c_gid[d]*gid_d
    + sum_k c_iter[k]*i_k elements of array `array_id` (Eq 5)."""
    c_gid: Tuple[int, int, int]
    c_iter: Tuple[int, ...]
    base: int = 0
    elem_bytes: int = 4
    flags: int = 0
    array_id: int = 0


@dataclass
class Loop:
    refs: List[Ref]
    trips: Tuple[int, ...]
    block: Tuple[int, int, int]
    grid: Tuple[int, int, int]
    extent: Tuple[int, int, int] = (0, 0, 0)
    regs: int = 0
    smem: int = 0
    mode: int = MODE_UNION
    force_carveout_kb: int = -1


def titan_v() -> Dict:
    """Table 1 + P:48 (64 warps/SM) + P:208 (0/8/16/32/64/96 KB
    shared memory, the rest of 128 KB is L1D)."""
    carve = [0, 8, 16, 32, 64, 96]
    return dict(num_sms=80, max_warps_sm=64, max_ctas_sm=32, regs_sm=65536,
                reg_alloc_unit=256, warp_size=32, smem_alloc_unit=256,
                reserved_smem_cta=0, line_bytes=128,
                carveout_kb=carve, l1d_bytes=[(128 - c) * 1024 for c in carve])


class Unlaunchable(ValueError):
    pass


def _ceil_div(a: int, b: int) -> int:
    return -(-a // b)


def _round_up(a: int, b: int) -> int:
    return _ceil_div(a, b) * b


# ---------------------------------------------------------------- a1 (Eq 1-4)
def occupancy(loop: Loop, hw: Dict):
    """Returns (W, T, carveout_kb, l1d_bytes)."""
    bx, by, bz = loop.block
    threads = bx * by * bz
    W = _ceil_div(threads, hw["warp_size"])
    paper = loop.mode == MODE_PAPER
    if paper:
        smem_cta = loop.smem                                             # Eq 1 as printed
    else:
        smem_cta = _round_up(loop.smem + hw["reserved_smem_cta"], hw["smem_alloc_unit"])
    smem_max = max(hw["carveout_kb"]) * 1024
    limits = []
    if smem_cta > 0:
        limits.append(smem_max // smem_cta)                              # Eq 1
    if loop.regs > 0:
        if paper:
            limits.append(hw["regs_sm"] // (loop.regs * threads))         # Eq 2 as printed
        else:
            per_warp = _round_up(loop.regs * hw["warp_size"], hw["reg_alloc_unit"])
            warps = 4 * ((hw["regs_sm"] // 4) // per_warp)               # 4 sub-partitions
            limits.append(warps // W)
    limits.append(min(hw["max_ctas_sm"], hw["max_warps_sm"] // W))        # #TB_HW
    gx, gy, gz = loop.grid
    limits.append(_ceil_div(gx * gy * gz, hw["num_sms"]))                 # grid bound (R8)
    T = min(limits)                                                      # Eq 3
    if T < 1:
        raise Unlaunchable("no CTA fits on an SM")
    carve = list(hw["carveout_kb"])
    if loop.force_carveout_kb >= 0:
        if loop.force_carveout_kb not in carve:
            raise Unlaunchable("forced carveout is not a configurable option")
        idx = carve.index(loop.force_carveout_kb)
        if smem_cta > 0:
            T = min(T, carve[idx] * 1024 // smem_cta)
        if T < 1:
            raise Unlaunchable("forced carveout holds no CTA")
    else:
        need = T * smem_cta                                              # Eq 4
        idx = next(i for i, c in enumerate(carve) if c * 1024 >= need)
    return W, T, carve[idx], hw["l1d_bytes"][idx]


# ---------------------------------------------------------------- a2/a3 helpers
def _coords(lin: int, dims: Sequence[int]) -> Tuple[int, int, int]:
    x = lin % dims[0]
    y = (lin // dims[0]) % dims[1]
    z = lin // (dims[0] * dims[1])
    return x, y, z


def _lane_gids(loop: Loop, b: int, w: int, warp_size: int) -> List[Tuple[int, int, int]]:
    """Global thread coordinates of the valid lanes of warp w of block b."""
    bx, by, bz = loop.block
    threads = bx * by * bz
    bc = _coords(b, loop.grid)
    out = []
    for lane in range(warp_size):
        t = w * warp_size + lane
        if t >= threads:
            break
        tc = _coords(t, loop.block)
        g = tuple(bc[d] * loop.block[d] + tc[d] for d in range(3))
        if any(loop.extent[d] > 0 and g[d] >= loop.extent[d] for d in range(3)):
            continue
        out.append(g)
    return out


def has_locality(ref: Ref, trips: Sequence[int], line: int) -> bool:
    """Eq 6 with the trip counts: some line of the reference is
    re-touched by the same thread (a level with |C_i|*e < line that actually
    iterates, trip >= 2)."""
    return any(abs(ref.c_iter[k]) * ref.elem_bytes < line and trips[k] >= 2 for k in range(len(trips)))


def _reuse_levels(ref: Ref, trips: Sequence[int], line: int):
    return [k for k in range(len(trips)) if abs(ref.c_iter[k]) * ref.elem_bytes < line and trips[k] >= 2]


def retouches(ref: Ref, trips: Sequence[int], line: int) -> int:
    """R23: how many times one thread touches a line of the reference before
    leaving it: line / (|C_i| * e) consecutive iterations, capped by the trip
    count; an outer-level reuse (C_i = 0) re-touches once per iteration of that
    level. Maximum over the reuse levels (0 without reuse)."""
    return max([trips[k] if ref.c_iter[k] == 0 else min(trips[k], line // (abs(ref.c_iter[k]) * ref.elem_bytes))
                for k in _reuse_levels(ref, trips, line)] or [0])


def reuse_trip(ref: Ref, trips: Sequence[int], line: int) -> int:
    """R23: the longest trip count among the loops that carry the reuse."""
    return max([trips[k] for k in _reuse_levels(ref, trips, line)] or [0])


def _window(ref: Ref, trips: Sequence[int], line: int):
    """Iteration vectors whose lines the warp retains until the reuse, as a
    function of the phase k of the innermost loop (Eq 6; R10, R11).

    Returns (per_phase, iters): if per_phase, the ref is evaluated at the
    single vector (0, .., 0, k) -- consecutive-iteration reuse (the line is
    re-touched next iteration) or no reuse (the line lives one iteration);
    otherwise `iters` is the fixed window of an outer-level reuse: all inner
    iteration vectors with the outer indices at 0."""
    n = len(trips)
    if n == 0:
        return True, None
    L = n - 1
    if abs(ref.c_iter[L]) * ref.elem_bytes < line:        # consecutive-iteration reuse
        return True, None
    for k in range(L - 1, -1, -1):
        if abs(ref.c_iter[k]) * ref.elem_bytes < line:    # reuse across level-k iterations
            inner = [range(trips[d]) for d in range(k + 1, n)]
            size = math.prod(len(r) for r in inner)
            if size > MAX_WINDOW:
                raise Unlaunchable("reuse window too large to enumerate")
            return False, [(0,) * (k + 1) + tuple(v) for v in itertools.product(*inner)]
    return True, None                                     # no reuse: one iteration's lines


def _phase_iter(trips: Sequence[int], k: int):
    n = len(trips)
    return [()] if n == 0 else [(0,) * (n - 1) + (k,)]


def _lines(ref: Ref, gids, iters, line: int, irregular_as_unit: bool = True):
    c_gid = (1, 0, 0) if (ref.flags & REF_IRREGULAR and irregular_as_unit) else ref.c_gid
    out = set()
    for g in gids:
        off = ref.base + c_gid[0] * g[0] + c_gid[1] * g[1] + c_gid[2] * g[2]
        for it in iters:
            idx = off + sum(ref.c_iter[k] * it[k] for k in range(len(it)))
            out.add((ref.array_id, (idx * ref.elem_bytes) // line))
    return out


# ---------------------------------------------------------------- a3 paper mode (Eq 7)
def req_warp_paper(ref: Ref, loop: Loop, hw: Dict) -> int:
    if ref.flags & REF_NOT_L1:
        return 0
    line, ws, e = hw["line_bytes"], hw["warp_size"], ref.elem_bytes
    if loop.block[0] % ws == 0 or ref.flags & REF_IRREGULAR:
        c = 1 if ref.flags & REF_IRREGULAR else abs(ref.c_gid[0])
        if c == 0:
            return 1
        return min(ws, _ceil_div(ws * c * e, line))
    # warps span several rows of a multi-dimensional block: examine every address
    gids = _lane_gids(loop, 0, 0, ws)
    it0 = [(0,) * len(loop.trips)]
    return max(1, len(_lines(ref, gids, it0, line)))


# ---------------------------------------------------------------- footprint model
class Model:
    def __init__(self, loop: Loop, hw: Dict):
        self.loop, self.hw = loop, hw
        self.W, self.T, self.carveout_kb, self.l1d_bytes = occupancy(loop, hw)
        self.line = hw["line_bytes"]
        self.paper = loop.mode == MODE_PAPER
        self.divergent = True
        self.streams = 0
        # contention is measured only "for loops where cache locality presents"
        self.locality = any(has_locality(r, loop.trips, self.line) for r in loop.refs
                            if not (r.flags & REF_NOT_L1))
        if self.paper:
            self.req = sum(req_warp_paper(r, loop, hw) for r in loop.refs)
            self.lines_per_warp_iter = self.req
            self.reuse_span = self.req
        else:
            self.refs = [r for r in loop.refs if not (r.flags & (REF_NOT_L1 | REF_STORE))]
            self.win = [_window(r, loop.trips, self.line) for r in self.refs]
            gx, gy, gz = loop.grid
            nblocks = gx * gy * gz
            # CTAs resident on SM 0 in the first wave: 0, #SM, 2*#SM, ...
            self.blocks = [k * hw["num_sms"] for k in range(self.T) if k * hw["num_sms"] < nblocks]
            # phases of the innermost loop over which per-phase lines are
            # evaluated: one line's worth of 4-byte steps covers every
            # alignment of a row start (R11)
            per_phase = any(pp for pp, _ in self.win)
            self.phases = min(loop.trips[-1], hw["line_bytes"] // 4) if (per_phase and loop.trips) else 1
            self._R = {}
            gids00 = _lane_gids(loop, 0, 0, hw["warp_size"])
            it0 = [(0,) * len(loop.trips)]
            per_ref = [len(_lines(r, gids00, it0, self.line)) for r in self.refs]
            self.lines_per_warp_iter = sum(per_ref)
            div = hw.get("divergent_lines", 0)
            rt, rtrip = hw.get("min_retouch", 0), hw.get("min_reuse_trip", 0)
            # R32 (hw key private_streams): a load whose lines warp 1 requests
            # exactly as warp 0 does is shared by the CTA's warps, not a stream
            gids01 = _lane_gids(loop, 0, 1, hw["warp_size"]) if (hw.get("private_streams", 0) > 0 and self.W >= 2) else None
            shared = [gids01 is not None and n >= div and _lines(r, gids01, it0, self.line) == _lines(r, gids00, it0, self.line)
                      for r, n in zip(self.refs, per_ref)]
            hot = [n >= div and not sh and retouches(r, loop.trips, self.line) >= rt and reuse_trip(r, loop.trips, self.line) >= rtrip
                   for r, n, sh in zip(self.refs, per_ref, shared) if has_locality(r, loop.trips, self.line)]
            self.streams = sum(hot)                   # R29: memory-divergent reused loads
            self.divergent = (div <= 0 and rt <= 0 and rtrip <= 0 and hw.get("max_stream_pct", 0) <= 0) or any(hot)
            # R24: bytes per lane and iteration of streams L1 cannot serve again
            pct = hw.get("max_stream_pct", 0)
            if pct > 0:
                mem = [r for r in loop.refs if not (r.flags & REF_NOT_L1)]
                total = sum(r.elem_bytes for r in mem)
                stream = sum(r.elem_bytes for r in mem
                             if (r.flags & REF_STORE) or not has_locality(r, loop.trips, self.line))
                if 100 * stream > pct * total:
                    self.divergent = False
            self.reuse_span = len(self.retained(0, 0, 0))

    def retained(self, b: int, w: int, k: int):
        key = (b, w, k)
        if key not in self._R:
            gids = _lane_gids(self.loop, b, w, self.hw["warp_size"])
            s = set()
            for r, (pp, iters) in zip(self.refs, self.win):
                s |= _lines(r, gids, _phase_iter(self.loop.trips, k) if pp else iters, self.line)
            self._R[key] = s
        return self._R[key]

    def F(self, a: int, m: int) -> int:
        """Footprint in lines with a active warps per CTA and m CTAs per SM."""
        if self.paper:
            return self.req * a * m                                      # Eq 8 / Eq 9
        # any m consecutive CTAs of the SM's list may be co-resident (R9), any
        # of the warp groups of Fig 4 (warps g*a .. g*a+a-1) may be active, and
        # the innermost loop may be at any phase k (R11): take the maximum
        best = 0
        for s0 in range(max(1, len(self.blocks) - m + 1)):
            for g in range(_ceil_div(self.W, a)):
                for k in range(self.phases):
                    s = set()
                    for b in self.blocks[s0:s0 + m]:
                        for w in range(g * a, min(self.W, g * a + a)):
                            s |= self.retained(b, w, k)
                    best = max(best, len(s))
        return best

    def fits(self, lines: int) -> bool:
        return lines * self.line <= self.l1d_bytes


def analyse(loop: Loop, hw: Dict) -> Dict:
    """catt_footprint, the oracle version: returns the result fields."""
    M = Model(loop, hw)
    W, T = M.W, M.T
    full = M.F(W, T)
    res = dict(lines_per_warp_iter=M.lines_per_warp_iter, reuse_span=M.reuse_span,
               footprint_lines_full=full, l1d_bytes=M.l1d_bytes, base_warps=W, base_ctas=T,
               carveout_kb=M.carveout_kb)

    def done(a, m, lines, flag):
        res.update(active_warps=a, active_ctas=m, footprint_lines=lines,
                   footprint_bytes=lines * M.line, flags=flag)
        return res

    if M.fits(full) or not M.locality:
        return done(W, T, full, FIT_NONE_NEEDED)
    guards = not M.paper and any(hw.get(key, 0) > 0 for key in ("min_warps_sm", "divergent_lines", "min_retouch",
                                                                  "min_reuse_trip", "max_stream_pct"))
    if guards:
        # B200 rule (R18, R19): memory-divergent loops only; all (a, m) with a | W,
        # m <= T, by warps per SM descending, ties -> larger a (fewer CTAs);
        # not below min_warps_sm; else the most throttled pair that respects it
        if not M.divergent:
            return done(W, T, full, FIT_NONE_NEEDED | FIT_GUARDED)
        floor_w = hw.get("min_warps_sm", 0)
        if hw.get("stream_floor", 0) > 0 and T == 1 and M.streams >= 2:     # R29
            floor_w = _ceil_div(floor_w, M.streams)
        cands = [(a, m) for a in range(W, 0, -1) if W % a == 0 for m in range(T, 0, -1)
                 if (a, m) != (W, T) and a * m >= floor_w]
        cands.sort(key=lambda am: (-am[0] * am[1], -am[0]))

        def flag(a, m):
            return (FIT_WARP if a < W else 0) | (FIT_CTA if m < T else 0)

        for a, m in cands:
            f = M.F(a, m)
            if M.fits(f):
                return done(a, m, f, flag(a, m))
        if not cands:
            return done(W, T, full, FIT_NONE_NEEDED | FIT_GUARDED)
        least = min(a * m for a, m in cands)
        a, m = max((am for am in cands if am[0] * am[1] == least), key=lambda am: am[0])
        if hw.get("cta_fallback", 0) > 0 and T >= 2:
            # R27: several CTAs per SM -> cap whole CTAs, the smallest m with
            # floor <= W m <= 2 floor
            ms = [mm for mm in range(1, T + 1) if floor_w <= W * mm <= 2 * floor_w]
            if ms:
                if ms[0] == T:
                    return done(W, T, full, FIT_NONE_NEEDED | FIT_GUARDED)
                a, m = W, ms[0]
        return done(a, m, M.F(a, m), flag(a, m) | FIT_GUARDED)
    for N in range(2, W + 1):                     # Eq 9, warp level first
        if W % N:
            continue
        a = W // N
        f = M.F(a, T)
        if M.fits(f):
            return done(a, T, f, FIT_WARP)
    for m in range(T - 1, 0, -1):                 # then TB level with one warp per TB
        f = M.F(1, m)
        if M.fits(f):
            return done(1, m, f, FIT_CTA)
    return done(W, T, full, FIT_UNRESOLVABLE)     # P:244, P:395 (CORR): leave as is
