"""CPU ORACLE — the B200 throttle decision, measured on address traces.

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / reference legs may import this (see oracle/footprint.py).

Independent of oracle/footprint.py and of the library's analyser
(csrc/footprint.cpp): nothing here reads a loop descriptor. Every input of the
rule is measured on the loop body's address trace (oracle/lru.py `program`,
written from the kernels' source loops), and "fits" is the LRU L1D simulator's
verdict, not a footprint formula.

The rule (readings R17-R19, R23, R24, R27, R29, R32), restated on traces:

  reuse(I)        instruction I has same-thread locality: one thread touches one
                  line with I in two different iterations (Eq 6's intent,
                  P:218-221 "the fetched cache line is reused in the following
                  iteration"; a loop with no such instruction is not throttled,
                  P:212, R17)
  lines(I)        distinct lines of I's first warp-level access (Eq 7, P:223-235;
                  the memory divergence of P:32)
  retouch(I)      the most touches one thread makes to one line with I (R23)
  stream          bytes of stores and of loads without reuse over all traced
                  bytes of the loop body (R24)
  shared(I)       warp 1 of CTA 0 requests exactly warp 0's lines with I's
                  first access (the CTA's warps share I's lines; R32)
  divergent       some reused load has lines >= divergent_lines and retouch >=
                  min_retouch (and, when private_streams is on, is not shared),
                  and 100 * stream <= max_stream_pct * total (R18, R23, R24,
                  R32); S = the number of such loads
  floor           min_warps_sm, or ceil(min_warps_sm / S) when stream_floor is on,
                  T = 1 and S >= 2 (R29)
  fits(a, m)      zero intra-thread capacity misses when a warps per CTA and m
                  CTAs per SM run SM 0's first T CTAs through an LRU of the L1D's
                  lines (R12)

  decision        full TLP (W, T) if no reuse or fits(W, T); full TLP (guarded)
                  if not divergent; otherwise, over the admissible pairs A =
                  {(a, m): a | W, 1 <= m <= T, (a, m) != (W, T), a m >= floor}:
                  the fitting pair with the most warps per SM, ties to the larger
                  a (R19); if none fits, the pair with the fewest warps per SM
                  (ties to the larger a), replaced when T >= 2 and cta_fallback
                  by (W, m*) with m* the smallest m such that floor <= W m <=
                  2 floor (R27; m* = T means no throttle).

The B200 guard constants and the measured L1D per carveout are DESIGN.md's
(R18, R23, R24, R27; section 5 "Carveout and L1D on B200"), typed here from the
text, not read from the library.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Dict, List, Tuple

from . import lru

# DESIGN.md R18 (floor 8 warps/SM, >= 8 lines per request), R23 (>= 16
# re-touches), R24 (<= 25 % stream bytes), R27 (CTA fallback on), R29 (the
# floor divided by the divergent streams when T = 1), R32 (loads shared by
# the CTA's warps are not streams)
B200_GUARDS = dict(min_warps_sm=8, divergent_lines=8, min_retouch=16, max_stream_pct=25, cta_fallback=1,
                   stream_floor=1, private_streams=1)
# shared-memory options (KB) and the L1D each leaves (KB, measured)
B200_L1D_KB = {0: 218, 8: 218, 16: 218, 32: 218, 64: 186, 100: 150, 132: 118, 164: 86, 196: 53, 228: 21}


@dataclass
class TraceInputs:
    reuse: Dict[str, bool]
    lines: Dict[str, int]
    retouch: Dict[str, int]
    stored: Dict[str, bool]
    stream_bytes: int
    total_bytes: int
    shared: Dict[str, bool]

    @property
    def locality(self) -> bool:
        return any(r for i, r in self.reuse.items() if not self.stored[i])


def trace_inputs(kernel, line: int = lru.LINE) -> TraceInputs:
    """Measure the rule's inputs on warp 0 of CTA 0 (all its lanes)."""
    prog = kernel.program(0, 0)
    touches: Dict[Tuple[str, object, object], int] = {}
    first: Dict[str, int] = {}
    stored: Dict[str, bool] = {}
    nbytes: Dict[str, int] = {}
    for instr, st, nb, lanes in prog:
        stored[instr] = st
        nbytes[instr] = nbytes.get(instr, 0) + nb * len(lanes)
        if instr not in first:
            first[instr] = len({ln for ln, _ in lanes})
        for ln, tid in lanes:
            key = (instr, tid, ln)
            touches[key] = touches.get(key, 0) + 1
    retouch = {i: 0 for i in first}
    for (instr, _, _), c in touches.items():
        retouch[instr] = max(retouch[instr], c)
    reuse = {i: retouch[i] >= 2 for i in first}
    stream = sum(nbytes[i] for i in first if stored[i] or not reuse[i])
    # R32: the first request of each instruction in warp 1 of the same CTA
    first1: Dict[str, set] = {}
    for instr, _, _, lanes in (kernel.program(0, 1) if kernel.W >= 2 else []):
        if instr not in first1:
            first1[instr] = {ln for ln, _ in lanes}
    first0: Dict[str, set] = {}
    for instr, _, _, lanes in prog:
        if instr not in first0:
            first0[instr] = {ln for ln, _ in lanes}
    shared = {i: i in first1 and first1[i] == first0[i] for i in first}
    return TraceInputs(reuse=reuse, lines=first, retouch=retouch, stored=stored, stream_bytes=stream,
                       total_bytes=sum(nbytes.values()), shared=shared)


def divergent_loads(inp: TraceInputs, guards: Dict) -> int:
    """How many reused loads are memory-divergent (R18, R23): the streams of R29."""
    return sum(1 for i in inp.lines if inp.reuse[i] and not inp.stored[i] and inp.lines[i] >= guards["divergent_lines"]
               and inp.retouch[i] >= guards["min_retouch"] and not (guards.get("private_streams", 0) and inp.shared[i]))


def divergent(inp: TraceInputs, guards: Dict) -> bool:
    return divergent_loads(inp, guards) > 0 and 100 * inp.stream_bytes <= guards["max_stream_pct"] * inp.total_bytes


class _Loads(lru.Kernel):
    """The load events of a kernel's program (what L1 keeps), for lru.simulate."""

    def __init__(self, k):
        self.k, self.W, self.threads, self.nblocks = k, k.W, k.threads, k.nblocks

    def events(self, b, w):
        return [lanes for _, st, _, lanes in self.k.program(b, w) if not st]


def decide(kernel, W: int, T: int, l1d_lines: int, num_sms: int, guards: Dict = B200_GUARDS) -> Tuple[int, int, str]:
    """The B200 rule's (active warps per CTA, active CTAs per SM, how)."""
    inp = trace_inputs(kernel)
    loads = _Loads(kernel)
    blocks = lru.sm0_blocks(loads, num_sms, max(T, 1))
    memo: Dict[Tuple[int, int], bool] = {}

    def fits(a, m):
        if (a, m) not in memo:
            memo[(a, m)] = lru.simulate(loads, blocks, a, m, l1d_lines)["intra_thread_capacity_misses"] == 0
        return memo[(a, m)]

    if not inp.locality or fits(W, T):
        return W, T, "none"
    if not divergent(inp, guards):
        return W, T, "none(guard)"
    floor = guards["min_warps_sm"]
    S = divergent_loads(inp, guards)
    if guards.get("stream_floor", 0) and T == 1 and S >= 2:          # R29: S streams per warp
        floor = -(-floor // S)
    admissible = [(a, m) for a in range(1, W + 1) if W % a == 0 for m in range(1, T + 1)
                  if (a, m) != (W, T) and a * m >= floor]
    if not admissible:
        return W, T, "none(guard)"
    fitting = [am for am in admissible if fits(*am)]
    if fitting:
        a, m = max(fitting, key=lambda am: (am[0] * am[1], am[0]))
        return a, m, "fit"
    fewest = min(a * m for a, m in admissible)
    a, m = max((am for am in admissible if am[0] * am[1] == fewest), key=lambda am: am[0])
    if guards["cta_fallback"] and T >= 2:
        ms = [mm for mm in range(1, T + 1) if floor <= W * mm <= 2 * floor]
        if ms:
            return (W, T, "none(guard)") if ms[0] == T else (W, ms[0], "fallback(cta)")
    return a, m, "fallback"


def l1d_lines(carveout_kb: int, line: int = lru.LINE) -> int:
    return B200_L1D_KB[carveout_kb] * 1024 // line


def b200_hw(num_sms: int = 148) -> Dict:
    """The B200 table for oracle.footprint.occupancy (Eq 1-4): 148 SMs, 64
    warps / 32 CTAs / 64 K registers per SM, 128-byte shared-memory allocation
    unit, 1 KB reserved per CTA (SURVEY 8 header; pinned on the device by
    tests/test_gpu.py::test_occupancy_model_matches_cuda_occupancy_api), the
    carveout options and measured L1D of DESIGN.md section 5."""
    carve = sorted(B200_L1D_KB)
    return dict(num_sms=num_sms, max_warps_sm=64, max_ctas_sm=32, regs_sm=65536, reg_alloc_unit=256, warp_size=32,
                smem_alloc_unit=128, reserved_smem_cta=1024, line_bytes=128, carveout_kb=carve,
                l1d_bytes=[B200_L1D_KB[c] * 1024 for c in carve])
