"""CPU ORACLE — address traces of the hot-path loops and an LRU L1D simulator.

TEST INFRASTRUCTURE ONLY (see oracle/footprint.py header). Independent of the
descriptors: the traces below are written from the loop bodies themselves
(PolyBench/GPU and Rodinia kernels of Table 2; ATAX kernel 1 is
Fig 1), one event per warp-level memory instruction, so they pin
both the footprint model and the descriptors the library builds.

LRU model: fully associative, LRU, `line_bytes` lines.
Warps are interleaved round-robin, one memory instruction per turn. Only
`a` warps per CTA and `m` CTAs per SM are runnable; a finished warp's slot
goes to the next waiting warp of its CTA (semaphore semantics), a finished
CTA's slot to the next CTA of the SM's list. A miss is an *intra-thread
capacity miss* when the same thread touched that line before: the
intra-thread locality CATT protects ("the fetched cache line
is reused in the following iteration"). Compulsory misses and lines another
thread fetched (inter-thread reuse, e.g. the line a row ends in and the next
row starts in) do not count (reading R12).

An event is one warp-level memory instruction: a tuple of (line, thread id)
pairs, one per active lane.

`program(b, w)` is the same loop body with every access labelled: a list of
(instruction, is_store, bytes per lane, lanes) where lanes is the event tuple.
It follows the kernels' source order (csrc/k_gemv.cu row_thread_kernel: x[j],
then A[i*N + j], then B[i*N + j]) and includes the stores, which L1 does not
keep (write-through, no allocate) and `events` therefore leaves out. The
B200 decision rule's inputs are measured on it (oracle/b200_rule.py).
"""
from __future__ import annotations

from collections import OrderedDict, deque
from typing import Dict, List, Sequence, Tuple

LINE = 128
E = 4  # fp32


def _line(arr: str, idx: int, line: int = LINE) -> Tuple[str, int]:
    return (arr, (idx * E) // line)


class Kernel:
    """nblocks CTAs of W warps; events(b, w) -> list of events."""
    nblocks: int
    W: int
    threads: int

    def lanes(self, b: int, w: int):
        for lane in range(32):
            t = 32 * w + lane
            if t < self.threads:
                yield t


class RowKernel(Kernel):
    """Thread i = blockIdx.x*cta + threadIdx.x owns row i (i < M):
         for j (step vec): for each matrix X: acc += X[i*N + j] * x[j]
    vec = 4 models float4 loads (one 16-byte access per thread). With
    with_tmp=True the accumulator is the global tmp[i] read every iteration
    (Fig 1 literally)."""

    def __init__(self, M, N, cta, vec=1, matrices=("A",), with_tmp=False):
        self.M, self.N, self.vec, self.matrices, self.with_tmp = M, N, vec, matrices, with_tmp
        self.threads = cta
        self.W = (cta + 31) // 32
        self.nblocks = (M + cta - 1) // cta

    def events(self, b, w):
        rows = [b * self.threads + t for t in self.lanes(b, w)]
        rows = [i for i in rows if i < self.M]
        ev = []
        if not rows:
            return ev
        for j in range(0, self.N, self.vec):
            if self.with_tmp:
                ev.append(tuple((_line("tmp", i), i) for i in rows))
            for X in self.matrices:
                ev.append(tuple((_line(X, i * self.N + j), i) for i in rows))
                ev.append(tuple((_line("x", j), i) for i in rows))
        return ev

    def program(self, b, w):
        rows = [i for i in (b * self.threads + t for t in self.lanes(b, w)) if i < self.M]
        out = []
        if not rows:
            return out
        nb = 4 * self.vec
        for j in range(0, self.N, self.vec):
            if self.with_tmp:
                out.append(("tmp", False, 4, tuple((_line("tmp", i), i) for i in rows)))
            out.append(("x", False, nb, tuple((_line("x", j), i) for i in rows)))
            for X in self.matrices:
                out.append((X, False, nb, tuple((_line(X, i * self.N + j), i) for i in rows)))
        return out


class ColKernel(Kernel):
    """Thread j owns column j (j < N):  for i < M: acc += A[i*N + j] * v[i]."""

    def __init__(self, M, N, cta):
        self.M, self.N = M, N
        self.threads = cta
        self.W = (cta + 31) // 32
        self.nblocks = (N + cta - 1) // cta

    def events(self, b, w):
        cols = [b * self.threads + t for t in self.lanes(b, w)]
        cols = [j for j in cols if j < self.N]
        ev = []
        if not cols:
            return ev
        for i in range(self.M):
            ev.append(tuple((_line("A", i * self.N + j), j) for j in cols))
            ev.append(tuple((_line("v", i), j) for j in cols))
        return ev

    def program(self, b, w):
        cols = [j for j in (b * self.threads + t for t in self.lanes(b, w)) if j < self.N]
        out = []
        for i in range(self.M if cols else 0):
            out.append(("A", False, 4, tuple((_line("A", i * self.N + j), j) for j in cols)))
            out.append(("v", False, 4, tuple((_line("v", i), j) for j in cols)))
        return out


class SyrkKernel(Kernel):
    """PolyBench/GPU syrk, block (32, 8): j = bx*32 + tx, i = by*8 + ty,
    for k < Mk: c += alpha * a[i*Mk + k] * a[j*Mk + k] (c in a register)."""

    def __init__(self, N, Mk, bdim=(32, 8)):
        self.N, self.Mk, self.bdim = N, Mk, bdim
        self.threads = bdim[0] * bdim[1]
        self.W = (self.threads + 31) // 32
        self.gx = (N + bdim[0] - 1) // bdim[0]
        self.gy = (N + bdim[1] - 1) // bdim[1]
        self.nblocks = self.gx * self.gy

    def events(self, b, w):
        bx, by = b % self.gx, b // self.gx
        th = []
        for t in self.lanes(b, w):
            tx, ty = t % self.bdim[0], t // self.bdim[0]
            i, j = by * self.bdim[1] + ty, bx * self.bdim[0] + tx
            if i < self.N and j < self.N:
                th.append((i, j))
        ev = []
        if not th:
            return ev
        for k in range(self.Mk):
            ev.append(tuple((_line("a", i * self.Mk + k), (i, j)) for i, j in th))
            ev.append(tuple((_line("a", j * self.Mk + k), (i, j)) for i, j in th))
        return ev

    def _ij(self, b, w):
        bx, by = b % self.gx, b // self.gx
        th = []
        for t in self.lanes(b, w):
            tx, ty = t % self.bdim[0], t // self.bdim[0]
            i, j = by * self.bdim[1] + ty, bx * self.bdim[0] + tx
            if i < self.N and j < self.N:
                th.append((i, j))
        return th

    def program(self, b, w):
        th = self._ij(b, w)
        out = []
        for k in range(self.Mk if th else 0):
            out.append(("a_i", False, 4, tuple((_line("a", i * self.Mk + k), (i, j)) for i, j in th)))
            out.append(("a_j", False, 4, tuple((_line("a", j * self.Mk + k), (i, j)) for i, j in th)))
        return out


class Syr2kKernel(SyrkKernel):
    """PolyBench/GPU syr2k, block (32, 8), same thread map as syrk; for k < Mk:
    c += alpha*a[i*Mk + k]*b[j*Mk + k] + alpha*b[i*Mk + k]*a[j*Mk + k]."""

    def events(self, b, w):
        bx, by = b % self.gx, b // self.gx
        th = []
        for t in self.lanes(b, w):
            tx, ty = t % self.bdim[0], t // self.bdim[0]
            i, j = by * self.bdim[1] + ty, bx * self.bdim[0] + tx
            if i < self.N and j < self.N:
                th.append((i, j))
        ev = []
        if not th:
            return ev
        for k in range(self.Mk):
            for X, row in (("a", 0), ("b", 0), ("b", 1), ("a", 1)):
                ev.append(tuple((_line(X, (i, j)[row] * self.Mk + k), (i, j)) for i, j in th))
        return ev

    def program(self, b, w):
        th = self._ij(b, w)
        out = []
        for k in range(self.Mk if th else 0):
            for X, row in (("a", 0), ("b", 0), ("b", 1), ("a", 1)):
                out.append((f"{X}_{'ij'[row]}", False, 4,
                            tuple((_line(X, (i, j)[row] * self.Mk + k), (i, j)) for i, j in th)))
        return out


class GemmKernel(Kernel):
    """PolyBench/GPU gemm, block (32, 8): j = bx*32 + tx, i = by*8 + ty,
    for k < nk: c += alpha * a[i*nk + k] * b[k*nj + j]."""

    def __init__(self, ni, nj, nk, bdim=(32, 8)):
        self.ni, self.nj, self.nk, self.bdim = ni, nj, nk, bdim
        self.threads = bdim[0] * bdim[1]
        self.W = (self.threads + 31) // 32
        self.gx = (nj + bdim[0] - 1) // bdim[0]
        self.gy = (ni + bdim[1] - 1) // bdim[1]
        self.nblocks = self.gx * self.gy

    def events(self, b, w):
        bx, by = b % self.gx, b // self.gx
        th = []
        for t in self.lanes(b, w):
            tx, ty = t % self.bdim[0], t // self.bdim[0]
            i, j = by * self.bdim[1] + ty, bx * self.bdim[0] + tx
            if i < self.ni and j < self.nj:
                th.append((i, j))
        ev = []
        if not th:
            return ev
        for k in range(self.nk):
            ev.append(tuple((_line("a", i * self.nk + k), (i, j)) for i, j in th))
            ev.append(tuple((_line("b", k * self.nj + j), (i, j)) for i, j in th))
        return ev

    def program(self, b, w):
        bx, by = b % self.gx, b // self.gx
        th = []
        for t in self.lanes(b, w):
            tx, ty = t % self.bdim[0], t // self.bdim[0]
            i, j = by * self.bdim[1] + ty, bx * self.bdim[0] + tx
            if i < self.ni and j < self.nj:
                th.append((i, j))
        out = []
        for k in range(self.nk if th else 0):
            out.append(("a", False, 4, tuple((_line("a", i * self.nk + k), (i, j)) for i, j in th)))
            out.append(("b", False, 4, tuple((_line("b", k * self.nj + j), (i, j)) for i, j in th)))
        return out


class KmeansKernel(Kernel):
    """Rodinia kmeansPoint, feature-major: thread p (p < npoints):
    for c < k: for f < nf: diff = feat[f*ld + p] - clusters[c*nf + f]
    (clusters are staged in shared memory, so not traced)."""

    def __init__(self, npoints, nf, k, ld, cta):
        self.npoints, self.nf, self.k, self.ld = npoints, nf, k, ld
        self.threads = cta
        self.W = (cta + 31) // 32
        self.nblocks = (npoints + cta - 1) // cta

    def events(self, b, w):
        pts = [b * self.threads + t for t in self.lanes(b, w)]
        pts = [p for p in pts if p < self.npoints]
        ev = []
        if not pts:
            return ev
        for c in range(self.k):
            for f in range(self.nf):
                ev.append(tuple((_line("F", f * self.ld + p), p) for p in pts))
        return ev

    def program(self, b, w):
        return [("F", False, 4, ev) for ev in self.events(b, w)]


class TransposeKernel(Kernel):
    """Rodinia invert_mapping (KM's other loop, csrc/k_kmeans_iter.cu LITERAL):
    thread p (p < npoints): for f < nf: out[f*ld + p] = in[p*nf + f]."""

    def __init__(self, npoints, nf, ld, cta):
        self.npoints, self.nf, self.ld = npoints, nf, ld
        self.threads = cta
        self.W = (cta + 31) // 32
        self.nblocks = (npoints + cta - 1) // cta

    def program(self, b, w):
        pts = [p for p in (b * self.threads + t for t in self.lanes(b, w)) if p < self.npoints]
        out = []
        for f in range(self.nf if pts else 0):
            out.append(("in", False, 4, tuple((_line("in", p * self.nf + f), p) for p in pts)))
            out.append(("out", True, 4, tuple((_line("out", f * self.ld + p), p) for p in pts)))
        return out

    def events(self, b, w):
        return [lanes for _, st, _, lanes in self.program(b, w) if not st]


class CorrKernel(Kernel):
    """PolyBench/GPU correlation, the thread-per-column loop (csrc/k_corr.cu
    corr_thread_kernel): thread j1 (j1 < m): for j2 in j1+1 .. m-1: for i < n:
    s += data[i*m + j1] * data[i*m + j2]; then symmat[j1*m + j2] = s and
    symmat[j2*m + j1] = s. Lane j1 starts its j2 loop at j1 + 1, so the warp's
    lanes are at different j2 in the same step."""

    def __init__(self, m, n, cta):
        self.m, self.n = m, n
        self.threads = cta
        self.W = (cta + 31) // 32
        self.nblocks = (m + cta - 1) // cta

    def program(self, b, w):
        cols = [j for j in (b * self.threads + t for t in self.lanes(b, w)) if j < self.m]
        out = []
        if not cols:
            return out
        # the lanes run the j2 loop in lockstep from their own start: at step
        # q lane j1 is at j2 = j1 + 1 + q, and is done once j2 reaches m
        for q in range(self.m - min(cols) - 1):
            act = [(j1, j1 + 1 + q) for j1 in cols if j1 + 1 + q < self.m]
            for i in range(self.n):
                out.append(("d_j1", False, 4, tuple((_line("d", i * self.m + j1), j1) for j1, j2 in act)))
                out.append(("d_j2", False, 4, tuple((_line("d", i * self.m + j2), j1) for j1, j2 in act)))
            out.append(("sym_12", True, 4, tuple((_line("sym", j1 * self.m + j2), j1) for j1, j2 in act)))
            out.append(("sym_21", True, 4, tuple((_line("sym", j2 * self.m + j1), j1) for j1, j2 in act)))
        return out

    def events(self, b, w):
        return [lanes for _, st, _, lanes in self.program(b, w) if not st]


def simulate(kernel: Kernel, sm_blocks: Sequence[int], a: int, m: int, capacity: int) -> Dict:
    """Run the warps of the CTAs in sm_blocks (in order) with at most a active
    warps per CTA and m active CTAs; LRU of `capacity` lines."""
    cache: "OrderedDict" = OrderedDict()
    seen: Dict[object, set] = {}
    stats = dict(accesses=0, hits=0, misses=0, intra_thread_capacity_misses=0)
    pending = deque(sm_blocks)
    rotation: deque = deque()          # entries: [b, w, events, pos]
    cta_wait: Dict[int, deque] = {}
    cta_left: Dict[int, int] = {}

    def start_cta():
        b = pending.popleft()
        ws = deque(range(kernel.W))
        cta_wait[b] = ws
        cta_left[b] = kernel.W
        for _ in range(min(a, kernel.W)):
            w = ws.popleft()
            rotation.append([b, w, kernel.events(b, w), 0])

    active_ctas = 0
    while pending and active_ctas < m:
        start_cta()
        active_ctas += 1
    while rotation:
        ent = rotation.popleft()
        b, w, ev, pos = ent
        if pos < len(ev):
            by_line: Dict[Tuple[str, int], list] = {}
            for ln, tid in ev[pos]:
                by_line.setdefault(ln, []).append(tid)
            # one warp request: every tag is looked up first (hits refresh
            # their lines), then the missing lines are filled, evicting LRU
            # lines not touched by this request
            missing = []
            for ln, tids in by_line.items():
                stats["accesses"] += 1
                if ln in cache:
                    cache.move_to_end(ln)
                    stats["hits"] += 1
                else:
                    missing.append((ln, tids))
            for ln, tids in missing:
                stats["misses"] += 1
                if any(ln in seen.get(t, ()) for t in tids):
                    stats["intra_thread_capacity_misses"] += 1
                cache[ln] = True
                if len(cache) > capacity:
                    cache.popitem(last=False)
            for ln, tids in by_line.items():
                for t in tids:
                    seen.setdefault(t, set()).add(ln)
            ent[3] = pos + 1
        if ent[3] < len(ev):
            rotation.append(ent)
            continue
        # warp done: refill its slot from its CTA
        cta_left[b] -= 1
        if cta_wait[b]:
            w2 = cta_wait[b].popleft()
            rotation.append([b, w2, kernel.events(b, w2), 0])
        elif cta_left[b] == 0 and pending:
            start_cta()
    return stats


def sm0_blocks(kernel: Kernel, num_sms: int, limit: int = 1 << 30) -> List[int]:
    """Blocks the round-robin distribution gives SM 0: 0, #SM, 2*#SM, ..."""
    return list(range(0, kernel.nblocks, num_sms))[:limit]


def decide_by_lru(kernel: Kernel, W: int, T: int, capacity: int, num_sms: int, limit_blocks=None) -> Tuple[int, int, str]:
    """Walk the Eq 9 candidate order and return the
    first throttle with zero intra-thread capacity misses."""
    blocks = sm0_blocks(kernel, num_sms, limit_blocks or max(T, 1))

    def ok(a, m):
        return simulate(kernel, blocks, a, m, capacity)["intra_thread_capacity_misses"] == 0

    if ok(W, T):
        return W, T, "none"
    for N in range(2, W + 1):
        if W % N == 0 and ok(W // N, T):
            return W // N, T, "warp"
    for m in range(T - 1, 0, -1):
        if ok(1, m):
            return 1, m, "cta"
    return W, T, "unresolvable"
