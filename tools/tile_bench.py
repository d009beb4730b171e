"""A/B timing of the FP32 tile kernels (SYRK / SYR2K / CORR / GEMM STAGED) for
one kernel choice per process (the CATT_TILED_* switches are read once), and a
digest of every output so two processes can be compared bit for bit.

    CATT_TILED_T2=0 python tools/tile_bench.py [--n 2048] [--reps 20]

Prints one JSON line: per workload the mean / min event time of the kernel,
TFLOP/s (2 n^2 m for SYRK, 4 n^2 m for SYR2K, the SYRK part of CORR) and the
sha1 of the result."""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402


def digest(t):
    return hashlib.sha1(t.detach().cpu().numpy().tobytes()).hexdigest()[:16]


def timeit(fn, reps, setup=None):
    s = torch.cuda.current_stream()
    ts = []
    for i in range(reps + 3):
        if setup:
            setup()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda._sleep(200_000)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        if i >= 3:
            ts.append(e0.elapsed_time(e1))
    return sum(ts) / len(ts), min(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=2048)
    ap.add_argument("--m", type=int, default=0)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--only", default="syrk,syr2k,corr")
    a = ap.parse_args()
    n, m = a.n, a.m or a.n
    out = {"n": n, "m": m, "env": {k: v for k, v in os.environ.items() if k.startswith("CATT_TILED")}}
    hw = catt.hw_query()
    def planned(prob):   # the CATT plan of the STAGED kernel, as bench.py launches it (Eq 4 picks the carveout)
        t, r = catt.plan(prob, catt.Throttle(variant="staged"), hw)
        out.setdefault("plans", {})[str(prob.loop)] = dict(carveout_kb=r["carveout_kb"], base=[r["base_warps"], r["base_ctas"]],
                                                          throttle=[t.active_warps, t.active_ctas])
        return t
    A = torch.empty(n * m, device="cuda")
    B = torch.empty(n * m, device="cuda")
    C0 = torch.empty(n * n, device="cuda")
    catt.fill_hash(A, 11)
    catt.fill_hash(B, 12)
    catt.fill_hash(C0, 13)
    A, B, C0 = A.view(n, m), B.view(n, m), C0.view(n, n)
    C = C0.clone()
    only = a.only.split(",")
    if "syrk" in only:
        st = planned(catt.problem(catt.K_SYRK, n=n, k=m))
        res = C0.clone()
        catt.syrk(A, res, 1.5, 1.2, t=st)
        mean, mn = timeit(lambda: catt.syrk(A, C, 1.5, 1.2, t=st), a.reps, lambda: C.copy_(C0))
        out["syrk"] = dict(ms=mean, min_ms=mn, tflops=2.0 * n * n * m / mean / 1e9, sha=digest(res))
    if "syr2k" in only:
        st = planned(catt.problem(catt.K_SYR2K, n=n, k=m))
        res = C0.clone()
        catt.syr2k(A, B, res, 1.5, 1.2, t=st)
        mean, mn = timeit(lambda: catt.syr2k(A, B, C, 1.5, 1.2, t=st), a.reps, lambda: C.copy_(C0))
        out["syr2k"] = dict(ms=mean, min_ms=mn, tflops=4.0 * n * n * m / mean / 1e9, sha=digest(res))
    if "corr" in only:
        D0 = torch.empty(m * n, device="cuda")
        catt.fill_hash(D0, 14)
        D0 = D0.view(m, n)      # m rows (observations) x n columns
        D = D0.clone()
        work = torch.empty(m * n, device="cuda")
        st = planned(catt.problem(catt.K_CORR, n=n, k=m))
        sym, _, _ = catt.corr(D, work=work, t=st)
        h = digest(sym)
        mean, mn = timeit(lambda: catt.corr(D, work=work, t=st), a.reps, lambda: D.copy_(D0))
        # the SYRK part: n(n+1)/2 outputs of m fmas (upper tiles: 136 of 256 at 2048)
        out["corr"] = dict(ms=mean, min_ms=mn, tflops=1.0 * n * (n + 1) * m / mean / 1e9, sha=h)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
