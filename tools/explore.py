"""Exploration timings (not the bench): each loop x variant x launch, CUDA
events, L2 flushed before every rep; prints GB/s of algorithmic bytes."""
import json
import sys
import time

import torch

import paper_conf_icpp_kimhlsh19_b200 as catt

torch.cuda.init()
dev = torch.device("cuda")
flush_buf = torch.empty(64 * 1024 * 1024, dtype=torch.int32, device=dev)   # 256 MiB > L2


def timeit(fn, reps=10, flush=True):
    ts = []
    for r in range(reps + 2):
        if flush:
            flush_buf.zero_()
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        if r >= 2:
            ts.append(s.elapsed_time(e))
    ts.sort()
    return ts[len(ts) // 2]


out = []


def report(name, ms, nbytes, extra=""):
    gbs = nbytes / (ms * 1e-3) / 1e9
    out.append(dict(name=name, ms=ms, gbs=gbs, extra=extra))
    print(f"{name:60s} {ms * 1e3:9.1f} us {gbs:8.0f} GB/s {extra}", flush=True)


def gemv_4096():
    n = 4096
    A = torch.empty(n, n, device=dev)
    catt.fill_hash(A, 2)
    x = torch.rand(n, device=dev)
    y = torch.empty(n, device=dev)
    nbytes = n * n * 4
    for var, ctas in [("literal", [32, 64, 128, 256, 1024]), ("vec4", [32, 64, 128, 256]),
                      ("staged", [32, 64, 128]), ("coop", [256])]:
        for c in ctas:
            t = catt.Throttle(cta_threads=c, variant=var)
            ms = timeit(lambda: catt.rows(A, x, y, t=t))
            report(f"rows 4096 {var} cta={c}", ms, nbytes)
    for var, ctas in [("literal", [32, 64, 128, 256]), ("vec4", [32, 64, 128]), ("staged", [32, 64, 128]), ("coop", [256])]:
        for c in ctas:
            t = catt.Throttle(cta_threads=c, variant=var)
            ms = timeit(lambda: catt.cols(A, x, y, t=t))
            report(f"cols 4096 {var} cta={c}", ms, nbytes)
    # throttle on the literal row loop at the contended carveout
    for carve in (0, 196, 228):
        for aw in (8, 4, 2, 1):
            t = catt.Throttle(cta_threads=256, active_warps=aw, carveout_kb=carve)
            ms = timeit(lambda: catt.rows(A, x, y, t=t))
            report(f"rows 4096 literal cta=256 carve={carve} warps={aw}", ms, nbytes)
    for carve in (0, 132, 196, 228):
        for aw in (32, 16, 8, 4):
            t = catt.Throttle(cta_threads=1024, active_warps=aw, carveout_kb=carve)
            ms = timeit(lambda: catt.rows(A, x, y, t=t))
            report(f"rows 4096 literal cta=1024 carve={carve} warps={aw}", ms, nbytes)


def kmeans():
    npts, nf, k = 494020, 34, 5
    hw = catt.hw_query()
    for ld in (494020, 494048):
        feat = torch.empty(nf * ld, device=dev)
        catt.fill_hash(feat, 4)
        clusters = feat.view(nf, ld)[:, :k].t().contiguous()
        memb = torch.empty(npts, dtype=torch.int32, device=dev)
        nbytes = npts * nf * 4 + npts * 4
        prob = catt.problem(catt.K_KMEANS, m=npts, n=nf, k=k, ld=ld)
        for carve in (0, 100, 228):
            tc, r = catt.plan(prob, catt.Throttle(carveout_kb=carve), hw)
            best = None
            for aw in (8, 4, 2, 1):
                for m in (8, 6, 4, 3, 2, 1):
                    if aw < 8 and m < 8 and aw != 1:
                        continue
                    t = catt.Throttle(active_warps=aw, active_ctas=m if m < 8 else 0, carveout_kb=carve)
                    ms = timeit(lambda: catt.kmeans_assign(feat, ld, npts, nf, clusters, memb, t=t))
                    tag = " <- CATT" if (aw == (tc.active_warps or 8) and m == (tc.active_ctas or 8)) else ""
                    report(f"kmeans ld={ld} carve={carve} ({aw},{m})", ms, nbytes, tag)
                    if best is None or ms < best[0]:
                        best = (ms, aw, m)
            print(f"   CATT pick {tc} flags={catt.FLAG_NAMES[r['flags']]}  best swept {best}")
        for var in ("regs",):
            for c in (128, 256):
                t = catt.Throttle(cta_threads=c, variant=var)
                ms = timeit(lambda: catt.kmeans_assign(feat, ld, npts, nf, clusters, memb, t=t))
                report(f"kmeans ld={ld} {var} cta={c}", ms, nbytes)


def syrk():
    n = 2048
    A = torch.empty(n, n, device=dev)
    C = torch.empty(n, n, device=dev)
    catt.fill_hash(A, 6)
    flops = 2 * n * n * n
    for var in ("literal", "staged"):
        t = catt.Throttle(variant=var)
        ms = timeit(lambda: catt.syrk(A, C, 1.5, 1.2, t=t), reps=5)
        report(f"syrk 2048 {var}", ms, flops, f"{flops / ms / 1e9:.1f} TFLOP/s")


def gesummv():
    n = 8192
    A = torch.empty(n, n, device=dev)
    B = torch.empty(n, n, device=dev)
    catt.fill_hash(A, 5)
    catt.fill_hash(B, 6)
    x = torch.rand(n, device=dev)
    y, tmp = torch.empty(n, device=dev), torch.empty(n, device=dev)
    nbytes = 2 * n * n * 4
    for var, ctas in [("literal", [64, 256]), ("vec4", [64, 256]), ("staged", [32, 64]), ("coop", [256])]:
        for c in ctas:
            t = catt.Throttle(cta_threads=c, variant=var)
            ms = timeit(lambda: catt.gesummv(A, B, x, 1.5, 1.2, y, tmp, t=t))
            report(f"gesummv 8192 {var} cta={c}", ms, nbytes)


def atax_big():
    m, n = 65536, 16384
    A = torch.empty(m, n, device=dev)
    catt.fill_hash(A, 7)
    x = torch.rand(n, device=dev)
    tmp, y = torch.empty(m, device=dev), torch.empty(n, device=dev)
    nbytes = m * n * 4
    for var, c in [("literal", 256), ("vec4", 256), ("staged", 32), ("staged", 64), ("coop", 256)]:
        t = catt.Throttle(cta_threads=c, variant=var)
        ms = timeit(lambda: catt.rows(A, x, tmp, t=t), reps=5)
        report(f"rows 65536x16384 {var} cta={c}", ms, nbytes)
    for var, c in [("literal", 256), ("vec4", 256), ("staged", 32), ("staged", 64), ("coop", 256)]:
        t = catt.Throttle(cta_threads=c, variant=var)
        ms = timeit(lambda: catt.cols(A, tmp, y, t=t), reps=5)
        report(f"cols 65536x16384 {var} cta={c}", ms, nbytes)


def staged_only():
    n = 4096
    A = torch.empty(n, n, device=dev)
    catt.fill_hash(A, 2)
    x = torch.rand(n, device=dev)
    y = torch.empty(n, device=dev)
    for c in (32, 64):
        for kind in ("rows", "cols"):
            t = catt.Throttle(cta_threads=c, variant="staged")
            f = (lambda: catt.rows(A, x, y, t=t)) if kind == "rows" else (lambda: catt.cols(A, x, y, t=t))
            report(f"{kind} 4096 staged cta={c}", timeit(f), n * n * 4)
    for kind in ("rows", "cols"):
        t = catt.Throttle(variant="coop")
        f = (lambda: catt.rows(A, x, y, t=t)) if kind == "rows" else (lambda: catt.cols(A, x, y, t=t))
        report(f"{kind} 4096 coop", timeit(f), n * n * 4)


if __name__ == "__main__":
    which = sys.argv[1:] or ["gemv", "kmeans", "syrk", "gesummv", "atax"]
    fns = dict(gemv=gemv_4096, kmeans=kmeans, syrk=syrk, gesummv=gesummv, atax=atax_big,
               staged=lambda: staged_only())
    for w in which:
        fns[w]()
    json.dump(out, open("gpurun_out/explore.json", "w"), indent=1)
