"""Held-out study 12 (round 2, closing): an out-of-sample check of the final
library rule (R18 ... R29, R32), no rule change under test. New launches
only (none of the 195 stored sweeps), spread over every loop family: row
loops with one, two and three divergent streams, the 2-D block SYRK / SYR2K,
the KMEANS assignment and transpose, and the GEMM control, at shapes, CTA
sizes and carveouts not measured before. The picks of the library's rule and
of the paper's Eq 9 are written BEFORE any timing (--predict prints them
without a GPU; the committed predictions file is that output).

For each launch: every (a, m) of the literal loop, timed cold (L2 flushed,
then a GPU sleep), median of `reps`.
usage: python tools/heldout12_study.py [--predict] [--reps R]
Writes gpurun_out/heldout12/heldout12_study.json."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

P = catt.problem
# (name, problem, [(CTA threads, carveout KB)])
CASES = [
    ("atax1 literal 24576x3072", P(catt.K_ATAX_1, m=24576, n=3072), [(256, 228), (1024, 164)]),
    ("bicg2 literal m=20480 n=1536", P(catt.K_BICG_2, m=20480, n=1536), [(512, 196), (384, 164)]),
    ("mvt1 literal 7168", P(catt.K_MVT_1, n=7168), [(768, 228), (256, 196)]),
    ("gesummv literal 9216", P(catt.K_GESUMMV, n=9216), [(1024, 132), (256, 196)]),
    ("rows3 literal 12288x3072", P(catt.K_ROWS3, m=12288, n=3072), [(512, 196)]),
    ("syrk literal 2560x1024", P(catt.K_SYRK, n=2560, k=1024), [(256, 196), (128, 228)]),
    ("syr2k literal 1792", P(catt.K_SYR2K, n=1792, k=1792), [(256, 228), (512, 196)]),
    ("kmeans assign 250000x24 k=6", P(catt.K_KMEANS, m=250000, n=24, k=6, ld=250000), [(256, 228), (512, 64)]),
    ("kmeans transpose 300000x20", P(catt.K_KMEANS_T, m=300000, n=20, ld=300000), [(256, 32)]),
    ("gemm literal 768", P(catt.K_GEMM, m=768, n=768, k=768), [(256, 228)]),
]


def picks(prob, cta, carve):
    hw = catt.hw_b200()
    launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant="literal")
    out = {}
    for name in ("b200", "paper"):
        h = hw if name == "b200" else catt.paper_rule(hw)
        t, r = catt.plan(prob, launch, h)
        W, T = r["base_warps"], r["base_ctas"]
        out[name] = [t.active_warps or W, t.active_ctas or T]
        out["base"] = [W, T]
        out["footprint"], out["l1d_lines"] = r["footprint_lines_full"], r["l1d_bytes"] // 128
    return out


def make_fn(torch, prob):
    dev = torch.device("cuda")
    L = prob.loop
    if L in (catt.K_SYRK, catt.K_SYR2K):
        n, k = prob.n, prob.k
        A = torch.empty(n, k, device=dev); catt.fill_hash(A, 6)
        B = torch.empty(n, k, device=dev); catt.fill_hash(B, 8)
        C = torch.empty(n, n, device=dev); catt.fill_hash(C, 106)
        if L == catt.K_SYRK:
            return lambda th: (lambda: catt.syrk(A, C, 1.5, 1.2, t=th))
        return lambda th: (lambda: catt.syr2k(A, B, C, 1.5, 1.2, t=th))
    if L == catt.K_GEMM:
        n = prob.n
        A = torch.empty(n, n, device=dev); catt.fill_hash(A, 6)
        B = torch.empty(n, n, device=dev); catt.fill_hash(B, 8)
        C = torch.empty(n, n, device=dev); catt.fill_hash(C, 106)
        return lambda th: (lambda: catt.gemm(A, B, C, 1.5, 1.2, t=th))
    if L == catt.K_KMEANS:
        npts, nf, ld, kc = prob.m, prob.n, prob.ld, prob.k
        fm = torch.empty(nf * ld, device=dev); catt.fill_hash(fm, 44)
        cl = fm.view(nf, ld)[:, :kc].t().contiguous()
        memb = torch.empty(npts, dtype=torch.int32, device=dev)
        return lambda th: (lambda: catt.kmeans_assign(fm, ld, npts, nf, cl, memb, t=th))
    if L == catt.K_KMEANS_T:
        npts, nf, ld = prob.m, prob.n, prob.ld
        pm = torch.empty(npts * nf, device=dev); catt.fill_hash(pm, 41)
        fm = torch.empty(nf * ld, device=dev)
        return lambda th: (lambda: catt.kmeans_transpose(pm, npts, nf, fm, ld, t=th))
    if L == catt.K_GESUMMV:
        n = prob.n
        A = torch.empty(n, n, device=dev); catt.fill_hash(A, 5)
        B = torch.empty(n, n, device=dev); catt.fill_hash(B, 105)
        x = torch.empty(n, device=dev); catt.fill_hash(x, 205)
        y, tmp = torch.empty(n, device=dev), torch.empty(n, device=dev)
        return lambda th: (lambda: catt.rows(A, x, y, catt.ROWS_GESUMMV, B=B, tmp=tmp, alpha=1.5, beta=1.2, t=th))
    if L == catt.K_ROWS3:
        m, n = prob.m, prob.n
        A = torch.empty(m, n, device=dev); catt.fill_hash(A, 5)
        BC = torch.empty(2 * m, n, device=dev); catt.fill_hash(BC, 105)
        x = torch.empty(n, device=dev); catt.fill_hash(x, 205)
        y = torch.empty(m, device=dev)
        return lambda th: (lambda: catt.rows(A, x, y, catt.ROWS_SUM3, B=BC, t=th))
    m = prob.m if L in (catt.K_BICG_2, catt.K_ATAX_1) else prob.n
    n = prob.n
    A = torch.empty(m, n, device=dev); catt.fill_hash(A, 2)
    x = torch.empty(n, device=dev); catt.fill_hash(x, 102)
    y = torch.empty(m, device=dev)
    mode = catt.ROWS_ACCUM if L == catt.K_MVT_1 else catt.ROWS_STORE
    return lambda th: (lambda: catt.rows(A, x, y, mode, t=th))


def main():
    if "--predict" in sys.argv:
        for name, prob, launches in CASES:
            for cta, carve in launches:
                print(name, cta, carve, picks(prob, cta, carve))
        return
    reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 3
    import torch
    dev = torch.device("cuda")
    flush_buf = torch.empty(64 * 1024 * 1024, dtype=torch.int32, device=dev)
    clean_buf = torch.zeros(64 * 1024 * 1024, dtype=torch.int32, device=dev)

    def med(fn):
        ts = []
        for r in range(reps + 1):
            flush_buf.zero_()
            clean_buf.sum()
            torch.cuda._sleep(400_000)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize()
            if r:
                ts.append(a.elapsed_time(b))
        return statistics.median(ts)

    res = []
    for name, prob, launches in CASES:
        make = make_fn(torch, prob)
        for cta, carve in launches:
            pk = picks(prob, cta, carve)
            W, T = pk["base"]
            launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant="literal")
            times = {}
            for a in [d for d in range(W, 0, -1) if W % d == 0]:
                for m in range(T, 0, -1):
                    times[(a, m)] = med(make(launch.copy(active_warps=a, active_ctas=m if m < T else 0)))
            best = min(times, key=times.get)
            row = dict(loop=name, prob=dict(loop=prob.loop, m=prob.m, n=prob.n, k=prob.k, ld=prob.ld), variant="literal",
                       cta=cta, carveout_kb=carve, base=[W, T], footprint=pk["footprint"], l1d_lines=pk["l1d_lines"],
                       b200=pk["b200"], paper=pk["paper"], best=list(best),
                       best_ms=round(times[best], 4), full_ms=round(times[(W, T)], 4),
                       **{f"{k}_over_best": round(times[tuple(pk[k])] / times[best], 3) for k in ("b200", "paper")},
                       swept={f"{a},{m}": round(v, 4) for (a, m), v in times.items()})
            print(json.dumps({k: v for k, v in row.items() if k != "swept"}), flush=True)
            res.append(row)
    os.makedirs("gpurun_out/heldout12", exist_ok=True)
    json.dump(res, open("gpurun_out/heldout12/heldout12_study.json", "w"), indent=1)


if __name__ == "__main__":
    main()
