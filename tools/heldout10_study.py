"""Held-out study 10 (round 2): tests the candidate R29 -- with one CTA per SM,
a loop with S >= 2 memory-divergent reused loads gets the TLP floor
ceil(8 / S) instead of 8 ("the number of divergent
streams"). New launches only (none of the 160 stored sweeps): 2-stream rows
(GESUMMV) and 3-stream rows (CATT_ROWS_SUM3) at shapes and CTA sizes not
measured before, plus 1-stream controls where R29 must not act.

For each launch: every (a, m) of the literal loop, timed cold (L2 flushed:
write + clean read, then a GPU sleep so enqueue cost stays out of the
events), median of `reps`; the picks of the library's rule (R29 off), of the
rule with R29 and of the paper's Eq 9 are written BEFORE any timing
(--predict prints them without a GPU; the committed predictions file is that
output). Adoption rule: geomean better and worst case no
worse on this set.
usage: python tools/heldout10_study.py [--predict] [--reps R]
Writes gpurun_out/heldout10/heldout10_study.json."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

P = catt.problem
# (name, problem, [(CTA threads, carveout KB)]); every launch has T = 1 (<= 148 CTAs)
CASES = [
    ("gesummv literal 5120", P(catt.K_GESUMMV, n=5120), [(256, 196), (512, 132), (320, 228)]),
    ("gesummv literal 7168", P(catt.K_GESUMMV, n=7168), [(1024, 164), (448, 196)]),
    ("gesummv literal 10240", P(catt.K_GESUMMV, n=10240), [(640, 228), (768, 164)]),
    ("gesummv literal 3072", P(catt.K_GESUMMV, n=3072), [(384, 164)]),
    ("rows3 literal 8192x4096", P(catt.K_ROWS3, m=8192, n=4096), [(256, 196), (512, 228), (1024, 132)]),
    ("rows3 literal 16384x2048", P(catt.K_ROWS3, m=16384, n=2048), [(1024, 164), (768, 196)]),
    ("rows3 literal 6144x6144", P(catt.K_ROWS3, m=6144, n=6144), [(384, 196), (640, 100)]),
    ("rows3 literal 4096x8192", P(catt.K_ROWS3, m=4096, n=8192), [(320, 228)]),
    # 1-stream controls (R29 must not act)
    ("bicg2 literal m=8192 n=4096", P(catt.K_BICG_2, m=8192, n=4096), [(512, 164)]),
    ("mvt1 literal 6144 w20", P(catt.K_MVT_1, n=6144), [(640, 196)]),
]


def picks(prob, cta, carve):
    hw = catt.hw_b200()
    launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant="literal")
    out = {}
    for name in ("b200", "r29", "paper"):
        h = catt.Hw.from_dict(hw.as_dict())
        if name == "r29":
            h.stream_floor = 1
        if name == "paper":
            h = catt.paper_rule(hw)
        t, r = catt.plan(prob, launch, h)
        W, T = r["base_warps"], r["base_ctas"]
        out[name] = [t.active_warps or W, t.active_ctas or T]
        out["base"] = [W, T]
        out["footprint"], out["l1d_lines"] = r["footprint_lines_full"], r["l1d_bytes"] // 128
    return out


def make_fn(torch, prob):
    dev = torch.device("cuda")
    if prob.loop == catt.K_GESUMMV:
        n = prob.n
        A = torch.empty(n, n, device=dev); catt.fill_hash(A, 5)
        B = torch.empty(n, n, device=dev); catt.fill_hash(B, 105)
        x = torch.empty(n, device=dev); catt.fill_hash(x, 205)
        y, tmp = torch.empty(n, device=dev), torch.empty(n, device=dev)
        return lambda th: (lambda: catt.rows(A, x, y, catt.ROWS_GESUMMV, B=B, tmp=tmp, alpha=1.5, beta=1.2, t=th))
    if prob.loop == catt.K_ROWS3:
        m, n = prob.m, prob.n
        A = torch.empty(m, n, device=dev); catt.fill_hash(A, 5)
        BC = torch.empty(2 * m, n, device=dev); catt.fill_hash(BC, 105)
        x = torch.empty(n, device=dev); catt.fill_hash(x, 205)
        y = torch.empty(m, device=dev)
        return lambda th: (lambda: catt.rows(A, x, y, catt.ROWS_SUM3, B=BC, t=th))
    m = prob.m if prob.loop in (catt.K_BICG_2, catt.K_ATAX_1) else prob.n
    n = prob.n
    A = torch.empty(m, n, device=dev); catt.fill_hash(A, 2)
    x = torch.empty(n, device=dev); catt.fill_hash(x, 102)
    y = torch.empty(m, device=dev)
    mode = catt.ROWS_ACCUM if prob.loop == catt.K_MVT_1 else catt.ROWS_STORE
    return lambda th: (lambda: catt.rows(A, x, y, mode, t=th))


def main():
    if "--predict" in sys.argv:
        for name, prob, launches in CASES:
            for cta, carve in launches:
                print(name, cta, carve, picks(prob, cta, carve))
        return
    reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 5
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
                       b200=pk["b200"], r29=pk["r29"], paper=pk["paper"], best=list(best),
                       best_ms=round(times[best], 4), full_ms=round(times[(W, T)], 4),
                       **{f"{k}_over_best": round(times[tuple(pk[k])] / times[best], 3) for k in ("b200", "r29", "paper")},
                       swept={f"{a},{m}": round(v, 4) for (a, m), v in times.items()})
            print(json.dumps({k: v for k, v in row.items() if k != "swept"}), flush=True)
            res.append(row)
    os.makedirs("gpurun_out/heldout10", exist_ok=True)
    json.dump(res, open("gpurun_out/heldout10/heldout10_study.json", "w"), indent=1)


if __name__ == "__main__":
    main()
