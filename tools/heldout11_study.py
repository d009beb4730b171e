"""Held-out study 11 (round 2): tests the candidate R32 -- a memory-divergent
reused load whose lines every warp of the CTA requests as well (SYRK's and
SYR2K's a[j][k] / b[j][k] in a 2-D block: the warps differ in i, the lanes in
j) counts neither as divergent nor as a stream. On the stored sweeps no
throttle ever beat full TLP by more than 5 % on a 2-D block loop, and the
library's rule loses 1.17x (SYR2K 2048, 228 KB) and 1.06x (SYR2K 768) there.
New launches only (none of the 178 stored sweeps): SYRK and SYR2K at shapes,
CTA sizes (2-D blocks 32 x 4 .. 32 x 32) and carveouts not measured before,
chosen where the two rules pick differently, plus 1-stream row controls
where R32 must not act.

For each launch: every (a, m) of the literal loop, timed cold (L2 flushed,
then a GPU sleep so enqueue cost stays out of the events), median of `reps`.
The picks of the library's rule, of the rule with R32 and of the paper's
Eq 9 are written BEFORE any timing (--predict prints them without a GPU; the
committed predictions file is that output). Adoption rule:
geomean better and worst case no worse on this set.
usage: python tools/heldout11_study.py [--predict] [--reps R]
Writes gpurun_out/heldout11/heldout11_study.json."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

P = catt.problem
# (name, problem, [(CTA threads, carveout KB)])
CASES = [
    ("syrk literal 3072", P(catt.K_SYRK, n=3072, k=3072), [(256, 228), (128, 196)]),
    ("syrk literal 2048x512", P(catt.K_SYRK, n=2048, k=512), [(256, 228), (512, 228), (128, 228)]),
    ("syrk literal 1280", P(catt.K_SYRK, n=1280, k=1280), [(128, 228), (512, 228)]),
    ("syr2k literal 1536", P(catt.K_SYR2K, n=1536, k=1536), [(256, 228), (128, 196), (512, 228)]),
    ("syr2k literal 2048x768", P(catt.K_SYR2K, n=2048, k=768), [(256, 196), (1024, 228), (128, 132)]),
    ("syr2k literal 2560", P(catt.K_SYR2K, n=2560, k=2560), [(256, 228), (128, 164)]),
    # 1-stream row controls (lanes are rows: nothing is CTA-shared, R32 must not act)
    ("bicg2 literal m=12288 n=2048", P(catt.K_BICG_2, m=12288, n=2048), [(1024, 196), (512, 228)]),
]


def picks(prob, cta, carve):
    hw = catt.hw_b200()
    launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant="literal")
    out = {}
    for name in ("b200", "r32", "paper"):
        h = catt.Hw.from_dict(hw.as_dict())
        if name == "r32":
            h.private_streams = 1
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
    if prob.loop in (catt.K_SYRK, catt.K_SYR2K):
        n, k = prob.n, prob.k
        A = torch.empty(n, k, device=dev); catt.fill_hash(A, 6)
        B = torch.empty(n, k, device=dev); catt.fill_hash(B, 8)
        C = torch.empty(n, n, device=dev); catt.fill_hash(C, 106)
        if prob.loop == catt.K_SYRK:
            return lambda th: (lambda: catt.syrk(A, C, 1.5, 1.2, t=th))
        return lambda th: (lambda: catt.syr2k(A, B, C, 1.5, 1.2, t=th))
    m, n = prob.m, prob.n
    A = torch.empty(m, n, device=dev); catt.fill_hash(A, 2)
    x = torch.empty(n, device=dev); catt.fill_hash(x, 102)
    y = torch.empty(m, device=dev)
    return lambda th: (lambda: catt.rows(A, x, y, catt.ROWS_STORE, t=th))


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
                       b200=pk["b200"], r32=pk["r32"], paper=pk["paper"], best=list(best),
                       best_ms=round(times[best], 4), full_ms=round(times[(W, T)], 4),
                       **{f"{k}_over_best": round(times[tuple(pk[k])] / times[best], 3) for k in ("b200", "r32", "paper")},
                       swept={f"{a},{m}": round(v, 4) for (a, m), v in times.items()})
            print(json.dumps({k: v for k, v in row.items() if k != "swept"}), flush=True)
            res.append(row)
    os.makedirs("gpurun_out/heldout11", exist_ok=True)
    json.dump(res, open("gpurun_out/heldout11/heldout11_study.json", "w"), indent=1)


if __name__ == "__main__":
    main()
