"""Held-out study 14 (round 2, last session): a third out-of-sample check of
the final library rule (R18 ... R29, R32), no rule change under test. New
launches only (none of the 229 stored sweeps): every loop family at shapes,
CTA sizes and carveouts not measured before. The picks of the library's rule
and of the paper's Eq 9 are written BEFORE any timing (--predict prints them
without a GPU; profiles/r2/heldout14/heldout14_predictions.txt is that output,
committed before the measuring run). Timing as held-out study 12 (every
(a, m) of the literal loop, cold L2, GPU sleep, median of `reps`).
usage: python tools/heldout14_study.py [--predict] [--reps R]
Writes gpurun_out/heldout14/heldout14_study.json."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402
from heldout12_study import make_fn, picks  # noqa: E402

P = catt.problem
CASES = [
    ("atax1 literal 98304x1536", P(catt.K_ATAX_1, m=98304, n=1536), [(384, 196), (1024, 132)]),
    ("bicg2 literal m=40960 n=3072", P(catt.K_BICG_2, m=40960, n=3072), [(512, 164)]),
    ("bicg2 literal m=24576 n=2048", P(catt.K_BICG_2, m=24576, n=2048), [(768, 228)]),
    ("mvt1 literal 5632", P(catt.K_MVT_1, n=5632), [(768, 164)]),
    ("gesummv literal 6656", P(catt.K_GESUMMV, n=6656), [(256, 164), (1024, 228)]),
    ("gesummv literal 10240", P(catt.K_GESUMMV, n=10240), [(512, 100)]),
    ("rows3 literal 10240x2560", P(catt.K_ROWS3, m=10240, n=2560), [(512, 132)]),
    ("syrk literal 2816x1024", P(catt.K_SYRK, n=2816, k=1024), [(512, 196)]),
    ("syr2k literal 2560x768", P(catt.K_SYR2K, n=2560, k=768), [(128, 228)]),
    ("kmeans assign 300000x28 k=4", P(catt.K_KMEANS, m=300000, n=28, k=4, ld=300000), [(512, 196)]),
    ("kmeans transpose 250000x24", P(catt.K_KMEANS_T, m=250000, n=24, ld=250000), [(384, 100)]),
    ("gemm literal 896", P(catt.K_GEMM, m=896, n=896, k=896), [(128, 164)]),
]
OUT = "gpurun_out/heldout14"


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
            os.makedirs(OUT, exist_ok=True)
            json.dump(res, open(os.path.join(OUT, "heldout14_study.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
