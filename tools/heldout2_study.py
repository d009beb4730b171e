"""Second held-out throttle study (after R23 was fixed): loops and launches
used neither to fit R18/R19 nor to choose R23's thresholds. For each launch:
every (a, m) of the literal loop, timed cold (L2 flushed: write + clean read),
median of `reps`; the picks of the B200 rule (R18+R19+R23), of R18 alone and
of the paper's rule are recorded BEFORE the timings (--predict prints them
without a GPU). Rows carry their problem, so tools/rule_replay.py can re-plan
them. Writes gpurun_out/heldout2_study.json.
usage: python tools/heldout2_study.py [--predict] [--set3|...|--set9]   (--set3: the third held-out set, after
R24; --set4: the fourth, testing the candidate R25; --set5: the fifth, new shapes; --set6: the sixth, testing
the candidate R26; --set7: the seventh, testing the candidate R27; --set8: the
eighth, R27 as adopted)"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

P = catt.problem
CASES = [
    # KM transpose (Rodinia invert_mapping) at other feature counts: trip 16 / 64 / 128 / 256
    ("kmeans transpose nf=16", P(catt.K_KMEANS_T, m=262144, n=16, ld=262144), "literal", [(256, 16), (256, 228), (1024, 196)]),
    ("kmeans transpose nf=64", P(catt.K_KMEANS_T, m=262144, n=64, ld=262144), "literal", [(256, 16), (256, 228), (1024, 196)]),
    ("kmeans transpose nf=128", P(catt.K_KMEANS_T, m=262144, n=128, ld=262144), "literal", [(256, 16), (256, 228), (1024, 196)]),
    ("kmeans transpose nf=256", P(catt.K_KMEANS_T, m=131072, n=256, ld=131072), "literal", [(256, 16), (1024, 196)]),
    # VEC4 row loops (8 re-touches per line) at launches not studied before
    ("mvt1 vec4", P(catt.K_MVT_1, n=4096), "vec4", [(1024, 228), (512, 196), (1024, 132)]),
    ("gesummv vec4", P(catt.K_GESUMMV, n=8192), "vec4", [(1024, 196), (256, 228)]),
    # scalar row loops with short rows: trip 96 (< 128) and 256
    ("bicg2 literal n=96", P(catt.K_BICG_2, m=262144, n=96), "literal", [(1024, 196), (1024, 228), (256, 228)]),
    ("bicg2 literal n=256", P(catt.K_BICG_2, m=131072, n=256), "literal", [(1024, 196), (1024, 228), (256, 228)]),
]

# Third held-out set (after R24 was fixed on the second): new shapes and launches
CASES3 = [
    ("kmeans transpose nf=34 512thr", P(catt.K_KMEANS_T, m=494020, n=34, ld=494020), "literal", [(512, 16), (512, 196)]),
    ("kmeans transpose nf=96", P(catt.K_KMEANS_T, m=262144, n=96, ld=262144), "literal", [(256, 100), (512, 228)]),
    ("atax1 literal n=192", P(catt.K_ATAX_1, m=131072, n=192), "literal", [(1024, 196), (512, 228)]),
    ("mvt1 literal n=2048", P(catt.K_MVT_1, n=2048), "literal", [(512, 196), (1024, 228)]),
    ("bicg2 literal n=512", P(catt.K_BICG_2, m=65536, n=512), "literal", [(512, 228), (1024, 132)]),
    ("bicg2 vec4 n=96", P(catt.K_BICG_2, m=262144, n=96), "vec4", [(1024, 196)]),
    ("syr2k literal 1024", P(catt.K_SYR2K, n=1024, k=1024), "literal", [(512, 196), (128, 228)]),
    ("syrk literal 1024", P(catt.K_SYRK, n=1024, k=1024), "literal", [(512, 228), (128, 164)]),
]

# Fourth held-out set (after R24; tests the candidate R25 before it enters the
# library): launches of 512- and 1024-thread CTAs where R25 (TLP floor of 16
# warps per SM for CTAs of >= 16 warps, 8 otherwise) and the library's rule
# pick differently, plus four where they agree
CASES4 = [
    ("gesummv literal 8192", P(catt.K_GESUMMV, n=8192), "literal", [(1024, 228), (512, 196), (512, 228), (512, 100)]),
    ("atax1 literal 65536x16384", P(catt.K_ATAX_1, m=65536, n=16384), "literal", [(512, 196), (1024, 228), (512, 228)]),
    ("mvt1 literal 8192", P(catt.K_MVT_1, n=8192), "literal", [(1024, 196), (1024, 228), (512, 228), (1024, 132)]),
    ("bicg2 literal m=131072 n=128", P(catt.K_BICG_2, m=131072, n=128), "literal", [(1024, 196), (512, 228), (1024, 164)]),
    ("bicg2 literal m=32768 n=1024", P(catt.K_BICG_2, m=32768, n=1024), "literal", [(1024, 228), (512, 196)]),
    ("syr2k literal 1024 wide", P(catt.K_SYR2K, n=1024, k=1024), "literal", [(1024, 228)]),
]

# Fifth held-out set (no rule change under test): loop shapes and launches of
# every literal family not studied before -- KMEANS assign at other feature /
# centre counts, CTAs of 384, 640 and 768 threads (W = 12, 20, 24: divisors
# that are not powers of two), other matrix sizes -- to check that the
# library's rule generalises
CASES5 = [
    ("kmeans assign nf=16 k=8", P(catt.K_KMEANS, m=262144, n=16, k=8, ld=262144), "literal", [(256, 100), (512, 228)]),
    ("kmeans assign nf=64 k=4", P(catt.K_KMEANS, m=131072, n=64, k=4, ld=131072), "literal", [(256, 32), (1024, 196)]),
    ("atax1 literal 32768x2048", P(catt.K_ATAX_1, m=32768, n=2048), "literal", [(256, 196), (768, 228)]),
    ("gesummv literal 4096", P(catt.K_GESUMMV, n=4096), "literal", [(384, 196), (1024, 100)]),
    ("mvt1 literal 6000", P(catt.K_MVT_1, n=6000), "literal", [(512, 164), (256, 132)]),
    ("syrk literal 1536", P(catt.K_SYRK, n=1536, k=1536), "literal", [(256, 196), (1024, 100)]),
    ("syr2k literal 768", P(catt.K_SYR2K, n=768, k=768), "literal", [(256, 228)]),
    ("bicg2 literal m=65536 n=384", P(catt.K_BICG_2, m=65536, n=384), "literal", [(640, 196)]),
    ("kmeans transpose nf=48", P(catt.K_KMEANS_T, m=262144, n=48, ld=262144), "literal", [(256, 64), (384, 228)]),
]

# Sixth held-out set: tests the candidate R26 (the TLP floor is the largest
# warp count per SM not above 8 that the launch can reach, a | W times m <= T;
# the library's floor of 8 rounds up to W when W = 12, 20 or 28), at CTAs of
# 384, 640, 768 and 896 threads; six launches where the two rules differ and
# six where they agree
CASES6 = [
    ("gesummv literal 4096", P(catt.K_GESUMMV, n=4096), "literal", [(384, 228), (384, 132)]),
    ("atax1 literal 65536x2048", P(catt.K_ATAX_1, m=65536, n=2048), "literal", [(384, 196), (384, 228)]),
    ("mvt1 literal 6000 w12", P(catt.K_MVT_1, n=6000), "literal", [(384, 196)]),
    ("bicg2 literal m=65536 n=1024", P(catt.K_BICG_2, m=65536, n=1024), "literal", [(640, 228)]),
    ("gesummv literal 8192 w20", P(catt.K_GESUMMV, n=8192), "literal", [(640, 196), (384, 196)]),
    ("atax1 literal 32768x2048 w24", P(catt.K_ATAX_1, m=32768, n=2048), "literal", [(768, 196)]),
    ("mvt1 literal 8192 w28", P(catt.K_MVT_1, n=8192), "literal", [(896, 196), (896, 228)]),
    ("bicg2 literal m=131072 n=128 w12", P(catt.K_BICG_2, m=131072, n=128), "literal", [(384, 228)]),
]

# Seventh held-out set: tests the candidate R27 (in the floor fallback -- no
# pair at or above the TLP floor fits -- cap whole CTAs, (W, m) with the
# smallest m such that floor <= W m <= 2 floor, when such an m exists, instead
# of gating warps down to the floor), fitted on stored sweeps where it changed
# 10 picks and lost none; new shapes at 320- to 512-thread CTAs
CASES7 = [
    ("gesummv literal 6144", P(catt.K_GESUMMV, n=6144), "literal", [(512, 228), (512, 196), (320, 196)]),
    ("mvt1 literal 5120", P(catt.K_MVT_1, n=5120), "literal", [(512, 228), (512, 196)]),
    ("atax1 literal 131072x1024", P(catt.K_ATAX_1, m=131072, n=1024), "literal", [(384, 228), (512, 228), (384, 196)]),
    ("bicg2 literal m=98304 n=768", P(catt.K_BICG_2, m=98304, n=768), "literal", [(512, 228), (1024, 196)]),
    ("atax1 literal 49152x4096", P(catt.K_ATAX_1, m=49152, n=4096), "literal", [(512, 228), (320, 228)]),
    ("bicg2 literal m=131072 n=256 w12", P(catt.K_BICG_2, m=131072, n=256), "literal", [(384, 228)]),
]

# Eighth held-out set: the library's rule (with R27 for T >= 2) against the
# same rule without R27, on launches with several CTAs per SM where the floor
# fallback applies and W = 12 or 16 (the only CTA sizes where the two differ
# under the 8-warp floor); recorded before measuring
CASES8 = [
    ("bicg2 literal m=163840 n=512", P(catt.K_BICG_2, m=163840, n=512), "literal", [(512, 228), (384, 228)]),
    ("bicg2 literal m=131072 n=512 w12", P(catt.K_BICG_2, m=131072, n=512), "literal", [(384, 196), (384, 228)]),
    ("atax1 literal 196608x256", P(catt.K_ATAX_1, m=196608, n=256), "literal", [(512, 196), (384, 228), (512, 228)]),
    ("bicg2 literal m=262144 n=128", P(catt.K_BICG_2, m=262144, n=128), "literal", [(512, 164), (512, 228)]),
    ("atax1 literal 131072x640", P(catt.K_ATAX_1, m=131072, n=640), "literal", [(512, 196), (512, 228)]),
    ("bicg2 literal m=98304 n=1024 w12", P(catt.K_BICG_2, m=98304, n=1024), "literal", [(384, 228)]),
]

# Ninth held-out set: tests the candidate R28 (one CTA per SM, 8 < W < 16, W
# even: the TLP floor becomes W / 2 instead of rounding up to W -- the W = 12
# misses of held-out sets 5 and 6, where 6 warps were best) at CTAs of 320,
# 384 and 448 threads (W = 10, 12, 14)
CASES9 = [
    ("gesummv literal 6144 w10", P(catt.K_GESUMMV, n=6144), "literal", [(320, 228)]),
    ("mvt1 literal 8192 w10", P(catt.K_MVT_1, n=8192), "literal", [(320, 196)]),
    ("atax1 literal 16384x4096 w10", P(catt.K_ATAX_1, m=16384, n=4096), "literal", [(320, 228)]),
    ("bicg2 literal m=32768 n=2048 w10", P(catt.K_BICG_2, m=32768, n=2048), "literal", [(320, 196)]),
    ("gesummv literal 6144 w12", P(catt.K_GESUMMV, n=6144), "literal", [(384, 196)]),
    ("mvt1 literal 8192 w12", P(catt.K_MVT_1, n=8192), "literal", [(384, 228)]),
    ("bicg2 literal m=40960 n=1024 w12", P(catt.K_BICG_2, m=40960, n=1024), "literal", [(384, 196)]),
    ("gesummv literal 6144 w14", P(catt.K_GESUMMV, n=6144), "literal", [(448, 228)]),
    ("atax1 literal 32768x1024 w14", P(catt.K_ATAX_1, m=32768, n=1024), "literal", [(448, 196)]),
    ("mvt1 literal 6000 w14", P(catt.K_MVT_1, n=6000), "literal", [(448, 228)]),
]


def r28_pick(prob, launch, hw):
    """The library's rule with R28 (see CASES9)."""
    t, r = catt.plan(prob, launch, hw)
    W, T = r["base_warps"], r["base_ctas"]
    if T == 1 and 8 < W < 16 and W % 2 == 0:
        h = catt.Hw.from_dict(hw.as_dict())
        h.min_warps_sm = W // 2
        t, r = catt.plan(prob, launch, h)
    return [t.active_warps or W, t.active_ctas or T]


def r27_pick(prob, launch, hw):
    """R27 applied to the library's pick (see CASES7)."""
    t, r = catt.plan(prob, launch, hw)
    W, T = r["base_warps"], r["base_ctas"]
    pick = [t.active_warps or W, t.active_ctas or T]
    if (r["flags"] & catt.FIT_GUARDED) and pick != [W, T] and r["footprint_bytes"] > r["l1d_bytes"]:
        floor = hw.min_warps_sm
        ms = [m for m in range(1, T + 1) if floor <= W * m <= 2 * floor]
        if ms:
            pick = [W, min(ms)]
    return pick


def r26_floor(W, T):
    """R26's TLP floor: the largest a * m <= 8 with a | W and m <= T."""
    return max(a * m for a in range(1, W + 1) if W % a == 0 for m in range(1, T + 1) if a * m <= 8)


def picks(prob, var, cta, carve):
    b200 = catt.hw_query() if catt_gpu() else catt.hw_b200()
    r18 = catt.Hw.from_dict(b200.as_dict())
    r18.min_retouch, r18.min_reuse_trip, r18.max_stream_pct = 0, 0, 0
    r23 = catt.Hw.from_dict(r18.as_dict())
    r23.min_retouch, r23.min_reuse_trip = 16, 128
    out = {}
    r25 = catt.Hw.from_dict(b200.as_dict())
    r25.min_warps_sm = 16 if cta // 32 >= 16 else 8
    r24 = catt.Hw.from_dict(b200.as_dict())
    r24.cta_fallback = 0
    r26 = catt.Hw.from_dict(b200.as_dict())
    _, base = catt.plan(prob, catt.Throttle(cta_threads=cta, carveout_kb=carve, variant=var), b200)
    r26.min_warps_sm = r26_floor(base["base_warps"], base["base_ctas"])
    for name, hw in (("b200", b200), ("r23", r23), ("r18", r18), ("paper", catt.paper_rule(b200)), ("r25", r25),
                     ("r26", r26), ("r24", r24)):
        launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant=var)
        t, r = catt.plan(prob, launch, hw)
        W, T = r["base_warps"], r["base_ctas"]
        out[name] = [t.active_warps or W, t.active_ctas or T]
        out["base"], out["carveout_kb"] = [W, T], r["carveout_kb"]
        out["footprint"], out["l1d_lines"] = r["footprint_lines_full"], r["l1d_bytes"] // 128
    out["r27"] = r27_pick(prob, catt.Throttle(cta_threads=cta, carveout_kb=carve, variant=var), b200)
    out["r28"] = r28_pick(prob, catt.Throttle(cta_threads=cta, carveout_kb=carve, variant=var), b200)
    return out


def catt_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def main():
    predict = "--predict" in sys.argv
    third = "--set3" in sys.argv
    fourth = "--set4" in sys.argv
    fifth = "--set5" in sys.argv
    sixth = "--set6" in sys.argv
    seventh = "--set7" in sys.argv
    eighth = "--set8" in sys.argv
    ninth = "--set9" in sys.argv
    cases = CASES9 if ninth else CASES8 if eighth else CASES7 if seventh else CASES6 if sixth else CASES5 if fifth else CASES4 if fourth else CASES3 if third else CASES
    if predict:
        for name, prob, var, launches in cases:
            for cta, carve in launches:
                print(name, cta, carve, picks(prob, var, cta, carve))
        return
    import torch
    dev = torch.device("cuda")
    flush_buf = torch.empty(64 * 1024 * 1024, dtype=torch.int32, device=dev)
    clean_buf = torch.zeros(64 * 1024 * 1024, dtype=torch.int32, device=dev)

    def med(fn, reps):
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
    for name, prob, var, launches in cases:
        if prob.loop == catt.K_KMEANS:
            npts, nf, ld, kc = prob.m, prob.n, prob.ld, prob.k
            fm = torch.empty(nf * ld, device=dev)
            catt.fill_hash(fm, 44)
            cl = fm.view(nf, ld)[:, :kc].t().contiguous()          # centres = the first k points
            memb = torch.empty(npts, dtype=torch.int32, device=dev)
            make = lambda th: (lambda: catt.kmeans_assign(fm, ld, npts, nf, cl, memb, t=th))
        elif prob.loop == catt.K_KMEANS_T:
            npts, nf, ld = prob.m, prob.n, prob.ld
            pm = torch.empty(npts * nf, device=dev)
            catt.fill_hash(pm, 41)
            fm = torch.empty(nf * ld, device=dev)
            make = lambda th: (lambda: catt.kmeans_transpose(pm, npts, nf, fm, ld, t=th))
        elif prob.loop in (catt.K_SYRK, catt.K_SYR2K):
            n = prob.n
            A = torch.empty(n, n, device=dev); catt.fill_hash(A, 6)
            B2 = torch.empty(n, n, device=dev); catt.fill_hash(B2, 8)
            C = torch.empty(n, n, device=dev); catt.fill_hash(C, 106)
            if prob.loop == catt.K_SYRK:
                make = lambda th: (lambda: catt.syrk(A, C, 1.5, 1.2, t=th))
            else:
                make = lambda th: (lambda: catt.syr2k(A, B2, C, 1.5, 1.2, t=th))
        elif prob.loop == catt.K_GESUMMV:
            n = prob.n
            A = torch.empty(n, n, device=dev); catt.fill_hash(A, 5)
            B = torch.empty(n, n, device=dev); catt.fill_hash(B, 105)
            x = torch.empty(n, device=dev); catt.fill_hash(x, 205)
            y, tmp = torch.empty(n, device=dev), torch.empty(n, device=dev)
            make = lambda th: (lambda: catt.rows(A, x, y, catt.ROWS_GESUMMV, B=B, tmp=tmp, alpha=1.5, beta=1.2, t=th))
        else:
            m = prob.m if prob.loop in (catt.K_BICG_2, catt.K_ATAX_1) else prob.n
            n = prob.n
            A = torch.empty(m, n, device=dev); catt.fill_hash(A, 2)
            x = torch.empty(n, device=dev); catt.fill_hash(x, 102)
            y = torch.empty(m, device=dev)
            mode = catt.ROWS_ACCUM if prob.loop == catt.K_MVT_1 else catt.ROWS_STORE
            make = lambda th: (lambda: catt.rows(A, x, y, mode, t=th))
        for cta, carve in launches:
            pk = picks(prob, var, cta, carve)
            W, T = pk["base"]
            launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant=var)
            times = {}
            for a in [d for d in range(W, 0, -1) if W % d == 0]:
                for m in range(T, 0, -1):
                    th = launch.copy(active_warps=a, active_ctas=m if m < T else 0)
                    times[(a, m)] = med(make(th), 3)
            best = min(times, key=times.get)
            row = dict(loop=name, prob=dict(loop=prob.loop, m=prob.m, n=prob.n, k=prob.k, ld=prob.ld), variant=var,
                       cta=cta, carveout_kb=carve, base=[W, T], footprint=pk["footprint"], l1d_lines=pk["l1d_lines"],
                       b200=pk["b200"], r23=pk["r23"], r18=pk["r18"], paper=pk["paper"], best=list(best),
                       best_ms=round(times[best], 4), full_ms=round(times[(W, T)], 4),
                       **{f"{k}_over_best": round(times[tuple(pk[k])] / times[best], 3)
                          for k in ("b200", "r23", "r18", "paper", "r25", "r26", "r27", "r24", "r28")},
                       r25=pk["r25"], r26=pk["r26"], r27=pk["r27"], r24=pk["r24"], r28=pk["r28"],
                       swept={f"{a},{m}": round(v, 4) for (a, m), v in times.items()})
            print(json.dumps({k: v for k, v in row.items() if k != "swept"}), flush=True)
            res.append(row)
    os.makedirs("gpurun_out", exist_ok=True)
    out = "heldout9" if ninth else "heldout8" if eighth else "heldout7" if seventh else "heldout6" if sixth else "heldout5" if fifth else "heldout4" if fourth else "heldout3" if third else "heldout2"
    json.dump(res, open(f"gpurun_out/{out}_study.json", "w"), indent=1)


if __name__ == "__main__":
    main()
