"""Held-out throttle study: loops / launches NOT used to choose the B200 rule
(R18, R19). For each: every (a, m), the CATT pick under the paper rule and the
B200 rule, full TLP, best swept. L2 flushed (write + clean read) before each
timed launch; median of `reps`. Writes gpurun_out/heldout_study.json."""
import json
import statistics
import sys

import torch

import paper_conf_icpp_kimhlsh19_b200 as catt

dev = torch.device("cuda")
flush_buf = torch.empty(64 * 1024 * 1024, dtype=torch.int32, device=dev)
clean_buf = torch.zeros(64 * 1024 * 1024, dtype=torch.int32, device=dev)
hw = catt.hw_query()
paper = catt.paper_rule(hw)


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


def study(name, prob, launches, make_fn, reps=3):
    out = []
    for cta, carve in launches:
        launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant="literal")
        t, r = catt.plan(prob, launch, hw)
        tp, rp = catt.plan(prob, launch, paper)
        W, T = r["base_warps"], r["base_ctas"]
        times = {}
        for a in [d for d in range(W, 0, -1) if W % d == 0]:
            for m in range(T, 0, -1):
                th = launch.copy(active_warps=a, active_ctas=m if m < T else 0)
                times[(a, m)] = med(make_fn(th), reps)
        pick = (t.active_warps or W, t.active_ctas or T)
        pp = (tp.active_warps or W, tp.active_ctas or T)
        best = min(times, key=times.get)
        row = dict(loop=name, cta=cta, carveout_kb=r["carveout_kb"], base=[W, T],
                   footprint=r["footprint_lines_full"], l1d_lines=r["l1d_bytes"] // 128,
                   b200=list(pick), b200_over_best=round(times[pick] / times[best], 3),
                   b200_over_full=round(times[pick] / times[(W, T)], 3),
                   paper=list(pp), paper_over_best=round(times[pp] / times[best], 3),
                   best=list(best), best_ms=round(times[best], 4), full_ms=round(times[(W, T)], 4),
                   swept={f"{a},{m}": round(v, 4) for (a, m), v in times.items()})
        print(json.dumps({k: v for k, v in row.items() if k != "swept"}), flush=True)
        out.append(row)
    return out


res = []
# SYRK 2048 literal: 2-D CTAs (32 x BY)
n = 2048
A = torch.empty(n, n, device=dev); catt.fill_hash(A, 6)
C = torch.empty(n, n, device=dev); catt.fill_hash(C, 106)
res += study("syrk2048 literal", catt.problem(catt.K_SYRK, n=n, k=n), [(256, 0), (256, 228), (1024, 196)],
             lambda th: (lambda: catt.syrk(A, C, 1.5, 1.2, t=th)), reps=2)
# row loops at CTA sizes not in the fitting set
n = 4096
B = torch.empty(n, n, device=dev); catt.fill_hash(B, 2)
x = torch.rand(n, device=dev); y = torch.empty(n, device=dev)
res += study("mvt1 literal", catt.problem(catt.K_MVT_1, n=n), [(512, 100), (512, 196), (512, 228), (128, 228)],
             lambda th: (lambda: catt.rows(B, x, y, catt.ROWS_ACCUM, t=th)))
res += study("bicg2 vec4", catt.problem(catt.K_BICG_2, m=n, n=n), [(1024, 196)],
             lambda th: (lambda: catt.rows(B, x, y, t=th.copy(variant=catt.VAR_VEC4))))
# KMEANS with the padded leading dimension, 512-thread CTAs
npts, nf, k, ld = 494020, 34, 5, 494048
feat = torch.empty(nf * ld, device=dev); catt.fill_hash(feat, 4)
cl = feat.view(nf, ld)[:, :k].t().contiguous()
memb = torch.empty(npts, dtype=torch.int32, device=dev)
res += study("kmeans ld=494048", catt.problem(catt.K_KMEANS, m=npts, n=nf, k=k, ld=ld), [(512, 100), (128, 228)],
             lambda th: (lambda: catt.kmeans_assign(feat, ld, npts, nf, cl, memb, t=th)))
json.dump(res, open("gpurun_out/heldout_study.json", "w"), indent=1)
