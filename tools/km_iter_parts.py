"""Where the one-launch k-means iteration's time goes (KMEANS 494020 x 34,
k = 5, the bench shape): CUDA-event time per launch, cold L2 as bench.py, of
  assign       catt_kmeans_assign (STAGED): the distances and the argmin only
  accumulate   catt_kmeans_accumulate: + the exact sums into acc (no rounding)
  step         catt_kmeans_step: + the last CTA's rounding of the new centres
The centres and memberships are restored before every timed launch.
usage: python tools/km_iter_parts.py [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 30
npts, nf, k, ld = 494020, 34, 5, 494020
feat = torch.empty(nf * ld, device="cuda")
catt.fill_hash(feat, 4)
cl0 = feat.view(nf, ld)[:, :k].t().contiguous()
cl = cl0.clone()
memb = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
acc = torch.zeros(catt.kmeans_acc_words(k, nf), dtype=torch.int64, device="cuda")
fl, cb = torch.empty(64 << 20, dtype=torch.int32, device="cuda"), torch.zeros(64 << 20, dtype=torch.int32, device="cuda")


def timed(name, fn):
    ts = []
    for r in range(reps + 3):
        cl.copy_(cl0)
        memb.fill_(-1)
        acc.zero_()
        fl.zero_()
        cb.sum()
        torch.cuda._sleep(400_000)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        if r >= 3:
            ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    print(f"{name:12s} median {ts[len(ts) // 2]:7.2f} us  min {ts[0]:7.2f}", flush=True)


timed("assign", lambda: catt.kmeans_assign(feat, ld, npts, nf, cl, memb, t=catt.Throttle(variant="staged")))
timed("accumulate", lambda: catt.kmeans_accumulate(feat, ld, npts, nf, cl, memb, acc))
timed("step", lambda: catt.kmeans_step(feat, ld, npts, nf, cl, memb, acc))
timed("acc+final", lambda: (catt.kmeans_accumulate(feat, ld, npts, nf, cl, memb, acc), catt.kmeans_finalize(acc, cl)))
