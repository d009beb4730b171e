"""KMEANS assign at the Rodinia shape: CUDA-event time per launch (cold L2,
as bench.py) of each variant x carveout preference.
usage: python tools/km_variants.py [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 30
npts, nf, k, ld = 494020, 34, 5, 494020
feat = torch.empty(nf * ld, device="cuda")
catt.fill_hash(feat, 4)
cl = feat.view(nf, ld)[:, :k].t().contiguous()
memb = torch.empty(npts, dtype=torch.int32, device="cuda")
ref = catt.kmeans_assign(feat, ld, npts, nf, cl, t=catt.Throttle(variant="regs")).clone()
fl, cb = torch.empty(64 << 20, dtype=torch.int32, device="cuda"), torch.zeros(64 << 20, dtype=torch.int32, device="cuda")
for var in ("staged", "coop", "regs"):
    for carve in (16, 0, -1, 100, 228):
        t = catt.Throttle(cta_threads=256, variant=var, carveout_kb=carve)
        ts = []
        for r in range(reps + 3):
            fl.zero_()
            cb.sum()
            torch.cuda._sleep(400_000)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            catt.kmeans_assign(feat, ld, npts, nf, cl, memb, t=t)
            e1.record()
            torch.cuda.synchronize()
            if r >= 3:
                ts.append(e0.elapsed_time(e1) * 1e3)
        ok = bool(torch.equal(memb, ref))
        print(f"{var:7s} carveout {carve:4d}: mean {sum(ts) / len(ts):6.2f} us  min {min(ts):6.2f}  exact {ok}", flush=True)
