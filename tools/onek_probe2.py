"""Loop-1 time per CTA (residency probe, warm) of the standalone literal row
kernel (catt.rows) and of the one-kernel ATAX (catt_atax_onekernel) at several
launches: is the one-kernel form's faster loop 1 an L1 effect?"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

n = 4096
A = torch.empty(n, n, device="cuda")
catt.fill_hash(A, 1)
x = torch.ones(n, device="cuda")
y = torch.empty(n, device="cuda")
for cta, carve, aw in ((1024, 196, 0), (1024, 196, 8), (1024, 0, 0), (1024, 228, 0), (256, 228, 0), (256, 0, 0)):
    ncta, W = n // cta, cta // 32
    res = {}
    for name in ("rows", "onekernel"):
        ts = []
        for rep in range(4):
            pr = torch.zeros(ncta * W * 3, dtype=torch.int64, device="cuda")
            t = catt.Throttle(cta_threads=cta, carveout_kb=carve, active_warps=aw, probe=pr.data_ptr())
            if name == "rows":
                catt.rows(A, x, y, catt.ROWS_STORE, t=t)
            else:
                catt.atax_onekernel(A, x, k1=t)
            torch.cuda.synchronize()
            rec = pr.cpu().numpy().reshape(ncta, W, 3)
            if rep:
                ts.append(np.median([(rec[c, :, 2].max() - rec[c, :, 1].min()) / 1e6 for c in range(ncta)]))
        res[name] = round(float(np.median(ts)), 3)
    print(f"cta {cta} carve {carve} warps {aw or W}: loop-1 ms per CTA  rows {res['rows']}  onekernel {res['onekernel']}  "
          f"ratio {res['rows'] / res['onekernel']:.3f}", flush=True)
