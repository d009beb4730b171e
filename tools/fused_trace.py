"""Where the FUSED single-read BICG+MVT launch spends its time: per-CTA
%globaltimer stamps (catt_fused_trace) after a cold-L2 flush, as in bench.py.
usage: CATT_FUSED_TRACE=1 python tools/fused_trace.py [n] [reps]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("CATT_FUSED_TRACE", "1")
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
T = lambda k: torch.empty(k, device="cuda")
Ab, Am = T(n * n).view(n, n), T(n * n).view(n, n)
catt.fill_hash(Ab, 2)
catt.fill_hash(Am, 3)
v = [T(n) for _ in range(8)]
for i, t in enumerate(v):
    catt.fill_hash(t, 200 + i)
group = [dict(A=Ab, xr=v[0], xc=v[1], yr=v[2], yc=v[3]),
         dict(A=Am, xr=v[4], xc=v[5], yr=v[6], yc=v[7], row_accumulate=True, col_accumulate=True)]
fl, cl = torch.empty(64 << 20, dtype=torch.int32, device="cuda"), torch.zeros(64 << 20, dtype=torch.int32, device="cuda")
names = ["first stage", "stream end", "partials", "barrier", "end"]
for r in range(reps + 1):
    fl.zero_()
    cl.sum()
    torch.cuda._sleep(400_000)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    catt.dual_group(group)
    e1.record()
    torch.cuda.synchronize()
    tr = catt.fused_trace(148).astype(np.int64)
    tr = tr[tr[:, 0] > 0]
    t0 = tr[:, 0].min()
    rel = (tr - t0) / 1e3
    if r == 0:
        continue
    line = f"event {e0.elapsed_time(e1) * 1e3:7.1f} us | start spread {rel[:, 0].max():5.1f}"
    for k, nm in enumerate(names, 1):
        line += f" | {nm} med {np.median(rel[:, k]):6.1f} max {rel[:, k].max():6.1f}"
    print(line, flush=True)
