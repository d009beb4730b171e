"""Fused single-read BICG+MVT 4096^2 (the bicg_mvt bench step) under the
library's tuning knobs: CUDA-event time after the bench's L2 flush (median of
reps) and the per-CTA phase stamps (catt_fused_trace), one line per config.
usage: python tools/fused_sweep.py [n] [reps]"""
import os
import statistics
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 15
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
nbytes = 2 * n * n * 4 + 4 * 10 * n
CONFIGS = [("default", {}), ("stage16", {"CATT_FUSED_STAGE_KB": "16"}), ("stage32", {"CATT_FUSED_STAGE_KB": "32"}),
           ("stage128", {"CATT_FUSED_STAGE_KB": "128"}), ("smem160", {"CATT_FUSED_SMEM_KB": "160"}),
           ("bands", {"CATT_FUSED_INTERLEAVE": "0"}), ("barrier1", {"CATT_FUSED_BARRIER": "1"}),
           ("noredpf", {"CATT_FUSED_REDPF": "0"})]
only = os.environ.get("SWEEP_ONLY")
names = ["first stage", "stream end", "partials", "barrier", "end"]


def flush():
    fl.zero_()
    cl.sum()
    torch.cuda._sleep(400_000)


for name, env in CONFIGS:
    if only and name not in only.split(","):
        continue
    for k in ("CATT_FUSED_STAGE_KB", "CATT_FUSED_SMEM_KB", "CATT_FUSED_INTERLEAVE", "CATT_FUSED_BARRIER",
              "CATT_FUSED_REDPF", "CATT_FUSED_TRACE"):
        os.environ.pop(k, None)
    os.environ.update(env)
    ts = []
    for r in range(reps + 2):
        flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        catt.dual_group(group)
        e1.record()
        torch.cuda.synchronize()
        if r >= 2:
            ts.append(e0.elapsed_time(e1) * 1e3)
    med = statistics.median(ts)
    os.environ["CATT_FUSED_TRACE"] = "1"
    phases = []
    for r in range(6):
        flush()
        catt.dual_group(group)
        torch.cuda.synchronize()
        tr = catt.fused_trace(148).astype(np.int64)
        tr = tr[tr[:, 0] > 0]
        rel = (tr - tr[:, 0].min()) / 1e3
        if r:
            phases.append([rel[:, 0].max()] + [np.median(rel[:, k]) for k in range(1, 6)] + [rel[:, 5].max()])
    ph = np.median(np.array(phases), axis=0)
    print(f"{name:10s} event {med:6.1f} us ({nbytes / med / 1e3:6.0f} GB/s) | start spread {ph[0]:4.1f} | " +
          " | ".join(f"{nm} {ph[k + 1]:5.1f}" for k, nm in enumerate(names)) + f" | last end {ph[6]:5.1f}", flush=True)
