"""Does the relative placement of GESUMMV's A and B rows matter at a launch
the footprint model calls uncontended (GESUMMV 4096, 384-thread CTAs, 132 KB
carveout: 769 lines at full TLP vs 944 L1D lines, yet 6 of 12 warps ran 1.21x
faster, held-out 6)? B is placed at several byte offsets after A in one
allocation; full TLP and (6, 1) are timed warm (median of 7)."""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

n = 4096
x = torch.empty(n, device="cuda")
catt.fill_hash(x, 205)
y, tmp = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
buf = torch.empty(2 * n * n + (1 << 20), device="cuda")
catt.fill_hash(buf, 5)
A = buf[:n * n].view(n, n)


def t_of(fn):
    ts = []
    for r in range(8):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        if r:
            ts.append(a.elapsed_time(b))
    return statistics.median(ts)


for cta, carve in ((384, 132), (384, 228), (256, 132)):
    for off_bytes in (0, 128, 256, 1024, 4096, 32768, 65536, 4096 + 128):
        o = n * n + off_bytes // 4
        B = buf[o:o + n * n].view(n, n)
        res = []
        W = cta // 32
        for a in (W, W // 2):
            th = catt.Throttle(cta_threads=cta, carveout_kb=carve, active_warps=a)
            res.append(t_of(lambda: catt.rows(A, x, y, catt.ROWS_GESUMMV, B=B, tmp=tmp, alpha=1.5, beta=1.2, t=th)))
        print(f"cta {cta} carve {carve} B offset {off_bytes:6d} B: full {res[0]:.3f} ms  half warps {res[1]:.3f} ms  "
              f"full/half {res[0] / res[1]:.3f}", flush=True)
