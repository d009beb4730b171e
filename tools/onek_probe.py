"""One launch each of the literal ATAX row loop (catt_atax) and the one-kernel
ATAX (catt_atax_onekernel) at (1024 threads, 196 KB carveout), for an ncu
launch-statistics check of the shared-memory configuration the driver chose."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

n = 4096
A = torch.empty(n, n, device="cuda")
catt.fill_hash(A, 1)
x = torch.ones(n, device="cuda")
L = catt.Throttle(cta_threads=1024, carveout_kb=196)
for a in (32, 8):
    catt.atax(A, x, k1=L.copy(active_warps=a), k2=catt.Throttle(cta_threads=1024, carveout_kb=196))
    catt.atax_onekernel(A, x, k1=L.copy(active_warps=a))
torch.cuda.synchronize()
