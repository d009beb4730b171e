"""Launch the SYRK and SYR2K tiled kernels at 2048 once each (for ncu)."""
import torch
import paper_conf_icpp_kimhlsh19_b200 as catt

dev = torch.device("cuda")
n = 2048
A, B, C = (torch.empty(n, n, device=dev) for _ in range(3))
for i, t in enumerate((A, B, C)):
    catt.fill_hash(t, 40 + i)
T = catt.Throttle(variant="staged")
catt.syrk(A, C, 1.5, 1.2, t=T)
catt.syr2k(A, B, C, 1.5, 1.2, t=T)
torch.cuda.synchronize()
