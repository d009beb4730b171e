"""One launch each of: STAGED rows, STAGED cols, COOP cols (cluster), COOP cols (1024-thread CTA) at 4096^2."""
import torch
import paper_conf_icpp_kimhlsh19_b200 as catt
n = 4096
A = torch.empty(n, n, device="cuda"); catt.fill_hash(A, 2)
x = torch.rand(n, device="cuda"); y = torch.empty(n, device="cuda")
catt.rows(A, x, y, t=catt.Throttle(variant="staged", cta_threads=32))
catt.cols(A, x, y, t=catt.Throttle(variant="staged", cta_threads=32))
catt.cols(A, x, y, t=catt.Throttle(variant="coop"))
catt.cols(A, x, y, t=catt.Throttle(variant="coop", cta_threads=1024, active_ctas=1))   # capped -> col_warp_kernel path
torch.cuda.synchronize()
