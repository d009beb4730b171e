"""Launch each CATT study case once (for ncu). Prints the case order."""
import sys
import torch
import paper_conf_icpp_kimhlsh19_b200 as catt

dev = torch.device("cuda")
n = 4096
A = torch.empty(n, n, device=dev); catt.fill_hash(A, 2)
x = torch.rand(n, device=dev); y = torch.empty(n, device=dev)
npts, nf, k, ld = 494020, 34, 5, 494020
feat = torch.empty(nf * ld, device=dev); catt.fill_hash(feat, 4)
cl = feat.view(nf, ld)[:, :k].t().contiguous()
memb = torch.empty(npts, dtype=torch.int32, device=dev)
T = catt.Throttle
cases = [
    ("kmeans (8,8) carve16", lambda: catt.kmeans_assign(feat, ld, npts, nf, cl, memb, t=T(carveout_kb=16))),
    ("kmeans (4,8) carve16", lambda: catt.kmeans_assign(feat, ld, npts, nf, cl, memb, t=T(active_warps=4, carveout_kb=16))),
    ("kmeans (8,4) carve16", lambda: catt.kmeans_assign(feat, ld, npts, nf, cl, memb, t=T(active_ctas=4, carveout_kb=16))),
    ("kmeans (8,8) carve228", lambda: catt.kmeans_assign(feat, ld, npts, nf, cl, memb, t=T(carveout_kb=228))),
    ("kmeans (1,2) carve228", lambda: catt.kmeans_assign(feat, ld, npts, nf, cl, memb, t=T(active_warps=1, active_ctas=2, carveout_kb=228))),
    ("kmeans regs", lambda: catt.kmeans_assign(feat, ld, npts, nf, cl, memb, t=T(variant="regs", cta_threads=128))),
    ("rows cta1024 carve196 (32,1)", lambda: catt.rows(A, x, y, t=T(cta_threads=1024, carveout_kb=196))),
    ("rows cta1024 carve196 (16,1)", lambda: catt.rows(A, x, y, t=T(cta_threads=1024, active_warps=16, carveout_kb=196))),
    ("rows cta1024 carve196 (8,1)", lambda: catt.rows(A, x, y, t=T(cta_threads=1024, active_warps=8, carveout_kb=196))),
    ("rows cta1024 carve0 (32,1)", lambda: catt.rows(A, x, y, t=T(cta_threads=1024, carveout_kb=0))),
    ("rows cta256 carve228 (8,1)", lambda: catt.rows(A, x, y, t=T(carveout_kb=228))),
    ("rows cta256 carve228 (4,1)", lambda: catt.rows(A, x, y, t=T(active_warps=4, carveout_kb=228))),
    ("rows cta256 carve0 (8,1)", lambda: catt.rows(A, x, y, t=T(carveout_kb=0))),
    ("rows staged cta32", lambda: catt.rows(A, x, y, t=T(variant="staged", cta_threads=32))),
]
for name, fn in cases:
    fn()
torch.cuda.synchronize()
for i, (name, fn) in enumerate(cases):
    print(i, name, flush=True)
    fn()
torch.cuda.synchronize()
