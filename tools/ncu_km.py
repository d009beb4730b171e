"""Launch the KMEANS-iteration kernels once each at the BASELINE shape (for ncu)."""
import torch
import paper_conf_icpp_kimhlsh19_b200 as catt

npts, nf, k = 494020, 34, 5
feat = torch.empty(nf * npts, device="cuda"); catt.fill_hash(feat, 4)
cl = feat.view(nf, npts)[:, :k].t().contiguous()
memb = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
acc = torch.zeros(catt.kmeans_acc_words(k, nf), dtype=torch.int64, device="cuda")
pm = torch.empty(npts * nf, device="cuda"); catt.fill_hash(pm, 9)
out = torch.empty(nf * npts, device="cuda")
catt.kmeans_accumulate(feat, npts, npts, nf, cl, memb, acc)
catt.kmeans_finalize(acc, cl)
catt.kmeans_transpose(pm, npts, nf, out, npts, t=catt.Throttle(variant="coop"))
catt.kmeans_transpose(pm, npts, nf, out, npts, t=catt.Throttle(variant="literal"))
torch.cuda.synchronize()
