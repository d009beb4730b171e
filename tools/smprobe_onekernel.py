import os, sys, torch, numpy as np
sys.path.insert(0, os.getcwd())
import paper_conf_icpp_kimhlsh19_b200 as catt
n = 4096
A = torch.empty(n, n, device="cuda"); catt.fill_hash(A, 1)
x = torch.ones(n, device="cuda")
for name, fn in (("row_thread (catt_atax k1)", lambda pr: catt.atax(A, x, k1=catt.Throttle(cta_threads=1024, carveout_kb=196, probe=pr.data_ptr()))),
                 ("onekernel", lambda pr: catt.atax_onekernel(A, x, k1=catt.Throttle(cta_threads=1024, carveout_kb=196, probe=pr.data_ptr())))):
    for rep in range(3):
        pr = torch.zeros(4 * 32 * 3, dtype=torch.int64, device="cuda")
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(pr); e1.record(); torch.cuda.synchronize()
        rec = pr.cpu().numpy().reshape(4, 32, 3)
        sms = [sorted(set(int(s) for s in rec[c, :, 0])) for c in range(4)]
        dur = [(rec[c, :, 2].max() - rec[c, :, 1].min()) / 1e6 for c in range(4)]
        print(name, rep, "ms", round(e0.elapsed_time(e1), 3), "SM per CTA", sms, "loop ms per CTA", [round(d, 2) for d in dur])
