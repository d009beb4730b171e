"""Does the bench protocol's idle gap before the timed region cost bandwidth?
Read-only sum of S MB, timed with CUDA events after:
  A  flush (256 MiB write + 256 MiB clean read), then a 200 us GPU sleep (current bench order)
  B  the GPU sleep first, then the flush (HBM busy right up to the timed kernel)
Both keep L2 cold and every launch queued before the GPU reaches it."""
import statistics
import torch

dev = torch.device("cuda")
fb = torch.empty(64 << 20, dtype=torch.int32, device=dev)
cb = torch.zeros(64 << 20, dtype=torch.int32, device=dev)


def flush():
    fb.zero_()
    cb.sum()


def timed(fn, order, reps=9):
    ts = []
    for r in range(reps + 1):
        if order == "A":
            flush(); torch.cuda._sleep(400_000)
        else:
            torch.cuda._sleep(400_000); flush()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        if r:
            ts.append(a.elapsed_time(b))
    return statistics.median(ts)


for mb in (32, 64, 134, 256, 512, 2048):
    x = torch.ones(mb * (1 << 20) // 4, device=dev)
    ta, tb = timed(lambda: x.sum(), "A"), timed(lambda: x.sum(), "B")
    g = lambda t: mb * 1.048576e-3 / t * 1e3
    print(f"{mb:5d} MB  A(flush,sleep): {ta*1e3:8.1f} us {g(ta):6.0f} GB/s   B(sleep,flush): {tb*1e3:8.1f} us {g(tb):6.0f} GB/s",
          flush=True)
    del x
