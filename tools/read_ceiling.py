"""Read-only and copy bandwidth vs size with the bench protocol (write+clean-read
flush, GPU sleep so launches are queued, CUDA events)."""
import statistics
import torch
dev = torch.device("cuda")
fb = torch.empty(64 << 20, dtype=torch.int32, device=dev)
cb = torch.zeros(64 << 20, dtype=torch.int32, device=dev)
def timed(fn, reps=7):
    ts = []
    for r in range(reps + 1):
        fb.zero_(); cb.sum(); torch.cuda._sleep(400_000)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        if r: ts.append(a.elapsed_time(b))
    return statistics.median(ts)
for mb in (16, 32, 64, 69, 128, 256, 512, 1024, 2048):
    n = mb * (1 << 20) // 4
    x = torch.ones(n, device=dev)
    y = torch.empty(n // 2, device=dev); z = torch.empty(n // 2, device=dev)
    tr = timed(lambda: x.sum())
    tc = timed(lambda: z.copy_(y))
    print(f"{mb:5d} MB  read-only sum: {tr*1e3:8.1f} us {mb*1.048576e-3/tr*1e3:7.0f} GB/s   copy(same bytes moved): {tc*1e3:8.1f} us {mb*1.048576e-3/tc*1e3:7.0f} GB/s", flush=True)
    del x, y, z
