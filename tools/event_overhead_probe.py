import torch, statistics, sys
sys.path.insert(0, '.')
import paper_conf_icpp_kimhlsh19_b200 as catt
flush_buf = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
clean_buf = torch.zeros(64 << 20, dtype=torch.int32, device="cuda")
x = torch.empty(1 << 20, device="cuda")
def flush():
    flush_buf.zero_(); clean_buf.sum(); torch.cuda._sleep(400_000)
def tiny():
    catt.fill_hash(x[:32], 1)
def timed(pre, fn, reps=30):
    ts = []
    for r in range(reps + 3):
        pre()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        if r >= 3: ts.append(a.elapsed_time(b) * 1e3)
    ts.sort(); return ts[len(ts)//2], ts[0]
g = torch.cuda.CUDAGraph()
s = torch.cuda.Stream()
with torch.cuda.stream(s):
    tiny(); torch.cuda.synchronize()
    with torch.cuda.graph(g): tiny()
torch.cuda.synchronize()
print("tiny after flush+sleep          ", timed(flush, tiny))
print("tiny after sleep only           ", timed(lambda: torch.cuda._sleep(400_000), tiny))
print("tiny, idle GPU                  ", timed(torch.cuda.synchronize, tiny))
print("graph tiny after flush+sleep    ", timed(flush, g.replay))
print("two tiny after flush+sleep      ", timed(flush, lambda: (tiny(), tiny())))
print("nothing after flush+sleep       ", timed(flush, lambda: None))
print("nothing idle                    ", timed(torch.cuda.synchronize, lambda: None))
