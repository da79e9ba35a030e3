import statistics, sys, time
import torch
for mb in (0.25, 1, 4, 4.6, 8, 16, 64, 256):
    n = int(mb * 1e6)
    h = torch.empty(n, dtype=torch.uint8).pin_memory()
    d = torch.empty(n, dtype=torch.uint8, device="cuda")
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for i in range(20):
        torch.cuda.synchronize()
        e0.record(); d.copy_(h, non_blocking=True); e1.record(); e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts2 = []
    for i in range(20):
        torch.cuda.synchronize()
        e0.record(); h.copy_(d, non_blocking=True); e1.record(); e1.synchronize()
        ts2.append(e0.elapsed_time(e1) * 1e3)
    print(f"{mb:7.2f} MB  H2D {statistics.median(ts):8.1f} us ({n/statistics.median(ts)/1e3:6.1f} GB/s)   D2H {statistics.median(ts2):8.1f} us ({n/statistics.median(ts2)/1e3:6.1f} GB/s)", flush=True)
