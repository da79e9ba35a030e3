"""Where the e2e step's time goes (H2D of the flat weights, publish, digest D2H)."""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

name = sys.argv[1] if len(sys.argv) > 1 else "ptychonn"
specs = synth.model_specs(name)
offs, off = [], 0
for s_ in specs:
    offs.append(off)
    off = (off + synth.nbytes_of(s_) + 255) // 256 * 256
flat = torch.empty(off, dtype=torch.uint8, device="cuda")
dt = {synth.F32: torch.float32, synth.BF16: torch.bfloat16, synth.F16: torch.float16}
pt = [flat[o:o + synth.nbytes_of(s_)].view(dt[s_[1]]).view(s_[2]) for o, s_ in zip(offs, specs)]
ct = G.alloc_model(specs)
host = flat.cpu().pin_memory()
c = V.Model("e2eb", V.CONSUMER, ct)
p = V.Model("e2eb", V.PRODUCER, pt)
st = torch.cuda.current_stream()
_, sp, n = p.debug_buffers()
digest = torch.empty(2 * n, dtype=torch.int64).pin_memory()
T = {k: [] for k in ("h2d_enqueue", "publish", "debug_buffers", "digest", "total", "h2d_dev")}
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for i in range(40):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    e0.record(st)
    flat.copy_(host, non_blocking=True)
    e1.record(st)
    t1 = time.perf_counter()
    p.publish(i + 1, stream=st)
    t2 = time.perf_counter()
    _, sp, _ = p.debug_buffers()
    t3 = time.perf_counter()
    like = torch.empty(4 * n, dtype=torch.int32, device="cuda")
    digest.copy_(V._from_ptr(sp, like).view(torch.int64), non_blocking=True)
    torch.cuda.synchronize()
    t4 = time.perf_counter()
    if i >= 5:
        for k, v in zip(("h2d_enqueue", "publish", "debug_buffers", "digest", "total"),
                        (t1 - t0, t2 - t1, t3 - t2, t4 - t3, t4 - t0)):
            T[k].append(v * 1e6)
        T["h2d_dev"].append(e0.elapsed_time(e1) * 1e3)
for k, v in T.items():
    print(f"{k:14s} {statistics.median(v):8.1f} us")
c.close()
p.close()
