"""ASYNC in-process update latency decomposition (1-GPU loopback): producer
stall (publish return), publish -> update-thread pickup, and publish ->
installed (wait_installed), L2 flushed (write + read) before every update."""
import argparse
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="resnet50")
ap.add_argument("--steps", type=int, default=20)
ap.add_argument("--gap-ms", type=float, default=2.0, help="idle time between updates (the update thread sleeps)")
ap.add_argument("--tier", type=int, default=0, help="0 GPU, 1 DRAM")
a = ap.parse_args()
specs = synth.model_specs(a.config)
seed = synth.SEEDS[a.config]
pt, ct = G.alloc_model(specs), G.alloc_model(specs)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
c = V.Model("al", V.CONSUMER, ct, tier=a.tier)
p = V.Model("al", V.PRODUCER, pt, mode=V.ASYNC, tier=a.tier)
stall, done, pick, inst = [], [], [], []
for v in range(1, a.steps + 4):
    G.fill_model(pt, specs, seed, v)
    G.l2_flush(flush, clean=True)
    torch.cuda.synchronize()
    time.sleep(a.gap_ms * 1e-3)
    t0 = time.perf_counter()
    p.publish(v)
    t1 = time.perf_counter()
    c.wait_installed(v, timeout_us=5_000_000)
    t2 = time.perf_counter()
    if v > 3:
        s = c.stats()
        stall.append((t1 - t0) * 1e6)
        done.append((t2 - t0) * 1e6)
        pick.append(s["t_notify_us"])
        inst.append(s["t_install_us"])
c.close()
p.close()
med = statistics.median
print(f"{a.config} tier={a.tier} ASYNC: publish returns {med(stall):.1f} us | pickup {med(pick):.1f} us | "
      f"install (launch->done) {med(inst):.1f} us | publish -> installed {med(done):.1f} us")
