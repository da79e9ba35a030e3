"""Kernel-only times of pack_seal / install_verify: the stream is kept busy
with a sleep kernel while publish() enqueues, so the library's CUDA events
bracket back-to-back device work (no host launch gaps inside)."""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="ptychonn")
ap.add_argument("--steps", type=int, default=20)
ap.add_argument("--flush", type=int, default=1)
a = ap.parse_args()
specs = synth.model_specs(a.config)
seed = synth.SEEDS[a.config]
pt, ct = G.alloc_model(specs), G.alloc_model(specs)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
c = V.Model("kt", V.CONSUMER, ct, flags=V.FLAG_TIMING)
p = V.Model("kt", V.PRODUCER, pt, flags=V.FLAG_TIMING)
st = torch.cuda.current_stream()
pk, ins, tot = [], [], []
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for v in range(1, a.steps + 6):
    G.fill_model(pt, specs, seed, v, stream=st)
    if a.flush:
        G.l2_flush(flush, stream=st)
    torch.cuda._sleep(200_000)   # ~100 us: publish() enqueues behind it
    e0.record(st)
    p.publish(v, stream=st)
    e1.record(st)
    e1.synchronize()
    if v > 5:
        pk.append(p.stats()["t_pack_dev_us"])
        ins.append(c.stats()["t_install_dev_us"])
        tot.append(e0.elapsed_time(e1) * 1e3)
S = synth.model_bytes(a.config)
print(f"{a.config}: pack {statistics.median(pk):.2f} us ({2*S/statistics.median(pk)/1e3:.0f} GB/s)  "
      f"install {statistics.median(ins):.2f} us ({2*S/statistics.median(ins)/1e3:.0f} GB/s)  "
      f"pack+install back-to-back {statistics.median(tot):.2f} us  flush={a.flush}")
c.close()
p.close()
