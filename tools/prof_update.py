"""Run a few SYNC model updates of one config (for ncu captures; no timing)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="ptychonn")
ap.add_argument("--steps", type=int, default=5)
ap.add_argument("--flush", action="store_true")
ap.add_argument("--tier", type=int, default=0)
ap.add_argument("--nofuse", action="store_true")
ap.add_argument("--flags", type=int, default=0, help="extra VIPER_FLAG_* bits for the producer")
ap.add_argument("--cflags", type=int, default=0, help="VIPER_FLAG_* bits for the consumer")
ap.add_argument("--mode", type=int, default=0, help="0 SYNC, 1 ASYNC (the consumer's update thread installs)")
ap.add_argument("--view-seals", action="store_true", help="seal the consumer's installed slot after every update")
a = ap.parse_args()
specs = synth.model_specs(a.config)
seed = synth.SEEDS[a.config]
pt, ct = G.alloc_model(specs), G.alloc_model(specs)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda") if a.flush else None
c = V.Model("prof", V.CONSUMER, ct, tier=a.tier, flags=a.cflags)
p = V.Model("prof", V.PRODUCER, pt, tier=a.tier, flags=(V.FLAG_NO_FUSE if a.nofuse else 0) | a.flags, mode=a.mode)
for v in range(1, a.steps + 1):
    G.fill_model(pt, specs, seed, v)
    if flush is not None:
        G.l2_flush(flush)
    p.publish(v)
    if a.mode == V.ASYNC:
        c.wait_installed(v)
    if a.view_seals:
        view = c.acquire_latest()
        buf = torch.empty(16 * c.stats()["nchunks"], dtype=torch.uint8, device="cuda")
        c.view_seals(view, buf)
        torch.cuda.synchronize()
        c.release(view)
torch.cuda.synchronize()
c.close()
p.close()
print("done", a.config, a.steps)
