"""DRAM-tier (pinned host staging) update latency vs GPU tier, 1-GPU loopback."""
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
ap.add_argument("--steps", type=int, default=4)
ap.add_argument("--dram-only", action="store_true", help="only the DRAM-tier update (piece sweeps)")
a = ap.parse_args()
specs = synth.model_specs(a.config)
S = synth.model_bytes(a.config)
pt, ct = G.alloc_model(specs), G.alloc_model(specs)
for tier in ((V.TIER_DRAM,) if a.dram_only else (V.TIER_DRAM, V.TIER_GPU)):
    c = V.Model(f"d{tier}", V.CONSUMER, ct, tier=tier)
    p = V.Model(f"d{tier}", V.PRODUCER, pt, tier=tier)
    lat = []
    for v in range(1, a.steps + 3):
        G.fill_model(pt, specs, synth.SEEDS[a.config], v)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        p.publish(v)
        lat.append((time.perf_counter() - t0) * 1e3)
    lat = lat[2:]
    print(f"{a.config} tier={'dram' if tier else 'gpu'}: {statistics.mean(lat):.3f} ms/update  "
          f"({S / (statistics.mean(lat) * 1e-3) / 1e9:.1f} GB/s)", flush=True)
    c.close()
    p.close()
if a.dram_only:
    sys.exit(0)
# raw pinned copy rates
h = torch.empty(S, dtype=torch.uint8).pin_memory()
d = torch.empty(S, dtype=torch.uint8, device="cuda")
for name, fn in (("D2H", lambda: h.copy_(d, non_blocking=True)), ("H2D", lambda: d.copy_(h, non_blocking=True))):
    fn(); torch.cuda.synchronize()
    t0 = time.perf_counter(); fn(); torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    print(f"pinned {name} {S/1e9:.2f} GB: {S / dt / 1e9:.1f} GB/s", flush=True)

# bidirectional: a D2H and an H2D of the same size at once on two streams
# (the DRAM tier's steady state: the producer's D2H of piece i overlaps the
# consumer's H2D of piece i-1)
nb = min(S, 4 << 30)
ha, hb = G.PinnedBuffer(nb), G.PinnedBuffer(nb)
da = torch.empty(nb, dtype=torch.uint8, device="cuda")
db = torch.empty(nb, dtype=torch.uint8, device="cuda")
sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
for rep in range(2):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ha.from_device_ptr(da.data_ptr(), nb, stream=sa)
    hb.to_device(db, stream=sb)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
print(f"pinned D2H || H2D {nb/1e9:.2f} GB each: {nb / dt / 1e9:.1f} GB/s per direction, {2 * nb / dt / 1e9:.1f} GB/s total",
      flush=True)
for name, fn in (("D2H", lambda: ha.from_device_ptr(da.data_ptr(), nb, stream=sa)), ("H2D", lambda: hb.to_device(db, stream=sa))):
    fn(); torch.cuda.synchronize()
    t0 = time.perf_counter(); fn(); torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    print(f"raw pinned {name} {nb/1e9:.2f} GB alone: {nb / dt / 1e9:.1f} GB/s", flush=True)
ha.close(); hb.close()
