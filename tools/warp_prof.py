"""Per-warp timeline of publish_fused_kernel (profiling build, VP_WARP_PROF=1):
when each warp started and finished, how many items / bytes it moved, and when
the last block finished the swap.  Shows the launch ramp and the tail.

  python tools/warp_prof.py --build            # here: builds tune/libviper_prof.so
  python tools/warp_prof.py --config resnet50  # on the GPU box
"""
import argparse
import ctypes as C
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
LIBP = os.path.join(ROOT, "tune", "libviper_prof.so")

ap = argparse.ArgumentParser()
ap.add_argument("--build", action="store_true")
ap.add_argument("--config", default="resnet50")
ap.add_argument("--steps", type=int, default=5)
ap.add_argument("--defines", default="")
ap.add_argument("--lib", default=LIBP)
ap.add_argument("--clean", action="store_true", help="write + read L2 flush (bench.py default)")
a = ap.parse_args()
if a.build:
    from paper_conf_icpp_yecrbypnmskn24_b200 import build as B
    B.build_viper(force=True, out=a.lib, defines=["VP_WARP_PROF=1"] + [d for d in a.defines.split(",") if d])
    sys.exit(0)
os.environ["VIPER_LIB_PATH"] = a.lib
import numpy as np
import torch

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

specs = synth.model_specs(a.config)
seed = synth.SEEDS[a.config]
pt, ct = G.alloc_model(specs), G.alloc_model(specs)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
lib = C.CDLL(a.lib)
lib.vp_debug_warp_prof.argtypes = [C.c_void_p, C.c_int]
NW = 296 * 8
c = V.Model("wp", V.CONSUMER, ct, flags=V.FLAG_TIMING | V.FLAG_NO_TMA)
p = V.Model("wp", V.PRODUCER, pt, flags=V.FLAG_TIMING | V.FLAG_NO_TMA)
st = torch.cuda.current_stream()
rows = []
for v in range(1, a.steps + 4):
    G.fill_model(pt, specs, seed, v, stream=st)
    G.l2_flush(flush if a.clean else flush[:256 << 20], stream=st, clean=a.clean)
    torch.cuda._sleep(400_000)
    buf = np.zeros(NW * 4 + 1, dtype=np.uint64)
    p.publish(v, stream=st)
    torch.cuda.synchronize()
    assert lib.vp_debug_warp_prof(buf.ctypes.data, NW) == 0
    if v <= 3:
        continue
    w = buf[:NW * 4].reshape(NW, 4).astype(np.int64)
    used = w[:, 2] > 0
    w = w[used]
    t0 = w[:, 0].min()
    start = (w[:, 0] - t0) / 1e3
    end = (w[:, 1] - t0) / 1e3
    kend = (int(buf[-1]) - t0) / 1e3
    ev = p.stats()["t_fused_dev_us"]
    rows.append((ev, start, end, kend, w))
    print(f"v{v}: events {ev:.2f} us | warps {used.sum()} | start spread p50 {np.median(start):.2f} "
          f"p99 {np.percentile(start, 99):.2f} max {start.max():.2f} | end min {end.min():.2f} p10 "
          f"{np.percentile(end, 10):.2f} p50 {np.median(end):.2f} p90 {np.percentile(end, 90):.2f} "
          f"max {end.max():.2f} | last block done {kend:.2f} | items/warp {w[:, 2].min()}..{w[:, 2].max()} "
          f"bytes/warp {w[:, 3].min()}..{w[:, 3].max()}", flush=True)
S = synth.model_bytes(a.config)
ev, start, end, kend, w = rows[-1]
# bandwidth timeline: bytes moved (3 per byte of item) assuming each warp moved its bytes uniformly
print(f"{a.config}: 3S = {3 * S / 1e6:.1f} MB; span first-start -> last-block {kend:.2f} us = "
      f"{3 * S / (kend * 1e-6) / 1e9:.0f} GB/s; events {ev:.2f} us")
c.close()
p.close()
