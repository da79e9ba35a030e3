"""Kernel-only times: fused SYNC kernel and separate pack / install kernels.
The stream is kept busy with a sleep kernel while publish() enqueues, so the
library's CUDA events bracket back-to-back device work (no host launch gaps)."""
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
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--flush", type=int, default=1)
a = ap.parse_args()
specs = synth.model_specs(a.config)
seed = synth.SEEDS[a.config]
pt, ct = G.alloc_model(specs), G.alloc_model(specs)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")  # --flush 1: write 256 MiB; 2: + read 256 MiB
S = synth.model_bytes(a.config)
res = {}
for label, flags in (("fused", V.FLAG_NO_TMA), ("fused_tma", V.FLAG_FUSED_TMA), ("sep", V.FLAG_NO_FUSE | V.FLAG_NO_TMA),
                     ("tma", V.FLAG_TMA)):
    cflags = {"sep": V.FLAG_NO_TMA, "tma": V.FLAG_TMA}.get(label, 0)
    c = V.Model("kt" + label, V.CONSUMER, ct, flags=V.FLAG_TIMING | cflags)
    p = V.Model("kt" + label, V.PRODUCER, pt, flags=V.FLAG_TIMING | flags)
    st = torch.cuda.current_stream()
    fu, pk, ins = [], [], []
    for v in range(1, a.steps + 4):
        G.fill_model(pt, specs, seed, v, stream=st)
        if a.flush == 1:
            G.l2_flush(flush[:256 << 20], stream=st)
        elif a.flush == 2:
            G.l2_flush(flush, stream=st, clean=True)
        torch.cuda._sleep(400_000)
        p.publish(v, stream=st)
        torch.cuda.synchronize()
        if v > 3:
            s = p.stats()
            fu.append(s["t_fused_dev_us"])
            pk.append(s["t_pack_dev_us"])
            ins.append(c.stats()["t_install_dev_us"])
    c.close()
    p.close()
    if label in ("fused", "fused_tma"):
        res[label] = statistics.median(fu)
    elif label == "sep":
        res["pack"], res["install"] = statistics.median(pk), statistics.median(ins)
    else:
        res["tma"] = statistics.median(pk)
        res["install_tma"] = statistics.median(ins)
lib = os.path.basename(os.environ.get("VIPER_LIB_PATH", "libviper.so"))
print(f"{lib:28s} {a.config:9s} fused {res['fused']:9.2f} us ({3*S/res['fused']/1e3/6550.4:.3f})  "
      f"fused_tma {res['fused_tma']:9.2f} us ({3*S/res['fused_tma']/1e3/6550.4:.3f})  "
      f"pack {res['pack']:9.2f} us ({2*S/res['pack']/1e3/6550.4:.3f})  "
      f"install {res['install']:9.2f} us ({2*S/res['install']/1e3/6550.4:.3f})  "
      f"pack_tma {res['tma']:9.2f} us ({2*S/res['tma']/1e3/6550.4:.3f})  "
      f"install_tma {res['install_tma']:9.2f} us ({2*S/res['install_tma']/1e3/6550.4:.3f})", flush=True)
