"""The item-granular pipeline on one GPU: a SYNC publish with separate pack
and install kernels (VIPER_FLAG_NO_FUSE), the install launched with
programmatic dependent launch right behind the pack and waiting per item on
the seals the pack releases -- the same mechanism the cross-GPU early-notified
pipeline uses.  Prints, per model, the update latency (CUDA events around
publish, L2 flushed before each update) for: the fused kernel (default), the
PDL pipeline, and the pack + install run back to back without overlap
(VIPER_FLAG_TIMING disables PDL), beside the kernel times of the latter."""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G


def run(name, flags, steps=15, warmup=5):
    specs = synth.model_specs(name)
    seed = synth.SEEDS[name]
    pt, ct = G.alloc_model(specs), G.alloc_model(specs)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    c = V.Model(f"po-{name}-{flags}", V.CONSUMER, ct, flags=flags & V.FLAG_TIMING)
    p = V.Model(f"po-{name}-{flags}", V.PRODUCER, pt, flags=flags)
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    lat, pk, ins = [], [], []
    for v in range(1, warmup + steps + 1):
        G.fill_model(pt, specs, seed, v, stream=st)
        G.l2_flush(flush, stream=st, clean=True)
        torch.cuda.synchronize()
        e0.record(st)
        p.publish(v, stream=st)
        e1.record(st)
        e1.synchronize()
        if v > warmup:
            lat.append(e0.elapsed_time(e1) * 1e3)
            pk.append(p.stats()["t_pack_dev_us"])
            ins.append(c.stats()["t_install_dev_us"])
    view = c.acquire_latest()
    ok = view.version == warmup + steps and all(
        torch.equal(g.view(torch.uint8), q.view(torch.uint8)) for g, q in zip(view.tensors(ct), pt))
    c.release(view)
    c.close()
    p.close()
    return statistics.median(lat), statistics.median(pk), statistics.median(ins), ok


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="resnet50,vit_b16,gpt2_xl")
    a = ap.parse_args()
    for nm in a.configs.split(","):
        fused = run(nm, 0)
        pdl = run(nm, V.FLAG_NO_FUSE | V.FLAG_NO_TMA)
        serial = run(nm, V.FLAG_NO_FUSE | V.FLAG_NO_TMA | V.FLAG_TIMING)
        print(f"{nm:9s} update latency: fused {fused[0]:8.1f} us | PDL pipeline {pdl[0]:8.1f} us | "
              f"pack then install {serial[0]:8.1f} us (pack {serial[1]:7.1f} + install {serial[2]:7.1f} us) "
              f"parity {fused[3] and pdl[3] and serial[3]}", flush=True)
