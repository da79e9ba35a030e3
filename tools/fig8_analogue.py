"""the paper's Fig. 8 (end-to-end model update latency,
P:1865-2009) re-run on one B200 with synthetic checkpoints of the paper's sizes.

  file baseline : torch.save(state_dict) to local disk + fsync, then
                  torch.load(map_location=cuda) and copy into the inference
                  replica (the paper's baseline is h5py on Lustre; this is the
                  local-disk analogue, context only)
  Viper GPU     : publish() SYNC, GPU tier (fused pack + install + swap)
  Viper DRAM    : publish() SYNC, pinned-DRAM tier (piece-pipelined D2H/H2D)

Latency = producer checkpoint + consumer load, the paper's definition
(P:2056-2060).  Prints one JSON object."""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

out = {}
path = os.environ.get("FIG8_FILE", "/tmp/viper_fig8.pt")
for name in synth.PAPER_SIZED:
    specs = synth.model_specs(name)
    S = synth.model_bytes(name)
    seed = synth.SEEDS[name]
    pt, ct = G.alloc_model(specs), G.alloc_model(specs)
    G.fill_model(pt, specs, seed, 1)
    torch.cuda.synchronize()
    row = {"bytes": S}
    # file baseline
    fl = []
    for rep in range(2):
        t0 = time.perf_counter()
        torch.save({s[0]: t for s, t in zip(specs, pt)}, path)
        with open(path, "rb") as f:
            os.fsync(f.fileno())
        t1 = time.perf_counter()
        sd = torch.load(path, map_location="cuda")
        for s, t in zip(specs, ct):
            t.copy_(sd[s[0]])
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        del sd
        fl.append((t1 - t0, t2 - t1))
    os.remove(path)
    ok = all(torch.equal(a.view(torch.uint8), b.view(torch.uint8)) for a, b in zip(pt, ct))
    row["file_save_s"] = round(min(x[0] for x in fl), 4)
    row["file_load_s"] = round(min(x[1] for x in fl), 4)
    row["file_s"] = round(min(x[0] + x[1] for x in fl), 4)
    row["file_ok"] = ok
    for tier, label in ((V.TIER_GPU, "gpu"), (V.TIER_DRAM, "dram")):
        c = V.Model(f"f8{label}{name}", V.CONSUMER, ct, tier=tier)
        p = V.Model(f"f8{label}{name}", V.PRODUCER, pt, tier=tier)
        lat = []
        for v in range(1, 5):
            G.fill_model(pt, specs, seed, v)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            p.publish(v)
            lat.append(time.perf_counter() - t0)
        view = c.acquire_latest()
        row[f"viper_{label}_ok"] = view.version == 4 and all(
            torch.equal(a.view(torch.uint8), b.view(torch.uint8)) for a, b in zip(view.tensors(ct), pt))
        c.release(view)
        c.close()
        p.close()
        row[f"viper_{label}_s"] = round(statistics.mean(lat[1:]), 5)
    row["speedup_gpu_vs_file"] = round(row["file_s"] / row["viper_gpu_s"], 1)
    row["speedup_dram_vs_file"] = round(row["file_s"] / row["viper_dram_s"], 1)
    out[name] = row
    del pt, ct
    torch.cuda.empty_cache()
    print(name, json.dumps(row), flush=True)
out["paper_context"] = ("Fig. 8 (Polaris A100, inter-node, h5py on Lustre): GPU-to-GPU ~9x (TC1 Async 9.3x, NT3.A 12x, "
                        "PtychoNN 15x) and Host-to-Host ~3x (TC1 Async 3.4x) faster than the file baseline")
print(json.dumps(out))
