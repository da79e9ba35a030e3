"""Failure detection: a consumer process dies without unregistering; the SYNC
producer must keep publishing (no 60 s stall) and the surviving consumer must
keep installing.  rank 0 producer, rank 1 survivor, rank 2 dies after v2."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import torch.distributed as dist

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

dist.init_process_group("gloo")
rank, world = dist.get_rank(), dist.get_world_size()
torch.cuda.set_device(0)
specs = [(f"t{i}", synth.F32, (50_000 + i,)) for i in range(5)]
seed = 0xFA11
ts = G.alloc_model(specs)
m = V.Model("fail", V.PRODUCER if rank == 0 else V.CONSUMER, ts, bootstrap=V.Bootstrap(rank, world, 0))
dist.barrier()  # last collective: from here a rank may vanish
if rank == 2:
    m.wait_installed(2, timeout_us=20_000_000)
    os._exit(0)  # crash without viper_unregister
if rank == 0:
    time0 = time.monotonic()
    results = []
    for v in range(1, 7):
        G.fill_model(ts, specs, seed, v)
        torch.cuda.synchronize()
        try:
            m.publish(v)
            results.append(0)
        except V.ViperError as e:
            results.append(e.status)
        time.sleep(0.2)
    took = time.monotonic() - time0
    ok = took < 15 and all(r in (0, V.E_PEER) for r in results)
    print(f"FAIL_PRODUCER results={results} took={took:.2f}s ok={ok}", flush=True)
    time.sleep(1.0)
    os._exit(0 if ok else 1)
if rank == 1:
    m.wait_installed(6, timeout_us=30_000_000)
    view = m.acquire_latest()
    good = view.version == 6 and all(
        np.array_equal(g.contiguous().view(torch.uint8).reshape(-1).cpu().numpy(),
                       synth.vgen_numpy(seed, 6, i, s[1], synth.nelem_of(s)))
        for i, (g, s) in enumerate(zip(view.tensors(ts), specs)))
    m.release(view)
    print(f"FAIL_SURVIVOR version={view.version} good={good}", flush=True)
    os._exit(0 if good else 1)
