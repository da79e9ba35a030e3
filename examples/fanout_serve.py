"""One trainer, N-1 inference processes: the cross-process model update
(one process per GPU, the paper's GPU-to-GPU channel s4.4 P:1677-1696,
fanned out to several consumers).

    torchrun --nproc-per-node 4 examples/fanout_serve.py [--fanout sa|chain|direct|push|nvls] [--steps 30]

Rank 0 trains a small MLP and publishes its state dict every step (ASYNC:
the trainer pays only for the snapshot).  Every other rank serves from the
latest installed version in a loop and, at the end, proves its replica: the
chunk seals of what it installed, computed on its own GPU
(viper_view_seals), must equal the producer's chunk seals of the same
version, and its logits on a probe batch must equal the trainer's bit for
bit.  On a box with fewer GPUs than ranks, ranks share GPUs (NVLS then
reports VIPER_E_UNSUPPORTED, and the example falls back to direct pulls)."""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import torch.distributed as dist
from torch.func import functional_call

from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V

FANOUTS = {"direct": V.FANOUT_DIRECT, "chain": V.FANOUT_CHAIN, "sa": V.FANOUT_SCATTER_ALLGATHER,
           "push": V.FANOUT_PUSH, "nvls": V.FANOUT_NVLS}


def seals_of(m, view, dev):
    n = m.stats()["nchunks"]
    buf = torch.empty(16 * n, dtype=torch.uint8, device=dev)
    m.view_seals(view, buf)
    torch.cuda.synchronize(dev)
    return buf.view(torch.int64).cpu().numpy().view(np.uint64).reshape(n, 2)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--fanout", default="sa", choices=sorted(FANOUTS))
    ap.add_argument("--steps", type=int, default=30)
    a = ap.parse_args()
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = torch.device("cuda", rank % torch.cuda.device_count())
    torch.cuda.set_device(dev)
    torch.manual_seed(0)  # same initial weights everywhere; the consumers' are overwritten anyway
    net = torch.nn.Sequential(torch.nn.Linear(256, 1024), torch.nn.GELU(), torch.nn.Linear(1024, 10)).to(dev)
    names = list(net.state_dict().keys())
    tensors = list(net.state_dict().values())
    bs = V.Bootstrap(rank, world, producer_rank=0)
    role = V.PRODUCER if rank == 0 else V.CONSUMER
    fanout = FANOUTS[a.fanout]
    try:
        m = V.Model("mlp", role, tensors, fanout=fanout, mode=V.ASYNC, bootstrap=bs, names=names, device=dev.index)
    except V.ViperError as e:
        if e.status != V.E_UNSUPPORTED:
            raise
        if rank == 0:
            print(f"fan-out {a.fanout} unavailable here ({e.detail}); using direct pulls", flush=True)
        fanout = V.FANOUT_DIRECT
        m = V.Model("mlp", role, tensors, fanout=fanout, mode=V.ASYNC, bootstrap=bs, names=names, device=dev.index)
    probe = torch.randn(16, 256, device=dev, generator=torch.Generator(device=dev).manual_seed(1))
    ok = True
    if rank == 0:
        opt = torch.optim.SGD(net.parameters(), lr=0.01)
        for step in range(1, a.steps + 1):
            x = torch.randn(64, 256, device=dev)
            loss = net(x).square().mean()
            opt.zero_grad()
            loss.backward()
            opt.step()
            m.publish(step)  # ASYNC: returns once the snapshot is enqueued on the current stream
        torch.cuda.synchronize(dev)
        _, sp, n = m.debug_buffers()
        like = torch.empty(4 * n, dtype=torch.int32, device=dev)
        ref_seals = V._from_ptr(sp, like).view(torch.int64).cpu().numpy().view(np.uint64).reshape(n, 2)
        with torch.no_grad():
            ref_logits = net(probe).cpu()
        shared = [ref_seals, ref_logits]
    else:
        served, t0 = 0, time.time()
        with torch.no_grad():
            while time.time() - t0 < 60:
                try:
                    view = m.acquire_latest(timeout_us=100_000)
                except V.ViperError:
                    continue
                functional_call(net, dict(zip(names, view.tensors(tensors))), (probe,))
                served += 1
                last = view.version
                m.release(view, stream=torch.cuda.current_stream())
                if last == a.steps:
                    break
        shared = [None, None]
    dist.broadcast_object_list(shared, src=0)
    if rank != 0:
        m.wait_installed(a.steps, timeout_us=30_000_000)
        view = m.acquire_latest()
        mine = seals_of(m, view, dev)
        with torch.no_grad():
            logits = functional_call(net, dict(zip(names, view.tensors(tensors))), (probe,)).cpu()
        m.release(view)
        ok = view.version == a.steps and np.array_equal(mine, shared[0]) and torch.equal(logits, shared[1])
        st = m.stats()
        print(f"[rank {rank}] served {served} inferences, installed {st['installs']} versions "
              f"(skipped {st['skipped']}), v{view.version}: seals match the producer's and logits match "
              f"the trainer's bit for bit: {ok}", flush=True)
    dist.barrier()
    if rank != 0:
        m.close()
    dist.barrier()
    if rank == 0:
        m.close()
    t = torch.tensor([0 if ok else 1])
    dist.all_reduce(t)
    if rank == 0:
        print(f"FANOUT_SERVE {'ok' if int(t.item()) == 0 else 'FAILED'} ({a.fanout})", flush=True)
    dist.destroy_process_group()
    sys.exit(int(t.item()) != 0)


if __name__ == "__main__":
    main()
