"""Worker for the cross-process tests (one process per "GPU"; on a 1-GPU box
every rank uses cuda:0 and CUDA-IPC maps the same device).

Rank 0 = producer, ranks 1.. = consumers; bootstrap over a gloo group.
Checks, for every version: each consumer's acquired view is byte-identical to
VGEN(version) computed on the host (synth.vgen_numpy), versions never go
backwards, and the producer's chunk seals equal the oracle's.
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch
import torch.distributed as dist

import synth
from oracle import transfer as T
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G


def host_bytes(t):
    return t.contiguous().view(torch.uint8).reshape(-1).cpu().numpy() if t.numel() else np.zeros(0, np.uint8)


def stress(m, rank, specs, seed, tensors, n, dev):
    """Producer: n ASYNC publishes back to back.  Consumers: acquire -> compare
    every byte of the view with VGEN(view.version) on the GPU -> release, until
    the last version is seen (torn / mixed-version reads and regressions count
    as errors)."""
    errors = 0
    dist.barrier()
    if rank == 0:
        st = torch.cuda.Stream()
        for v in range(1, n + 1):
            with torch.cuda.stream(st):
                G.fill_model(tensors, specs, seed, v, stream=st)
                m.publish(v, stream=st)
        st.synchronize()
    else:
        exp = G.alloc_model(specs, device=f"cuda:{dev}")
        s = torch.cuda.Stream()
        last, seen = 0, 0
        while last < n:
            try:
                view = m.acquire_latest(timeout_us=2_000_000)
            except V.ViperError:
                continue
            with torch.cuda.stream(s):
                G.fill_model(exp, specs, seed, view.version, stream=s)
                got = view.tensors(tensors)
                bad = sum(int((g.view(torch.uint8) != e.view(torch.uint8)).sum()) for g, e in zip(got, exp))
            m.release(view, stream=s)
            s.synchronize()
            if bad:
                print(f"[rank{rank}] torn view v{view.version}: {bad} bytes", flush=True)
                errors += 1
            if view.version < last:
                errors += 1
            last = view.version
            seen += 1
        print(f"[rank{rank}] stress: {seen} verified views, last v{last}, stats {m.stats()['installs']} installs "
              f"{m.stats()['skipped']} skipped", flush=True)
    dist.barrier()
    return errors


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="ptychonn")
    ap.add_argument("--tier", type=int, default=0)
    ap.add_argument("--mode", type=int, default=0)
    ap.add_argument("--fanout", type=int, default=0)
    ap.add_argument("--versions", type=int, default=6)
    ap.add_argument("--fault", type=int, default=0)
    ap.add_argument("--stress", type=int, default=0, help="ASYNC publishes while consumers verify every view")
    ap.add_argument("--nprod", type=int, default=1, help="data-parallel producers (ranks 0..nprod-1)")
    ap.add_argument("--delay-ms", type=float, default=0.0,
                    help="ASYNC: the producer's stream sleeps this long before each publish; consumers check "
                         "that their install did not start (and spin) before the stream reached the pack")
    ap.add_argument("--expect-tier", type=int, default=-1, help="check the tier in use after registration "
                    "(VIPER_TIER_AUTO resolved by the Transfer Selector)")
    ap.add_argument("--no-peer-rank", type=int, default=-1, help="this rank reports that it reaches no GPU "
                    "(VIPER_TEST_NO_PEER)")
    ap.add_argument("--allow-unsupported", action="store_true",
                    help="registration may fail with VIPER_E_UNSUPPORTED on EVERY rank (NVLS without multicast)")
    a = ap.parse_args()
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = rank % torch.cuda.device_count()
    torch.cuda.set_device(dev)
    specs = synth.model_specs(a.config) if a.config in synth.SEEDS else \
        [(f"t{i}", synth.F32, (1000 + 37 * i,)) for i in range(7)] + [("odd", synth.BYTES, (13,))]
    seed = synth.SEEDS.get(a.config, 0xC0FFEE)
    tensors = G.alloc_model(specs, device=f"cuda:{dev}")
    bs = V.Bootstrap(rank, world, producer_rank=0, nproducers=a.nprod)
    is_prod = rank < a.nprod
    role = V.PRODUCER if is_prod else V.CONSUMER
    if rank == a.no_peer_rank:
        os.environ["VIPER_TEST_NO_PEER"] = "1"
    try:
        m = V.Model(f"xp-{a.config}", role, tensors, tier=a.tier, mode=a.mode, fanout=a.fanout, device=dev,
                    bootstrap=bs)
    except V.ViperError as e:
        unsupported = e.status == V.E_UNSUPPORTED
        t = torch.tensor([0 if unsupported else 1])
        dist.all_reduce(t)
        if rank == 0:
            print(f"XPROC_UNSUPPORTED everywhere={int(t.item()) == 0}: {e.detail}", flush=True)
        dist.destroy_process_group()
        sys.exit(0 if (a.allow_unsupported and int(t.item()) == 0) else 1)
    errors = 0
    if a.expect_tier >= 0 and m.stats()["tier"] != a.expect_tier:
        print(f"[rank{rank}] tier {m.stats()['tier']}, want {a.expect_tier}", flush=True)
        errors += 1
    last = 0
    if a.stress:
        errors += stress(m, rank, specs, seed, tensors, a.versions, dev)
        a.versions = 0  # skip the lock-step loop
    for v in range(1, a.versions + 1):
        if a.fault and rank == 1 and v == 2:
            m.fault_next()
        dist.barrier()
        if is_prod:
            G.fill_model(tensors, specs, seed, v)
            torch.cuda.synchronize()
            if a.delay_ms:
                torch.cuda._sleep(int(a.delay_ms * 2.0e6))  # ~2 GHz SM clock
            try:
                m.publish(v)
            except V.ViperError as e:
                if not (a.fault and v == 2 and e.status == V.E_CHECKSUM):
                    print(f"[rank0] publish({v}) failed: {e}", flush=True)
                    errors += 1
            if a.mode == V.SYNC:
                _, sp, n = m.debug_buffers()
                like = torch.empty(4 * n, dtype=torch.int32, device=f"cuda:{dev}")
                seals = V._from_ptr(sp, like).view(torch.int64).cpu().numpy().view(np.uint64).reshape(n, 2)
                exp = [synth.vgen_numpy(seed, v, i, s[1], synth.nelem_of(s)) for i, s in enumerate(specs)]
                off, S = T.layout([e.size for e in exp], 256)
                ref = T.seal(T.pack(exp, off, S), 2 << 20, v)
                own = [c for c in range(n) if c % a.nprod == rank]  # data-parallel: this producer's chunks
                if not np.array_equal(seals[own], ref[own]):
                    print(f"[rank{rank}] seals differ at v{v}", flush=True)
                    errors += 1
        dist.barrier()
        if not is_prod and a.mode == V.SYNC:
            view = m.acquire_latest(timeout_us=5_000_000)
            want = 1 if (a.fault and rank == 1 and v == 2) else v
            if view.version != want:
                print(f"[rank{rank}] v{v}: acquired {view.version}, want {want}", flush=True)
                errors += 1
            if view.version < last:
                errors += 1
            last = view.version
            got = view.tensors(tensors)
            exp = [synth.vgen_numpy(seed, view.version, i, s[1], synth.nelem_of(s)) for i, s in enumerate(specs)]
            for i, (g, e) in enumerate(zip(got, exp)):
                if not np.array_equal(host_bytes(g), e):
                    print(f"[rank{rank}] tensor {i} differs at v{view.version}", flush=True)
                    errors += 1
                    break
            # the installed slot's chunk seals, computed on this GPU, == the oracle's
            n = m.stats()["nchunks"]
            sb = torch.empty(max(16 * n, 16), dtype=torch.uint8, device=f"cuda:{dev}")
            m.view_seals(view, sb)
            torch.cuda.synchronize()
            cs = sb.view(torch.int64).cpu().numpy().view(np.uint64).reshape(-1, 2)[:n]
            off, S = T.layout([e.size for e in exp], 256)
            if not np.array_equal(cs, T.seal(T.pack(exp, off, S), 2 << 20, view.version)):
                print(f"[rank{rank}] installed-slot seals differ from the oracle at v{view.version}", flush=True)
                errors += 1
            m.release(view)
        dist.barrier()
    if not is_prod and a.mode == V.ASYNC and not a.stress:
        m.wait_installed(a.versions, timeout_us=20_000_000)
        view = m.acquire_latest()
        if view.version != a.versions:
            errors += 1
        got = view.tensors(tensors)
        for i, (g, s) in enumerate(zip(got, specs)):
            if not np.array_equal(host_bytes(g), synth.vgen_numpy(seed, view.version, i, s[1], synth.nelem_of(s))):
                errors += 1
        m.release(view)
        st = m.stats()
        print(f"[rank{rank}] installs={st['installs']} skipped={st['skipped']} "
              f"last install {st['t_install_us']:.0f} us", flush=True)
        if a.delay_ms and st["t_install_us"] > a.delay_ms * 1e3 / 3:
            print(f"[rank{rank}] install started before the producer's stream reached the pack", flush=True)
            errors += 1
    dist.barrier()
    if not is_prod:
        m.close()
    dist.barrier()
    if is_prod:
        m.close()
    t = torch.tensor([errors])
    dist.all_reduce(t)
    if rank == 0:
        print(f"XPROC_RESULT errors={int(t.item())}", flush=True)
    dist.destroy_process_group()
    sys.exit(1 if int(t.item()) else 0)


if __name__ == "__main__":
    main()
