#!/usr/bin/env python
"""bench.py -- model-update latency of the Viper hot path on B200.

Default (N=1): BASELINE.json configs[1], the first configuration the metric
is quoted on, in 1-GPU form: ResNet-50 fp32 (161 tensors, 102 MB), 1 producer
-> 1 consumer on one GPU (in-process loopback: the NVLink hop of configs[1]
needs a second GPU; GPU tier, SYNC mode).  configs[0] (PtychoNN-sized, 4.6 MB)
is the small parity case; it is reported in the loopback sweep beside the
larger configs.  One step = one versioned model update: pack + seal (K2) ->
publish/notify -> install + verify (K6) -> device-side atomic version swap;
publish() returns once the consumer serves v.

Timing: per step, L2 is flushed (a 256 MiB write, then a 256 MiB read of another
buffer; each > the 126 MB L2) and the
producer's tensors are rewritten with VGEN(v) (the synthetic "optimizer step")
OUTSIDE the timed interval; each update is timed with CUDA events on the
publishing stream (start before publish, end after it returned) and with the
host clock (publish entry -> return = the swap is visible).  value = mean
device-event latency over the K timed steps.

Extra keys: roofline of the dominant kernel (library-recorded CUDA events,
VIPER_FLAG_TIMING), cpu_baseline (the oracle on host cores), e2e (host
buffers: H2D of the new weights + publish + D2H of the seal digest), clocks,
gpu_launches, and a 1-GPU loopback sweep over the other BASELINE.json model
sizes (not the headline).

--impl reference: the oracle (plain C, oracle/) on the host cores, same
config/metric -- the deliberately slow reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

HBM_NOMINAL_GBS = 7700.0  # B200 HGX HBM3e nominal (B200_PROFILING.md), context beside the measured copy peak
METRIC = "model-update latency (ms) and GB/s vs NVLink/HBM roofline at 1->1/3/7 GPUs"
# "dtype" is the arithmetic the path computes in: bytes moved as 128-bit words,
# sealed with u32 word checksums summed mod 2^64 (R16); the model's
# own element type, never interpreted, is reported as "model_dtype".


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def ncu_traffic(kernel, config):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch from the committed
    ncu --set full capture (profiles/ncu_traffic.json), or None."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            t = json.load(f)
        # template instances are named "<kernel><...>:<config>"; the newest capture of the kernel wins
        keys = [k for k in t if k.split("<")[0].split(":")[0] == kernel and k.endswith(f":{config}")]
        return t[sorted(keys, key=lambda k: "<" in k)[-1]].get("traffic_bytes") if keys else None
    except Exception:
        return None


LAUNCH_LISTS = {"resnet50": "profiles/r02/launches_bench_r50_summary.json",
                "ptychonn": "profiles/r01/launches_bench_c1_summary.json"}


def ncu_launches(config, kernel, alg_bytes, peak):
    """The committed ncu launch list of this bench command (`ncu --metrics
    gpu__time_duration.sum --clock-control none`): the kernel's mean cold,
    serialised duration and its share of the library's kernel time per update
    (fused kernel + side-stream seal reduction), or None."""
    try:
        with open(os.path.join(ROOT, LAUNCH_LISTS[config])) as f:
            t = json.load(f)
        k = t[next(n for n in t if n.split("<")[0] == kernel)]
        lib = k["total_us"] + t.get("seal_reduce_kernel", {}).get("total_us", 0.0) * k["launches"] / max(
            1, t.get("seal_reduce_kernel", {}).get("launches", 1))
        return {"file": LAUNCH_LISTS[config], "mean_us": k["mean_us"], "share_of_library_kernels":
                round(k["total_us"] / lib, 4), "frac_at_ncu_duration": round(alg_bytes / (k["mean_us"] * 1e3) / peak, 4)}
    except Exception:
        return None


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    def __init__(self, index=0):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 6:
                self.rows.append(parts)

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[2 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


# ---------------------------------------------------------------- GPU arm
FLUSH_BYTES = 512 << 20  # two halves, each > the 126 MB L2


def flush_l2(G, buf, stream=None, dirty=False):
    """Evict L2 before a timed update.  Default: write 256 MiB, then read
    another 256 MiB, so the written lines go back to HBM inside the flush and
    L2 holds clean unrelated data (the state ncu's cache control leaves).
    dirty=True: the write alone, leaving ~126 MB of dirty harness lines that
    the timed kernel must write back (reported beside the headline)."""
    if dirty:
        G.l2_flush(buf[:FLUSH_BYTES // 2], stream=stream)
    else:
        G.l2_flush(buf, stream=stream, clean=True)


def run_update_bench(V, G, synth, name, steps, warmup, flush_buf, mode=None, tier=None, kernel_timing=False,
                     extra_flags=0, ncons=1, dirty=False):
    """Producer + 1 consumer on this GPU; per-step update latency.

    kernel_timing=False: the headline pass -- nothing but the update inside
    the events.  kernel_timing=True: the library records CUDA events around
    its kernels (VIPER_FLAG_TIMING) and a sleep kernel keeps the stream busy
    while publish() enqueues, so those events bracket back-to-back device work
    (kernel-only times for the roofline; the latency of this pass is not used).
    """
    import torch
    specs = synth.model_specs(name)
    seed = synth.SEEDS[name]
    prod_t = G.alloc_model(specs)
    cons_ts = [G.alloc_model(specs) for _ in range(ncons)]
    cons_t = cons_ts[0]
    mname = f"bench-{name}-{os.getpid()}-{time.monotonic_ns()}"
    flags = (V.FLAG_TIMING if kernel_timing else 0) | extra_flags
    mode = V.SYNC if mode is None else mode
    tier = V.TIER_GPU if tier is None else tier
    conss = [V.Model(mname, V.CONSUMER, ct, flags=flags, tier=tier) for ct in cons_ts]
    cons = conss[0]
    prod = V.Model(mname, V.PRODUCER, prod_t, flags=flags, mode=mode, tier=tier)
    st = torch.cuda.current_stream()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    dev_ms, host_ms, pack_us, inst_us, fused_us = [], [], [], [], []
    try:
        for i in range(warmup + steps):
            v = i + 1
            G.fill_model(prod_t, specs, seed, v, stream=st)
            if flush_buf is not None:  # None: warm L2 (the optimizer's writes of v are still cached)
                flush_l2(G, flush_buf, st, dirty=dirty)
            if kernel_timing:
                torch.cuda._sleep(400_000)
            else:
                torch.cuda.synchronize()
            ev0.record(st)
            t0 = time.perf_counter()
            prod.publish(v, stream=st)
            t1 = time.perf_counter()
            ev1.record(st)
            ev1.synchronize()
            if i >= warmup:
                dev_ms.append(ev0.elapsed_time(ev1))
                host_ms.append((t1 - t0) * 1e3)
                if kernel_timing:
                    ps = prod.stats()
                    pack_us.append(ps["t_pack_dev_us"])
                    fused_us.append(ps["t_fused_dev_us"])
                    inst_us.append(cons.stats()["t_install_dev_us"])
        ok = True
        for c, ct in zip(conss, cons_ts):
            view = c.acquire_latest()
            ok = ok and view.version == warmup + steps and all(
                torch.equal(g.view(torch.uint8), p.view(torch.uint8)) for g, p in zip(view.tensors(ct), prod_t))
            c.release(view)
        s_packed = prod.stats()["s_packed"]
        nchunks = prod.stats()["nchunks"]
    finally:
        for c in conss:
            c.close()
        prod.close()
    return {"dev_ms": dev_ms, "host_ms": host_ms, "pack_us": pack_us, "install_us": inst_us, "fused_us": fused_us,
            "ok": ok,
            "s_packed": s_packed, "nchunks": nchunks, "bytes": synth.model_bytes(name), "tensors": len(specs)}


def run_back_to_back(V, G, synth, name, steps, warmup):
    """Steady state: K SYNC publishes issued back to back with
    nothing in between (no L2 flush, no optimizer write), one CUDA-event window
    around all K on the publishing stream: every update pays the deferred L2
    write-back of the one before it.  ms per update."""
    import torch
    specs = synth.model_specs(name)
    prod_t, cons_t = G.alloc_model(specs), G.alloc_model(specs)
    G.fill_model(prod_t, specs, synth.SEEDS[name], 1)
    mname = f"b2b-{name}-{os.getpid()}-{time.monotonic_ns()}"
    cons = V.Model(mname, V.CONSUMER, cons_t)
    prod = V.Model(mname, V.PRODUCER, prod_t)
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    try:
        for v in range(1, warmup + 1):
            prod.publish(v, stream=st)
        torch.cuda.synchronize()
        e0.record(st)
        for v in range(warmup + 1, warmup + steps + 1):
            prod.publish(v, stream=st)
        e1.record(st)
        e1.synchronize()
        view = cons.acquire_latest()
        ok = view.version == warmup + steps and all(
            torch.equal(g.view(torch.uint8), p.view(torch.uint8)) for g, p in zip(view.tensors(cons_t), prod_t))
        cons.release(view)
    finally:
        cons.close()
        prod.close()
    return e0.elapsed_time(e1) / steps, ok


def golden_check_local(V, G, synth, name):
    """The N = 1 headline config's bit-exact evidence against the oracle: publish
    VGEN(seed, synth.VCHECK) and compare the producer's chunk seals and the
    consumer's installed-slot seals (viper_view_seals) with the oracle-written
    tests/golden/seals/<name>.txt, plus every byte of the slot with VGEN."""
    import numpy as np
    import torch
    specs = synth.model_specs(name)
    gold = synth.golden_seals(name)
    prod_t, cons_t = G.alloc_model(specs), G.alloc_model(specs)
    G.fill_model(prod_t, specs, synth.SEEDS[name], synth.VCHECK)
    mname = f"gold-{name}-{os.getpid()}-{time.monotonic_ns()}"
    cons = V.Model(mname, V.CONSUMER, cons_t)
    prod = V.Model(mname, V.PRODUCER, prod_t)
    try:
        prod.publish(1)
        _, sp, n = prod.debug_buffers()
        like = torch.empty(4 * n, dtype=torch.int32, device="cuda")
        pseals = V._from_ptr(sp, like).view(torch.int64).cpu().numpy().view(np.uint64).reshape(n, 2)
        view = cons.acquire_latest()
        buf = torch.empty(16 * n, dtype=torch.uint8, device="cuda")
        cons.view_seals(view, buf)
        torch.cuda.synchronize()
        cseals = buf.view(torch.int64).cpu().numpy().view(np.uint64).reshape(n, 2)
        exp = G.alloc_model(specs)
        G.fill_model(exp, specs, synth.SEEDS[name], synth.VCHECK)
        bytes_ok = all(torch.equal(g.view(torch.uint8), e.view(torch.uint8)) for g, e in zip(view.tensors(cons_t), exp))
        cons.release(view)
    finally:
        cons.close()
        prod.close()
    g = np.array(gold[1], dtype=np.uint64) if gold else None
    return {"chunks": n, "producer_seals_ok": bool(g is not None and np.array_equal(pseals[:, 1], g)),
            "consumer_seals_ok": bool(g is not None and np.array_equal(cseals[:, 1], g) and (cseals[:, 0] == 1).all()),
            "bytes_ok": bool(bytes_ok),
            "how": "VGEN(seed, synth.VCHECK) published; every chunk seal of the snapshot and of the consumer's "
                   "installed slot (viper_view_seals) == the oracle's tests/golden/seals file; every slot byte == VGEN"}


def run_e2e(V, G, synth, name, steps, warmup, flush_buf):
    """Same update through the public API with HOST buffers: the trainer's
    parameters live in one flat device buffer (tensor views at 256-B aligned
    offsets); each step copies the new weights from a flat pinned host buffer
    (one cudaMemcpyAsync H2D), publishes, and reads the chunk-seal digest of
    the installed version back (D2H)."""
    import torch
    specs = synth.model_specs(name)
    seed = synth.SEEDS[name]
    offs, off = [], 0
    for s_ in specs:
        offs.append(off)
        off = (off + synth.nbytes_of(s_) + 255) // 256 * 256
    flat = torch.empty(max(off, 256), dtype=torch.uint8, device="cuda")
    dt = {synth.F32: torch.float32, synth.BF16: torch.bfloat16, synth.F16: torch.float16}
    prod_t = [flat[o:o + synth.nbytes_of(s_)].view(dt.get(s_[1], torch.uint8)).view(s_[2])
              for o, s_ in zip(offs, specs)]
    cons_t = G.alloc_model(specs)
    host = []
    for i in range(2):  # two host versions of the whole flat buffer, alternated
        G.fill_model(prod_t, specs, seed, 1000 + i)
        hb = G.PinnedBuffer(flat.numel())
        hb.view()[:] = flat.cpu().numpy()
        host.append(hb)
    mname = f"e2e-{name}-{os.getpid()}-{time.monotonic_ns()}"
    cons = V.Model(mname, V.CONSUMER, cons_t)
    prod = V.Model(mname, V.PRODUCER, prod_t)
    st = torch.cuda.current_stream()
    _, _, nchunks = prod.debug_buffers()
    digest = G.PinnedBuffer(16 * nchunks)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    times = []
    try:
        for i in range(warmup + steps):
            flush_l2(G, flush_buf, st)
            torch.cuda.synchronize()
            ev0.record(st)
            host[i % 2].to_device(flat, stream=st)
            prod.publish(i + 1, stream=st)
            _, seals_ptr, _ = prod.debug_buffers()
            digest.from_device_ptr(seals_ptr, 16 * nchunks, stream=st)
            ev1.record(st)
            ev1.synchronize()
            if i >= warmup:
                times.append(ev0.elapsed_time(ev1))
        d = digest.view().view("<u8").reshape(nchunks, 2)
        ok = bool((d[:, 0] == warmup + steps).all())
    finally:
        cons.close()
        prod.close()
        for hb in host:
            hb.close()
        digest.close()
    return {"ms": statistics.mean(times), "h2d": flat.numel(), "d2h": 16 * nchunks, "ok": ok}


def c3_concurrent(V, G, synth, seconds=1.5, period_ms=2.0, install_sms=0, reader_kind="verify"):
    """BASELINE.json configs[2] in 1-GPU loopback: ViT-B/16 bf16 consumer serving
    while ASYNC updates land.  A reader thread loops acquire -> read every weight
    byte and compare with VGEN(view.version) on the GPU (a bandwidth-heavy
    stand-in for inference) -> stream-ordered release.  Reports
    verified views/s without and with publishes every `period_ms`, torn views
    (must be 0) and the install latency seen by the consumer.
    reader_kind="gemm": a compute-bound stand-in instead -- per view, the 48
    linear layers of the 12 encoder blocks (in_proj, out_proj, mlp.0, mlp.3,
    bf16 tensor cores) over a batch of 64 images x 197 tokens, using the
    view's weights."""
    import threading
    import torch
    name = "vit_b16"
    specs = synth.model_specs(name)
    seed = synth.SEEDS[name]
    pt, ct = G.alloc_model(specs), G.alloc_model(specs)
    mname = f"c3-{os.getpid()}-{time.monotonic_ns()}"
    cons = V.Model(mname, V.CONSUMER, ct, install_sms=install_sms)
    prod = V.Model(mname, V.PRODUCER, pt, mode=V.ASYNC)
    G.fill_model(pt, specs, seed, 1)
    prod.publish(1)
    cons.wait_installed(1)
    stop = threading.Event()
    stats = {"views": 0, "torn": 0, "regress": 0}

    def reader():
        torch.cuda.set_device(torch.cuda.current_device())
        s = torch.cuda.Stream()
        exp = G.alloc_model(specs)
        last = 0
        lin = [i for i, sp in enumerate(specs) if len(sp[2]) == 2 and sp[2][1] in (768, 3072) and "encoder" in sp[0]]
        x0 = torch.randn(64 * 197, 768, dtype=torch.bfloat16, device="cuda") if reader_kind == "gemm" else None
        with torch.cuda.stream(s):
            while not stop.is_set() and reader_kind == "gemm":
                view = cons.acquire_latest(timeout_us=100_000)
                w = view.tensors(ct)
                x = x0
                for i in lin:  # x @ W^T through the encoder's linear layers (shapes chain per block)
                    y = x @ w[i].t()
                    x = y[:, :768] if y.shape[1] == 2304 else y
                cons.release(view, stream=s)
                s.synchronize()
                stats["views"] += 1
            while not stop.is_set() and reader_kind == "verify":
                view = cons.acquire_latest(timeout_us=100_000)
                G.fill_model(exp, specs, seed, view.version, stream=s)
                bad = torch.zeros((), dtype=torch.int64, device="cuda")
                for g, e in zip(view.tensors(ct), exp):
                    bad += (g.view(torch.uint8) != e.view(torch.uint8)).sum()
                cons.release(view, stream=s)
                torn = int(bad.item())
                stats["torn"] += int(torn > 0)
                stats["regress"] += int(view.version < last)
                last = view.version
                stats["views"] += 1

    def phase(publish):
        stats["views"] = 0
        th = threading.Thread(target=reader)
        th.start()
        t0 = time.perf_counter()
        v = prod.stats()["version"]
        ps = torch.cuda.Stream()
        n = 0
        while time.perf_counter() - t0 < seconds:
            if publish:
                v += 1
                with torch.cuda.stream(ps):
                    G.fill_model(pt, specs, seed, v, stream=ps)
                    prod.publish(v, stream=ps)
                n += 1
            time.sleep(period_ms / 1e3)
        stop.set()
        th.join()
        stop.clear()
        return stats["views"] / (time.perf_counter() - t0), n

    try:
        base, _ = phase(False)
        busy, npub = phase(True)
        cons.wait_installed(prod.stats()["version"])
        cst = cons.stats()
    finally:
        cons.close()
        prod.close()
    return {"workload": "vit_b16 bf16 1 producer -> 1 consumer (1-GPU loopback), ASYNC, publish every "
                        f"{period_ms} ms", "install_sms": install_sms or "all", "reader_kind": reader_kind,
            "reader": "acquire -> byte-compare every weight with VGEN -> release" if reader_kind == "verify" else
                      "acquire -> 48 encoder linears (bf16 GEMMs, 64 x 197 tokens) on the view's weights -> release",
            "views_per_s_idle": round(base, 1), "views_per_s_during_updates": round(busy, 1),
            "throughput_drop": round(1 - busy / base, 4) if base else None, "publishes": npub,
            "installs": cst["installs"], "skipped": cst["skipped"], "torn_views": stats["torn"],
            "version_regressions": stats["regress"], "last_install_us": round(cst["t_install_us"], 1),
            "last_pickup_us": round(cst["t_notify_us"], 1),
            "pickup_note": "publish -> update-thread pickup, includes waiting for the previous install"}


def c5_schedule(V, G, synth, flush, gpu_row):
    """BASELINE.json configs[4]: Llama-3 8B through the pinned-DRAM tier vs the
    GPU tier (1-GPU loopback here), each driving viper_schedule (the paper's
    IPP, s4.3) with the engine's measured costs: t_p = producer stall (the
    pack for the GPU tier; pack + host copy for DRAM), t_c =
    consumer load (the install / H2D + install), on a synthetic Exp3 warm-up
    loss curve with the paper's Fig. 6 time magnitudes."""
    import numpy as np
    d = run_update_bench(V, G, synth, "llama3_8b", 3, 2, flush, tier=V.TIER_DRAM)
    dram_ms = statistics.mean(d["dev_ms"])
    gpu_ms = gpu_row.get("latency_ms")
    rng = np.random.default_rng(5)
    x = np.arange(50.0)
    warm = list(2.5 * np.exp(-0.02 * x) + 0.8 + rng.normal(0, 0.01, 50))
    t_train, t_infer = 0.07, 0.006
    s_iter, e_iter = 50, 2000
    total = int((e_iter - s_iter) * t_train / t_infer)
    res = {"dram_update_ms": round(dram_ms, 3), "gpu_update_ms": gpu_ms,
           "dram_over_gpu": round(dram_ms / gpu_ms, 2) if gpu_ms else None,
           "paper_context": "TC1 Host-Async / GPU-Async latency 2.326 s / 0.856 s = 2.7x (Polaris, inter-node)"}
    for tier, t_p, t_c in (("gpu", gpu_row.get("pack_us", 0) * 1e-6, gpu_row.get("install_us", 0) * 1e-6),
                           ("dram", dram_ms * 1e-3 / 2, dram_ms * 1e-3 / 2)):
        sch = V.schedule(warm, s_iter=s_iter, e_iter=e_iter, total_infers=total, t_train=t_train, t_infer=t_infer,
                         t_p=t_p, t_c=t_c, x=list(x))
        gr = V.schedule(warm, s_iter=s_iter, e_iter=e_iter, total_infers=total, t_train=t_train, t_infer=t_infer,
                        t_p=t_p, t_c=t_c, x=list(x), algo=V.SCHED_GREEDY)
        res[tier] = {"t_p_s": t_p, "t_c_s": t_c, "family": ["Exp2", "Exp3", "Lin2", "Expd3"][sch["family"]],
                     "fixed_interval": sch["best_interval"], "fixed_cil": round(sch["predicted_cil"], 3),
                     "greedy_checkpoints": len(gr["sched"]), "greedy_cil": round(gr["predicted_cil"], 3)}
    return res


def schedule_from_costs(V, costs):
    """viper_schedule (the paper's IPP, s4.3) driven by measured update costs,
    on the synthetic Exp3 warm-up curve and Fig. 6 time magnitudes of
    c5_schedule: costs = {name: (t_p seconds, t_c seconds)}."""
    import numpy as np
    rng = np.random.default_rng(5)
    x = np.arange(50.0)
    warm = list(2.5 * np.exp(-0.02 * x) + 0.8 + rng.normal(0, 0.01, 50))
    t_train, t_infer = 0.07, 0.006
    s_iter, e_iter = 50, 2000
    total = int((e_iter - s_iter) * t_train / t_infer)
    out = {}
    for nm, (t_p, t_c) in costs.items():
        sch = V.schedule(warm, s_iter=s_iter, e_iter=e_iter, total_infers=total, t_train=t_train, t_infer=t_infer,
                         t_p=t_p, t_c=t_c, x=list(x))
        gr = V.schedule(warm, s_iter=s_iter, e_iter=e_iter, total_infers=total, t_train=t_train, t_infer=t_infer,
                        t_p=t_p, t_c=t_c, x=list(x), algo=V.SCHED_GREEDY)
        out[nm] = {"t_p_s": t_p, "t_c_s": t_c, "family": ["Exp2", "Exp3", "Lin2", "Expd3"][sch["family"]],
                   "fixed_interval": sch["best_interval"], "fixed_cil": round(sch["predicted_cil"], 3),
                   "greedy_checkpoints": len(gr["sched"]), "greedy_cil": round(gr["predicted_cil"], 3)}
    return out


def torch_copy_baseline(G, synth, name, flush_buf, steps=10, warmup=3):
    """the naive state-dict copy -- one torch copy_ per tensor from
    the producer's to the consumer's parameters (no snapshot, no seal, no
    verification, no atomic swap: a reader can see a torn model).  Timed like
    the update: CUDA events around the copies, L2 flushed before each."""
    import torch
    specs = synth.model_specs(name)
    pt, ct = G.alloc_model(specs), G.alloc_model(specs)
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ms = []
    for i in range(warmup + steps):
        flush_l2(G, flush_buf, st)
        torch.cuda.synchronize()
        e0.record(st)
        for d, s in zip(ct, pt):
            d.copy_(s)
        e1.record(st)
        e1.synchronize()
        if i >= warmup:
            ms.append(e0.elapsed_time(e1))
    del pt, ct
    return statistics.mean(ms)


def event_floor_us(G, reps=20):
    """An empty kernel bracketed exactly like the library's timing events."""
    import torch
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    out = []
    for _ in range(reps):
        torch.cuda._sleep(200_000)
        e0.record(st)
        G.empty_kernel(stream=st)
        e1.record(st)
        e1.synchronize()
        out.append(e0.elapsed_time(e1) * 1e3)
    return statistics.median(out)


def cpu_model():
    """Host CPU model, the cores this process may use, and its NUMA node."""
    model = "unknown"
    try:
        with open("/proc/cpuinfo") as f:
            model = next((l.split(":", 1)[1].strip() for l in f if l.startswith("model name")), model)
    except OSError:
        pass
    node = None
    try:
        import glob
        cpu0 = min(os.sched_getaffinity(0))
        node = next((int(p.split("node")[-1].split("/")[0]) for p in glob.glob(f"/sys/devices/system/cpu/cpu{cpu0}/node*")),
                    None)
    except (OSError, ValueError):
        pass
    return {"model": model, "affinity_cores": len(os.sched_getaffinity(0)), "numa_node": node}


class OracleUpdates:
    """The oracle (plain C, single thread, as it stands) set up once for one
    config: a producer + `ncons` consumers and two pre-generated versions.
    `subset`: only these tensor indices (the P-thread baseline gives each
    thread a disjoint subset, its own oracle channel)."""

    def __init__(self, synth, name, ncons=1, subset=None):
        from oracle import transfer as T
        self.T, self.name = T, name
        specs = synth.model_specs(name)
        seed = synth.SEEDS[name]
        idx = list(range(len(specs))) if subset is None else list(subset)
        nb = [synth.nbytes_of(specs[i]) for i in idx]
        self.versions = [[synth.vgen_numpy(seed, v, i, specs[i][1], synth.nelem_of(specs[i])) for i in idx]
                         for v in (1, 2)]
        self.cs = [self.T.Consumer(nb) for _ in range(ncons)]
        self.p = self.T.Producer(nb, self.cs)
        self.v = 0

    def one(self):
        self.v += 1
        st = self.p.publish(self.v, self.versions[self.v % 2])
        assert st == self.T.OK

    def run(self, budget_s, max_updates=100000):
        """Updates until the budget is spent; ms per update."""
        times = []
        t_start = time.perf_counter()
        while time.perf_counter() - t_start < budget_s and len(times) < max_updates:
            t0 = time.perf_counter()
            self.one()
            times.append((time.perf_counter() - t0) * 1e3)
        return times

    def close(self):
        self.p.close()
        for c in self.cs:
            c.close()


def oracle_parallel(synth, name, nthreads, budget_s, max_updates=100000):
    """P-thread oracle baseline: the model's tensors split into
    P disjoint subsets of about equal bytes, each its own oracle channel (plain
    C, single-threaded, unchanged) driven by its own thread; one update = every
    thread updating its subset (the ctypes calls release the GIL).  ms per
    whole-model update."""
    specs = synth.model_specs(name)
    order = sorted(range(len(specs)), key=lambda i: -synth.nbytes_of(specs[i]))
    groups, load = [[] for _ in range(nthreads)], [0] * nthreads
    for i in order:  # greedy: largest tensor to the lightest group
        k = load.index(min(load))
        groups[k].append(i)
        load[k] += synth.nbytes_of(specs[i])
    groups = [sorted(g) for g in groups if g]
    parts = [OracleUpdates(synth, name, subset=g) for g in groups]
    times = []
    try:
        t_start = time.perf_counter()
        while time.perf_counter() - t_start < budget_s and len(times) < max_updates:
            ths = [threading.Thread(target=o.one) for o in parts]
            t0 = time.perf_counter()
            for th in ths:
                th.start()
            for th in ths:
                th.join()
            times.append((time.perf_counter() - t0) * 1e3)
    finally:
        for o in parts:
            o.close()
    return times, len(parts)


def cpu_baseline(synth, name, budget_s=10.0, max_updates=100000):
    """The oracle timed on this host's cores on a bounded sample: repeated
    updates of the same config, on 1 thread (the value) and on P threads
    (P = the cores this process may use)."""
    o = OracleUpdates(synth, name)
    try:
        times = o.run(budget_s, max_updates)
    finally:
        o.close()
    cpu = cpu_model()
    ptimes, p = oracle_parallel(synth, name, cpu["affinity_cores"], budget_s, max_updates)
    return {"value": statistics.mean(times), "unit": "ms", "cores": 1, "kind": "oracle", "cpu": cpu,
            "sample": f"{len(times)} oracle updates of {name} (pack+seal+deliver+verify+install+swap, 1 consumer)",
            "p_threads": {"value": statistics.mean(ptimes), "unit": "ms", "cores": p, "kind": "oracle",
                          "sample": f"{len(ptimes)} whole-model updates of {name}, the tensors split into {p} "
                                    f"disjoint subsets of about equal bytes, one oracle channel and thread each"}}


N_CONFIG = {2: "resnet50", 4: "vit_b16", 8: "gpt2_xl"}  # BASELINE.json configs[1..3]
CONFIG_INDEX = {"ptychonn": 0, "resnet50": 1, "vit_b16": 2, "gpt2_xl": 3, "llama3_8b": 4}


def ce_baseline(rank, group, buf, steps, warmup):
    """SURVEY B2 (baseline only): copy-engine delivery.  Rank 0 shares its
    S-byte buffer through CUDA IPC (torch's own reduction), every consumer
    copies it into a local buffer at the same time (torch copy_ across devices:
    cudaMemcpyPeerAsync on the copy engine), device-timed per consumer.
    Returns this rank's mean ms (0 on the producer)."""
    import torch
    import torch.distributed as dist
    from torch.multiprocessing.reductions import reduce_tensor
    obj = [reduce_tensor(buf) if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    ms = []
    peer = local = None
    if rank != 0:
        fn, fargs = obj[0]
        peer = fn(*fargs)
        local = torch.empty_like(buf)
    for i in range(warmup + steps):
        torch.cuda.synchronize()
        dist.barrier(group=group)
        if rank != 0:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            local.copy_(peer, non_blocking=True)
            e1.record()
            e1.synchronize()
            if i >= warmup:
                ms.append(e0.elapsed_time(e1))
    del peer, local
    torch.cuda.synchronize()
    dist.barrier(group=group)  # the producer's buffer outlives every mapping
    return statistics.mean(ms) if ms else 0.0


def xproc_e2e(V, G, synth, name, rank, world, dev, group, fanout, flush_buf, steps, warmup):
    """The N > 1 update end to end through the public API with HOST buffers
    (the N = 1 run_e2e across processes).  Rank 0's parameters live in one flat
    device buffer; each step copies the step's weights from a pinned host
    buffer (one H2D of S bytes), publishes SYNC (returns after every consumer
    swapped), and reads the chunk-seal digest back (D2H).  Rank 0's host clock
    around the three; the consumers only take part in the publishes."""
    import torch
    import torch.distributed as dist
    specs = synth.model_specs(name)
    offs, off = [], 0
    for s_ in specs:
        offs.append(off)
        off = (off + synth.nbytes_of(s_) + 255) // 256 * 256
    dt = {synth.F32: torch.float32, synth.BF16: torch.bfloat16, synth.F16: torch.float16}
    flat = torch.empty(max(off, 256), dtype=torch.uint8, device="cuda")
    tensors = [flat[o:o + synth.nbytes_of(s_)].view(dt.get(s_[1], torch.uint8)).view(s_[2])
               for o, s_ in zip(offs, specs)]
    host, digest = [], None
    if rank == 0:
        for i in range(2):  # two host versions of the whole flat buffer, alternated
            G.fill_model(tensors, specs, synth.SEEDS[name], 1000 + i)
            hb = G.PinnedBuffer(flat.numel())
            hb.view()[:] = flat.cpu().numpy()
            host.append(hb)
    bs = V.Bootstrap(rank, world, producer_rank=0, group=group)
    m = V.Model(f"bench-x-e2e-{name}", V.PRODUCER if rank == 0 else V.CONSUMER, tensors, fanout=fanout,
                device=dev, bootstrap=bs)
    times, ok, nchunks = [], True, 0
    try:
        if rank == 0:
            _, _, nchunks = m.debug_buffers()
            digest = G.PinnedBuffer(16 * nchunks)
        st = torch.cuda.current_stream()
        for i in range(warmup + steps):
            flush_l2(G, flush_buf, st)
            torch.cuda.synchronize()
            dist.barrier(group=group)
            if rank == 0:
                t0 = time.perf_counter()
                host[i % 2].to_device(flat, stream=st)
                try:
                    m.publish(i + 1, stream=st)
                except V.ViperError:  # reported as digest_ok = false, the ranks stay in step
                    ok = False
                _, seals_ptr, _ = m.debug_buffers()
                digest.from_device_ptr(seals_ptr, 16 * nchunks, stream=st)
                st.synchronize()
                if i >= warmup:
                    times.append((time.perf_counter() - t0) * 1e3)
            dist.barrier(group=group)
        if rank == 0:
            d = digest.view().view("<u8").reshape(nchunks, 2)
            ok = ok and bool((d[:, 0] == warmup + steps).all())
    finally:
        if rank != 0:  # consumers first, as in xproc_arm
            m.close()
        dist.barrier(group=group)
        if rank == 0:
            m.close()
        for hb in host:
            hb.close()
        if digest is not None:
            digest.close()
    return {"ms": statistics.mean(times) if times else 0.0, "h2d": flat.numel(), "d2h": 16 * nchunks, "ok": ok}


# include/viper.h VIPER_FANOUT_*; "dram" (-1) = the pinned-DRAM tier (BASELINE configs[4]: DRAM-to-DRAM
# staging vs direct GPU-to-GPU), direct fan-out
FANOUTS = {"direct": 0, "chain": 1, "sa": 2, "nvls": 3, "push": 4, "nccl": 100, "ce": 101, "dram": -1}
FANOUT_NAMES = {0: "direct pull", 1: "pipelined chain", 2: "scatter-allgather", 3: "NVLS multicast",
                4: "push (producer stores into peer staging)", 100: "NCCL broadcast (engine baseline)",
                101: "copy engine (engine baseline)", -1: "pinned-DRAM tier (D2H -> shared host staging -> H2D)"}
NVLINK_GBS = 900.0  # NVLink 5 per direction per GPU (north_star / B200_PROFILING.md)


def log(msg):
    """Progress of the N > 1 arm on stderr (rank-tagged; the JSON line stays alone on stdout)."""
    print(f"[bench rank {os.environ.get('RANK', '0')} {time.strftime('%H:%M:%S')}] {msg}", file=sys.stderr, flush=True)


def verify_replicas(V, G, synth, m, name, rank, tensors, dev):
    """Bit-exact evidence for one cross-process run, without the oracle at bench
    time: the LAST published version carries VGEN(seed, synth.VCHECK), whose
    chunk checksums tools/make_golden_seals.py wrote with the oracle into
    tests/golden/seals/<name>.txt.  Each consumer computes the chunk seals of
    its installed slot on its GPU (viper_view_seals) and compares EVERY chunk
    with that file, then compares every byte of every tensor with VGEN
    regenerated on its GPU; the producer compares its snapshot seals.  Returns
    {"seals_ok", "bytes_ok", "chunks", "version"}."""
    import numpy as np
    import torch
    gold = synth.golden_seals(name)
    specs = synth.model_specs(name)
    out = {"seals_ok": None, "bytes_ok": None, "chunks": 0, "version": 0}
    if rank == 0:
        _, sp, n = m.debug_buffers()
        like = torch.empty(4 * n, dtype=torch.int32, device=f"cuda:{dev}")
        seals = V._from_ptr(sp, like).view(torch.int64).cpu().numpy().view(np.uint64).reshape(n, 2)
        out["version"] = int(seals[0, 0]) if n else 0
        if gold is not None:
            out["seals_ok"] = bool(n == gold[0]["nchunks"] and all(int(seals[c, 1]) == gold[1][c] for c in range(n)))
            out["chunks"] = n
        return out
    view = m.acquire_latest(timeout_us=30_000_000)
    try:
        n = m.stats()["nchunks"]
        buf = torch.empty(max(16 * n, 16), dtype=torch.uint8, device=f"cuda:{dev}")
        st = torch.cuda.current_stream()
        m.view_seals(view, buf, stream=st)
        st.synchronize()
        got = buf.view(torch.int64).cpu().numpy().view(np.uint64).reshape(-1, 2)[:n]
        out["version"] = int(view.version)
        out["chunks"] = n
        if gold is not None:
            out["seals_ok"] = bool(n == gold[0]["nchunks"] and (got[:, 0] == view.version).all()
                                   and all(int(got[c, 1]) == gold[1][c] for c in range(n)))
        exp = G.alloc_model(specs, device=f"cuda:{dev}")
        G.fill_model(exp, specs, synth.SEEDS[name], synth.VCHECK)
        out["bytes_ok"] = bool(all(torch.equal(g.view(torch.uint8), e.view(torch.uint8))
                                   for g, e in zip(view.tensors(tensors), exp)))
        del exp
    finally:
        m.release(view)
    return out


def xproc_updates(V, G, synth, name, rank, world, dev, gloo, fanout, flush, steps, warmup):
    """One fan-out, SYNC updates.  Per step (untimed): VGEN(v) into the
    producer's tensors, an L2 flush on every rank, barrier.  Timed: CUDA events
    on rank 0's stream around publish(v), which returns only once every
    consumer's install kernel swapped its version word (so the window holds the
    whole pack -> NVLink -> install pipeline); host clock beside it.  Consumers
    report their install kernel's CUDA-event time (VIPER_FLAG_TIMING).  Then the
    verification version (verify_replicas).  Returns this rank's dict, or
    {"unsupported": why} on every rank when registration says so (NVLS without
    multicast, ...)."""
    import torch
    import torch.distributed as dist
    specs = synth.model_specs(name)
    seed = synth.SEEDS[name]
    tensors = G.alloc_model(specs)
    bs = V.Bootstrap(rank, world, producer_rank=0, group=gloo)
    log(f"{name} fan-out {fanout}: registering")
    tier = V.TIER_DRAM if fanout == FANOUTS["dram"] else V.TIER_GPU
    try:
        m = V.Model(f"bench-x-{name}-{fanout}", V.PRODUCER if rank == 0 else V.CONSUMER, tensors,
                    fanout=max(fanout, 0), tier=tier, flags=V.FLAG_TIMING if rank else 0, device=dev, bootstrap=bs)
    except V.ViperError as e:
        log(f"fan-out {fanout}: {e.name}")
        del tensors
        torch.cuda.empty_cache()
        return {"unsupported": f"{e.name}: {e.detail}"[:300]}
    st = torch.cuda.current_stream()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    lat, host, inst, pick, ihost = [], [], [], [], []
    errors = []

    def any_error():  # every rank learns of any rank's failure, so all leave the loop together
        t = torch.tensor([1.0 if errors else 0.0])
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=gloo)
        return bool(t.item())

    ver = {"seals_ok": None, "bytes_ok": None, "chunks": 0, "version": 0}
    s_packed = 0
    # BENCH_TEST_FAULT=<fan-out name> (tests): consumer rank 1 corrupts its install of v2, so the line must
    # report that fan-out's error and carry on with the others
    fault = os.environ.get("BENCH_TEST_FAULT") == next((k for k, c in FANOUTS.items() if c == fanout), None)
    try:
        for i in range(warmup + steps):
            v = i + 1
            if fault and rank == 1 and v == 2:
                m.fault_next()
            if rank == 0:
                G.fill_model(tensors, specs, seed, v)
            flush_l2(G, flush)
            torch.cuda.synchronize()
            dist.barrier(group=gloo)
            if rank == 0:
                ev0.record(st)
                t0 = time.perf_counter()
                try:
                    m.publish(v, stream=st)
                except V.ViperError as e:  # reported in the line, never a hang or a lost line
                    errors.append(f"publish({v}): {e.name}: {e.detail}"[:300])
                t1 = time.perf_counter()
                ev1.record(st)
                ev1.synchronize()
                if i >= warmup:
                    lat.append(ev0.elapsed_time(ev1))
                    host.append((t1 - t0) * 1e3)
            dist.barrier(group=gloo)
            if rank != 0 and i >= warmup:
                cs = m.stats()
                inst.append(cs["t_install_dev_us"])
                pick.append(cs["t_pickup_us"])
                ihost.append(cs["t_install_us"])
                if cs["last_status"] != V.OK:
                    errors.append(f"install of v{v}: {V.lib().viper_strerror(cs['last_status']).decode()}")
            if any_error():
                break
        if not any_error():
            log(f"fan-out {fanout}: {steps} timed updates done; verification version")
            # verification version: the golden content
            if rank == 0:
                G.fill_model(tensors, specs, seed, synth.VCHECK)
                torch.cuda.synchronize()
            dist.barrier(group=gloo)
            if rank == 0:
                try:
                    m.publish(warmup + steps + 1, stream=st)
                except V.ViperError as e:
                    errors.append(f"verification publish: {e.name}: {e.detail}"[:300])
                st.synchronize()
            dist.barrier(group=gloo)
            try:
                ver = verify_replicas(V, G, synth, m, name, rank, tensors, dev)
            except V.ViperError as e:
                errors.append(f"verification: {e.name}: {e.detail}"[:300])
            ver["version_ok"] = ver["version"] == warmup + steps + 1
            log(f"fan-out {fanout}: verified {ver}")
        s_packed = m.stats()["s_packed"]
    finally:
        log(f"fan-out {fanout}: closing")
        dist.barrier(group=gloo)
        if rank != 0:  # consumers first: they read the producer's buffers
            m.close()
        dist.barrier(group=gloo)
        if rank == 0:
            m.close()
        del tensors
        torch.cuda.empty_cache()
        log(f"fan-out {fanout}: closed")
    return {"lat": lat, "host": host, "inst": inst, "pick": pick, "ihost": ihost, "verify": ver, "s_packed": s_packed,
            "errors": errors}


def gather_obj(obj, gloo):
    import torch.distributed as dist
    out = [None] * dist.get_world_size(group=gloo)
    dist.all_gather_object(out, obj, group=gloo)
    return out


def summarize_fanout(per_rank, S):
    """Rank 0's view of one fan-out: value = the max over ranks of each rank's
    device-timed update window (the producer's CUDA events bracket every
    consumer's swap; a consumer's own window is its install kernel)."""
    if any("unsupported" in r for r in per_rank):
        return {"unsupported": next(r["unsupported"] for r in per_rank if "unsupported" in r)}
    errs = [f"rank {i}: {e}" for i, r in enumerate(per_rank) for e in r.get("errors", [])]
    if errs or not per_rank[0]["lat"]:
        return {"error": errs[:4] or ["no timed update"], "parity_ok": False}
    p = per_rank[0]
    lat_ms = statistics.mean(p["lat"])
    inst_us = [statistics.median(r["inst"]) if r["inst"] else 0.0 for r in per_rank[1:]]
    win = max([lat_ms] + [u / 1e3 for u in inst_us])
    ver = [r["verify"] for r in per_rank]
    return {
        "latency_ms": round(win, 6), "latency_p50_ms": round(statistics.median(p["lat"]), 6),
        "latency_min_ms": round(min(p["lat"]), 6), "host_latency_ms": round(statistics.mean(p["host"]), 6),
        "update_gbps_per_consumer": round(S / (win * 1e-3) / 1e9, 3),
        "nvlink_frac": round(S / (win * 1e-3) / 1e9 / NVLINK_GBS, 4),
        "install_kernel_us_per_consumer": [round(u, 3) for u in inst_us],
        "host_path_us_per_consumer": [
            {"pickup": round(statistics.median(r["pick"]), 1) if r.get("pick") else None,
             "install_host": round(statistics.median(r["ihost"]), 1) if r.get("ihost") else None}
            for r in per_rank[1:]],
        "host_path_how": "median per consumer: pickup = producer's publish entry -> the consumer's update thread "
                         "picks v up; install_host = pickup -> install kernel done, seen by that thread",
        "install_kernel_nvlink_frac": round(S / (max(inst_us) * 1e-6) / 1e9 / NVLINK_GBS, 4) if max(inst_us) else None,
        "parity": {"producer_seals_ok": ver[0]["seals_ok"],
                   "consumers": [{"rank": i + 1, "seals_ok": v["seals_ok"], "bytes_ok": v["bytes_ok"],
                                  "chunks": v["chunks"], "version_ok": v["version_ok"]} for i, v in enumerate(ver[1:])]},
        "parity_ok": bool(ver[0]["seals_ok"] is not False and all(
            v["seals_ok"] and v["bytes_ok"] and v["version_ok"] for v in ver[1:])),
    }


def xproc_concurrent(V, G, synth, name, rank, world, dev, gloo, fanout, seconds=2.0, period_ms=2.0):
    """BASELINE.json configs[2] across processes: each consumer serves while
    ASYNC updates land.  A reader thread per consumer loops acquire -> compare
    every weight byte with VGEN(view.version) on its GPU -> stream-ordered
    release; the producer publishes every `period_ms`.  Counts views, torn
    views (must be 0) and version regressions; views/s idle vs during updates."""
    import threading
    import torch
    import torch.distributed as dist
    specs = synth.model_specs(name)
    seed = synth.SEEDS[name]
    tensors = G.alloc_model(specs)
    bs = V.Bootstrap(rank, world, producer_rank=0, group=gloo)
    try:
        m = V.Model(f"bench-xc-{name}", V.PRODUCER if rank == 0 else V.CONSUMER, tensors, fanout=fanout,
                    mode=V.ASYNC, device=dev, bootstrap=bs)
    except V.ViperError as e:
        return {"unsupported": f"{e.name}: {e.detail}"[:300]}
    res = {"views_idle": 0.0, "views_busy": 0.0, "torn": 0, "regress": 0, "publishes": 0, "installs": 0, "errors": []}

    def guarded(fn, *a, **k):  # a failure is reported in the line; the ranks stay in step
        try:
            return fn(*a, **k)
        except V.ViperError as e:
            res["errors"].append(f"{e.name}: {e.detail}"[:200])
            return None

    try:
        if rank == 0:
            G.fill_model(tensors, specs, seed, 1)
            guarded(m.publish, 1)
            torch.cuda.synchronize()
        else:
            guarded(m.wait_installed, 1, timeout_us=30_000_000)
        stop = threading.Event()
        cnt = {"views": 0, "torn": 0, "regress": 0}

        def reader():
            torch.cuda.set_device(dev)
            s = torch.cuda.Stream()
            exp = G.alloc_model(specs, device=f"cuda:{dev}")
            last = 0
            with torch.cuda.stream(s):
                while not stop.is_set():
                    try:
                        view = m.acquire_latest(timeout_us=100_000)
                    except V.ViperError:
                        continue
                    G.fill_model(exp, specs, seed, view.version, stream=s)
                    bad = torch.zeros((), dtype=torch.int64, device=f"cuda:{dev}")
                    for g, e in zip(view.tensors(tensors), exp):
                        bad += (g.view(torch.uint8) != e.view(torch.uint8)).sum()
                    m.release(view, stream=s)
                    cnt["torn"] += int(int(bad.item()) > 0)
                    cnt["regress"] += int(view.version < last)
                    last = view.version
                    cnt["views"] += 1

        for phase in ("idle", "busy"):
            log(f"concurrent acquire: {phase}")
            dist.barrier(group=gloo)
            cnt["views"] = 0
            th = threading.Thread(target=reader) if rank else None
            if th:
                th.start()
            t0 = time.perf_counter()
            if rank == 0:
                v = m.stats()["version"]
                ps = torch.cuda.Stream()
                while time.perf_counter() - t0 < seconds:
                    if phase == "busy":
                        v += 1
                        with torch.cuda.stream(ps):
                            G.fill_model(tensors, specs, seed, v, stream=ps)
                            guarded(m.publish, v, stream=ps)
                        res["publishes"] += 1
                    time.sleep(period_ms / 1e3)
                ps.synchronize()
                last_v = torch.tensor([float(v)])
            else:
                time.sleep(seconds)
                last_v = torch.tensor([0.0])
            dist.all_reduce(last_v, op=dist.ReduceOp.MAX, group=gloo)
            if rank:
                guarded(m.wait_installed, int(last_v.item()), timeout_us=60_000_000)
                stop.set()
                th.join()
                stop.clear()
                res[f"views_{phase}"] = cnt["views"] / (time.perf_counter() - t0)
        res["torn"], res["regress"] = cnt["torn"], cnt["regress"]
        if rank:
            res["installs"] = m.stats()["installs"]
    finally:
        dist.barrier(group=gloo)
        if rank != 0:
            m.close()
        dist.barrier(group=gloo)
        if rank == 0:
            m.close()
        del tensors
        torch.cuda.empty_cache()
    return res


def xproc_line(args, world, name, S, ndev, over, head, results, conc_all, t, e2e, clocks):
    """Rank 0's JSON line of the N > 1 arm.  t = [NCCL broadcast ms, CE pull ms,
    e2e ms, e2e digest failures], max over ranks.  A headline fan-out that
    failed or was unsupported has no latency: the line still prints (value
    null, its errors under `fanouts`)."""
    from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
    h = results[head]
    ok = "latency_ms" in h  # (an unsupported or failed fan-out has no latency: the line still prints)
    lat_ms = h["latency_ms"] if ok else None
    inst = max(h["install_kernel_us_per_consumer"]) if ok else None
    cons = [c for c in conc_all[1:] if "unsupported" not in c]
    out = {
        "metric": METRIC, "value": lat_ms, "unit": "ms", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": lat_ms, "higher_is_better": False, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32", "model_dtype": "f32" if name in ("ptychonn", "resnet50") else "bf16",
        "data": "synthetic (VGEN seeded random-init parameters, BASELINE.json shapes)",
        "config": {"workload": f"{name}: 1 producer -> {world - 1} consumer(s) "
                               f"{'sharing one GPU (code path only, no NVLink)' if over else 'over NVLink'} "
                               f"({FANOUT_NAMES[FANOUTS[head]]}), SYNC",
                   "baseline_config": f"BASELINE.json configs[{CONFIG_INDEX[name]}]", "fanout": head,
                   "model_bytes": S, "devices_visible": ndev, "oversubscribed": over,
                   "l2": "flushed on every rank before every update (256 MiB write + 256 MiB read)",
                   "parallelism": f"1 producer + {world - 1} consumers, one process per GPU"},
        "update_gbps_per_consumer": h.get("update_gbps_per_consumer"),
        "roofline": None if (over or not ok) else {
            "bound": "nvlink", "kernel": "update: pack -> NVLink delivery -> install + verify + swap (pipelined)",
            "achieved": round(S / (lat_ms * 1e-3) / 1e9, 2), "peak": NVLINK_GBS, "unit": "GB/s",
            "frac": round(S / (lat_ms * 1e-3) / 1e9 / NVLINK_GBS, 4), "traffic": None,
            "peak_kind": "NVLink 5 per direction per GPU (north_star; B200_PROFILING.md)",
            "algorithmic_bytes": S, "formula": "f_NVL = (S / L_update) / 900 GB/s (SURVEY s8(d))",
            "install_kernel": {"us": inst, "achieved": round(S / (inst * 1e-6) / 1e9, 2) if inst else None,
                               "frac": h["install_kernel_nvlink_frac"]}},
        "fanouts": results,
        "dram_over_gpu": (round(results["dram"]["latency_ms"] / lat_ms, 3)
                          if ok and "latency_ms" in results.get("dram", {}) else None),
        "dram_over_gpu_how": "BASELINE configs[4]: the pinned-DRAM tier's update latency over the headline "
                             "GPU-to-GPU fan-out, same bytes (paper context: TC1 Host-Async / GPU-Async 2.7x)",
        "schedule": (schedule_from_costs(V, {f: (results[f]["latency_ms"] * 1e-3, 0.0) for f in (head, "dram")
                                             if "latency_ms" in results.get(f, {})})
                     if ok else None),
        "schedule_how": "viper_schedule (IPP, s4.3) per channel with t_p = the measured SYNC update latency "
                        "(the publish returns after every consumer installed) and t_c = 0, on c5_schedule's "
                        "synthetic Exp3 warm-up curve (BASELINE configs[4]: schedule from viper_schedule)",
        "parity_ok": h.get("parity_ok", False),
        "parity": h.get("parity"),
        "nccl_broadcast_ms": None if over else round(float(t[0]), 6),
        "ce_pull_ms": round(float(t[1]), 6),
        "ce_pull_how": "SURVEY B2 baseline: every consumer pulls the producer's S bytes at once with the copy "
                       "engine (torch copy_ from the CUDA-IPC-mapped producer buffer = cudaMemcpyPeerAsync), "
                       "CUDA events, max over consumers",
        "concurrent_acquire": {
            "how": f"ASYNC publish every 2 ms for 2 s ({FANOUT_NAMES[FANOUTS[head]]}); per consumer a reader "
                   "thread acquires, compares every weight byte with VGEN(view.version) on its GPU, releases",
            "torn_views": sum(c["torn"] for c in cons), "version_regressions": sum(c["regress"] for c in cons),
            "views_per_s_idle": [round(c["views_idle"], 1) for c in cons],
            "views_per_s_during_updates": [round(c["views_busy"], 1) for c in cons],
            "publishes": conc_all[0].get("publishes"), "installs": [c["installs"] for c in cons],
            "errors": [e for c in conc_all for e in c.get("errors", [])][:4],
            **({"unsupported": conc_all[0]["unsupported"]} if "unsupported" in conc_all[0] else {})},
        "gpu_launches": (2 + (world - 1)) * args.steps,
        "gpu_launches_how": "per update: pack (+ push / NVLS stores) and seal_reduce on the producer, one "
                            "install per consumer",
        "clocks": clocks,
        "cpu_baseline": None,
        "cpu_baseline_note": "the oracle is timed on rank 0 at N = 1 only (task rule); see the N = 1 line",
        "e2e": {"value": round(float(t[2]), 6), "unit": "ms", "h2d_bytes_per_step": e2e["h2d"],
                "d2h_bytes_per_step": e2e["d2h"], "digest_ok": bool(float(t[3]) == 0.0),
                "how": "rank 0: pinned host -> device copy of the step's weights, SYNC publish (returns "
                       "after every consumer swapped), D2H of the chunk-seal digest; host clock"},
    }
    return out


def xproc_arm(args):
    """N > 1: one process per GPU (self-launched by main() when WORLD_SIZE is
    unset).  Rank 0 is the producer, ranks 1..N-1 the consumers.  The workload
    follows BASELINE.json: N = 2 -> configs[1] ResNet-50 1 -> 1, N = 4 ->
    configs[2] ViT-B/16 1 -> 3 with concurrent acquire, N = 8 -> configs[3]
    GPT-2 XL 1 -> 7 (other N: ResNet-50).  Every fan-out the engine has is
    timed on the same bytes (SYNC updates): the headline is NVLS where the box
    exposes multicast, else scatter-allgather (N > 2) / direct pull (N = 2);
    the others, push, chain, direct star and the engine's copy-engine baseline
    sit beside it, with an NCCL broadcast and a torch copy-engine pull of the
    same bytes as baselines.  Each fan-out's last version is verified on every
    consumer against the oracle's golden chunk seals and byte for byte
    (verify_replicas).  Roofline: f_NVL = (S / L_update) / 900 GB/s (SURVEY
    s8(d)), the install kernel's own S / t_install beside it."""
    import torch
    import torch.distributed as dist
    rank, world, local = dist_env()
    if os.environ.get("BENCH_WATCHDOG_S"):  # debugging: dump every thread's Python stack if the arm stalls
        import faulthandler
        faulthandler.dump_traceback_later(int(os.environ["BENCH_WATCHDOG_S"]), repeat=True)
    if not torch.cuda.is_available() or torch.cuda.device_count() == 0:
        # no GPU (CPU plumbing check of the launcher): rendezvous, max over
        # ranks, one line from rank 0 -- and no number
        dist.init_process_group("gloo")
        t = torch.tensor([float(rank)])
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        if rank == 0:
            print(json.dumps({"metric": METRIC, "value": None, "unit": "ms", "n_gpus": world, "steps": args.steps,
                              "warmup": args.warmup, "higher_is_better": False, "scaling": "weak",
                              "ranks_seen": int(t.item()) + 1,
                              "unavailable": "no CUDA device visible: launcher / rendezvous / max-over-ranks "
                                             "plumbing only, nothing measured"}), flush=True)
        dist.barrier()
        dist.destroy_process_group()
        return
    import synth
    from synth import gpu as G
    from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
    ndev = torch.cuda.device_count()
    over = ndev < world
    if over and not args.oversubscribe:
        raise SystemExit(f"bench.py: {world} ranks but {ndev} visible GPU(s); pass --oversubscribe to run the "
                         f"code path with ranks sharing GPUs (no NVLink is measured then)")
    dev = local % ndev
    torch.cuda.set_device(dev)
    if over:
        dist.init_process_group("gloo")
    else:
        dist.init_process_group("cpu:gloo,cuda:nccl", device_id=torch.device("cuda", dev))
    gloo = dist.new_group(backend="gloo")
    name = args.config if args.config_explicit else N_CONFIG.get(world, "resnet50")
    S = synth.model_bytes(name)
    flush = torch.empty(FLUSH_BYTES, dtype=torch.uint8, device="cuda")
    # the fan-outs to time: headline first
    if args.fanout != "auto":
        order = [args.fanout]
    elif world == 2:
        order = ["direct", "push", "nvls", "ce", "nccl", "dram"]
    else:
        order = ["nvls", "sa", "chain", "push", "direct", "ce", "nccl", "dram"]
    if over and args.fanout == "auto":  # ranks time-slice one GPU: peer waits only serialise
        order = ["direct", "push", "ce", "nccl", "dram"]
    results = {}
    with ClockSampler(dev) as clk:
        for f in order:
            if f == "push" and world - 1 > 8:
                continue
            r = xproc_updates(V, G, synth, name, rank, world, dev, gloo, FANOUTS[f], flush, args.steps, args.warmup)
            per_rank = gather_obj(r, gloo)  # collective: every rank
            results[f] = summarize_fanout(per_rank, S) if rank == 0 else None
            dist.barrier(group=gloo)
    # headline: the first fan-out in preference order that ran and verified bit-exact (rank 0 decides)
    head = None
    if rank == 0:
        engine = [f for f in order if f not in ("dram", "nccl", "ce")]  # the baselines never headline
        head = next((f for f in engine if results[f].get("parity_ok")), None)
        head = head or next((f for f in engine if "latency_ms" in results[f]), engine[0] if engine else order[0])
    head = gather_obj(head, gloo)[0]
    log(f"fan-outs timed, headline {head}; baselines")
    # baselines on the same bytes: NCCL broadcast (device time, max over ranks) and a torch copy-engine pull
    buf = torch.empty(S, dtype=torch.uint8, device="cuda")
    nccl_ms = []
    for i in range(0 if over else args.warmup + args.steps):
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        dist.broadcast(buf, src=0)
        e1.record()
        e1.synchronize()
        if i >= args.warmup:
            nccl_ms.append(e0.elapsed_time(e1))
    ce_ms = ce_baseline(rank, gloo, buf, args.steps, args.warmup)
    del buf
    torch.cuda.empty_cache()
    log("concurrent acquire")
    conc = xproc_concurrent(V, G, synth, name, rank, world, dev, gloo, FANOUTS[head])
    conc_all = gather_obj(conc, gloo)
    log("e2e")
    e2e = xproc_e2e(V, G, synth, name, rank, world, dev, gloo, FANOUTS[head], flush, args.steps, args.warmup)
    t = torch.tensor([statistics.mean(nccl_ms) if nccl_ms else 0.0, ce_ms, e2e["ms"], float(1 - e2e["ok"])],
                     dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=gloo)
    if rank == 0:
        out = xproc_line(args, world, name, S, ndev, over, head, results, conc_all, [float(x) for x in t], e2e,
                         clk.summary())
        print(json.dumps(out), flush=True)
    dist.barrier(group=gloo)
    dist.destroy_process_group()


def gpu_arm(args):
    import torch
    rank, world, local = dist_env()
    if world > 1:
        return xproc_arm(args)
    torch.cuda.set_device(local)
    import synth
    from synth import gpu as G
    from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    name = args.config
    peak, peak_kind = load_peaks()
    flush = torch.empty(FLUSH_BYTES, dtype=torch.uint8, device="cuda")
    # ---- headline
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        r = run_update_bench(V, G, synth, name, args.steps, args.warmup, flush)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    mean_ms = statistics.mean(r["dev_ms"])
    if world > 1:
        t = torch.tensor([mean_ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        mean_ms = float(t.item())
    warm = run_update_bench(V, G, synth, name, args.steps, args.warmup, None)  # cold and warm
    # kernel-only times: the fused SYNC kernel (what the headline runs) and,
    # for reference, the separate pack / install kernels (VIPER_FLAG_NO_FUSE)
    kt = run_update_bench(V, G, synth, name, args.steps, args.warmup, flush, kernel_timing=True)
    ks = run_update_bench(V, G, synth, name, args.steps, args.warmup, flush, kernel_timing=True,
                          extra_flags=V.FLAG_NO_FUSE)
    # the same headline after a write-only flush (dirty harness lines in L2)
    rd = run_update_bench(V, G, synth, name, args.steps, args.warmup, flush, dirty=True)
    ktd = run_update_bench(V, G, synth, name, args.steps, args.warmup, flush, kernel_timing=True, dirty=True)
    fused_dirty = statistics.median(ktd["fused_us"])
    fused = statistics.median(kt["fused_us"])
    pack = statistics.median(ks["pack_us"])
    inst = statistics.median(ks["install_us"])
    alg = 3 * r["bytes"]  # HBM minimum: read the tensors + write the snapshot + write the slot
                          # (the install's read-back of the snapshot is served by L2 by design)
    dom, dom_us = "publish_fused (pack_seal + install_verify + swap)", fused
    achieved = alg / (dom_us * 1e-6) / 1e9
    calib = event_floor_us(G)
    b2b_ms, b2b_ok = run_back_to_back(V, G, synth, name, args.steps, args.warmup)
    gold = golden_check_local(V, G, synth, name)
    out = {
        "metric": METRIC, "value": round(mean_ms, 6), "unit": "ms", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(mean_ms, 6), "higher_is_better": False,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "model_dtype": "f32" if name in ("ptychonn", "resnet50") else "bf16",
        "data": "synthetic (VGEN seeded random-init parameters, BASELINE.json shapes)",
        "config": {"workload": f"{name}: 1 producer -> 1 consumer, 1-GPU loopback "
                               f"(BASELINE.json configs[{CONFIG_INDEX[name]}]"
                               f"{'' if name == 'ptychonn' else ' without its NVLink hop'})",
                   "tensors": r["tensors"], "model_bytes": r["bytes"], "packed_bytes": r["s_packed"],
                   "tier": "gpu", "mode": "sync",
                   "l2": "flushed before every timed update: a 256 MiB write, then a read of another 256 MiB "
                         "(the written lines go back to HBM inside the flush; L2 is left holding clean unrelated "
                         "data, as ncu's cache control does). dirty_l2 repeats the headline with the write alone",
                   "parallelism": "replicas" if world > 1 else "single GPU"},
        "update_gbps": round(r["bytes"] / (mean_ms * 1e-3) / 1e9, 3),
        "host_latency_ms": round(statistics.mean(r["host_ms"]), 6),
        "latency_p50_ms": round(statistics.median(r["dev_ms"]), 6),
        "latency_p90_ms": round(sorted(r["dev_ms"])[max(0, int(0.9 * len(r["dev_ms"]) + 0.5) - 1)], 6),
        "latency_min_ms": round(min(r["dev_ms"]), 6),
        "latency_warm_l2_ms": round(statistics.mean(warm["dev_ms"]), 6),
        "dirty_l2": {"latency_ms": round(statistics.mean(rd["dev_ms"]), 6),
                     "publish_fused_us": round(fused_dirty, 3),
                     "fused_hbm_frac": round(alg / (fused_dirty * 1e-6) / 1e9 / peak, 4),
                     "how": "write-only 256 MiB flush: ~126 MB of dirty harness lines stay in L2 and are written "
                            "back during the timed kernel", "parity_ok": rd["ok"] and ktd["ok"]},
        "latency_back_to_back_ms": round(b2b_ms, 6),
        "back_to_back": {"hbm_frac": round(alg / (b2b_ms * 1e-3) / 1e9 / peak, 4), "parity_ok": b2b_ok,
                         "how": "K SYNC publishes issued back to back, one CUDA-event window around all K (no flush, "
                                "no optimizer write): each update pays the deferred L2 write-back of the previous "
                                "one; 3S algorithmic bytes per update vs measured HBM"},
        "parity_golden": gold,
        "kernels_us": {"publish_fused": round(fused, 3), "pack_seal": round(pack, 3),
                       "install_verify": round(inst, 3), "event_bracket_floor": round(calib, 3),
                       "how": "library CUDA events around each kernel, stream kept busy (no host gaps); "
                              "event_bracket_floor = an empty kernel timed the same way"},
        "roofline": {"bound": "hbm", "kernel": dom, "achieved": round(achieved, 2), "peak": peak,
                     "unit": "GB/s", "frac": round(achieved / peak, 4),
                     "traffic": ncu_traffic("publish_fused_kernel", name),
                     "traffic_source": "profiles/ncu_traffic.json (ncu --set full, cold caches)",
                     "peak_kind": peak_kind, "algorithmic_bytes": alg,
                     "duration": "CUDA events around each launch on its stream (includes the event_bracket_floor)",
                     "ncu_launch_list": ncu_launches(name, "publish_fused_kernel", alg, peak),
                     "frac_of_nominal_7700": round(achieved / HBM_NOMINAL_GBS, 4)},
        "parity_ok": bool(r["ok"] and gold["producer_seals_ok"] and gold["consumer_seals_ok"] and gold["bytes_ok"]),
        "gpu_launches": 2 * args.steps,  # publish_fused + seal_reduce per update
    }
    out["clocks"] = clk.summary()
    if rank == 0:
        e = run_e2e(V, G, synth, name, max(3, args.steps // 2), args.warmup, flush)
        out["e2e"] = {"value": round(e["ms"], 6), "unit": "ms", "h2d_bytes_per_step": e["h2d"],
                      "d2h_bytes_per_step": e["d2h"], "digest_ok": e["ok"]}
        if not args.no_sweep:
            sweep = {}
            for nm in ["ptychonn", "resnet50", "vit_b16", "gpt2_xl", "llama3_8b"]:
                if nm == name:
                    continue
                try:
                    s = run_update_bench(V, G, synth, nm, 5, 3, flush)
                    k = run_update_bench(V, G, synth, nm, 5, 3, flush, kernel_timing=True)
                    k2 = run_update_bench(V, G, synth, nm, 5, 3, flush, kernel_timing=True,
                                          extra_flags=V.FLAG_NO_FUSE)
                    fu = statistics.median(k["fused_us"])
                    pk, ins = statistics.median(k2["pack_us"]), statistics.median(k2["install_us"])
                    lat = statistics.mean(s["dev_ms"])
                    sweep[nm] = {"latency_ms": round(lat, 4), "fused_us": round(fu, 2), "pack_us": round(pk, 2),
                                 "install_us": round(ins, 2),
                                 "fused_hbm_frac": round(3 * s["bytes"] / (fu * 1e-6) / 1e9 / peak, 4),
                                 "fused_frac_of_nominal_7700": round(3 * s["bytes"] / (fu * 1e-6) / 1e9 /
                                                                     HBM_NOMINAL_GBS, 4),
                                 "pack_hbm_frac": round(2 * s["bytes"] / (pk * 1e-6) / 1e9 / peak, 4),
                                 "install_hbm_frac": round(2 * s["bytes"] / (ins * 1e-6) / 1e9 / peak, 4),
                                 "update_gbps": round(s["bytes"] / (lat * 1e-3) / 1e9, 2),
                                 "parity_ok": s["ok"] and k["ok"] and k2["ok"]}
                except Exception as ex:  # report, never hide
                    sweep[nm] = {"error": str(ex)[:200]}
                torch.cuda.empty_cache()
            out["loopback_sweep"] = sweep
            fan = {}
            for nm, nc in (("vit_b16", 3), ("gpt2_xl", 3)):  # BASELINE configs[2] / [3] consumers on one GPU
                try:
                    s = run_update_bench(V, G, synth, nm, 5, 3, flush, ncons=nc)
                    k = run_update_bench(V, G, synth, nm, 5, 3, flush, kernel_timing=True, ncons=nc)
                    fu = statistics.median(k["fused_us"])
                    lat = statistics.mean(s["dev_ms"])
                    fan[f"{nm}_1to{nc}"] = {
                        "latency_ms": round(lat, 4), "fused_us": round(fu, 2),
                        "algorithmic_bytes": (2 + nc) * s["bytes"],
                        "fused_hbm_frac": round((2 + nc) * s["bytes"] / (fu * 1e-6) / 1e9 / peak, 4),
                        "parity_ok": s["ok"] and k["ok"]}
                except Exception as ex:  # report, never hide
                    fan[f"{nm}_1to{nc}"] = {"error": str(ex)[:200]}
                torch.cuda.empty_cache()
            out["loopback_fanout"] = {
                "how": "in-process SYNC, 1 producer -> N consumers on this GPU: one fused kernel reads the "
                       "tensors once and writes the snapshot + N slots ((2+N)*S bytes)", **fan}
            try:
                out["c3_concurrent"] = c3_concurrent(V, G, synth)
                out["c3_concurrent_gemm"] = c3_concurrent(V, G, synth, reader_kind="gemm")  # compute-bound reader
            except Exception as ex:
                out["c3_concurrent"] = {"error": str(ex)[:200]}
            try:
                out["c5_schedule"] = c5_schedule(V, G, synth, flush, sweep.get("llama3_8b", {}))
            except Exception as ex:
                out["c5_schedule"] = {"error": str(ex)[:200]}
        try:
            base = {name: round(torch_copy_baseline(G, synth, name, flush), 6)}
            if not args.no_sweep:
                for nm in ["ptychonn", "resnet50", "vit_b16", "gpt2_xl"]:
                    if nm == name:
                        continue
                    base[nm] = round(torch_copy_baseline(G, synth, nm, flush), 6)
            out["baseline_torch_state_dict_copy_ms"] = base
        except Exception as ex:
            out["baseline_torch_state_dict_copy_ms"] = {"error": str(ex)[:200]}
        out["cpu_baseline"] = cpu_baseline(synth, name, budget_s=args.cpu_budget)
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def reference_arm(args):
    """The oracle on the host cores, on this arm's config: at N > 1 rank 0
    alone runs it with the same 1 -> N-1 fan-out (N-1 oracle consumers, as
    many as fit in 40% of the host's available memory; the sample says how
    many), the other ranks exit without work."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import synth
    name = args.config if (args.config_explicit or world == 1) else N_CONFIG.get(world, "resnet50")
    ncons = max(1, world - 1)
    try:
        avail = os.sysconf("SC_AVPHYS_PAGES") * os.sysconf("SC_PAGE_SIZE")
        fit = int((0.4 * avail / synth.model_bytes(name) - 3) // 3)  # producer + 2 versions; 3 S per consumer
        ncons = max(1, min(ncons, fit))
    except (ValueError, OSError):
        pass
    o = OracleUpdates(synth, name, ncons=ncons)
    res = []
    try:
        for i in range(args.warmup + args.steps):
            t = o.run(max(0.2, args.cpu_budget / max(args.steps, 1)), max_updates=20)
            if i >= args.warmup:
                res.append(statistics.mean(t))
    finally:
        o.close()
    v = statistics.mean(res)
    out = {"impl": "reference", "metric": METRIC, "value": round(v, 4), "unit": "ms", "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(v, 4), "higher_is_better": False,
           "scaling": "weak", "vs_baseline": None, "dtype": "u32", "model_dtype": "f32" if name in ("ptychonn", "resnet50") else "bf16",
           "data": "synthetic (VGEN)", "config": {"workload": f"{name}: 1 producer -> {ncons} consumer(s), the oracle on "
                                                     f"host cores (BASELINE.json configs[{CONFIG_INDEX[name]}])"},
           "cpu_baseline": {"value": round(v, 4), "unit": "ms", "cores": 1, "kind": "oracle", "cpu": cpu_model(),
                            "sample": f"each step = up to 20 oracle updates to {ncons} consumer(s), mean ms per update"},
           "e2e": {"value": round(v, 4), "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def free_port() -> int:
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def launch_ranks(args) -> int:
    """`--gpus N` (N > 1) without a launcher: start N ranks of this script with
    torch.distributed.run on 127.0.0.1 (the same command the driver uses), one
    per GPU.  Fails loudly when fewer than N GPUs are visible, unless
    --oversubscribe (ranks then share GPUs: a code-path run, no NVLink)."""
    ndev = 0
    try:
        import torch
        ndev = torch.cuda.device_count() if torch.cuda.is_available() else 0
    except Exception:
        pass
    if ndev < args.gpus and not args.oversubscribe:
        print(f"bench.py: --gpus {args.gpus} but {ndev} GPU(s) visible (pass --oversubscribe to share GPUs)",
              file=sys.stderr, flush=True)
        return 2
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.run(cmd).returncode


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="viper", choices=["viper", "reference"])
    ap.add_argument("--config", default=None, choices=["ptychonn", "resnet50", "vit_b16", "gpt2_xl", "llama3_8b"])
    ap.add_argument("--fanout", default="auto", choices=["auto"] + sorted(FANOUTS),
                    help="N > 1: time only this fan-out (auto: every fan-out, headline NVLS where available, else "
                         "scatter-allgather for N > 2 and direct pull for N = 2)")
    ap.add_argument("--oversubscribe", action="store_true",
                    help="N > 1 with fewer visible GPUs than ranks: ranks share GPUs (code path only, no NVLink)")
    ap.add_argument("--no-sweep", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=10.0)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    args.config_explicit = args.config is not None
    if args.config is None:
        args.config = "resnet50"  # BASELINE.json configs[1] (1-GPU loopback)
    if args.gpus < 1:
        raise SystemExit("bench.py: --gpus must be >= 1")
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(launch_ranks(args))  # one process per GPU, then each rank re-enters main()
    _, world, _ = dist_env()
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")
    if args.impl == "reference":
        reference_arm(args)
    else:
        gpu_arm(args)


if __name__ == "__main__":
    main()
