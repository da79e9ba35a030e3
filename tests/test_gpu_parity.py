"""GPU parity: the CUDA path (through the C-ABI) against the oracle, element by
element on the same seeded VGEN inputs, plus the protocol invariants
 on the device path.  Bit-exact throughout: this is
byte work."""
import os
import threading
import time

import numpy as np
import pytest
import torch

import synth
from oracle import transfer as T
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

pytestmark = pytest.mark.gpu
_uid = [0]


def uname(p="m"):
    _uid[0] += 1
    return f"{p}-{_uid[0]}-{time.monotonic_ns()}"


def host_bytes(t):
    return t.detach().contiguous().view(torch.uint8).reshape(-1).cpu().numpy() if t.numel() else np.zeros(0, np.uint8)


def expect(specs, seed, v):
    return [synth.vgen_numpy(seed, v, i, s[1], synth.nelem_of(s)) for i, s in enumerate(specs)]


def oracle_packed_and_seals(specs, seed, v, chunk_bytes, align=256):
    ts = expect(specs, seed, v)
    off, s = T.layout([t.size for t in ts], align)
    p = T.pack(ts, off, s)
    return p, T.seal(p, chunk_bytes, v), off


def _raw_u64(ptr, count):
    """`count` uint64 words at device pointer ptr (as an int64 tensor)."""
    like = torch.empty(2 * max(count, 1), dtype=torch.int32, device="cuda")
    return V._from_ptr(ptr, like).view(torch.int64)[:count]


def device_packed_and_seals(prod):
    p, s, n = prod.debug_buffers()
    S, _ = prod.layout()
    torch.cuda.synchronize()
    packed = V._from_ptr(p, torch.empty(S, dtype=torch.uint8, device="cuda")) if S else torch.empty(0, dtype=torch.uint8)
    seals = _raw_u64(s, 2 * n)
    return host_bytes(packed), seals.cpu().numpy().view(np.uint64).reshape(n, 2)


def view_seals_host(c, view):
    """viper_view_seals: the installed slot's chunk seals, computed on the GPU."""
    n = c.stats()["nchunks"]
    buf = torch.empty(max(16 * n, 16), dtype=torch.uint8, device="cuda")
    c.view_seals(view, buf)
    torch.cuda.synchronize()
    return buf.view(torch.int64).cpu().numpy().view(np.uint64).reshape(-1, 2)[:n]


def check_slot(view, cons_like, specs, seed, v):
    got = view.tensors(cons_like)
    exp = expect(specs, seed, v)
    for i, (g, e) in enumerate(zip(got, exp)):
        assert np.array_equal(host_bytes(g), e), f"tensor {i} differs at version {v}"


def make_pair(specs, seed, ncons=1, **kw):
    prod_t = G.alloc_model(specs)
    cons_t = [G.alloc_model(specs) for _ in range(ncons)]
    name = uname()
    ckw = {k: v for k, v in kw.items() if k in ("tier", "chunk_bytes", "align")}
    cons = [V.Model(name, V.CONSUMER, ct, **ckw) for ct in cons_t]
    prod = V.Model(name, V.PRODUCER, prod_t, **kw)
    return prod, prod_t, cons, cons_t


def close_all(prod, cons):
    for c in cons:
        c.close()
    prod.close()


# ------------------------------------------------------------------ C1 (BJ configs[0])
@pytest.mark.parametrize("tier,mode,flags", [(V.TIER_GPU, V.SYNC, 0), (V.TIER_GPU, V.SYNC, V.FLAG_NO_FUSE),
                                              (V.TIER_GPU, V.SYNC, V.FLAG_FUSED_TMA),
                                              (V.TIER_GPU, V.SYNC, V.FLAG_TMA), (V.TIER_GPU, V.ASYNC, V.FLAG_TMA),
                                              (V.TIER_GPU, V.ASYNC, 0), (V.TIER_DRAM, V.SYNC, 0),
                                              (V.TIER_DRAM, V.ASYNC, 0)])
def test_c1_ptychonn_10_versions(tier, mode, flags):
    specs = synth.model_specs("ptychonn")
    seed = synth.SEEDS["ptychonn"]
    prod, prod_t, cons, cons_t = make_pair(specs, seed, tier=tier, mode=mode, flags=flags)
    try:
        for v in range(1, 11):
            G.fill_model(prod_t, specs, seed, v)
            prod.publish(v)
            if mode == V.ASYNC:
                cons[0].wait_installed(v)
            # producer snapshot and seals == oracle pack/seal of the same version
            if mode == V.SYNC or v == 10:
                p_dev, s_dev = device_packed_and_seals(prod)
                p_or, s_or, _ = oracle_packed_and_seals(specs, seed, v, 2 << 20)
                assert np.array_equal(p_dev, p_or)
                assert np.array_equal(s_dev, s_or)
            view = cons[0].acquire_latest(min_version=v, timeout_us=5_000_000)
            assert view.version == v
            check_slot(view, cons_t[0], specs, seed, v)
            cons[0].release(view)
        st = cons[0].stats()
        assert st["installs"] >= 1 and st["failures"] == 0
    finally:
        close_all(prod, cons)


# ----------------------------------------------------- ragged lists, several consumers
@pytest.mark.parametrize("seed", range(6))
def test_ragged_tensor_lists_many_chunks(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 40))
    specs = []
    for i in range(n):
        dt = int(rng.choice([synth.F32, synth.BF16, synth.F16, synth.BYTES]))
        ne = int(rng.choice([0, 1, 3, 7, 255, 1023, int(rng.integers(1, 70000))]))
        specs.append((f"t{i}", dt, (ne,)))
    chunk = int(rng.choice([256, 4096, 65536]))
    align = int(rng.choice([16, 256]))
    flags = [0, V.FLAG_NO_FUSE, V.FLAG_TMA, V.FLAG_FUSED_TMA][seed % 4]
    ncons = 3 if seed < 4 else 6   # > kMaxFused local consumers -> separate kernels
    prod, prod_t, cons, cons_t = make_pair(specs, seed, ncons=ncons, chunk_bytes=chunk, align=align, flags=flags)
    try:
        for v in (1, 2, 5):
            G.fill_model(prod_t, specs, 77 + seed, v)
            prod.publish(v)
            p_dev, s_dev = device_packed_and_seals(prod)
            p_or, s_or, _ = oracle_packed_and_seals(specs, 77 + seed, v, chunk, align)
            assert np.array_equal(p_dev, p_or)
            assert np.array_equal(s_dev, s_or)
            for c, ct in zip(cons, cons_t):
                view = c.acquire_latest()
                assert view.version == v
                check_slot(view, ct, specs, 77 + seed, v)
                assert np.array_equal(view_seals_host(c, view), s_or)  # installed-slot seals == oracle
                c.release(view)
    finally:
        close_all(prod, cons)


def test_unaligned_tensor_pointers():
    """Tensors that are byte-offset views (not 16-B aligned) take the word path."""
    specs = [("a", synth.BYTES, (1001,)), ("b", synth.BYTES, (4099,)), ("c", synth.BYTES, (37,))]
    base_p = torch.empty(6000, dtype=torch.uint8, device="cuda")
    base_c = torch.empty(6000, dtype=torch.uint8, device="cuda")
    prod_t = [base_p[1:1002], base_p[1003:5102], base_p[5103:5140]]
    cons_t = [base_c[3:1004], base_c[1005:5104], base_c[5105:5142]]
    name = uname()
    cons = V.Model(name, V.CONSUMER, cons_t, chunk_bytes=1024)
    prod = V.Model(name, V.PRODUCER, prod_t, chunk_bytes=1024)
    try:
        for v in (1, 2, 3):
            G.fill_model(prod_t, specs, 5, v)
            prod.publish(v)
            p_dev, s_dev = device_packed_and_seals(prod)
            p_or, s_or, _ = oracle_packed_and_seals(specs, 5, v, 1024)
            assert np.array_equal(p_dev, p_or) and np.array_equal(s_dev, s_or)
            view = cons.acquire_latest()
            # slot 0 is the unaligned caller view, slot 1 the library copy
            check_slot(view, cons_t, specs, 5, v)
            cons.release(view)
    finally:
        close_all(prod, [cons])


def test_empty_model():
    name = uname()
    cons = V.Model(name, V.CONSUMER, [], device=0)
    prod = V.Model(name, V.PRODUCER, [], device=0)
    try:
        prod.publish(1)
        view = cons.acquire_latest()
        assert view.version == 1 and view.ptrs == []
        cons.release(view)
    finally:
        close_all(prod, [cons])


# ------------------------------------------------------ in-process tier agreement
@pytest.mark.parametrize("first,second", [(V.TIER_GPU, V.TIER_DRAM), (V.TIER_DRAM, V.TIER_GPU)])
def test_in_process_endpoints_must_share_a_tier(first, second):
    """A DRAM-tier consumer reads the producer's host staging, which a GPU-tier
    producer never fills: registration with mixed tiers is refused (E_INVAL),
    whichever side registers first, and the channel stays usable."""
    specs = synth.model_specs("ptychonn")
    seed = synth.SEEDS["ptychonn"]
    name = uname()
    pt, ct, ct2 = G.alloc_model(specs), G.alloc_model(specs), G.alloc_model(specs)
    cons = V.Model(name, V.CONSUMER, ct, tier=first)
    try:
        with pytest.raises(V.ViperError) as ei:
            V.Model(name, V.PRODUCER, pt, tier=second)
        assert ei.value.status == V.E_INVAL
        with pytest.raises(V.ViperError) as ei:
            V.Model(name, V.CONSUMER, ct2, tier=second)
        assert ei.value.status == V.E_INVAL
        prod = V.Model(name, V.PRODUCER, pt, tier=first)
        try:
            G.fill_model(pt, specs, seed, 1)
            prod.publish(1)
            view = cons.acquire_latest(min_version=1, timeout_us=5_000_000)
            check_slot(view, ct, specs, seed, 1)
            cons.release(view)
        finally:
            prod.close()
    finally:
        cons.close()


@pytest.mark.parametrize("first", [V.TIER_AUTO, V.TIER_DRAM, V.TIER_GPU])
def test_in_process_transfer_selector(first):
    """VIPER_TIER_AUTO in process: the tier of the model's existing endpoints,
    else the GPU tier when this GPU reaches every visible GPU (here: the only
    one).  The producer registers with AUTO after a consumer asked for
    `first`; both report the same resolved tier and the update is bit-exact."""
    import torch
    specs = synth.model_specs("ptychonn")
    seed = synth.SEEDS["ptychonn"]
    name = uname()
    pt, ct = G.alloc_model(specs), G.alloc_model(specs)
    cons = V.Model(name, V.CONSUMER, ct, tier=first)
    prod = V.Model(name, V.PRODUCER, pt, tier=V.TIER_AUTO)
    try:
        solo = torch.cuda.device_count() == 1
        want = first if first != V.TIER_AUTO else (V.TIER_GPU if solo else cons.stats()["tier"])
        assert cons.stats()["tier"] == want and prod.stats()["tier"] == want
        for v in (1, 2):
            G.fill_model(pt, specs, seed, v)
            prod.publish(v)
        view = cons.acquire_latest(min_version=2, timeout_us=5_000_000)
        check_slot(view, ct, specs, seed, 2)
        cons.release(view)
    finally:
        close_all(prod, [cons])


# ---------------------------------------------------------------- protocol on device
@pytest.mark.parametrize("flags", [0, V.FLAG_NO_FUSE, V.FLAG_FUSED_TMA, V.FLAG_NO_TMA])
def test_fault_injection_keeps_old_version(flags):
    specs = synth.model_specs("ptychonn")
    seed = 11
    prod, prod_t, cons, cons_t = make_pair(specs, seed, flags=flags)
    try:
        G.fill_model(prod_t, specs, seed, 1)
        prod.publish(1)
        cons[0].fault_next()
        G.fill_model(prod_t, specs, seed, 2)
        with pytest.raises(V.ViperError) as ei:
            prod.publish(2)
        assert ei.value.status == V.E_CHECKSUM
        view = cons[0].acquire_latest()
        assert view.version == 1
        check_slot(view, cons_t[0], specs, seed, 1)
        cons[0].release(view)
        assert cons[0].stats()["failures"] == 1
        G.fill_model(prod_t, specs, seed, 3)
        prod.publish(3)
        view = cons[0].acquire_latest()
        assert view.version == 3
        check_slot(view, cons_t[0], specs, seed, 3)
        cons[0].release(view)
    finally:
        close_all(prod, cons)


def test_version_and_view_errors():
    specs = [("w", synth.F32, (1000,))]
    prod, prod_t, cons, cons_t = make_pair(specs, 1)
    try:
        with pytest.raises(V.ViperError) as ei:
            cons[0].acquire_latest(timeout_us=0)
        assert ei.value.status == V.E_NOVERSION
        with pytest.raises(V.ViperError) as ei:
            prod.publish(0)
        assert ei.value.status == V.E_VERSION
        prod.publish(4)
        for bad in (4, 3):
            with pytest.raises(V.ViperError) as ei:
                prod.publish(bad)
            assert ei.value.status == V.E_VERSION
        view = cons[0].acquire_latest()
        cons[0].release(view)
        with pytest.raises(V.ViperError) as ei:
            cons[0].release(view)
        assert ei.value.status == V.E_STATE
        with pytest.raises(V.ViperError) as ei:
            cons[0].publish(9)
        assert ei.value.status == V.E_STATE
        with pytest.raises(V.ViperError) as ei:
            cons[0].acquire_latest(min_version=5, timeout_us=20_000)
        assert ei.value.status == V.E_TIMEOUT
    finally:
        close_all(prod, cons)


def test_writer_waits_for_pinned_slot():
    """A reader pinning v keeps v's slot intact while v+1 and v+2 are published;
    v+2 (which needs that slot) waits for the release (a7)."""
    specs = [("w", synth.F32, (300_000,)), ("b", synth.F32, (77,))]
    seed = 3
    prod, prod_t, cons, cons_t = make_pair(specs, seed)
    try:
        G.fill_model(prod_t, specs, seed, 1)
        prod.publish(1)
        view = cons[0].acquire_latest()
        G.fill_model(prod_t, specs, seed, 2)
        prod.publish(2)                      # other slot: no wait
        def late_release():
            time.sleep(0.2)
            check_slot(view, cons_t[0], specs, seed, 1)  # still v1 while pinned
            cons[0].release(view)
        th = threading.Thread(target=late_release)
        th.start()
        G.fill_model(prod_t, specs, seed, 3)
        t0 = time.monotonic()
        prod.publish(3)                      # needs view's slot
        waited = time.monotonic() - t0
        th.join()
        assert waited > 0.15
        assert cons[0].stats()["writer_wait_us"] > 1.5e5
        v3 = cons[0].acquire_latest()
        assert v3.version == 3
        check_slot(v3, cons_t[0], specs, seed, 3)
        cons[0].release(v3)
    finally:
        close_all(prod, cons)


def test_stream_ordered_release():
    specs = [("w", synth.F32, (4096,))]
    prod, prod_t, cons, cons_t = make_pair(specs, 2)
    try:
        G.fill_model(prod_t, specs, 2, 1)
        prod.publish(1)
        s = torch.cuda.Stream()
        view = cons[0].acquire_latest()
        with torch.cuda.stream(s):
            torch.cuda._sleep(20_000_000)  # ~10 ms of reader work on the slot's stream
        cons[0].release(view, stream=s)
        G.fill_model(prod_t, specs, 2, 2)
        prod.publish(2)
        G.fill_model(prod_t, specs, 2, 3)
        prod.publish(3)  # waits until the stream passed the release
        s.synchronize()
        v = cons[0].acquire_latest()
        assert v.version == 3
        cons[0].release(v)
    finally:
        close_all(prod, cons)


def test_no_torn_reads_under_async_publishes():
    """Readers acquire -> compare every byte of the view with VGEN(view.version)
    on the GPU -> release, while the producer publishes back to back (ASYNC)."""
    specs = [(f"t{i}", synth.F32, (50_000 + 13 * i,)) for i in range(8)]
    seed = 99
    prod, prod_t, cons, cons_t = make_pair(specs, seed, mode=V.ASYNC)
    stop = threading.Event()
    errors, seen = [], []

    def reader():
        torch.cuda.set_device(0)
        s = torch.cuda.Stream()
        exp_t = G.alloc_model(specs)
        last = 0
        with torch.cuda.stream(s):
            while not stop.is_set():
                try:
                    view = cons[0].acquire_latest(timeout_us=100_000)
                except V.ViperError:
                    continue
                if view.version < last:
                    errors.append(("regress", last, view.version))
                last = view.version
                G.fill_model(exp_t, specs, seed, view.version, stream=s)
                got = view.tensors(cons_t[0])
                bad = sum(int((g.view(torch.uint8) != e.view(torch.uint8)).sum()) for g, e in zip(got, exp_t))
                if bad:
                    errors.append(("torn", view.version, bad))
                seen.append(view.version)
                cons[0].release(view, stream=s)
                s.synchronize()

    ths = [threading.Thread(target=reader) for _ in range(2)]
    try:
        for th in ths:
            th.start()
        ps = torch.cuda.Stream()
        for v in range(1, 301):
            with torch.cuda.stream(ps):
                G.fill_model(prod_t, specs, seed, v, stream=ps)
                prod.publish(v, stream=ps)
            if v % 50 == 0:
                time.sleep(0.01)
        cons[0].wait_installed(300)
        time.sleep(0.05)
        stop.set()
        for th in ths:
            th.join()
        assert not errors, errors[:5]
        assert len(seen) >= 20
        assert cons[0].acquire_latest().version == 300
    finally:
        stop.set()
        close_all(prod, cons)


# ----------------------------------------------- BJ-sized models in 1-GPU loopback
@pytest.mark.parametrize("name,flags,tier", [("resnet50", 0, V.TIER_GPU), ("vit_b16", 0, V.TIER_GPU),
                                             ("gpt2_xl", 0, V.TIER_GPU), ("llama3_8b", 0, V.TIER_GPU),
                                             ("gpt2_xl", V.FLAG_TMA, V.TIER_GPU), ("resnet50", 0, V.TIER_DRAM),
                                             ("resnet50", V.FLAG_FUSED_TMA, V.TIER_GPU),
                                             ("resnet50", V.FLAG_NO_TMA, V.TIER_GPU),
                                             ("gpt2_xl", V.FLAG_FUSED_TMA, V.TIER_GPU),
                                             ("gpt2_xl", 0, V.TIER_DRAM),
                                             # register pack + PDL register install: > one round of items per
                                             # warp, so both work counters hand out items (kernels.cu WorkQueue)
                                             ("resnet50", V.FLAG_NO_FUSE, V.TIER_GPU),
                                             ("vit_b16", V.FLAG_NO_FUSE | V.FLAG_NO_TMA, V.TIER_GPU)])
def test_full_size_loopback_sampled(name, flags, tier):
    """Full BASELINE.json model sizes, single-GPU loopback (the launch config
    bench.py times): every seal's version; sampled chunk seals recomputed by the
    oracle; sampled tensor byte ranges vs VGEN; all slot tensors == producer
    tensors (replica identity at any size)."""
    specs = synth.model_specs(name)
    seed = synth.SEEDS[name]
    prod, prod_t, cons, cons_t = make_pair(specs, seed, mode=V.SYNC, flags=flags, tier=tier)
    try:
        for v in (1, 2):
            G.fill_model(prod_t, specs, seed, v)
            prod.publish(v)
        torch.cuda.synchronize()
        S, offsets = prod.layout()
        p, sp, n = prod.debug_buffers()
        seals = _raw_u64(sp, 2 * n).cpu().numpy().view(np.uint64).reshape(n, 2)
        assert np.all(seals[:, 0] == 2)
        rng = np.random.default_rng(0)
        # every chunk seal where the oracle finishes in seconds, else a sample
        every = S <= 256 << 20
        for c in (range(n) if every else sorted({0, n - 1, *rng.integers(0, n, 4).tolist()})):
            assert int(seals[c, 1]) == T.expected_chunk_seal(specs, seed, 2, offsets, S, 2 << 20, c), c
        view = cons[0].acquire_latest()
        assert view.version == 2
        got = view.tensors(cons_t[0])
        for g, pt in zip(got, prod_t):
            assert torch.equal(g.view(torch.uint8), pt.view(torch.uint8))
        for i in sorted({0, len(specs) - 1, *rng.integers(0, len(specs), 6).tolist()}):
            nb = synth.nbytes_of(specs[i])
            lo = int(rng.integers(0, max(nb - 4096, 1)))
            hi = min(nb, lo + 4096)
            b = host_bytes(got[i].view(torch.uint8).reshape(-1)[lo:hi])
            assert np.array_equal(b, synth.vgen_bytes_range(seed, 2, i, specs[i][1], lo, hi))
        cons[0].release(view)
    finally:
        close_all(prod, cons)
        torch.cuda.empty_cache()


@pytest.mark.parametrize("mode", [V.SYNC, V.ASYNC])
def test_dram_tier_many_pieces(mode, monkeypatch):
    """The DRAM tier's D2H -> H2D piece pipeline with the maximum piece count
    (256 pieces of whole 4 KiB chunks): bytes and chunk seals equal the oracle's."""
    monkeypatch.setenv("VIPER_DRAM_PIECE", "1")  # -> S/256 per piece, rounded to whole chunks
    rng = np.random.default_rng(11)
    specs = [(f"t{i}", synth.F32 if i % 3 else synth.BYTES, (int(rng.integers(1, 70_000)),)) for i in range(40)]
    seed = 0x91EC
    prod, prod_t, cons, cons_t = make_pair(specs, seed, ncons=2, mode=mode, tier=V.TIER_DRAM, chunk_bytes=4096)
    try:
        for v in range(1, 5):
            G.fill_model(prod_t, specs, seed, v)
            prod.publish(v)
        for c, ct in zip(cons, cons_t):
            c.wait_installed(4, timeout_us=20_000_000)
            view = c.acquire_latest()
            assert view.version == 4
            check_slot(view, ct, specs, seed, 4)
            c.release(view)
        p_dev, s_dev = device_packed_and_seals(prod)
        p_or, s_or, _ = oracle_packed_and_seals(specs, seed, 4, 4096)
        assert np.array_equal(p_dev, p_or) and np.array_equal(s_dev, s_or)
    finally:
        close_all(prod, cons)


@pytest.mark.parametrize("install_sms,cflags,tier", [(1, 0, V.TIER_GPU), (3, V.FLAG_NO_TMA, V.TIER_GPU),
                                                    (2, 0, V.TIER_DRAM), (500, V.FLAG_NO_TMA, V.TIER_GPU)])
def test_install_sms_cap(install_sms, cflags, tier):
    """viper_config.install_sms: ASYNC installs on a capped number of SMs (TMA
    and register kernels, GPU and DRAM tiers; a cap above the SM count = all)
    stay byte-exact at ResNet-50 size, where the capped grid runs many rounds
    of work-counter claims per warp."""
    specs = synth.model_specs("resnet50")
    seed = synth.SEEDS["resnet50"]
    prod_t, cons_t = G.alloc_model(specs), G.alloc_model(specs)
    name = uname()
    cons = V.Model(name, V.CONSUMER, cons_t, tier=tier, flags=cflags, install_sms=install_sms)
    prod = V.Model(name, V.PRODUCER, prod_t, tier=tier, mode=V.ASYNC)
    try:
        for v in (1, 2, 3):
            G.fill_model(prod_t, specs, seed, v)
            prod.publish(v)
            cons.wait_installed(v, timeout_us=20_000_000)
            view = cons.acquire_latest()
            assert view.version == v
            assert all(torch.equal(g.view(torch.uint8), p.view(torch.uint8))
                       for g, p in zip(view.tensors(cons_t), prod_t))
            cons.release(view)
        assert cons.stats()["failures"] == 0
    finally:
        close_all(prod, [cons])
    with pytest.raises(V.ViperError):
        V.Model(uname(), V.CONSUMER, cons_t, install_sms=-1)


def test_teardown_races_in_process():
    """Unregistering a producer while its consumers' update threads install
    (ASYNC), and consumers while publishes run, never crashes or hangs."""
    specs = [(f"t{i}", synth.F32, (200_000,)) for i in range(4)]
    for rep in range(5):
        prod, prod_t, cons, cons_t = make_pair(specs, 1, ncons=3, mode=V.ASYNC)
        stop = threading.Event()

        def publisher():
            v = 0
            while not stop.is_set():
                v += 1
                try:
                    prod.publish(v)
                except V.ViperError:
                    break

        th = threading.Thread(target=publisher)
        th.start()
        time.sleep(0.01)
        cons[rep % 3].close()          # a consumer leaves mid-stream
        time.sleep(0.01)
        stop.set()
        th.join()
        prod.close()                   # producer leaves while others may install
        time.sleep(0.005)
        for i, c in enumerate(cons):
            if i != rep % 3:
                c.close()


def test_update_log_jsonl(tmp_path):
    """VIPER_LOG: one JSON line per publish / install (SURVEY s5 metrics)."""
    import json
    import subprocess
    import sys
    log = tmp_path / "viper.jsonl"
    code = (
        "import sys; sys.path.insert(0, '.');"
        "import synth; from synth import gpu as G; from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V;"
        "s=synth.model_specs('ptychonn'); pt,ct=G.alloc_model(s),G.alloc_model(s);"
        "c=V.Model('lg',V.CONSUMER,ct); p=V.Model('lg',V.PRODUCER,pt);"
        "[p.publish(v) for v in (1,2,3)]; c.close(); p.close()")
    env = dict(os.environ, VIPER_LOG=str(log))
    r = subprocess.run([sys.executable, "-c", code], cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                       env=env, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True, timeout=120)
    assert r.returncode == 0, r.stdout[-2000:]
    rows = [json.loads(l) for l in log.read_text().splitlines()]
    prod = [x for x in rows if x["role"] == "producer"]
    cons = [x for x in rows if x["role"] == "consumer"]
    assert [x["version"] for x in prod] == [1, 2, 3] and all(x["status"] == 0 for x in rows)
    assert [x["version"] for x in cons] == [1, 2, 3] and prod[0]["bytes"] == 4618496


def test_beyond_16_gib_word_index_wraps():
    """S > 16 GiB: the CKS word index g is taken mod 2^32 (R16); the
    chunks straddling g = 2^32 must match the oracle bit for bit."""
    specs = [("a", synth.BF16, (9 << 29,)), ("b", synth.BF16, (15 << 28,)), ("c", synth.F32, (12345,))]  # 16.5 GiB
    seed = 0xB16
    prod, prod_t, cons, cons_t = make_pair(specs, seed)
    try:
        G.fill_model(prod_t, specs, seed, 1)
        prod.publish(1)
        S, offsets = prod.layout()
        assert S > (16 << 30)
        p, sp, n = prod.debug_buffers()
        seals = _raw_u64(sp, 2 * n).cpu().numpy().view(np.uint64).reshape(n, 2)
        wrap = (16 << 30) // (2 << 20)  # first chunk whose words have g >= 2^32
        for c in (0, wrap - 1, wrap, wrap + 1, n - 1):
            assert int(seals[c, 1]) == T.expected_chunk_seal(specs, seed, 1, offsets, S, 2 << 20, c), c
        view = cons[0].acquire_latest()
        for g, pt in zip(view.tensors(cons_t[0]), prod_t):
            assert torch.equal(g.view(torch.uint8), pt.view(torch.uint8))
        cons[0].release(view)
    finally:
        close_all(prod, cons)
        del prod_t, cons_t
        torch.cuda.empty_cache()


@pytest.mark.parametrize("seed", range(8))
def test_randomized_configurations(seed):
    """Random tensor lists x {SYNC, ASYNC} x {GPU, DRAM} x {fused, separate,
    TMA} x {1..5 consumers} x chunk/align choices: every consumer ends
    byte-identical to VGEN(last version)."""
    rng = np.random.default_rng(1000 + seed)
    specs = []
    for i in range(int(rng.integers(1, 25))):
        dt = int(rng.choice([synth.F32, synth.BF16, synth.F16, synth.BYTES]))
        ne = int(rng.choice([0, 1, 5, 4097, int(rng.integers(1, 300_000))]))
        specs.append((f"t{i}", dt, (ne,)))
    mode = int(rng.choice([V.SYNC, V.ASYNC]))
    tier = int(rng.choice([V.TIER_GPU, V.TIER_DRAM]))
    flags = int(rng.choice([0, V.FLAG_NO_FUSE, V.FLAG_TMA, V.FLAG_NO_TMA, V.FLAG_FUSED_TMA]))
    chunk = int(rng.choice([4096, 65536, 2 << 20]))
    align = int(rng.choice([16, 256]))
    ncons = int(rng.integers(1, 6))
    prod, prod_t, cons, cons_t = make_pair(specs, seed, ncons=ncons, mode=mode, tier=tier, flags=flags,
                                           chunk_bytes=chunk, align=align)
    try:
        last = int(rng.integers(2, 6))
        for v in range(1, last + 1):
            G.fill_model(prod_t, specs, 7 * seed, v)
            prod.publish(v)
        for c, ct in zip(cons, cons_t):
            c.wait_installed(last, timeout_us=20_000_000)
            view = c.acquire_latest()
            assert view.version == last
            check_slot(view, ct, specs, 7 * seed, last)
            c.release(view)
        p_dev, s_dev = device_packed_and_seals(prod)
        p_or, s_or, _ = oracle_packed_and_seals(specs, 7 * seed, last, chunk, align)
        assert np.array_equal(p_dev, p_or) and np.array_equal(s_dev, s_or)
    finally:
        close_all(prod, cons)


def test_example_train_and_serve():
    """examples/train_and_serve.py: real ResNet-18 training publishes ASYNC while
    an inference thread serves; the served logits equal the trainer's."""
    import importlib.util
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    spec = importlib.util.spec_from_file_location("tas", os.path.join(root, "examples", "train_and_serve.py"))
    tas = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(tas)
    same, served = tas.main(steps=30, every=3, verbose=False)
    assert same
    assert served["n"] > 0 and len(served["versions"]) >= 2


# ------------------------------------------------------------ round 2 additions
def test_view_seals_unaligned_and_errors():
    """viper_view_seals on byte-offset (unaligned) slot tensors == the oracle's
    chunk seals; a released view or a producer is rejected (VIPER_E_STATE)."""
    specs = [("a", synth.BYTES, (1001,)), ("b", synth.BYTES, (4099,)), ("c", synth.BYTES, (37,))]
    base_p = torch.empty(6000, dtype=torch.uint8, device="cuda")
    base_c = torch.empty(6000, dtype=torch.uint8, device="cuda")
    prod_t = [base_p[1:1002], base_p[1003:5102], base_p[5103:5140]]
    cons_t = [base_c[3:1004], base_c[1005:5104], base_c[5105:5142]]
    name = uname()
    cons = V.Model(name, V.CONSUMER, cons_t, chunk_bytes=1024)
    prod = V.Model(name, V.PRODUCER, prod_t, chunk_bytes=1024)
    try:
        for v in (1, 2):
            G.fill_model(prod_t, specs, 0xAB, v)
            prod.publish(v)
            view = cons.acquire_latest()
            _, s_or, _ = oracle_packed_and_seals(specs, 0xAB, v, 1024)
            assert np.array_equal(view_seals_host(cons, view), s_or)
            cons.release(view)
        buf = torch.empty(16 * 16, dtype=torch.uint8, device="cuda")
        with pytest.raises(V.ViperError) as e:
            cons.view_seals(view, buf)  # released
        assert e.value.status == V.E_STATE
    finally:
        cons.close()
        prod.close()


@pytest.mark.parametrize("name", ["resnet50", "vit_b16"])
def test_golden_seals_full_size_in_process(name):
    """At BASELINE.json full size: VGEN(seed, VCHECK) published SYNC and ASYNC;
    the snapshot's and the installed slot's chunk seals == the oracle-written
    tests/golden/seals file, every chunk."""
    specs = synth.model_specs(name)
    hdr, gold = synth.golden_seals(name)
    for mode in (V.SYNC, V.ASYNC):
        prod, prod_t, cons, cons_t = make_pair(specs, synth.SEEDS[name], mode=mode)
        try:
            G.fill_model(prod_t, specs, synth.SEEDS[name], synth.VCHECK)
            prod.publish(3)
            cons[0].wait_installed(3)
            _, s_dev = device_packed_and_seals(prod)
            assert [int(x) for x in s_dev[:, 1]] == gold
            view = cons[0].acquire_latest()
            cs = view_seals_host(cons[0], view)
            assert (cs[:, 0] == 3).all() and [int(x) for x in cs[:, 1]] == gold
            cons[0].release(view)
        finally:
            close_all(prod, cons)


@pytest.mark.parametrize("fanout", [V.FANOUT_NVLS, V.FANOUT_PUSH, V.FANOUT_CE, V.FANOUT_NCCL])
def test_cross_process_only_fanouts_rejected_in_process(fanout):
    specs = synth.model_specs("ptychonn")
    t = G.alloc_model(specs)
    with pytest.raises(V.ViperError) as e:
        V.Model(uname(), V.PRODUCER, t, fanout=fanout)
    assert e.value.status == V.E_UNSUPPORTED


def test_consumer_records_are_reused():
    """consumers that unregister free their control record, so
    a long-lived producer serves more than kMaxConsumers (16) consumers over
    its life; each new one installs the next version bit-exactly."""
    specs = [("w", synth.F32, (4096,)), ("b", synth.F32, (7,))]
    prod_t = G.alloc_model(specs)
    name = uname()
    prod = V.Model(name, V.PRODUCER, prod_t)
    try:
        for k in range(20):
            ct = G.alloc_model(specs)
            c = V.Model(name, V.CONSUMER, ct)
            G.fill_model(prod_t, specs, 0x5E, k + 1)
            prod.publish(k + 1)
            view = c.acquire_latest()
            assert view.version == k + 1
            check_slot(view, ct, specs, 0x5E, k + 1)
            c.release(view)
            c.close()
        assert prod.stats()["nconsumers"] <= 2
    finally:
        prod.close()


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs two GPUs (in-process cross-device update)")
@pytest.mark.parametrize("mode,flags", [(V.SYNC, 0), (V.SYNC, V.FLAG_NO_FUSE), (V.SYNC, V.FLAG_TMA),
                                        (V.ASYNC, 0)])
def test_two_gpus_in_process(mode, flags):
    """producer on cuda:0, consumer on cuda:1 in one process.  SYNC
    installs run on the producer's stream and write the peer slot (the TMA
    install's shared-memory opt-in and the grid size are keyed on the
    launching GPU; the swap is fenced at system scope); ASYNC installs run on
    the consumer's GPU and pull the peer snapshot.  Bit-exact slots and
    installed-slot seals == the oracle's."""
    specs = synth.model_specs("resnet50")
    seed = synth.SEEDS["resnet50"]
    prod_t = G.alloc_model(specs, device="cuda:0")
    cons_t = G.alloc_model(specs, device="cuda:1")
    name = uname()
    torch.cuda.set_device(0)
    cons = V.Model(name, V.CONSUMER, cons_t, device=1)
    assert torch.cuda.current_device() == 0  # public calls leave the caller's device alone
    prod = V.Model(name, V.PRODUCER, prod_t, device=0, mode=mode, flags=flags)
    try:
        for v in (1, 2, 3):
            G.fill_model(prod_t, specs, seed, v)
            torch.cuda.set_device(1)
            prod.publish(v)
            assert torch.cuda.current_device() == 1
            torch.cuda.set_device(0)
            cons.wait_installed(v)
            view = cons.acquire_latest()
            assert view.version == v
            check_slot(view, cons_t, specs, seed, v)
            n = cons.stats()["nchunks"]
            buf = torch.empty(16 * n, dtype=torch.uint8, device="cuda:1")
            cons.view_seals(view, buf)
            assert torch.cuda.current_device() == 0
            torch.cuda.synchronize(1)
            _, s_or, _ = oracle_packed_and_seals(specs, seed, v, 2 << 20)
            assert np.array_equal(buf.view(torch.int64).cpu().numpy().view(np.uint64).reshape(n, 2), s_or)
            cons.release(view, stream=torch.cuda.current_stream(1))
            assert torch.cuda.current_device() == 0
    finally:
        cons.close()
        prod.close()
    assert torch.cuda.current_device() == 0
