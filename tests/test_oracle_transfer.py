"""Pins for the transfer oracle (oracle/viper_oracle.c), CPU only.

Each pin comes from something other than the oracle itself: a closed form, a
property that uniquely determines the definition, the plain state-dict-copy
definition, or an invariant of the double-buffer protocol
(P:1214-1227).  Plausible mistakes each fail at least one:
wrong alignment / padding -> layout properties; dropped XOR / wrong word
index base / wrong multiplier / 32-bit accumulation -> CKS closed forms;
wrong offset or length in pack/unpack -> byte equality with VGEN; a writer
that ignores readers or a non-atomic swap -> torn-read stress.
"""
import json
import os
import threading
import time

import numpy as np
import pytest

import synth
from oracle import transfer as T

GOLD = os.path.join(os.path.dirname(__file__), "golden")
K = 0x9E3779B1


# ------------------------------------------------------------------ LAY pins
@pytest.mark.parametrize("seed", range(40))
def test_layout_properties_bruteforce(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 10))
    nb = [int(x) for x in rng.integers(0, 68, n)]
    align = int(rng.choice([4, 16, 256]))
    off, s = T.layout(nb, align)
    # The layout is the unique one with: off_0 = 0, every offset aligned, the
    # next tensor starts at the FIRST aligned byte at/after the previous end.
    assert off[0] == 0
    ends = [int(o) + b for o, b in zip(off, nb)]
    for i in range(n):
        assert off[i] % align == 0
        nxt = s if i == n - 1 else int(off[i + 1])
        assert ends[i] <= nxt < ends[i] + align
    assert s % align == 0


def test_layout_empty():
    off, s = T.layout([], 256)
    assert s == 0 and len(off) == 0


def test_packed_sizes_match_survey():
    gold = json.load(open(os.path.join(GOLD, "model_sizes.json")))
    for name in synth.CONFIGS:
        off, s = T.layout([synth.nbytes_of(x) for x in synth.model_specs(name)], 256)
        assert s == gold[name]["packed"], name
        assert T.nchunks(s, 2 << 20) == gold[name]["chunks_2MiB"], name


# ------------------------------------------------------------------ CKS pins
def _weights(n, g0):
    return [((2 * ((g0 + i) & 0xFFFFFFFF) + 1) * K) & 0xFFFFFFFF for i in range(n)]


def test_cks_closed_forms():
    n, g0 = 3000, 123457
    m = _weights(n, g0)
    # all-zero words -> 0
    assert T.cks_words(np.zeros(n, dtype=np.uint32), g0) == 0
    # w_g = m_g^{-1} mod 2^32 -> every term is exactly 1 -> cks = n
    inv = np.array([pow(x, -1, 1 << 32) for x in m], dtype=np.uint32)
    assert T.cks_words(inv, g0) == n
    # w_g = 1 -> the sum of the weights; (2g+1)K mod 2^32 by python big ints
    assert T.cks_words(np.ones(n, dtype=np.uint32), g0) == sum(m)
    # w_g = -m_g^{-1} -> every term is 2^32 - 1: the sum must not wrap at 32 bits
    assert T.cks_words((-inv.astype(np.int64)).astype(np.uint32), g0) == n * 0xFFFFFFFF


def test_cks_word_index_wraps_mod_2_32():
    g0 = (1 << 32) - 3
    m = _weights(8, g0)
    inv = np.array([pow(x, -1, 1 << 32) for x in m], dtype=np.uint32)
    assert T.cks_words(inv, g0) == 8


def test_cks_additive_over_ranges():
    rng = np.random.default_rng(1)
    w = rng.integers(0, 1 << 32, 999, dtype=np.uint64).astype(np.uint32)
    whole = T.cks_words(w, 77)
    parts = T.cks_words(w[:400], 77) + T.cks_words(w[400:], 77 + 400)
    assert whole == parts


def test_cks_detects_every_single_bit_flip():
    rng = np.random.default_rng(2)
    w = rng.integers(0, 1 << 32, 64, dtype=np.uint64).astype(np.uint32)
    base = T.cks_words(w, 0)
    b = w.view(np.uint8)
    for i in range(b.size * 8):
        b2 = b.copy()
        b2[i // 8] ^= np.uint8(1 << (i % 8))
        assert T.cks_words(b2.view(np.uint32), 0) != base


def test_cks_detects_word_swaps():
    rng = np.random.default_rng(3)
    w = rng.integers(0, 1 << 32, 256, dtype=np.uint64).astype(np.uint32)
    base = T.cks_words(w, 0)
    hits = trials = 0
    for _ in range(200):
        i, j = rng.integers(0, 256, 2)
        if i == j or w[i] == w[j]:
            continue
        w2 = w.copy()
        w2[i], w2[j] = w[j], w[i]
        trials += 1
        hits += T.cks_words(w2, 0) != base
    assert trials > 150 and hits == trials


# ------------------------------------------------------- pack / seal / unpack
def _tensors(specs, seed, v):
    return [synth.vgen_numpy(seed, v, t, s[1], synth.nelem_of(s)) for t, s in enumerate(specs)]


@pytest.mark.parametrize("seed", range(12))
def test_pack_is_layout_copy_and_unpack_inverts(seed):
    rng = np.random.default_rng(100 + seed)
    specs = synth.random_specs(rng, int(rng.integers(1, 10)))
    ts = _tensors(specs, seed, 1)
    nb = [t.size for t in ts]
    off, s = T.layout(nb, 256)
    p = T.pack(ts, off, s)
    covered = np.zeros(s, dtype=bool)
    for t, o in zip(ts, off):
        assert np.array_equal(p[int(o): int(o) + t.size], t)
        covered[int(o): int(o) + t.size] = True
    assert not p[~covered].any()  # padding is zero
    back = T.unpack(p, nb, off)
    assert all(np.array_equal(a, b) for a, b in zip(back, ts))


def test_seal_chunks_and_verify():
    specs = synth.model_specs("ptychonn")
    ts = _tensors(specs, synth.SEEDS["ptychonn"], 3)
    off, s = T.layout([t.size for t in ts], 256)
    p = T.pack(ts, off, s)
    for cb in (4096, 65536, 2 << 20):
        seals = T.seal(p, cb, 3)
        assert seals.shape == (-(-s // cb), 2) and np.all(seals[:, 0] == 3)
        # chunk cks add up to the whole-buffer cks (additivity over ranges)
        assert int(seals[:, 1].astype(object).sum()) == T.cks_words(p, 0)
        assert T.verify(p, cb, 3, seals) == T.OK
        assert T.verify(p, cb, 4, seals) == T.E_VERSION
        q = p.copy()
        q[s - 7] ^= 0x40
        assert T.verify(q, cb, 3, seals) == T.E_CHECKSUM


def test_expected_chunk_matches_full_pack():
    specs = synth.model_specs("ptychonn")
    seed = synth.SEEDS["ptychonn"]
    ts = _tensors(specs, seed, 5)
    off, s = T.layout([t.size for t in ts], 256)
    p = T.pack(ts, off, s)
    cb = 1 << 20
    for c in range(T.nchunks(s, cb)):
        e = T.expected_chunk(specs, seed, 5, off, s, cb, c)
        assert np.array_equal(e, p[c * cb: min((c + 1) * cb, s)])
    assert T.expected_chunk_seal(specs, seed, 5, off, s, cb, 2) == int(T.seal(p, cb, 5)[2, 1])


# ------------------------------------------------ end-to-end oracle updates
def test_publish_installs_byte_exact_copy_10_versions():
    specs = synth.model_specs("ptychonn")
    seed = synth.SEEDS["ptychonn"]
    nb = [synth.nbytes_of(s) for s in specs]
    cons = [T.Consumer(nb), T.Consumer(nb)]
    prod = T.Producer(nb, cons)
    try:
        for v in range(1, 11):
            ts = _tensors(specs, seed, v)
            assert prod.publish(v, ts) == T.OK
            for c in cons:
                assert c.state >> 1 == v
                got = c.read_slot(c.state & 1)
                assert all(np.array_equal(a, b) for a, b in zip(got, ts))
        assert prod.publish(10, ts) == T.E_VERSION
        assert prod.publish(3, ts) == T.E_VERSION
    finally:
        prod.close()
        for c in cons:
            c.close()


def test_fault_injection_keeps_old_version():
    specs = synth.random_specs(np.random.default_rng(7), 6, max_bytes=3000)
    nb = [synth.nbytes_of(s) for s in specs]
    c = T.Consumer(nb, chunk_bytes=1024)
    p = T.Producer(nb, [c], chunk_bytes=1024)
    try:
        t1 = _tensors(specs, 1, 1)
        assert p.publish(1, t1) == T.OK
        c.corrupt_next()
        assert p.publish(2, _tensors(specs, 1, 2)) == T.E_CHECKSUM
        assert c.state >> 1 == 1
        got = c.read_slot(c.state & 1)
        assert all(np.array_equal(a, b) for a, b in zip(got, t1))
        assert p.publish(3, _tensors(specs, 1, 3)) == T.OK and c.state >> 1 == 3
    finally:
        p.close()
        c.close()


def test_acquire_release_errors():
    c = T.Consumer([16])
    try:
        assert c.acquire()[0] == T.E_NOVERSION
        assert c.release(0) == T.E_STATE
        assert c.release(5) == T.E_INVAL
    finally:
        c.close()


def test_no_torn_reads_under_concurrent_publish():
    """Readers verify every byte of the view they hold against VGEN(view.version)
    while the producer publishes back to back (P:1214-1227 'swapped atomically')."""
    specs = [(f"t{i}", synth.F32, (4096 + 7 * i,)) for i in range(6)]
    seed = 0xABC
    nb = [synth.nbytes_of(s) for s in specs]
    cache = {}

    def expect(v):
        if v not in cache:
            cache[v] = _tensors(specs, seed, v)
        return cache[v]

    for v in range(1, 61):
        expect(v)
    c = T.Consumer(nb, chunk_bytes=8192)
    p = T.Producer(nb, [c], chunk_bytes=8192)
    stop = threading.Event()
    errors, seen = [], []

    def reader():
        last = 0
        while not stop.is_set():
            st, v, slot = c.acquire()
            if st != T.OK:
                continue
            if v < last:
                errors.append(("regress", last, v))
            last = v
            got = c.read_slot(slot)
            exp = expect(v)
            if not all(np.array_equal(a, b) for a, b in zip(got, exp)):
                errors.append(("torn", v))
            seen.append(v)
            assert c.release(slot) == T.OK

    ths = [threading.Thread(target=reader) for _ in range(3)]
    try:
        for th in ths:
            th.start()
        for v in range(1, 61):
            assert p.publish(v, expect(v)) == T.OK
            time.sleep(0.002)  # let readers interleave (the GIL serialises them)
        stop.set()
        for th in ths:
            th.join()
        assert not errors, errors[:5]
        assert len(seen) > 20
        assert c.writes_while_pinned() == 0
        assert c.state >> 1 == 60
    finally:
        stop.set()
        p.close()
        c.close()
