"""Background flush of published versions
and the verified restore.  The flushed file's packed bytes and chunk seals are
compared with the oracle's pack/seal of the same VGEN version."""
import glob
import os
import struct
import time

import numpy as np
import pytest
import torch

import synth
from oracle import transfer as T
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

pytestmark = pytest.mark.gpu


def read_flush(path):
    raw = open(path, "rb").read()
    magic = raw[:8]
    version, s_packed, nitems, nchunks, chunk_bytes, item_max = struct.unpack_from("<6Q", raw, 8)
    align, n = struct.unpack_from("<Ii", raw, 56)
    o = 64
    nbytes = np.frombuffer(raw, np.uint64, n, o); o += 8 * n
    offsets = np.frombuffer(raw, np.uint64, n, o); o += 8 * n
    o += 16 * nitems
    seals = np.frombuffer(raw, np.uint64, 2 * nchunks, o).reshape(nchunks, 2); o += 16 * nchunks
    packed = np.frombuffer(raw, np.uint8, s_packed, o)
    return dict(magic=magic, version=version, s_packed=s_packed, chunk_bytes=chunk_bytes, nbytes=nbytes,
                offsets=offsets, seals=seals, packed=packed, packed_off=o)


def expect(specs, seed, v):
    return [synth.vgen_numpy(seed, v, i, s[1], synth.nelem_of(s)) for i, s in enumerate(specs)]


@pytest.mark.parametrize("tier", [V.TIER_GPU, V.TIER_DRAM])
def test_flush_every_version_matches_oracle_and_restores(tmp_path, tier):
    specs = synth.model_specs("ptychonn")
    seed = synth.SEEDS["ptychonn"]
    pt, ct = G.alloc_model(specs), G.alloc_model(specs)
    name = f"fl{tier}-{time.monotonic_ns()}"
    c = V.Model(name, V.CONSUMER, ct, tier=tier)
    p = V.Model(name, V.PRODUCER, pt, tier=tier, flush_dir=str(tmp_path))
    for v in range(1, 6):
        G.fill_model(pt, specs, seed, v)
        p.publish(v)
        time.sleep(0.05)  # let storage keep up (a busy flusher skips, by design)
    c.close()
    st = p.stats()
    p.close()  # drains the flush queue
    files = sorted(glob.glob(str(tmp_path / f"{name}.v*.viper")))
    assert st["flushed"] + st["flush_skipped"] == 5 and st["flushed"] >= 3
    assert len(files) == st["flushed"]
    for f in files:
        d = read_flush(f)
        assert d["magic"] == b"VIPERCK1"
        exp = expect(specs, seed, d["version"])
        off, S = T.layout([e.size for e in exp], 256)
        p_or = T.pack(exp, off, S)
        assert d["s_packed"] == S and np.array_equal(d["offsets"], off)
        assert np.array_equal(d["packed"], p_or)
        assert np.array_equal(d["seals"], T.seal(p_or, d["chunk_bytes"], d["version"]))
    # restore the newest into fresh tensors
    fresh = G.alloc_model(specs)
    v = V.restore(files[-1], fresh)
    assert v == read_flush(files[-1])["version"]
    for g, e in zip(fresh, expect(specs, seed, v)):
        assert np.array_equal(g.contiguous().view(torch.uint8).reshape(-1).cpu().numpy(), e)


def test_restore_detects_corruption_and_mismatch(tmp_path):
    specs = [("a", synth.F32, (10_000,)), ("b", synth.BF16, (777,)), ("c", synth.BYTES, (13,))]
    pt, ct = G.alloc_model(specs), G.alloc_model(specs)
    name = f"flc-{time.monotonic_ns()}"
    c = V.Model(name, V.CONSUMER, ct)
    p = V.Model(name, V.PRODUCER, pt, flush_dir=str(tmp_path))
    G.fill_model(pt, specs, 4, 1)
    p.publish(1)
    c.close()
    p.close()
    f = glob.glob(str(tmp_path / f"{name}.v*.viper"))[0]
    d = read_flush(f)
    bad = str(tmp_path / "bad.viper")
    raw = bytearray(open(f, "rb").read())
    raw[d["packed_off"] + 20011] ^= 0x04
    open(bad, "wb").write(bytes(raw))
    with pytest.raises(V.ViperError) as ei:
        V.restore(bad, G.alloc_model(specs))
    assert ei.value.status == V.E_CHECKSUM
    with pytest.raises(V.ViperError) as ei:
        V.restore(f, G.alloc_model(specs[:2]))
    assert ei.value.status == V.E_INVAL
    ok = G.alloc_model(specs)
    assert V.restore(f, ok) == 1
