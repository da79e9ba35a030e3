"""The golden chunk seals (tests/golden/seals/*.txt) that multi-GPU bench
lines and GPU tests compare every consumer against: written by
tools/make_golden_seals.py from the ORACLE only.  These CPU checks re-derive
sampled chunks with the oracle (first, last, and random ones) and the header
facts from the layout, so a stale or hand-edited file fails here."""
import random

import pytest

import synth
from oracle import transfer as T

MODELS = ["ptychonn", "resnet50", "vit_b16", "gpt2_xl", "llama3_8b"]


@pytest.mark.parametrize("name", MODELS)
def test_golden_header_matches_layout(name):
    hdr, cks = synth.golden_seals(name)
    specs = synth.model_specs(name)
    _, s = T.layout([synth.nbytes_of(sp) for sp in specs], 256)
    assert hdr["model"] == name and int(hdr["seed"], 16) == synth.SEEDS[name]
    assert hdr["s_packed"] == s and hdr["nchunks"] == T.nchunks(s, hdr["chunk_bytes"]) == len(cks)
    assert hdr["content_version"] == synth.VCHECK


@pytest.mark.parametrize("name", MODELS)
def test_golden_chunks_are_the_oracles(name):
    hdr, cks = synth.golden_seals(name)
    specs = synth.model_specs(name)
    off, s = T.layout([synth.nbytes_of(sp) for sp in specs], 256)
    n = len(cks)
    rng = random.Random(sum(map(ord, name)))
    sample = sorted({0, n - 1} | {rng.randrange(n) for _ in range(3)})
    for c in sample:
        assert T.expected_chunk_seal(specs, synth.SEEDS[name], synth.VCHECK, off, s, hdr["chunk_bytes"], c) == cks[c]


def test_golden_small_model_whole_packed_buffer():
    """PtychoNN: the whole packed buffer through the oracle's pack + seal equals
    the file (the chunk-by-chunk builder and the whole-buffer path agree)."""
    hdr, cks = synth.golden_seals("ptychonn")
    specs = synth.model_specs("ptychonn")
    ts = [synth.vgen_numpy(synth.SEEDS["ptychonn"], synth.VCHECK, i, sp[1], synth.nelem_of(sp))
          for i, sp in enumerate(specs)]
    off, s = T.layout([t.size for t in ts], 256)
    seals = T.seal(T.pack(ts, off, s), hdr["chunk_bytes"], 99)
    assert [int(x) for x in seals[:, 1]] == cks and (seals[:, 0] == 99).all()
