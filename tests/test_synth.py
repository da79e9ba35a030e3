"""Input generator checks (synth/): VGEN against published SplitMix64 outputs,
workload tensor lists against torchvision / transformers, sizes vs SURVEY s8(d)."""
import json
import os

import numpy as np
import pytest

import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_splitmix64_published_vectors():
    vals = [int(l, 16) for l in open(os.path.join(GOLD, "splitmix64_seed0.txt")) if l.startswith("0x")]
    got = [synth.splitmix64((n * synth.GOLDEN) & synth.MASK64) for n in range(len(vals))]
    assert got == vals


def test_vgen_numpy_matches_scalar():
    seed, v, t = 0x5EED0001, 7, 3
    k = synth.tensor_key(seed, v, t)
    raw = synth.vgen_numpy(seed, v, t, synth.F32, 64).view(np.uint32)
    for e in range(64):
        h = synth.splitmix64((k + e) & synth.MASK64)
        bits = (h >> 63) << 31 | (119 + ((h >> 32) & 3)) << 23 | (h & 0x7FFFFF)
        assert int(raw[e]) == bits


@pytest.mark.parametrize("dt", [synth.F32, synth.BF16, synth.F16])
def test_vgen_value_range(dt):
    raw = synth.vgen_numpy(0x5EED0003, 1, 0, dt, 4096)
    if dt == synth.F32:
        x = raw.view(np.float32).astype(np.float64)
    elif dt == synth.F16:
        x = raw.view(np.float16).astype(np.float64)
    else:
        x = (raw.view(np.uint16).astype(np.uint32) << 16).view(np.float32).astype(np.float64)
    a = np.abs(x)
    assert np.all(np.isfinite(x)) and np.all(a >= 2.0 ** -8) and np.all(a < 2.0 ** -4)
    assert 0.4 < np.mean(x > 0) < 0.6


def test_vgen_ranges_consistent():
    whole = synth.vgen_numpy(1, 2, 3, synth.BF16, 1000)
    part = synth.vgen_bytes_range(1, 2, 3, synth.BF16, 101, 1377)
    assert np.array_equal(whole[101:1377], part)


def test_versions_and_tensors_differ():
    a = synth.vgen_numpy(9, 1, 0, synth.F32, 256)
    b = synth.vgen_numpy(9, 2, 0, synth.F32, 256)
    c = synth.vgen_numpy(9, 1, 1, synth.F32, 256)
    assert (a != b).mean() > 0.9 and (a != c).mean() > 0.9


def test_model_sizes_match_survey():
    gold = json.load(open(os.path.join(GOLD, "model_sizes.json")))
    for name in synth.CONFIGS:
        specs = synth.model_specs(name)
        assert len(specs) == gold[name]["tensors"], name
        assert synth.model_bytes(name) == gold[name]["bytes"], name


def _torch_shapes(model):
    return [(n, tuple(p.shape)) for n, p in model.named_parameters()]


def test_resnet50_vit_match_torchvision():
    tv = pytest.importorskip("torchvision")
    import torch
    with torch.device("meta"):
        r = tv.models.resnet50()
        v = tv.models.vit_b_16()
    assert _torch_shapes(r) == [(n, s) for n, _, s in synth.model_specs("resnet50")]
    assert _torch_shapes(v) == [(n, s) for n, _, s in synth.model_specs("vit_b16")]


def test_gpt2_llama_match_transformers():
    tr = pytest.importorskip("transformers")
    import torch
    with torch.device("meta"):
        g = tr.GPT2LMHeadModel(tr.GPT2Config(n_embd=1600, n_layer=48, n_head=25))
        l = tr.LlamaForCausalLM(tr.LlamaConfig(hidden_size=4096, intermediate_size=14336, num_hidden_layers=32,
                                               num_attention_heads=32, num_key_value_heads=8, vocab_size=128256,
                                               tie_word_embeddings=False))
    assert _torch_shapes(g) == [(n, s) for n, _, s in synth.model_specs("gpt2_xl")]
    assert _torch_shapes(l) == [(n, s) for n, _, s in synth.model_specs("llama3_8b")]
