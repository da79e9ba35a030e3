"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no layout, no checksum, no
version protocol).  It only answers two questions, identically for both sides:

1. *Which tensors does a workload have?*  -- ``model_specs(name)`` returns the
   ordered (name, dtype, shape) list of the parameter sets named by
   BASELINE.json ``configs`` (PtychoNN-sized, ResNet-50, ViT-B/16, GPT-2 XL,
   Llama-3 8B).  Shapes are written out from each architecture's definition
   (no torchvision / transformers import at run time); ``tests/test_synth.py``
   checks them against torchvision / transformers where those are importable.

2. *What bytes does producer tensor t hold at version v?*  -- VGEN, a
   counter-based generator (splitmix64, Steele/Lea/Flood 2014) so the CPU side
   (``vgen_numpy`` here) and the GPU side (``synth/vgen.cu``, a harness kernel
   standing in for the training step's optimizer write) produce the same bits
   without sharing code or state:

       k = splitmix64(seed ^ splitmix64((v << 20) ^ t))
       h = splitmix64(k + e)                       (e = element index)
       fp32 bits = (h>>63)<<31 | (119 + ((h>>32)&3))<<23 | (h & 0x7FFFFF)
       bf16 bits = (h>>63)<<15 | (119 + ((h>>32)&3))<<7  | (h & 0x7F)
       fp16 bits = (h>>63)<<15 | (7   + ((h>>32)&3))<<10 | (h & 0x3FF)
       byte      = h & 0xFF

   i.e. |x| in [2^-8, 2^-4) with random sign and random mantissa (finite,
   normal, incompressible), the scale of freshly initialised weights.
   Recipe per DESIGN.md "Input recipe"; seeds 0x5EED0001..0x5EED0005 per config.
"""
from __future__ import annotations

import numpy as np

MASK64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15

# dtype codes follow include/viper.h (viper_dtype)
F32, BF16, F16, BYTES = 0, 1, 2, 3
DTYPE_SIZE = {F32: 4, BF16: 2, F16: 2, BYTES: 1}
DTYPE_NAME = {F32: "f32", BF16: "bf16", F16: "f16", BYTES: "u8"}

SEEDS = {
    "ptychonn": 0x5EED0001,
    "resnet50": 0x5EED0002,
    "vit_b16": 0x5EED0003,
    "gpt2_xl": 0x5EED0004,
    "llama3_8b": 0x5EED0005,
    "nt3a_600mb": 0x5EED0006,
    "tc1_4p7gb": 0x5EED0007,
    "ptychonn_4p5gb": 0x5EED0008,
}


# --------------------------------------------------------------------------
# VGEN
# --------------------------------------------------------------------------
def splitmix64(x: int) -> int:
    """Scalar splitmix64 mix of x (python ints, exact)."""
    z = (x + GOLDEN) & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def _splitmix64_np(x: np.ndarray) -> np.ndarray:
    z = x + np.uint64(GOLDEN)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def tensor_key(seed: int, version: int, t: int) -> int:
    return splitmix64((seed ^ splitmix64(((version << 20) ^ t) & MASK64)) & MASK64)


def vgen_numpy(seed: int, version: int, t: int, dtype: int, nelem: int,
               e0: int = 0) -> np.ndarray:
    """Raw little-endian bytes of elements [e0, e0+nelem) of tensor t at version v."""
    k = tensor_key(seed, version, t)
    with np.errstate(over="ignore"):
        e = np.arange(e0, e0 + nelem, dtype=np.uint64)
        h = _splitmix64_np(e + np.uint64(k))
    sign = h >> np.uint64(63)
    ex = (h >> np.uint64(32)) & np.uint64(3)
    if dtype == F32:
        bits = (sign << np.uint64(31)) | ((np.uint64(119) + ex) << np.uint64(23)) | (h & np.uint64(0x7FFFFF))
        return bits.astype(np.uint32).view(np.uint8)
    if dtype == BF16:
        bits = (sign << np.uint64(15)) | ((np.uint64(119) + ex) << np.uint64(7)) | (h & np.uint64(0x7F))
        return bits.astype(np.uint16).view(np.uint8)
    if dtype == F16:
        bits = (sign << np.uint64(15)) | ((np.uint64(7) + ex) << np.uint64(10)) | (h & np.uint64(0x3FF))
        return bits.astype(np.uint16).view(np.uint8)
    if dtype == BYTES:
        return (h & np.uint64(0xFF)).astype(np.uint8)
    raise ValueError(f"bad dtype {dtype}")


def vgen_bytes_range(seed: int, version: int, t: int, dtype: int,
                     byte_lo: int, byte_hi: int) -> np.ndarray:
    """Bytes [byte_lo, byte_hi) of tensor t at version v (for sampled checks)."""
    es = DTYPE_SIZE[dtype]
    e0 = byte_lo // es
    e1 = (byte_hi + es - 1) // es
    raw = vgen_numpy(seed, version, t, dtype, e1 - e0, e0)
    return raw[byte_lo - e0 * es: byte_hi - e0 * es]


# --------------------------------------------------------------------------
# Workload tensor lists (BASELINE.json configs)
# --------------------------------------------------------------------------
def _ptychonn():
    """PtychoNN conv stack (20 conv3x3 weights + 20 biases, fp32).

    Encoder 1-32-32-64-64-128-128, two decoders 128-128-128-64-64-32-32-1.
    1,154,210 parameters."""
    out = []
    enc = [1, 32, 32, 64, 64, 128, 128]
    dec = [128, 128, 128, 64, 64, 32, 32, 1]
    for i in range(len(enc) - 1):
        out.append((f"encoder.{i}.weight", F32, (enc[i + 1], enc[i], 3, 3)))
        out.append((f"encoder.{i}.bias", F32, (enc[i + 1],)))
    for d in ("decoder1", "decoder2"):
        for i in range(len(dec) - 1):
            out.append((f"{d}.{i}.weight", F32, (dec[i + 1], dec[i], 3, 3)))
            out.append((f"{d}.{i}.bias", F32, (dec[i + 1],)))
    return out


def _resnet50():
    """torchvision resnet50() named_parameters order (161 tensors, fp32)."""
    out = [("conv1.weight", F32, (64, 3, 7, 7)), ("bn1.weight", F32, (64,)), ("bn1.bias", F32, (64,))]
    inp = 64
    for li, (nblocks, w) in enumerate(zip((3, 4, 6, 3), (64, 128, 256, 512)), start=1):
        for b in range(nblocks):
            p = f"layer{li}.{b}."
            out += [
                (p + "conv1.weight", F32, (w, inp, 1, 1)), (p + "bn1.weight", F32, (w,)), (p + "bn1.bias", F32, (w,)),
                (p + "conv2.weight", F32, (w, w, 3, 3)), (p + "bn2.weight", F32, (w,)), (p + "bn2.bias", F32, (w,)),
                (p + "conv3.weight", F32, (4 * w, w, 1, 1)), (p + "bn3.weight", F32, (4 * w,)), (p + "bn3.bias", F32, (4 * w,)),
            ]
            if b == 0:
                out += [(p + "downsample.0.weight", F32, (4 * w, inp, 1, 1)),
                        (p + "downsample.1.weight", F32, (4 * w,)), (p + "downsample.1.bias", F32, (4 * w,))]
            inp = 4 * w
    out += [("fc.weight", F32, (1000, 2048)), ("fc.bias", F32, (1000,))]
    return out


def _vit_b16():
    """torchvision vit_b_16() named_parameters order (152 tensors, bf16)."""
    d, mlp = 768, 3072
    out = [("class_token", BF16, (1, 1, d)), ("conv_proj.weight", BF16, (d, 3, 16, 16)),
           ("conv_proj.bias", BF16, (d,)), ("encoder.pos_embedding", BF16, (1, 197, d))]
    for i in range(12):
        p = f"encoder.layers.encoder_layer_{i}."
        out += [
            (p + "ln_1.weight", BF16, (d,)), (p + "ln_1.bias", BF16, (d,)),
            (p + "self_attention.in_proj_weight", BF16, (3 * d, d)), (p + "self_attention.in_proj_bias", BF16, (3 * d,)),
            (p + "self_attention.out_proj.weight", BF16, (d, d)), (p + "self_attention.out_proj.bias", BF16, (d,)),
            (p + "ln_2.weight", BF16, (d,)), (p + "ln_2.bias", BF16, (d,)),
            (p + "mlp.0.weight", BF16, (mlp, d)), (p + "mlp.0.bias", BF16, (mlp,)),
            (p + "mlp.3.weight", BF16, (d, mlp)), (p + "mlp.3.bias", BF16, (d,)),
        ]
    out += [("encoder.ln.weight", BF16, (d,)), ("encoder.ln.bias", BF16, (d,)),
            ("heads.head.weight", BF16, (1000, d)), ("heads.head.bias", BF16, (1000,))]
    return out


def _gpt2_xl():
    """HF GPT2LMHeadModel(n_embd=1600, n_layer=48, vocab 50257), tied head: 580 tensors, bf16."""
    d, L, V, P = 1600, 48, 50257, 1024
    out = [("transformer.wte.weight", BF16, (V, d)), ("transformer.wpe.weight", BF16, (P, d))]
    for i in range(L):
        p = f"transformer.h.{i}."
        out += [
            (p + "ln_1.weight", BF16, (d,)), (p + "ln_1.bias", BF16, (d,)),
            (p + "attn.c_attn.weight", BF16, (d, 3 * d)), (p + "attn.c_attn.bias", BF16, (3 * d,)),
            (p + "attn.c_proj.weight", BF16, (d, d)), (p + "attn.c_proj.bias", BF16, (d,)),
            (p + "ln_2.weight", BF16, (d,)), (p + "ln_2.bias", BF16, (d,)),
            (p + "mlp.c_fc.weight", BF16, (d, 4 * d)), (p + "mlp.c_fc.bias", BF16, (4 * d,)),
            (p + "mlp.c_proj.weight", BF16, (4 * d, d)), (p + "mlp.c_proj.bias", BF16, (d,)),
        ]
    out += [("transformer.ln_f.weight", BF16, (d,)), ("transformer.ln_f.bias", BF16, (d,))]
    return out


def _llama3_8b():
    """HF LlamaForCausalLM (hidden 4096, inter 14336, 32 layers, 8 KV heads, vocab 128256, untied): 291 tensors, bf16."""
    d, ff, L, V, kv = 4096, 14336, 32, 128256, 1024
    out = [("model.embed_tokens.weight", BF16, (V, d))]
    for i in range(L):
        p = f"model.layers.{i}."
        out += [
            (p + "self_attn.q_proj.weight", BF16, (d, d)), (p + "self_attn.k_proj.weight", BF16, (kv, d)),
            (p + "self_attn.v_proj.weight", BF16, (kv, d)), (p + "self_attn.o_proj.weight", BF16, (d, d)),
            (p + "mlp.gate_proj.weight", BF16, (ff, d)), (p + "mlp.up_proj.weight", BF16, (ff, d)),
            (p + "mlp.down_proj.weight", BF16, (d, ff)),
            (p + "input_layernorm.weight", BF16, (d,)), (p + "post_attention_layernorm.weight", BF16, (d,)),
        ]
    out += [("model.norm.weight", BF16, (d,)), ("lm_head.weight", BF16, (V, d))]
    return out


def _paper_sized(total_bytes: int, n_conv: int, dense_in: int):
    """fp32 parameter set of a given checkpoint size, shaped like the paper's
    1D-CNN workloads (CANDLE NT3/TC1: a few conv1d kernels, then dense layers
    holding almost all bytes; PAPER.md s5.2 P:2016-2054, sizes P:2115-2117)."""
    out = []
    ch = 1
    for i in range(n_conv):
        out.append((f"conv{i}.weight", F32, (128, ch, 20)))
        out.append((f"conv{i}.bias", F32, (128,)))
        ch = 128
    used = sum(nbytes_of(s) for s in out)
    left = (total_bytes - used) // 4
    # two dense layers: dense_in -> h (the bulk), h -> 200, then the head
    h = max(1, (left - 200 * 2 - 2) // (dense_in + 200 + 1))
    out += [("dense0.weight", F32, (h, dense_in)), ("dense0.bias", F32, (h,)),
            ("dense1.weight", F32, (200, h)), ("dense1.bias", F32, (200,)),
            ("head.weight", F32, (2, 200)), ("head.bias", F32, (2,))]
    return out


PAPER_SIZED = {  # PAPER.md P:2115-2117 checkpoint sizes (GB = 1e9 B, reading R18)
    "nt3a_600mb": lambda: _paper_sized(600_000_000, 2, 60483 * 2),
    "tc1_4p7gb": lambda: _paper_sized(4_700_000_000, 2, 60483 * 8),
    "ptychonn_4p5gb": lambda: _paper_sized(4_500_000_000, 4, 65536 * 4),
}

_RECIPES = {
    "ptychonn": _ptychonn,
    "resnet50": _resnet50,
    "vit_b16": _vit_b16,
    "gpt2_xl": _gpt2_xl,
    "llama3_8b": _llama3_8b,
}

# BASELINE.json configs index -> workload name
CONFIGS = ["ptychonn", "resnet50", "vit_b16", "gpt2_xl", "llama3_8b"]


def model_specs(name: str):
    """Ordered [(tensor_name, dtype, shape)] for a workload."""
    if name in PAPER_SIZED:
        return list(PAPER_SIZED[name]())
    return list(_RECIPES[name]())


def nbytes_of(spec) -> int:
    _, dt, shape = spec
    n = 1
    for s in shape:
        n *= s
    return n * DTYPE_SIZE[dt]


def nelem_of(spec) -> int:
    n = 1
    for s in spec[2]:
        n *= s
    return n


def model_bytes(name: str) -> int:
    return sum(nbytes_of(s) for s in model_specs(name))


def random_specs(rng: np.random.Generator, n: int, max_bytes: int = 67, dtypes=(F32, BF16, F16, BYTES)):
    """Small ragged tensor lists for brute-force tests (sizes may be 0)."""
    out = []
    for i in range(n):
        dt = int(rng.choice(dtypes))
        es = DTYPE_SIZE[dt]
        ne = int(rng.integers(0, max_bytes // es + 1))
        out.append((f"t{i}", dt, (ne,)))
    return out


# --------------------------------------------------------------------------
# Verification content (golden seals)
# --------------------------------------------------------------------------
# The VGEN version whose packed chunk checksums tools/make_golden_seals.py
# wrote into tests/golden/seals/<model>.txt with the ORACLE.  Multi-GPU bench
# runs and GPU tests publish this content as their last version and compare
# every consumer's installed seals against that file.
VCHECK = 7


def golden_seals(name: str):
    """(header dict, list of chunk cks ints) from tests/golden/seals/<name>.txt
    (values written by the oracle; this only parses the file), or None."""
    import os
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests", "golden", "seals",
                        f"{name}.txt")
    if not os.path.exists(path):
        return None
    with open(path) as f:
        head = f.readline().lstrip("#").split()
        hdr = {k: v for k, v in (kv.split("=", 1) for kv in head)}
        cks = [int(line, 16) for line in f if line.strip()]
    for k in ("content_version", "chunk_bytes", "s_packed", "nchunks"):
        hdr[k] = int(hdr[k])
    if hdr["nchunks"] != len(cks) or hdr["content_version"] != VCHECK:
        raise ValueError(f"{path}: malformed golden seal file")
    return hdr, cks
