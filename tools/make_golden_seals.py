#!/usr/bin/env python
"""Write tests/golden/seals/<model>.txt: the oracle's chunk checksums of one
fixed synthetic version of every BASELINE.json model.

The values come from the ORACLE only (oracle/transfer.py: LAY + CKS of
DESIGN.md R16, built chunk by chunk from synth's seeded input generator), never
from the CUDA path.  bench.py's N > 1 arm and the GPU tests publish exactly
this content (VGEN(seed, CONTENT_VERSION)) as their verification version and
compare every consumer's installed-slot seals (viper_view_seals) and the
producer's snapshot seals against these files, so a multi-GPU bench line
carries its own bit-exact evidence without running the oracle at bench time.

File format: a header line
    # model=<name> seed=<hex> content_version=<v> chunk_bytes=<b> s_packed=<S> nchunks=<n>
then n lines, chunk c's cks as 16 hex digits (the seal's version field is the
version it is published under, not part of the content).

Usage: python tools/make_golden_seals.py [model ...]   (default: all five)
"""
from __future__ import annotations

import multiprocessing as mp
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CONTENT_VERSION = 7  # VGEN version of the verification content (synth.VCHECK)
CHUNK_BYTES = 2 << 20
OUT_DIR = os.path.join(ROOT, "tests", "golden", "seals")


def _work(args):
    name, lo, hi = args
    import synth
    from oracle import transfer as T
    specs = synth.model_specs(name)
    off, s = T.layout([synth.nbytes_of(sp) for sp in specs], 256)
    return [T.expected_chunk_seal(specs, synth.SEEDS[name], CONTENT_VERSION, off, s, CHUNK_BYTES, c)
            for c in range(lo, hi)]


def make(name: str, procs: int) -> str:
    import synth
    from oracle import transfer as T
    assert synth.VCHECK == CONTENT_VERSION
    specs = synth.model_specs(name)
    _, s = T.layout([synth.nbytes_of(sp) for sp in specs], 256)
    n = T.nchunks(s, CHUNK_BYTES)
    step = max(1, (n + 4 * procs - 1) // (4 * procs))
    jobs = [(name, lo, min(n, lo + step)) for lo in range(0, n, step)]
    with mp.get_context("spawn").Pool(procs) as pool:
        cks = [c for part in pool.map(_work, jobs) for c in part]
    os.makedirs(OUT_DIR, exist_ok=True)
    path = os.path.join(OUT_DIR, f"{name}.txt")
    with open(path, "w") as f:
        f.write(f"# model={name} seed={synth.SEEDS[name]:#x} content_version={CONTENT_VERSION} "
                f"chunk_bytes={CHUNK_BYTES} s_packed={s} nchunks={n}\n")
        for c in cks:
            f.write(f"{c:016x}\n")
    return path


if __name__ == "__main__":
    names = sys.argv[1:] or ["ptychonn", "resnet50", "vit_b16", "gpt2_xl", "llama3_8b"]
    for nm in names:
        print(make(nm, os.cpu_count() or 4), flush=True)
