"""ctypes wrapper of oracle/viper_oracle.c -- ORACLE, test infrastructure only.

See oracle/__init__.py for who may import this.  The C file holds the
arithmetic; this module only marshals numpy arrays and builds the library with
gcc on first use (``build()``).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "viper_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

OK, E_INVAL, E_VERSION, E_CHECKSUM, E_NOVERSION, E_STATE = 0, -1, -4, -5, -7, -8

u64p = C.POINTER(C.c_uint64)


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain -O2; it is never tuned)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            L = C.CDLL(build())
            L.or_layout.restype = C.c_uint64
            L.or_layout.argtypes = [C.c_int32, u64p, C.c_uint32, u64p]
            L.or_cks_words.restype = C.c_uint64
            L.or_cks_words.argtypes = [C.c_void_p, C.c_uint64, C.c_uint64]
            L.or_nchunks.restype = C.c_uint64
            L.or_nchunks.argtypes = [C.c_uint64, C.c_uint64]
            L.or_seal.restype = None
            L.or_seal.argtypes = [C.c_void_p, C.c_uint64, C.c_uint64, C.c_uint64, u64p]
            L.or_pack.restype = None
            L.or_pack.argtypes = [C.c_int32, C.POINTER(C.c_void_p), u64p, u64p, C.c_void_p, C.c_uint64]
            L.or_unpack.restype = None
            L.or_unpack.argtypes = [C.c_int32, C.POINTER(C.c_void_p), u64p, u64p, C.c_void_p]
            L.or_verify.restype = C.c_int32
            L.or_verify.argtypes = [C.c_void_p, C.c_uint64, C.c_uint64, C.c_uint64, u64p]
            L.or_consumer_new.restype = C.c_void_p
            L.or_consumer_new.argtypes = [C.c_int32, u64p, C.c_uint32, C.c_uint64]
            L.or_consumer_free.argtypes = [C.c_void_p]
            L.or_producer_new.restype = C.c_void_p
            L.or_producer_new.argtypes = [C.c_int32, u64p, C.c_uint32, C.c_uint64, C.c_int32, C.POINTER(C.c_void_p)]
            L.or_producer_free.argtypes = [C.c_void_p]
            L.or_producer_packed.restype = C.c_void_p
            L.or_producer_packed.argtypes = [C.c_void_p]
            L.or_producer_seals.restype = C.c_void_p
            L.or_producer_seals.argtypes = [C.c_void_p]
            L.or_producer_s_packed.restype = C.c_uint64
            L.or_producer_s_packed.argtypes = [C.c_void_p]
            L.or_consumer_corrupt_next.argtypes = [C.c_void_p]
            L.or_consumer_state.restype = C.c_uint64
            L.or_consumer_state.argtypes = [C.c_void_p]
            L.or_consumer_writes_while_pinned.restype = C.c_uint64
            L.or_consumer_writes_while_pinned.argtypes = [C.c_void_p]
            L.or_consumer_slot_ptr.restype = C.c_void_p
            L.or_consumer_slot_ptr.argtypes = [C.c_void_p, C.c_int32, C.c_int32]
            L.or_install.restype = C.c_int32
            L.or_install.argtypes = [C.c_void_p, C.c_uint64]
            L.or_publish.restype = C.c_int32
            L.or_publish.argtypes = [C.c_void_p, C.c_uint64, C.POINTER(C.c_void_p)]
            L.or_acquire.restype = C.c_int32
            L.or_acquire.argtypes = [C.c_void_p, C.c_uint64, u64p, C.POINTER(C.c_int32)]
            L.or_release.restype = C.c_int32
            L.or_release.argtypes = [C.c_void_p, C.c_int32]
            _lib = L
    return _lib


def _u64arr(vals):
    a = np.ascontiguousarray(np.asarray(vals, dtype=np.uint64))
    return a, a.ctypes.data_as(u64p)


# ----------------------------------------------------------------- plain steps
def layout(nbytes, align: int = 256):
    """(offsets, S_packed) per DESIGN.md reading R16 (LAY)."""
    nb, nbp = _u64arr(nbytes)
    off = np.zeros(max(len(nb), 1), dtype=np.uint64)
    s = lib().or_layout(len(nb), nbp, align, off.ctypes.data_as(u64p))
    return off[: len(nb)].copy(), int(s)


def cks_words(buf: np.ndarray, g0: int = 0) -> int:
    """CKS of a little-endian u32 word buffer whose first word has global index g0."""
    w = np.ascontiguousarray(buf).view(np.uint32)
    return int(lib().or_cks_words(w.ctypes.data, w.size, g0))


def nchunks(s_packed: int, chunk_bytes: int) -> int:
    return int(lib().or_nchunks(s_packed, chunk_bytes))


def pack(tensors, offsets, s_packed: int) -> np.ndarray:
    """tensors: list of uint8 numpy arrays (raw bytes)."""
    ts = [np.ascontiguousarray(t, dtype=np.uint8) for t in tensors]
    out = np.empty(max(s_packed, 1), dtype=np.uint8)
    ptrs = (C.c_void_p * max(len(ts), 1))(*[t.ctypes.data for t in ts])
    nb, nbp = _u64arr([t.size for t in ts])
    off, offp = _u64arr(offsets)
    lib().or_pack(len(ts), ptrs, nbp, offp, out.ctypes.data, s_packed)
    return out[:s_packed]


def seal(packed: np.ndarray, chunk_bytes: int, version: int) -> np.ndarray:
    """(nchunks, 2) uint64 array of {version, cks}."""
    s = packed.size
    n = nchunks(s, chunk_bytes)
    out = np.zeros((max(n, 1), 2), dtype=np.uint64)
    lib().or_seal(packed.ctypes.data, s, chunk_bytes, version, out.ctypes.data_as(u64p))
    return out[:n]


def verify(packed: np.ndarray, chunk_bytes: int, version: int, seals: np.ndarray) -> int:
    s = np.ascontiguousarray(seals, dtype=np.uint64)
    return int(lib().or_verify(packed.ctypes.data, packed.size, chunk_bytes, version, s.ctypes.data_as(u64p)))


def unpack(packed: np.ndarray, nbytes, offsets):
    outs = [np.empty(int(n), dtype=np.uint8) for n in nbytes]
    ptrs = (C.c_void_p * max(len(outs), 1))(*[o.ctypes.data for o in outs])
    nb, nbp = _u64arr(nbytes)
    off, offp = _u64arr(offsets)
    lib().or_unpack(len(outs), ptrs, nbp, offp, packed.ctypes.data)
    return outs


# ------------------------------------------------------------- update engine
class Consumer:
    def __init__(self, nbytes, align=256, chunk_bytes=2 << 20):
        self.nbytes = [int(n) for n in nbytes]
        nb, nbp = _u64arr(self.nbytes)
        self.h = lib().or_consumer_new(len(nb), nbp, align, chunk_bytes)

    def close(self):
        if self.h:
            lib().or_consumer_free(self.h)
            self.h = None

    @property
    def state(self) -> int:
        return int(lib().or_consumer_state(self.h))

    def writes_while_pinned(self) -> int:
        return int(lib().or_consumer_writes_while_pinned(self.h))

    def corrupt_next(self):
        lib().or_consumer_corrupt_next(self.h)

    def read_slot(self, slot: int):
        out = []
        for t, n in enumerate(self.nbytes):
            p = lib().or_consumer_slot_ptr(self.h, slot, t)
            out.append(np.ctypeslib.as_array((C.c_uint8 * max(n, 1)).from_address(p))[:n].copy())
        return out

    def acquire(self, min_version: int = 0):
        v = C.c_uint64(0)
        s = C.c_int32(-1)
        st = lib().or_acquire(self.h, min_version, C.byref(v), C.byref(s))
        return st, int(v.value), int(s.value)

    def release(self, slot: int) -> int:
        return int(lib().or_release(self.h, slot))


class Producer:
    def __init__(self, nbytes, consumers, align=256, chunk_bytes=2 << 20):
        self.nbytes = [int(n) for n in nbytes]
        nb, nbp = _u64arr(self.nbytes)
        cs = (C.c_void_p * max(len(consumers), 1))(*[c.h for c in consumers])
        self.h = lib().or_producer_new(len(nb), nbp, align, chunk_bytes, len(consumers), cs)
        self.s_packed = int(lib().or_producer_s_packed(self.h))
        self.chunk_bytes = chunk_bytes

    def close(self):
        if self.h:
            lib().or_producer_free(self.h)
            self.h = None

    def publish(self, version: int, tensors) -> int:
        ts = [np.ascontiguousarray(t, dtype=np.uint8) for t in tensors]
        ptrs = (C.c_void_p * max(len(ts), 1))(*[t.ctypes.data for t in ts])
        return int(lib().or_publish(self.h, version, ptrs))

    def packed(self) -> np.ndarray:
        p = lib().or_producer_packed(self.h)
        return np.ctypeslib.as_array((C.c_uint8 * max(self.s_packed, 1)).from_address(p))[: self.s_packed].copy()

    def seals(self) -> np.ndarray:
        n = nchunks(self.s_packed, self.chunk_bytes)
        p = lib().or_producer_seals(self.h)
        return np.ctypeslib.as_array((C.c_uint64 * max(2 * n, 1)).from_address(p))[: 2 * n].reshape(n, 2).copy()


# ------------------------------------------------- sampled chunk seals (VGEN)
def expected_chunk(specs, seed: int, version: int, offsets, s_packed: int, chunk_bytes: int, c: int):
    """Packed bytes of chunk c of VGEN(seed, version) laid out by LAY, built one
    tensor range at a time (for configs too large to pack whole on the host)."""
    import synth

    lo = c * chunk_bytes
    hi = min(lo + chunk_bytes, s_packed)
    buf = np.zeros(hi - lo, dtype=np.uint8)
    for t, spec in enumerate(specs):
        n = synth.nbytes_of(spec)
        a, b = int(offsets[t]), int(offsets[t]) + n
        if b <= lo or a >= hi or n == 0:
            continue
        x0, x1 = max(a, lo), min(b, hi)
        buf[x0 - lo: x1 - lo] = synth.vgen_bytes_range(seed, version, t, spec[1], x0 - a, x1 - a)
    return buf


def expected_chunk_seal(specs, seed, version, offsets, s_packed, chunk_bytes, c) -> int:
    buf = expected_chunk(specs, seed, version, offsets, s_packed, chunk_bytes, c)
    return cks_words(buf, (c * chunk_bytes) // 4)
