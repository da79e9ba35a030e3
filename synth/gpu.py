"""GPU side of the input generator: ctypes wrapper of synth/libvgen.so (harness
kernel writing VGEN bits into producer tensors; see synth/__init__.py)."""
from __future__ import annotations

import ctypes as C
import os

_LIB = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libvgen.so")
_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB):
            raise ImportError(f"{_LIB} missing -- run __graft_entry__.build()")
        _lib = C.CDLL(_LIB)
        _lib.vgen_fill.argtypes = [C.c_void_p, C.c_uint64, C.c_uint64, C.c_uint64, C.c_int32, C.c_uint64, C.c_void_p]
        _lib.vgen_fill.restype = C.c_int
        _lib.l2_flush.argtypes = [C.c_void_p, C.c_uint64, C.c_void_p]
        _lib.l2_flush.restype = C.c_int
        _lib.l2_flush_clean.argtypes = [C.c_void_p, C.c_uint64, C.c_void_p]
        _lib.l2_flush_clean.restype = C.c_int
        _lib.launch_empty.argtypes = [C.c_void_p]
        _lib.launch_empty.restype = C.c_int
        _lib.host_alloc.argtypes = [C.c_uint64]
        _lib.host_alloc.restype = C.c_void_p
        _lib.host_free.argtypes = [C.c_void_p]
        _lib.copy_async.argtypes = [C.c_void_p, C.c_void_p, C.c_uint64, C.c_int, C.c_void_p]
        _lib.copy_async.restype = C.c_int
    return _lib


def _sp(stream):
    return None if stream is None else C.c_void_p(stream.cuda_stream)


def fill(t, seed: int, version: int, index: int, dtype: int, stream=None):
    """Write VGEN(seed, version, index, e) into CUDA tensor t (raw bytes)."""
    from . import DTYPE_SIZE
    n = t.numel() * t.element_size() // DTYPE_SIZE[dtype]
    if lib().vgen_fill(C.c_void_p(t.data_ptr()), seed, version, index, dtype, n, _sp(stream)) != 0:
        raise RuntimeError("vgen_fill failed")


def fill_model(tensors, specs, seed: int, version: int, stream=None):
    for i, (t, s) in enumerate(zip(tensors, specs)):
        fill(t, seed, version, i, s[1], stream)


def alloc_model(specs, device=None):
    """Allocate one CUDA tensor per spec (torch dtype matching the spec), on
    `device` or else on the current CUDA device (one process per GPU)."""
    import torch
    device = device if device is not None else torch.device("cuda", torch.cuda.current_device())
    from . import F32, BF16, F16
    dt = {F32: torch.float32, BF16: torch.bfloat16, F16: torch.float16}
    return [torch.empty(s[2], dtype=dt.get(s[1], torch.uint8), device=device) for s in specs]


def l2_flush(buf, stream=None, clean=False):
    """Evict L2 between timed steps by writing `buf` (> L2).  clean=True: write
    its first half, then read its second half (each half > L2), so the dirty
    lines are written back inside the flush and L2 holds clean unrelated data
    (ncu's cache-control state) instead of ~126 MB of dirty harness lines that
    the next kernel would have to write back."""
    fn = lib().l2_flush_clean if clean else lib().l2_flush
    if fn(C.c_void_p(buf.data_ptr()), buf.numel() * buf.element_size(), _sp(stream)) != 0:
        raise RuntimeError("l2_flush failed")


def empty_kernel(stream=None):
    if lib().launch_empty(_sp(stream)) != 0:
        raise RuntimeError("launch_empty failed")


H2D, D2H = 1, 2


class PinnedBuffer:
    """cudaHostAlloc'ed host buffer (bench e2e leg) with raw async copies."""

    def __init__(self, nbytes: int):
        self.nbytes = nbytes
        self.ptr = lib().host_alloc(max(nbytes, 1))
        if not self.ptr:
            raise MemoryError("cudaHostAlloc failed")

    def view(self):
        import numpy as np
        return np.ctypeslib.as_array((C.c_uint8 * max(self.nbytes, 1)).from_address(self.ptr))[: self.nbytes]

    def to_device(self, dev_tensor, stream=None):
        if lib().copy_async(C.c_void_p(dev_tensor.data_ptr()), C.c_void_p(self.ptr), self.nbytes, H2D, _sp(stream)):
            raise RuntimeError("H2D failed")

    def from_device_ptr(self, dev_ptr: int, nbytes: int, stream=None):
        if lib().copy_async(C.c_void_p(self.ptr), C.c_void_p(dev_ptr), nbytes, D2H, _sp(stream)):
            raise RuntimeError("D2H failed")

    def close(self):
        if self.ptr:
            lib().host_free(C.c_void_p(self.ptr))
            self.ptr = None
