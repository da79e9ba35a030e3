"""Thin ctypes binding of libviper.so (include/viper.h).  Argument marshalling
only: every step of the model-update path runs in the library's CUDA kernels.
There is no fallback -- if libviper.so is missing or no GPU is visible, the
calls raise.
"""
from __future__ import annotations

import ctypes as C
import os
import threading

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("VIPER_LIB_PATH") or os.path.join(_HERE, "libviper.so")  # override: tuning variants

OK, E_INVAL, E_NOMEM, E_CUDA, E_VERSION, E_CHECKSUM, E_TIMEOUT, E_NOVERSION, E_STATE, E_UNSUPPORTED, E_PEER = (
    0, -1, -2, -3, -4, -5, -6, -7, -8, -9, -10)
PRODUCER, CONSUMER = 1, 2
F32, BF16, F16, BYTES = 0, 1, 2, 3
TIER_GPU, TIER_DRAM, TIER_AUTO = 0, 1, 2
FANOUT_DIRECT, FANOUT_CHAIN, FANOUT_SCATTER_ALLGATHER, FANOUT_NVLS, FANOUT_PUSH = 0, 1, 2, 3, 4
FANOUT_NCCL, FANOUT_CE = 100, 101  # baselines (include/viper.h)
SYNC, ASYNC = 0, 1
FLAG_TIMING = 2
FLAG_NO_FUSE = 4
FLAG_TMA = 8
FLAG_NO_TMA = 16
FLAG_FUSED_TMA = 32
SCHED_FIXED, SCHED_GREEDY = 0, 1


class viper_tensor(C.Structure):
    _fields_ = [("name", C.c_char_p), ("dtype", C.c_int32), ("ndim", C.c_int32),
                ("shape", C.POINTER(C.c_int64)), ("dev_ptr", C.c_void_p), ("nbytes", C.c_uint64)]


ALLGATHER_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p)


class viper_bootstrap(C.Structure):
    _fields_ = [("rank", C.c_int32), ("world", C.c_int32), ("producer_rank", C.c_int32),
                ("allgather", ALLGATHER_FN), ("user", C.c_void_p), ("nproducers", C.c_int32)]


class viper_config(C.Structure):
    _fields_ = [("tier", C.c_int32), ("fanout", C.c_int32), ("mode", C.c_int32), ("chunk_bytes", C.c_uint64),
                ("align", C.c_uint32), ("device", C.c_int32), ("slot1", C.POINTER(viper_tensor)),
                ("flags", C.c_int32), ("flush_dir", C.c_char_p), ("install_sms", C.c_int32)]


class viper_view(C.Structure):
    _fields_ = [("version", C.c_uint64), ("slot", C.c_int32), ("ntensors", C.c_int32),
                ("dev_ptrs", C.POINTER(C.c_void_p)), ("ticket", C.c_uint64)]


class viper_stats(C.Structure):
    _fields_ = [("version", C.c_uint64), ("s_packed", C.c_uint64), ("nchunks", C.c_uint64), ("nitems", C.c_uint64),
                ("installs", C.c_uint64), ("skipped", C.c_uint64), ("failures", C.c_uint64),
                ("t_publish_us", C.c_double), ("t_install_us", C.c_double), ("t_notify_us", C.c_double),
                ("writer_wait_us", C.c_double), ("t_pack_dev_us", C.c_double),
                ("t_install_dev_us", C.c_double), ("t_fused_dev_us", C.c_double), ("last_status", C.c_int32), ("nconsumers", C.c_int32),
                ("flushed", C.c_uint64), ("flush_skipped", C.c_uint64), ("flush_last", C.c_uint64),
                ("tier", C.c_int32), ("fanout", C.c_int32), ("t_pickup_us", C.c_double)]


class viper_sched_in(C.Structure):
    _fields_ = [("losses", C.POINTER(C.c_double)), ("x", C.POINTER(C.c_double)), ("n", C.c_int32),
                ("s_iter", C.c_int64), ("e_iter", C.c_int64), ("total_infers", C.c_int64),
                ("t_train", C.c_double), ("t_infer", C.c_double), ("s_model", C.c_double),
                ("bw_write", C.c_double), ("bw_read", C.c_double), ("t_p", C.c_double), ("t_c", C.c_double),
                ("algo", C.c_int32), ("thresh", C.c_double), ("family", C.c_int32), ("params", C.c_double * 3)]


class viper_sched_out(C.Structure):
    _fields_ = [("family", C.c_int32), ("params", C.c_double * 3), ("mse", C.c_double * 4), ("t_p", C.c_double),
                ("t_c", C.c_double), ("thresh", C.c_double), ("best_interval", C.c_int64),
                ("sched", C.POINTER(C.c_int64)), ("sched_cap", C.c_int64), ("sched_len", C.c_int64),
                ("predicted_cil", C.c_double)]


UPDATE_CB = C.CFUNCTYPE(None, C.c_uint64, C.c_int32, C.c_void_p)

# every symbol include/viper.h declares (checked by tests/test_abi.py)
EXPORTS = ["viper_register_model", "viper_publish", "viper_subscribe", "viper_acquire_latest", "viper_release",
           "viper_wait_installed", "viper_get_stats", "viper_layout", "viper_debug_buffers", "viper_debug_fault_next", "viper_unregister",
           "viper_view_seals",
           "viper_schedule", "viper_restore", "viper_strerror", "viper_last_error", "viper_version",
           "viper_debug_proto_create", "viper_debug_proto_open", "viper_debug_proto_close",
           "viper_debug_proto_publish", "viper_debug_proto_install", "viper_debug_proto_read",
           "viper_debug_resolve_tier", "viper_debug_fd_listen", "viper_debug_fd_serve", "viper_debug_fd_fetch"]

_lib = None
_lock = threading.Lock()
_fast = None  # CPython shim for publish / acquire / release (csrc/pyfast.c), same libviper.so symbols


class ViperError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        L = lib()
        self.name = L.viper_strerror(status).decode()
        self.detail = L.viper_last_error().decode()
        super().__init__(f"{where}: {self.name} ({status}): {self.detail}")


def lib() -> C.CDLL:
    """Load libviper.so (raises if it was not built: there is no fallback)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise ImportError(f"{LIB_PATH} missing -- run __graft_entry__.build() "
                                  f"(python paper_conf_icpp_yecrbypnmskn24_b200/build.py)")
            L = C.CDLL(LIB_PATH)
            L.viper_register_model.argtypes = [C.c_char_p, C.c_int32, C.POINTER(viper_tensor), C.c_int32,
                                               C.POINTER(viper_config), C.POINTER(viper_bootstrap),
                                               C.POINTER(C.c_void_p)]
            L.viper_publish.argtypes = [C.c_void_p, C.c_uint64, C.c_void_p]
            L.viper_subscribe.argtypes = [C.c_void_p, UPDATE_CB, C.c_void_p]
            L.viper_acquire_latest.argtypes = [C.c_void_p, C.c_uint64, C.c_int64, C.POINTER(viper_view)]
            L.viper_release.argtypes = [C.c_void_p, C.POINTER(viper_view), C.c_void_p]
            L.viper_wait_installed.argtypes = [C.c_void_p, C.c_uint64, C.c_int64]
            L.viper_get_stats.argtypes = [C.c_void_p, C.POINTER(viper_stats)]
            L.viper_layout.argtypes = [C.c_void_p, C.POINTER(C.c_uint64), C.POINTER(C.c_uint64), C.c_int32]
            L.viper_debug_buffers.argtypes = [C.c_void_p, C.POINTER(C.c_void_p), C.POINTER(C.c_void_p),
                                              C.POINTER(C.c_uint64)]
            L.viper_debug_fault_next.argtypes = [C.c_void_p]
            L.viper_view_seals.argtypes = [C.c_void_p, C.POINTER(viper_view), C.c_void_p, C.c_void_p]
            L.viper_unregister.argtypes = [C.c_void_p]
            L.viper_schedule.argtypes = [C.POINTER(viper_sched_in), C.POINTER(viper_sched_out)]
            L.viper_debug_proto_create.argtypes = [C.c_char_p, C.c_uint64, C.c_int32, C.POINTER(C.c_void_p)]
            L.viper_debug_proto_open.argtypes = [C.c_char_p, C.c_uint64, C.POINTER(C.c_void_p)]
            L.viper_debug_proto_close.argtypes = [C.c_void_p, C.c_int32, C.c_char_p]
            L.viper_debug_proto_publish.argtypes = [C.c_void_p, C.c_uint64]
            L.viper_debug_proto_install.argtypes = [C.c_void_p, C.c_int32, C.POINTER(C.c_uint64),
                                                    C.POINTER(C.c_uint64)]
            L.viper_debug_proto_read.argtypes = [C.c_void_p, C.c_int32, C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)]
            L.viper_debug_resolve_tier.argtypes = [C.c_void_p, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_int32,
                                                   C.POINTER(C.c_int32)]
            L.viper_restore.argtypes = [C.c_char_p, C.POINTER(viper_tensor), C.c_int32, C.c_int32, C.c_void_p,
                                        C.POINTER(C.c_uint64)]
            L.viper_debug_fd_listen.argtypes = [C.c_char_p, C.c_int32, C.POINTER(C.c_int32)]
            L.viper_debug_fd_serve.argtypes = [C.c_int32, C.c_int32, C.c_int32, C.c_int32]
            L.viper_debug_fd_fetch.argtypes = [C.c_char_p, C.POINTER(C.c_int32), C.c_int64]
            L.viper_strerror.argtypes = [C.c_int32]
            L.viper_strerror.restype = C.c_char_p
            L.viper_last_error.restype = C.c_char_p
            L.viper_version.restype = C.c_char_p
            for f in EXPORTS:
                fn = getattr(L, f)
                if fn.restype is C.c_int:  # default
                    fn.restype = C.c_int32
            global _fast
            try:
                from . import _fast as F
                F.init(LIB_PATH)
                _fast = F
            except ImportError:
                _fast = None
            _lib = L
    return _lib


def check(st: int, where: str):
    if st != OK:
        raise ViperError(st, where)


def _dtype_code(t) -> int:
    import torch
    return {torch.float32: F32, torch.bfloat16: BF16, torch.float16: F16}.get(t.dtype, BYTES)


def _tensor_descs(tensors, names=None):
    """torch tensors (contiguous, CUDA) -> viper_tensor array (+ keepalive)."""
    n = len(tensors)
    arr = (viper_tensor * max(n, 1))()
    keep = []
    for i, t in enumerate(tensors):
        if not t.is_contiguous():
            raise ValueError(f"tensor {i} is not contiguous")
        shape = (C.c_int64 * max(t.dim(), 1))(*t.shape)
        nm = (names[i] if names else f"t{i}").encode()
        keep += [shape, nm]
        arr[i] = viper_tensor(nm, _dtype_code(t), t.dim(), shape, C.c_void_p(t.data_ptr()), t.numel() * t.element_size())
    return arr, keep


class View:
    def __init__(self, model: "Model", raw: viper_view):
        self.model = model
        self.raw = raw
        self.version = int(raw.version)
        self.slot = int(raw.slot)
        self.ptrs = [int(raw.dev_ptrs[i] or 0) for i in range(raw.ntensors)]

    def tensors(self, like):
        """Zero-copy torch views of the pinned slot, shaped/typed like `like`."""
        return [_from_ptr(p, t) for p, t in zip(self.ptrs, like)]


class _CAI:
    def __init__(self, ptr, t):
        import torch
        typestr = {torch.float32: "<f4", torch.float16: "<f2", torch.float64: "<f8", torch.uint8: "|u1",
                   torch.int8: "|i1", torch.int16: "<i2", torch.int32: "<i4", torch.int64: "<i8",
                   torch.bool: "|b1"}[t.dtype if t.dtype != torch.bfloat16 else torch.int16]
        self.__cuda_array_interface__ = {"shape": tuple(t.shape), "typestr": typestr, "data": (ptr, False),
                                         "version": 3, "strides": None}


def _from_ptr(ptr, like):
    import torch
    if like.numel() == 0:
        return torch.empty_like(like)
    out = torch.as_tensor(_CAI(ptr, like), device=like.device)
    return out.view(torch.bfloat16) if like.dtype == torch.bfloat16 else out


class Model:
    """One endpoint (producer or consumer) of a model-update channel."""

    def __init__(self, name: str, role: int, tensors, *, tier=TIER_GPU, fanout=FANOUT_DIRECT, mode=SYNC,
                 chunk_bytes=0, align=0, device=None, slot1=None, flags=0, bootstrap=None, names=None,
                 flush_dir=None, install_sms=0):
        L = lib()
        self.tensors = list(tensors)
        self.role = role
        if device is None:
            device = self.tensors[0].device.index if self.tensors and self.tensors[0].is_cuda else 0
        descs, self._keep = _tensor_descs(self.tensors, names)
        self._flush_dir = flush_dir.encode() if flush_dir else None
        cfg = viper_config(tier, fanout, mode, chunk_bytes, align, device, None, flags, self._flush_dir, install_sms)
        if slot1 is not None:
            s1, k1 = _tensor_descs(slot1, names)
            self._keep += [s1, k1]
            cfg.slot1 = C.cast(s1, C.POINTER(viper_tensor))
        self._bs = None
        if bootstrap is not None:
            self._bs = bootstrap.struct()
        h = C.c_void_p()
        check(L.viper_register_model(name.encode(), role, descs, len(self.tensors), C.byref(cfg),
                                     C.byref(self._bs) if self._bs is not None else None, C.byref(h)),
              "viper_register_model")
        self.h = h
        self._cb = None

    # -- producer
    def publish(self, version: int, stream=None):
        if _fast is not None:
            st = _fast.publish(self.h.value, version, None if stream is None else
                               (stream if isinstance(stream, int) else stream.cuda_stream))
        else:
            st = lib().viper_publish(self.h, version, _stream_ptr(stream))
        if st:
            raise ViperError(st, f"viper_publish({version})")

    # -- consumer
    def subscribe(self, fn):
        self._cb = UPDATE_CB(lambda v, st, u: fn(int(v), int(st))) if fn else UPDATE_CB()
        check(lib().viper_subscribe(self.h, self._cb, None), "viper_subscribe")

    def acquire_latest(self, min_version=0, timeout_us=0) -> View:
        if _fast is not None:
            st, ver, slot, nt, ptrs, ticket = _fast.acquire(self.h.value, min_version, timeout_us)
            if st:
                raise ViperError(st, "viper_acquire_latest")
            v = viper_view(ver, slot, nt, C.cast(C.c_void_p(ptrs), C.POINTER(C.c_void_p)), ticket)
            return View(self, v)
        v = viper_view()
        check(lib().viper_acquire_latest(self.h, min_version, timeout_us, C.byref(v)), "viper_acquire_latest")
        return View(self, v)

    def release(self, view: View, stream=None):
        if _fast is not None:
            r = view.raw
            st = _fast.release(self.h.value, r.version, r.slot, r.ntensors,
                               C.cast(r.dev_ptrs, C.c_void_p).value or 0, r.ticket,
                               None if stream is None else (stream if isinstance(stream, int) else stream.cuda_stream))
            if st:
                raise ViperError(st, "viper_release")
            return
        check(lib().viper_release(self.h, C.byref(view.raw), _stream_ptr(stream)), "viper_release")

    def wait_installed(self, version: int, timeout_us: int = 10_000_000):
        check(lib().viper_wait_installed(self.h, version, timeout_us), f"viper_wait_installed({version})")

    def view_seals(self, view: View, out, stream=None):
        """Chunk seals {version, cks} of a pinned view's slot into `out` (a CUDA
        tensor of >= 16 * nchunks bytes), computed on the device."""
        check(lib().viper_view_seals(self.h, C.byref(view.raw), C.c_void_p(out.data_ptr()), _stream_ptr(stream)),
              "viper_view_seals")

    def fault_next(self):
        check(lib().viper_debug_fault_next(self.h), "viper_debug_fault_next")

    # -- both
    def stats(self) -> dict:
        s = viper_stats()
        check(lib().viper_get_stats(self.h, C.byref(s)), "viper_get_stats")
        return {f: getattr(s, f) for f, _ in viper_stats._fields_}

    def layout(self):
        s = C.c_uint64()
        n = len(self.tensors)
        off = (C.c_uint64 * max(n, 1))()
        check(lib().viper_layout(self.h, C.byref(s), off, n), "viper_layout")
        return int(s.value), [int(off[i]) for i in range(n)]

    def debug_buffers(self):
        p, s, n = C.c_void_p(), C.c_void_p(), C.c_uint64()
        check(lib().viper_debug_buffers(self.h, C.byref(p), C.byref(s), C.byref(n)), "viper_debug_buffers")
        return p.value or 0, s.value or 0, int(n.value)

    def close(self):
        if self.h:
            check(lib().viper_unregister(self.h), "viper_unregister")
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def _stream_ptr(stream):
    if stream is None:
        return None
    if isinstance(stream, int):
        return C.c_void_p(stream)
    return C.c_void_p(stream.cuda_stream)


class Bootstrap:
    """Cross-process bootstrap over a torch.distributed process group."""

    def __init__(self, rank: int, world: int, producer_rank: int = 0, group=None, nproducers: int = 1):
        """nproducers > 1: ranks producer_rank .. producer_rank+nproducers-1 are
        data-parallel producers, each packing its share of the chunks."""
        self.rank, self.world, self.producer_rank, self.group = rank, world, producer_rank, group
        self.nproducers = nproducers

    def _allgather(self, inp, out, nbytes, user):
        try:
            import torch
            import torch.distributed as dist
            src = bytes((C.c_char * nbytes).from_address(inp))
            t = torch.frombuffer(bytearray(src), dtype=torch.uint8)
            backend = dist.get_backend(self.group)
            dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")
            t = t.to(dev)
            outs = [torch.empty_like(t) for _ in range(self.world)]
            dist.all_gather(outs, t, group=self.group)
            blob = b"".join(bytes(o.cpu().numpy().tobytes()) for o in outs)
            C.memmove(out, blob, len(blob))
            return 0
        except Exception:  # never let a Python exception cross the C boundary
            return -1

    def struct(self) -> viper_bootstrap:
        self._fn = ALLGATHER_FN(self._allgather)
        return viper_bootstrap(self.rank, self.world, self.producer_rank, self._fn, None, self.nproducers)


def restore(path: str, tensors, device=None, stream=None) -> int:
    """Install a flushed version (viper_restore) into `tensors`; returns its version."""
    if device is None:
        device = tensors[0].device.index if tensors and tensors[0].is_cuda else 0
    descs, keep = _tensor_descs(list(tensors))
    v = C.c_uint64(0)
    check(lib().viper_restore(path.encode(), descs, len(tensors), device, _stream_ptr(stream), C.byref(v)),
          f"viper_restore({path})")
    return int(v.value)


def schedule(losses=None, *, s_iter, e_iter, total_infers, t_train, t_infer, t_p=-1.0, t_c=-1.0, s_model=0.0,
             bw_write=0.0, bw_read=0.0, algo=SCHED_FIXED, thresh=-1.0, x=None, family=-1, params=None) -> dict:
    L = lib()
    n = len(losses) if losses is not None else 0
    la = (C.c_double * max(n, 1))(*(losses if n else []))
    xa = (C.c_double * max(n, 1))(*x) if x is not None else None
    p3 = (C.c_double * 3)(*(list(params) + [0.0] * (3 - len(params)) if params is not None else [0, 0, 0]))
    si = viper_sched_in(la if n else None, xa, n, s_iter, e_iter, total_infers, t_train, t_infer, s_model,
                        bw_write, bw_read, t_p, t_c, algo, thresh, family, p3)
    so = viper_sched_out()
    so.sched = None
    so.sched_cap = 0
    st = L.viper_schedule(C.byref(si), C.byref(so))
    if st == E_INVAL and so.sched_len > 0:  # size query
        buf = (C.c_int64 * so.sched_len)()
        so.sched = buf
        so.sched_cap = so.sched_len
        st = L.viper_schedule(C.byref(si), C.byref(so))
    check(st, "viper_schedule")
    return {"family": so.family, "params": list(so.params), "mse": list(so.mse), "t_p": so.t_p, "t_c": so.t_c,
            "thresh": so.thresh, "best_interval": so.best_interval,
            "sched": [so.sched[i] for i in range(so.sched_len)] if so.sched_len else [],
            "predicted_cil": so.predicted_cil}
