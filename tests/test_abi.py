"""The C-ABI library loads and exports every symbol include/viper.h declares;
host-only entry points behave (no GPU needed); GPU entry points fail loudly
(no CPU fallback) when no device is visible."""
import ctypes as C
import os
import re

import pytest

from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "viper.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(viper_[a-z_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    fns = header_functions()
    for f in ["viper_register_model", "viper_publish", "viper_subscribe", "viper_acquire_latest",
              "viper_release", "viper_schedule"]:
        assert f in fns


def test_library_exports_every_declared_symbol():
    L = V.lib()
    for f in header_functions():
        assert hasattr(L, f), f
    assert sorted(V.EXPORTS) == header_functions()


def test_exports_are_c_symbols():
    out = os.popen(f"nm -D --defined-only {V.LIB_PATH}").read()
    for f in header_functions():
        assert re.search(rf"\bT {f}$", out, re.M), f


def test_strerror_and_version():
    L = V.lib()
    assert L.viper_strerror(V.E_CHECKSUM) == b"VIPER_E_CHECKSUM"
    assert L.viper_strerror(12345) == b"VIPER_E_UNKNOWN"
    assert L.viper_version().startswith(b"viper-b200")


def test_null_arguments_are_errors_not_crashes():
    L = V.lib()
    assert L.viper_publish(None, 1, None) == V.E_STATE
    assert L.viper_acquire_latest(None, 0, 0, None) == V.E_STATE
    assert L.viper_unregister(None) == V.E_INVAL
    assert L.viper_schedule(None, None) == V.E_INVAL
    h = C.c_void_p()
    assert L.viper_register_model(b"", V.PRODUCER, None, 0, None, None, C.byref(h)) == V.E_INVAL
    assert L.viper_register_model(b"m", 7, None, 0, None, None, C.byref(h)) == V.E_INVAL


@pytest.mark.skipif(os.environ.get("CUDA_VISIBLE_DEVICES", None) == "" and False, reason="")
def test_no_cpu_fallback_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is visible")
    L = V.lib()
    h = C.c_void_p()
    st = L.viper_register_model(b"m", V.PRODUCER, None, 0, None, None, C.byref(h))
    assert st == V.E_CUDA
    assert b"no CUDA device" in L.viper_last_error() or b"CUDA" in L.viper_last_error()
