"""Build libviper.so (the product) and synth/libvgen.so (harness) for sm_100a.

Plain nvcc, in-tree outputs (they travel to the GPU box with the repo snapshot).
Static cudart; libcuda is only dlopen'ed at the first CUDA call, so the
library also loads on a CPU-only box (for symbol checks).
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libviper.so")
VGEN_SRC = os.path.join(ROOT, "synth", "vgen.cu")
VGEN_LIB = os.path.join(ROOT, "synth", "libvgen.so")
SOURCES = ["kernels.cu", "runtime.cpp", "schedule.cpp", "xproc.cpp", "flush.cpp", "selftest.cpp", "nvls.cpp", "nccl_fanout.cpp"]
HEADERS = ["vp_internal.h", "runtime.h", "protocol.h", "selector.h"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nvcc() -> str:
    p = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
    if not os.path.exists(p):
        raise RuntimeError("nvcc not found: the CUDA toolkit is required to build libviper.so")
    return p


def _stale(target, deps) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build_viper(force: bool = False, verbose: bool = False, out: str = None, defines=()) -> str:
    """defines: extra -D flags (tuning experiments build side variants via `out`)."""
    target = out or LIB
    deps = [os.path.join(CSRC, s) for s in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "viper.h")]
    if not force and not _stale(target, deps):
        return target
    bdir = os.path.join(PKG, "build" if out is None else "build-" + os.path.basename(out))
    os.makedirs(bdir, exist_ok=True)
    common = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-Wall", "-I", os.path.join(ROOT, "include")]
    common += [f"-D{d}" for d in defines]
    procs, objs = [], []
    for s in SOURCES:
        o = os.path.join(bdir, s + ".o")
        objs.append(o)
        cmd = [nvcc()] + ARCH + common + ["-c", os.path.join(CSRC, s), "-o", o]
        if s.endswith(".cu"):
            cmd += ["-Xptxas", "-v"] if verbose else []
        procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
    for cmd, p in procs:
        log = p.communicate()[0].decode()
        if p.returncode != 0:
            raise RuntimeError("build failed:\n" + " ".join(cmd) + "\n" + log)
        if verbose and log.strip():
            print(log)
    tmp = target + f".tmp{os.getpid()}"
    cmd = [nvcc()] + ARCH + ["-shared", "-o", tmp] + objs + ["-lpthread", "-lrt", "-ldl"]
    r = subprocess.run(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)
    if r.returncode != 0:
        raise RuntimeError("link failed:\n" + r.stdout.decode())
    os.replace(tmp, target)
    return target


def build_fast(force: bool = False) -> str:
    """CPython shim for the per-update calls (publish / acquire / release)."""
    import sysconfig
    src = os.path.join(CSRC, "pyfast.c")
    out = os.path.join(PKG, "_fast" + sysconfig.get_config_var("EXT_SUFFIX"))
    if not force and not _stale(out, [src]):
        return out
    tmp = out + f".tmp{os.getpid()}"
    cmd = ["gcc", "-O2", "-shared", "-fPIC", "-I", sysconfig.get_paths()["include"], src, "-o", tmp, "-ldl"]
    r = subprocess.run(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)
    if r.returncode != 0:
        raise RuntimeError("pyfast build failed:\n" + r.stdout.decode())
    os.replace(tmp, out)
    return out


def build_vgen(force: bool = False) -> str:
    if not force and not _stale(VGEN_LIB, [VGEN_SRC]):
        return VGEN_LIB
    tmp = VGEN_LIB + f".tmp{os.getpid()}"
    cmd = [nvcc()] + ARCH + ["-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-shared", VGEN_SRC, "-o", tmp]
    r = subprocess.run(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)
    if r.returncode != 0:
        raise RuntimeError("vgen build failed:\n" + r.stdout.decode())
    os.replace(tmp, VGEN_LIB)
    return VGEN_LIB


def build_all(force: bool = False, verbose: bool = False):
    return build_viper(force, verbose), build_vgen(force), build_fast(force)


if __name__ == "__main__":
    print(build_all(force="--force" in sys.argv, verbose="-v" in sys.argv))
