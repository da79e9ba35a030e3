"""World-size-2 gloo worker (CPU): the descriptor hand-off NVLS registration
uses (abstract Unix socket + SCM_RIGHTS, nvls.cpp) through the library's test
hooks, with no CUDA.  Rank 0 serves a memfd holding known bytes; rank 1
fetches it and reads the bytes through its own descriptor.  Then rank 0 serves
to a fetcher that never comes and must fail with VIPER_E_PEER in bounded time."""
import os
import sys
import time
import ctypes as C

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch.distributed as dist

from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V

dist.init_process_group("gloo")
rank = dist.get_rank()
L = V.lib()
payload = b"viper multicast handle " * 100
ok = True
name = [None]
if rank == 0:
    fd = os.memfd_create("viper-test")
    os.write(fd, payload)
    buf = C.create_string_buffer(64)
    lfd = C.c_int32(-1)
    assert L.viper_debug_fd_listen(buf, 64, C.byref(lfd)) == V.OK
    name = [buf.value.decode()]
dist.broadcast_object_list(name, src=0)
if rank == 0:
    st = L.viper_debug_fd_serve(lfd.value, fd, 1, 20000)
    ok = st == V.OK
else:
    out = C.c_int32(-1)
    st = L.viper_debug_fd_fetch(name[0].encode(), C.byref(out), 20000)
    ok = st == V.OK and out.value >= 0
    if ok:
        os.lseek(out.value, 0, os.SEEK_SET)
        ok = os.read(out.value, len(payload) + 10) == payload
        os.close(out.value)
dist.barrier()
if rank == 0:  # nobody fetches: bounded failure
    buf = C.create_string_buffer(64)
    lfd = C.c_int32(-1)
    assert L.viper_debug_fd_listen(buf, 64, C.byref(lfd)) == V.OK
    t0 = time.monotonic()
    st = L.viper_debug_fd_serve(lfd.value, fd, 1, 300)
    ok = ok and st == V.E_PEER and time.monotonic() - t0 < 5
else:  # fetching a name nobody serves: bounded failure
    out = C.c_int32(-1)
    t0 = time.monotonic()
    st = L.viper_debug_fd_fetch(b"viper-nvls-nobody", C.byref(out), 200)
    ok = ok and st == V.E_PEER and time.monotonic() - t0 < 5
print(f"FDPASS rank{rank} ok={ok}", flush=True)
dist.barrier()
dist.destroy_process_group()
sys.exit(0 if ok else 1)
