"""CPU-only, world size 2 (gloo): rank 0 publishes versions 1..N through the
shared-memory version protocol; rank 1 installs them (one thread) while two
reader threads acquire / verify / release.  No GPU is involved: this is the
engine's cross-process host logic (protocol.h) on a real shm segment."""
import ctypes as C
import os
import random
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import torch.distributed as dist

from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V

N, WORDS = int(os.environ.get("PROTO_N", "3000")), 4096
dist.init_process_group("gloo")
rank = dist.get_rank()
L = V.lib()
obj = [f"/viper-proto-{os.getpid()}-{random.getrandbits(32):08x}" if rank == 0 else None]
dist.broadcast_object_list(obj, src=0)
path = obj[0].encode()
h = C.c_void_p()
if rank == 0:
    V.check(L.viper_debug_proto_create(path, WORDS, 1, C.byref(h)), "create")
dist.barrier()
if rank == 1:
    V.check(L.viper_debug_proto_open(path, WORDS, C.byref(h)), "open")
dist.barrier()
errors = 0
if rank == 0:
    rng = random.Random(1)
    for v in range(1, N + 1):
        V.check(L.viper_debug_proto_publish(h, v), f"publish {v}")
        if rng.random() < 0.3:
            time.sleep(rng.random() * 1e-4)
else:
    stop = threading.Event()
    stats = {"torn": 0, "reads": 0, "regress": 0, "installed": 0, "snap_torn": 0}
    lock = threading.Lock()

    def installer():
        last = 0
        while last < N:
            iv, tv = C.c_uint64(), C.c_uint64()
            V.check(L.viper_debug_proto_install(h, 0, C.byref(iv), C.byref(tv)), "install")
            with lock:
                stats["snap_torn"] += tv.value
            if iv.value:
                with lock:
                    stats["installed"] += 1
                    stats["regress"] += int(iv.value < last)
                last = max(last, iv.value)
        stop.set()

    def reader():
        last = 0
        while not stop.is_set():
            vv, tv = C.c_uint64(), C.c_uint64()
            V.check(L.viper_debug_proto_read(h, 0, C.byref(vv), C.byref(tv)), "read")
            if vv.value:
                with lock:
                    stats["reads"] += 1
                    stats["torn"] += int(tv.value > 0)
                    stats["regress"] += int(vv.value < last)
                last = vv.value

    ths = [threading.Thread(target=installer)] + [threading.Thread(target=reader) for _ in range(2)]
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    errors = stats["torn"] + stats["regress"] + stats["snap_torn"]
    print(f"PROTO rank1 {stats}", flush=True)
    if stats["reads"] < 10:
        errors += 1
dist.barrier()
t = torch.tensor([errors])
dist.all_reduce(t)
L.viper_debug_proto_close(h, 1 if rank == 0 else 0, path)
if rank == 0:
    print(f"PROTO_RESULT errors={int(t.item())}", flush=True)
dist.destroy_process_group()
sys.exit(1 if int(t.item()) else 0)
