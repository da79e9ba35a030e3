"""Host-side breakdown of one publish (debug trace timestamps).
Usage: trace_publish.py [config] [async]"""
import ctypes as C
import os

os.environ.setdefault("VIPER_TRACE", "1")
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

L = V.lib()
L.viper_debug_trace.argtypes = [C.POINTER(C.c_int64), C.c_int32]
specs = synth.model_specs(sys.argv[1] if len(sys.argv) > 1 else "ptychonn")
pt, ct = G.alloc_model(specs), G.alloc_model(specs)
c = V.Model("tr", V.CONSUMER, ct)
ASYNC = len(sys.argv) > 2 and sys.argv[2] == "async"
p = V.Model("tr", V.PRODUCER, pt, mode=V.ASYNC if ASYNC else V.SYNC)
st = torch.cuda.current_stream()
rows = []
buf = (C.c_int64 * 16)()
for v in range(1, 60):
    torch.cuda.synchronize()
    t0 = time.monotonic_ns()
    p.publish(v, stream=st)
    t1 = time.monotonic_ns()
    if ASYNC:
        c.wait_installed(v, timeout_us=5_000_000)
    L.viper_debug_trace(buf, 16)
    if v > 10:
        rows.append([buf[i] - buf[0] for i in range(8)] + [buf[0] - t0, t1 - buf[7], buf[8] - buf[0], buf[9] - buf[0]])
names = ["entry", "pinscan", "installs_prepared", "pack+install_launched", "reduce+events", "status_seen", "finish", "exit",
         "py->C", "C->py", "before_fused_launch", "after_fused_launch"]
for i, n in enumerate(names):
    print(f"{n:18s} {statistics.median(r[i] for r in rows) / 1e3:8.2f} us")
c.close()
p.close()
