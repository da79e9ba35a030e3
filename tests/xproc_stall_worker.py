"""a DRAM-tier install must not hang when the producer
names v and then never delivers it.  rank 0 = producer with
VIPER_TEST_DRAM_STALL=1 (its side stream never raises the pieces' flags, as a
producer that died mid-transfer), ASYNC; rank 1 = consumer.  The producer
publishes v1, waits 1 s and unregisters (then exits); the consumer's update
thread must notice the producer is gone, abort the install (VIPER_E_PEER, v1
not installed) and the consumer must unregister promptly."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import torch.distributed as dist

import synth
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V
from synth import gpu as G

dist.init_process_group("gloo")
rank, world = dist.get_rank(), dist.get_world_size()
if rank == 0:
    os.environ["VIPER_TEST_DRAM_STALL"] = "1"
dev = rank % torch.cuda.device_count()
torch.cuda.set_device(dev)
specs = [(f"t{i}", synth.F32, (3_000_000 + i,)) for i in range(4)]
ts = G.alloc_model(specs, device=f"cuda:{dev}")
m = V.Model("stall", V.PRODUCER if rank == 0 else V.CONSUMER, ts, tier=V.TIER_DRAM, mode=V.ASYNC, device=dev,
            bootstrap=V.Bootstrap(rank, world, 0))
dist.barrier()  # last collective
if rank == 0:
    G.fill_model(ts, specs, 0x57A1, 1)
    m.publish(1)
    torch.cuda.synchronize()
    time.sleep(1.0)
    m.close()
    print("STALL_PRODUCER closed", flush=True)
    time.sleep(0.5)
    os._exit(0)
t0 = time.monotonic()
print(f"STALL_CONSUMER waiting", flush=True)
status = 0
try:
    m.wait_installed(1, timeout_us=40_000_000)
except V.ViperError as e:
    status = e.status
took = time.monotonic() - t0
print(f"STALL_CONSUMER wait returned status={status} after {took:.2f}s", flush=True)
st = m.stats()
t1 = time.monotonic()
m.close()
closed = time.monotonic() - t1
ok = status == V.E_PEER and st["installs"] == 0 and took < 20 and closed < 10
print(f"STALL_CONSUMER status={status} installs={st['installs']} took={took:.2f}s close={closed:.2f}s ok={ok}",
      flush=True)
os._exit(0 if ok else 1)
