"""A rank that fails BEFORE the bootstrap (bad tensor / no device) must still
join the bootstrap collectives, so every other rank fails with an error
instead of waiting forever in the allgather.

Rank 1 registers host (CPU) memory, which the library rejects before the
bootstrap.  Rank 0 registers device memory when a GPU is visible, and then
gets VIPER_E_PEER.  On a CPU-only box both ranks fail with "no CUDA device",
which is also a pre-bootstrap failure."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import torch.distributed as dist

from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V

dist.init_process_group("gloo")
rank, world = dist.get_rank(), dist.get_world_size()
gpu = torch.cuda.is_available()
dev = "cuda" if (gpu and rank == 0) else "cpu"
tensors = [torch.zeros(1000, dtype=torch.float32, device=dev), torch.zeros(37, dtype=torch.uint8, device=dev)]
bs = V.Bootstrap(rank, world, producer_rank=0)
status = None
try:
    V.Model("abort-test", V.PRODUCER if rank == 0 else V.CONSUMER, tensors, bootstrap=bs, device=0)
except V.ViperError as e:
    status = e.status
want = (V.E_PEER if rank == 0 else V.E_INVAL) if gpu else V.E_CUDA
ok = status == want
print(f"[rank{rank}] status {status} (want {want})", flush=True)
t = torch.tensor([0 if ok else 1])
dist.all_reduce(t)
if rank == 0 and int(t.item()) == 0:
    print("ABORT_OK", flush=True)
dist.destroy_process_group()
sys.exit(0 if ok else 1)
