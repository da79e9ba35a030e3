"""CPU-only: the ctypes allgather callback of viper.Bootstrap over gloo."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch.distributed as dist

from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V

dist.init_process_group("gloo")
rank, world = dist.get_rank(), dist.get_world_size()
bs = V.Bootstrap(rank, world, producer_rank=0)
st = bs.struct()
n = 4096 + 3
inp = (C.c_uint8 * n)(*[(rank * 31 + i) & 0xFF for i in range(n)])
out = (C.c_uint8 * (n * world))()
rc = st.allgather(C.cast(inp, C.c_void_p), C.cast(out, C.c_void_p), n, None)
ok = rc == 0 and all(out[r * n + i] == ((r * 31 + i) & 0xFF) for r in range(world) for i in range(n))
dist.barrier()
if ok and rank == 0:
    print("BOOTSTRAP_OK", flush=True)
dist.destroy_process_group()
sys.exit(0 if ok else 1)
