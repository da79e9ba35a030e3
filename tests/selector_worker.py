"""CPU-only: Transfer Selector records exchanged through viper.Bootstrap's
allgather callback over gloo (world size 2), then resolved on every rank.
--blocked: the consumer (rank 1) reports that its GPU cannot reach the
producer's, so both ranks must pick the DRAM tier."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import torch.distributed as dist

import selector_util as S
from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V

dist.init_process_group("gloo")
rank, world = dist.get_rank(), dist.get_world_size()
blocked = "--blocked" in sys.argv
reach = [rank] if (blocked and rank == 1) else list(range(world))
me = S.record(S.AUTO, rank, reach)
bs = V.Bootstrap(rank, world, producer_rank=0).struct()
out = (S.TierRec * world)()
rc = bs.allgather(C.cast(C.byref(me), C.c_void_p), C.cast(out, C.c_void_p), C.sizeof(S.TierRec), None)
tier = C.c_int32(-1)
st = V.lib().viper_debug_resolve_tier(C.cast(out, C.c_void_p), world, 0, 1, S.DIRECT, S.AUTO, C.byref(tier))
ok = rc == 0 and st == V.OK and out[1 - rank].pci == S.pci(1 - rank)
print(f"SELECTOR {'GPU' if tier.value == S.GPU else 'DRAM'} rank={rank} ok={ok}", flush=True)
dist.barrier()
dist.destroy_process_group()
sys.exit(0 if ok else 1)
