"""Transfer Selector (VIPER_TIER_AUTO): the C decision
(selector.h, through viper_debug_resolve_tier) against an independent Python
reading of the rule on synthetic topologies, and the record exchange over a
world-size-2 gloo group (the bootstrap's allgather callback).  CPU only."""
import ctypes as C
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import selector_util as S  # noqa: E402

from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def resolve(recs, producer_rank=0, M=1, fanout=S.DIRECT, requested=S.AUTO):
    arr = (S.TierRec * len(recs))(*recs)
    out = C.c_int32(-1)
    st = V.lib().viper_debug_resolve_tier(C.cast(arr, C.c_void_p), len(recs), producer_rank, M, fanout, requested,
                                          C.byref(out))
    assert st == V.OK
    return out.value


def test_record_layout():
    assert C.sizeof(S.TierRec) == 288


def test_nvswitch_node_all_reach_all():
    recs = [S.record(S.AUTO, d, range(8)) for d in range(8)]
    for f in (S.DIRECT, S.CHAIN, S.SA):
        assert resolve(recs, fanout=f) == S.GPU


def test_one_consumer_cannot_reach_the_producer():
    recs = [S.record(S.AUTO, d, [x for x in range(8) if not (d == 3 and x == 0)]) for d in range(8)]
    assert resolve(recs) == S.DRAM


def test_consumers_reaching_each_other_only_matters_with_peer_fanout():
    # consumers 2 and 5 cannot reach each other; everybody reaches the producer (rank 0)
    reach = {d: [x for x in range(6) if {d, x} != {2, 5}] for d in range(6)}
    recs = [S.record(S.AUTO, d, reach[d]) for d in range(6)]
    assert resolve(recs, fanout=S.DIRECT) == S.GPU
    assert resolve(recs, fanout=S.SA) == S.DRAM
    assert resolve(recs, fanout=S.CHAIN) == S.DRAM


def test_the_producers_own_reach_does_not_decide():
    recs = [S.record(S.AUTO, 0, [])] + [S.record(S.AUTO, d, range(4)) for d in range(1, 4)]
    assert resolve(recs) == S.GPU


def test_explicit_tiers_are_kept():
    recs = [S.record(S.GPU, d, []) for d in range(3)]
    assert resolve(recs, requested=S.GPU) == S.GPU
    assert resolve(recs, requested=S.DRAM) == S.DRAM


def test_failed_ranks_decide_nothing():
    recs = [S.record(S.AUTO, d, range(4)) for d in range(4)]
    recs[2] = S.TierRec()  # magic 0: failed before the bootstrap
    assert resolve(recs, fanout=S.SA) == S.GPU


@pytest.mark.parametrize("seed", range(4))
def test_random_topologies_match_the_reference(seed):
    rng = np.random.default_rng(seed)
    for _ in range(150):
        world = int(rng.integers(1, 9))
        M = int(rng.integers(1, world + 1)) if world > 1 else 1
        M = min(M, 3)
        prank = int(rng.integers(0, world - M + 1))
        devs = [int(rng.integers(0, 8)) for _ in range(world)]  # several ranks may share a GPU
        reach = []
        for r in range(world):
            s = {devs[r]} if rng.random() < 0.9 else set()
            s |= {d for d in range(8) if rng.random() < 0.8}
            reach.append(sorted(s))
        failed = {r for r in range(world) if rng.random() < 0.05}
        requested = int(rng.choice([S.AUTO, S.AUTO, S.GPU, S.DRAM]))
        fanout = int(rng.choice([S.DIRECT, S.CHAIN, S.SA, S.PUSH, S.NVLS, S.CE]))
        recs = [S.TierRec() if r in failed else S.record(requested, devs[r], reach[r]) for r in range(world)]
        want = S.reference(recs, devs, reach, prank, M, fanout, requested, failed)
        assert resolve(recs, prank, M, fanout, requested) == want, (world, M, prank, devs, reach, fanout)


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("blocked,expect", [(False, "GPU"), (True, "DRAM")])
def test_records_over_gloo_world2(blocked, expect):
    """Each rank builds its record, the bootstrap's allgather callback
    exchanges them over gloo, and both ranks resolve the same tier."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2", "--master-addr",
           "127.0.0.1", "--master-port", str(free_port()), "tests/selector_worker.py"] + (["--blocked"] if blocked else [])
    r = subprocess.run(cmd, cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, timeout=120, text=True)
    assert r.returncode == 0, r.stdout[-3000:]
    assert r.stdout.count(f"SELECTOR {expect}") == 2, r.stdout[-3000:]


def test_push_needs_the_producer_to_reach_every_consumer():
    """Push / NVLS: the producer writes into the consumers' memory, so its GPU
    must reach theirs; for pulls (direct, copy engine) only the consumers'
    reach matters."""
    # rank 0 = producer reaches only itself; consumers reach everything
    recs = [S.record(S.AUTO, 0, [0]), S.record(S.AUTO, 1, [1, 0, 2]), S.record(S.AUTO, 2, [2, 0, 1])]
    assert resolve(recs, fanout=S.DIRECT) == S.GPU
    assert resolve(recs, fanout=S.CE) == S.GPU
    assert resolve(recs, fanout=S.PUSH) == S.DRAM
    assert resolve(recs, fanout=S.NVLS) == S.DRAM
    full = [S.record(S.AUTO, i, [i] + [j for j in range(3) if j != i]) for i in range(3)]
    assert resolve(full, fanout=S.PUSH) == S.GPU and resolve(full, fanout=S.NVLS) == S.GPU
