"""Transfer Selector records (selector.h TierRec) for the CPU tests, built in
Python from synthetic PCI bus ids, plus an independent reading of the rule
(DESIGN.md s1 "Transfer Selector"): AUTO -> GPU tier iff every consumer's GPU
reaches every producer's GPU and, with chain / scatter-allgather fan-out, every
other consumer's GPU; records of failed ranks (magic 0) decide nothing."""
import ctypes as C

MAGIC = 0x56495452
GPU, DRAM, AUTO = 0, 1, 2
DIRECT, CHAIN, SA, NVLS, PUSH, CE = 0, 1, 2, 3, 4, 101


class TierRec(C.Structure):
    _fields_ = [("magic", C.c_uint32), ("tier", C.c_int32), ("nreach", C.c_int32), ("pad", C.c_int32),
                ("pci", C.c_char * 16), ("reach", (C.c_char * 16) * 16)]


def pci(i):
    return f"0000:{0x18 + i:02X}:00.0".encode()


def record(tier, me, reach, magic=MAGIC):
    r = TierRec()
    r.magic, r.tier, r.nreach = magic, tier, len(reach)
    r.pci = pci(me)
    for k, d in enumerate(reach):
        r.reach[k].value = pci(d)
    return r


def reference(recs, devs, reach, producer_rank, M, fanout, requested, failed=()):
    if requested != AUTO:
        return requested
    world = len(devs)
    prods = set(range(producer_rank, producer_rank + M))
    for c in range(world):
        if c in prods:
            continue
        for r in range(world):
            if r == c or not (r in prods or fanout in (CHAIN, SA)):
                continue
            if c in failed or r in failed:
                continue
            if devs[r] not in reach[c]:
                return DRAM
        # push / NVLS: the producers write into every consumer's memory
        for p in prods:
            if fanout in (PUSH, NVLS) and c not in failed and p not in failed and devs[c] not in reach[p]:
                return DRAM
    return GPU
