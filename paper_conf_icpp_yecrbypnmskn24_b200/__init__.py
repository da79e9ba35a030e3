"""viper-b200: the model-update hot path of Viper (Ye et al., ICPP '24) on B200.

The product is libviper.so (csrc/, C-ABI in include/viper.h); this package is
its thin ctypes binding (viper.py).  It never imports ``oracle/``.
"""
from .viper import (  # noqa: F401
    ASYNC, BF16, BYTES, CONSUMER, E_CHECKSUM, E_INVAL, E_NOVERSION, E_STATE, E_TIMEOUT, E_UNSUPPORTED, E_VERSION,
    F16, F32, FANOUT_CHAIN, FANOUT_DIRECT, FANOUT_SCATTER_ALLGATHER, OK, PRODUCER, SCHED_FIXED, SCHED_GREEDY, SYNC, TIER_DRAM,
    TIER_GPU, Bootstrap, Model, View, ViperError, lib, schedule,
)
