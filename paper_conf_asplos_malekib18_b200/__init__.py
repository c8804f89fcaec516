"""B200-native PLR hot path: thin Python binding of the C ABI in include/plr.h.

Everything that computes runs in ``libplr_b200.so`` (hand-written sm_100a
CUDA + a C++ planner).  This module only marshals arguments: torch is used
for device memory, streams and ``torch.distributed``.  There is no CPU
fallback -- if the library is missing, import fails loudly.

    import paper_conf_asplos_malekib18_b200 as plr
    plan = plr.Plan((0.2,), (0.8,), "float32", n_max=1 << 30)
    y = plan(x)                       # x: CUDA tensor, float32

Names follow the paper (Maleki & Burtscher, ASPLOS'18): signature
(a0, a-1, ..., a-p : b-1, ..., b-k), recurrence Eq. (1).
"""
from __future__ import annotations

import ctypes
import os

from .binding import (  # noqa: F401
    LIB_PATH,
    PAYLOAD_BYTES,
    PLRError,
    Plan,
    ShardComm,
    abi_version,
    broadcast_bytes,
    gather_payloads,
    lib,
    shard_bounds,
)

__all__ = ["Plan", "PLRError", "ShardComm", "shard_bounds", "broadcast_bytes", "gather_payloads", "lib",
           "LIB_PATH", "PAYLOAD_BYTES", "abi_version"]
