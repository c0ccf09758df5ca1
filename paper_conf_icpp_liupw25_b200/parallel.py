"""Multi-GPU feature partitioning: host-side plumbing of the two exchanges.

Every rank owns a contiguous range of features, builds histograms and searches splits only for
them, and replicates everything else (y, yhat, g/h, row lists, node tables).  Per tree level:

1. ``exchange_keys``: MAX all-reduce of the packed split keys (one int64 per node).  A key is
   ``(bits(gain) & ~0xFFFFFF) | (0xFFFFFF - (f_global * B + b))`` (0 = no split), so the max is the
   largest gain with ties broken towards the smallest (feature, bin) (reading R16) — the same
   rule the single-GPU kernel applies with atomicMax, hence N GPUs pick exactly what 1 GPU picks.
2. ``exchange_records``: SUM all-reduce of the owners' split records (exact int64 left sums,
   counts, winner ids) and the row-direction bitmap; non-owners contribute zeros and the bits of
   different owners are disjoint, so SUM = the owners' values.

Both are plain NCCL (or gloo on CPU) all-reduces issued on the current stream; no host sync.
"""
from __future__ import annotations

import struct

import torch
import torch.distributed as dist


def shard_range(m: int, rank: int, world: int):
    """Contiguous feature range [f0, f1) of `rank` (balanced: every feature costs the same)."""
    return (m * rank) // world, (m * (rank + 1)) // world


def exchange_keys(keys: torch.Tensor, group=None) -> torch.Tensor:
    dist.all_reduce(keys, op=dist.ReduceOp.MAX, group=group)
    return keys


def exchange_records(xchg: torch.Tensor, group=None) -> torch.Tensor:
    dist.all_reduce(xchg, op=dist.ReduceOp.SUM, group=group)
    return xchg


def pack_key(gain: float, f_global: int, b: int, B: int) -> int:
    """Host-side copy of the kernel's key format (for tests and tree decoding)."""
    if not gain > 0.0:
        return 0
    bits = struct.unpack("<q", struct.pack("<d", gain))[0]
    return (bits & ~0xFFFFFF) | (0xFFFFFF - (f_global * B + b))


def unpack_key(key: int, B: int):
    """-> (f_global, bin, truncated gain) or None for key 0."""
    if key == 0:
        return None
    idx = 0xFFFFFF - (key & 0xFFFFFF)
    gain = struct.unpack("<d", struct.pack("<q", key & ~0xFFFFFF))[0]
    return idx // B, idx % B, gain
