"""Row-sharded multi-GPU execution (S8(e); the paper's "horizontal partitioning",
PAPER.md:407 Sec. 6.3).

One process per GPU.  The fact table is range-partitioned by row; every rank
caches its own rows and the (small) dimension tables, runs the same physical plans
on its shard, and the compacted partial group tables are exchanged with one
collective (``torch.distributed.all_gather_into_tensor``: NCCL on GPUs, gloo on CPU
in the tests).  Merging = host finalisation in libddq (``ddq_finalize_partials``:
exact int128 addition of equal packed keys, then ORDER BY / LIMIT).

Packed layout per query (int64 words): [n_groups, keys[cap], accs[cap * n_aggs * 2]].
"""
from __future__ import annotations

import numpy as np


def shard_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Rows [begin, end) of rank `rank` out of `world` (balanced, contiguous)."""
    return rank * n // world, (rank + 1) * n // world


def packed_words(cap: int, n_aggs: int) -> int:
    return 1 + cap + cap * n_aggs * 2


def pack_partials(keys: np.ndarray, accs: np.ndarray, cap: int, n_aggs: int) -> np.ndarray:
    g = keys.size
    if g > cap:
        raise ValueError("partial table exceeds its capacity")
    out = np.zeros(packed_words(cap, n_aggs), np.int64)
    out[0] = g
    out[1:1 + g] = keys
    out[1 + cap:1 + cap + g * n_aggs * 2] = np.asarray(accs, np.int64).reshape(-1)
    return out


def unpack_gathered(flat: np.ndarray, world: int, cap: int, n_aggs: int):
    """Concatenate the partial tables of all ranks (duplicates merged later)."""
    w = packed_words(cap, n_aggs)
    flat = np.asarray(flat).reshape(world, w)
    keys, accs = [], []
    for r in range(world):
        g = int(flat[r, 0])
        keys.append(flat[r, 1:1 + g])
        accs.append(flat[r, 1 + cap:1 + cap + g * n_aggs * 2])
    return np.concatenate(keys), np.concatenate(accs)


def all_gather_packed(packed, world: int):
    """all_gather of one packed int64 tensor per rank (torch.distributed plumbing)."""
    import torch
    import torch.distributed as dist
    out = torch.empty(world * packed.numel(), dtype=packed.dtype, device=packed.device)
    dist.all_gather_into_tensor(out, packed)
    return out
