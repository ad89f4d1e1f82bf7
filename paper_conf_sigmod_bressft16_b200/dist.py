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


def merge_finalized(root, rows_per_rank) -> "object":
    """Exact merge of one query's FINALISED results from several shards (the N > 1
    end-to-end path, where every rank runs ``ddq_submit`` / ``ddq_fetch`` on its own
    rows): each row's group keys are re-packed into the root AGGREGATE's key layout
    (key k at the sum of the earlier keys' bit lengths; 21 bits where the plan gives
    none, as libddq packs them), its integer aggregates split into int128 words, and
    libddq's host finalisation merges equal keys (SUM / COUNT add, MIN takes the
    minimum) and applies ORDER BY / LIMIT.  A shard's SQL-NULL row (an ungrouped
    aggregate over no rows, reading O7) contributes nothing.  Valid for aggregates
    that merge (SUM / COUNT / MIN) without AVG columns -- every SSB query."""
    from .engine import finalize_partials
    nk, na = int(root.n_keys), int(root.n_aggs)
    bits = [int(root.key_bits[k]) if int(root.key_bits[k]) > 0 else 21 for k in range(nk)]
    keys, lo, hi = [], [], []
    for rows in rows_per_rank:
        for r in rows:
            vals = r[nk:nk + na]
            if any(v is None for v in vals):
                continue
            p, sh = 0, 0
            for k in range(nk):
                p |= int(r[k]) << sh
                sh += bits[k]
            keys.append(p)
            for v in vals:
                v = int(v)
                lo.append(v & 0xFFFFFFFFFFFFFFFF)
                hi.append(v >> 64)
    accs = np.empty(2 * len(lo), np.int64)
    if lo:
        accs[0::2] = np.array(lo, np.uint64).view(np.int64)
        accs[1::2] = np.array(hi, np.int64)
    return finalize_partials(root, np.array(keys, np.int64), accs)
