"""Multi-process (world_size 2, gloo on CPU) check of the row-sharded path (S8(e)):
shard ranges, packing, the all_gather exchange and libddq's host merge +
finalisation (ddq_finalize_partials) reproduce the single-process result exactly.

The per-shard partial group tables come from the oracle evaluated on each rank's
rows (test infrastructure standing in for the GPU partials, which this CPU box
cannot compute); the merge and ORDER BY are the product's host code.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import datagen
import oracle

SF = 0.05
QUERIES = ["ssb1.1", "ssb2.1", "ssb3.2", "ssb4.1", "ssb4.3"]


class ShardView:
    """Dimension tables whole, lineorder rows [b, e)."""

    def __init__(self, data, b, e):
        self.data, self.b, self.e = data, b, e

    def __getitem__(self, c):
        a = self.data[c]
        return a[self.b:self.e] if c.startswith("lo_") else a


def to_partials(rows, nkeys, naggs):
    keys = np.zeros(len(rows), np.int64)
    accs = np.zeros((len(rows), naggs, 2), np.int64)
    for i, r in enumerate(rows):
        k = 0
        for j in range(nkeys):
            k |= int(r[j]) << (21 * j)
        keys[i] = k
        for a in range(naggs):
            v = int(r[nkeys + a]) & ((1 << 128) - 1)
            accs[i, a, 0] = np.int64(np.uint64(v & 0xFFFFFFFFFFFFFFFF).view(np.int64))
            accs[i, a, 1] = np.int64(np.uint64((v >> 64) & 0xFFFFFFFFFFFFFFFF).view(np.int64))
    return keys, accs.reshape(-1)


def _worker(rank, world, port, q, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_sigmod_bressft16_b200 import dist as D
    from paper_conf_sigmod_bressft16_b200.engine import Catalog, finalize_partials
    from paper_conf_sigmod_bressft16_b200.ssb import ssb_plan, STRING_DICTS
    data = datagen.SSB(SF)
    n = data.rows("lineorder")
    b, e = D.shard_range(n, rank, world)
    rows = oracle.run(ShardView(data, b, e), q)
    cat = Catalog({d: datagen.dictionary(d) for d in set(STRING_DICTS.values())})
    P = ssb_plan(cat, q)
    root = P.plan.ops[P.n - 1]
    nk, na = root.n_keys, root.n_aggs
    if q.startswith("ssb1"):
        rows = [r for r in rows if r[1] != 0]  # an empty shard has no group
    keys, accs = to_partials(rows, nk, na)
    cap = 4096
    packed = torch.from_numpy(D.pack_partials(keys, accs, cap, na))
    flat = D.all_gather_packed(packed, world).numpy()
    if rank == 0:
        k, a = D.unpack_gathered(flat, world, cap, na)
        res = finalize_partials(root, k, a)
        out.put(res.rows)
    dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("q", QUERIES)
def test_two_rank_shard_merge_equals_single(q):
    ctx = mp.get_context("spawn")
    out = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, out)) for r in range(2)]
    for p in procs:
        p.start()
    got = out.get(timeout=300)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    want = [tuple(r) for r in oracle.run(datagen.SSB(SF), q)]
    assert [tuple(r) for r in got] == want


def test_shard_ranges_partition_rows():
    from paper_conf_sigmod_bressft16_b200.dist import shard_range
    for n in (0, 1, 7, 120_000_000, 600_000_001):
        for w in (1, 2, 3, 8):
            rs = [shard_range(n, r, w) for r in range(w)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(w - 1))
            assert max(e - b for b, e in rs) - min(e - b for b, e in rs) <= 1
