"""Host finalisation (S8(a7)) through the C ABI, no GPU needed: ddq_finalize_partials
is the merge + ORDER BY / LIMIT step every query result passes through (P:256:
"once the root operator ... finished, the query result is returned").

Pins (closed forms, not a retyped formula):
  * the merge of per-shard partial groups equals the single-shard result: SUM / COUNT
    add, MIN takes the smaller (the merge used to add minima);
  * reading O7: an aggregate without GROUP BY over no rows is ONE row, COUNT 0 and
    SUM / MIN SQL NULL; a grouped aggregate over no rows is no row;
  * reading O10: AVG = sum / count / 10^scale as a double, NULL (NaN) at count 0,
    compared with exact rational arithmetic (fractions.Fraction) at rel 1e-15.
"""
import ctypes
import math
from fractions import Fraction

import numpy as np
import pytest


def _root(kinds, n_keys=0, key_bits=(), order_by=(), limit=0, avg=(), avg_count=-1):
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    op = A.Op()
    ctypes.memset(ctypes.addressof(op), 0, ctypes.sizeof(op))
    op.kind = A.OP_AGGREGATE
    op.input = -1
    op.n_keys = n_keys
    for k, b in enumerate(key_bits):
        op.key_bits[k] = b
    op.n_aggs = len(kinds)
    for a, k in enumerate(kinds):
        op.agg_kind[a] = k
    op.n_order = len(order_by)
    for i, o in enumerate(order_by):
        op.order_by[i] = o
    op.limit = limit
    op.n_avg = len(avg)
    op.avg_count = avg_count
    for k, (a, s) in enumerate(avg):
        op.avg_sum[k], op.avg_scale[k] = a, s
    return op


def _accs(rows):
    """rows: list of lists of Python ints (int128 each) -> int64 (lo, hi) words."""
    out = []
    for r in rows:
        for v in r:
            u = v & ((1 << 128) - 1)
            lo, hi = u & ((1 << 64) - 1), u >> 64
            out += [lo - (1 << 64) if lo >= 1 << 63 else lo, hi - (1 << 64) if hi >= 1 << 63 else hi]
    return np.array(out, np.int64)


def test_merge_per_aggregate_kind():
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.engine import finalize_partials
    root = _root([A.AGG_SUM, A.AGG_MIN, A.AGG_COUNT], n_keys=1, key_bits=[8], order_by=[1])
    # group 3 appears in three shards, group 5 in one; values beyond int64 to exercise int128
    keys = np.array([3, 5, 3, 3], np.int64)
    big = 1 << 70
    accs = _accs([[big, 40, 2], [7, -9, 1], [5, 12, 3], [-1, 17, 4]])
    r = finalize_partials(root, keys, accs)
    assert r.rows == [(3, big + 5 - 1, 12, 9), (5, 7, -9, 1)]


def test_ungrouped_empty_is_one_null_row():
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.engine import finalize_partials
    root = _root([A.AGG_SUM_MUL, A.AGG_COUNT, A.AGG_MIN])
    r = finalize_partials(root, np.zeros(0, np.int64), np.zeros(0, np.int64))
    assert r.rows == [(None, 0, None)]
    # non-empty: no NULLs
    r = finalize_partials(root, np.zeros(1, np.int64), _accs([[42, 3, -5]]))
    assert r.rows == [(42, 3, -5)]


def test_grouped_empty_has_no_rows():
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.engine import finalize_partials
    root = _root([A.AGG_SUM], n_keys=2, key_bits=[4, 4], order_by=[1, 2])
    r = finalize_partials(root, np.zeros(0, np.int64), np.zeros(0, np.int64))
    assert r.rows == []


def test_avg_columns():
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.engine import finalize_partials
    # TPC-H Q1 shape: sum_qty, sum_price, sum_disc, count; avg over scale-2 decimals
    root = _root([A.AGG_SUM, A.AGG_SUM, A.AGG_SUM, A.AGG_COUNT], n_keys=1, key_bits=[2], order_by=[1],
                 avg=[(0, 2), (1, 2), (2, 2)], avg_count=3)
    rng = np.random.default_rng(7)
    sums = [[int(rng.integers(1, 1 << 60)) * 1000 + 7, (1 << 66) + 12345, int(rng.integers(0, 1000)),
             int(rng.integers(1, 1 << 40))] for _ in range(3)]
    r = finalize_partials(root, np.arange(3, dtype=np.int64), _accs(sums))
    assert len(r.avgs) == 3
    for g, s in enumerate(sums):
        for k, a in enumerate((0, 1, 2)):
            exact = Fraction(s[a], s[3] * 100)
            assert r.avgs[g][k] == pytest.approx(float(exact), rel=1e-15)
    # count 0 -> NULL (NaN) for an ungrouped AVG
    root = _root([A.AGG_SUM, A.AGG_COUNT], avg=[(0, 2)], avg_count=1)
    r = finalize_partials(root, np.zeros(0, np.int64), np.zeros(0, np.int64))
    assert r.rows == [(None, 0)] and math.isnan(r.avgs[0][0])


def test_avg_operands_validated():
    from paper_conf_sigmod_bressft16_b200 import _abi as A, DDQError
    from paper_conf_sigmod_bressft16_b200.engine import finalize_partials
    root = _root([A.AGG_SUM, A.AGG_SUM], avg=[(0, 2)], avg_count=1)  # avg_count must be a COUNT
    with pytest.raises(DDQError):
        finalize_partials(root, np.zeros(1, np.int64), _accs([[1, 2]]))


def test_order_limit_with_ties():
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.engine import finalize_partials
    # ORDER BY agg desc, key asc; LIMIT 2 (TPC-H Q3 shape, reading O9)
    root = _root([A.AGG_SUM], n_keys=1, key_bits=[10], order_by=[-101, 1], limit=2)
    keys = np.array([9, 2, 7, 4], np.int64)
    r = finalize_partials(root, keys, _accs([[5], [8], [8], [1]]))
    assert r.rows == [(2, 8), (7, 8)]


def test_merge_is_partition_invariant():
    """Property (S8(e): sharding never changes results): for random groups split into
    random shards, merging the shards' partial tables equals finalising the unsplit
    table -- SUM / COUNT by exact int128 addition, MIN by minimum, any key order."""
    from hypothesis import given, settings, strategies as st
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.engine import finalize_partials

    root = _root([A.AGG_SUM, A.AGG_MIN, A.AGG_COUNT], n_keys=2, key_bits=[5, 6], order_by=[-101, 1, 2])
    big = st.integers(-(1 << 100), 1 << 100)

    @settings(max_examples=60, deadline=None)
    @given(st.lists(st.tuples(st.integers(0, 31), st.integers(0, 63), big, st.integers(-(1 << 62), 1 << 62)),
                    min_size=0, max_size=40),
           st.integers(1, 5), st.randoms())
    def check(rows, shards, rnd):
        exact = {}
        for k0, k1, v, m in rows:
            s, mn, c = exact.get((k0, k1), (0, None, 0))
            exact[(k0, k1)] = (s + v, m if mn is None else min(mn, m), c + 1)
        # the reference result: one row per group, ORDER BY SUM desc, keys asc
        want = sorted(((k0, k1, s, mn, c) for (k0, k1), (s, mn, c) in exact.items()),
                      key=lambda r: (-r[2], r[0], r[1]))
        # split every group's rows over random shards, each shard a partial table
        parts = {}
        for k0, k1, v, m in rows:
            sh = rnd.randrange(shards)
            s, mn, c = parts.get((sh, k0, k1), (0, None, 0))
            parts[(sh, k0, k1)] = (s + v, m if mn is None else min(mn, m), c + 1)
        items = list(parts.items())
        rnd.shuffle(items)
        keys = np.array([k0 | (k1 << 5) for (_, k0, k1), _ in items], np.int64)
        accs = _accs([[s, mn, c] for _, (s, mn, c) in items]) if items else np.zeros(0, np.int64)
        got = finalize_partials(root, keys, accs).rows
        assert got == want
    check()


def test_merge_finalized_shard_results():
    """dist.merge_finalized (bench.py's N > 1 end-to-end merge of ddq_fetch results):
    shard rows with unpacked keys re-pack into the root's key layout (here 2 keys of
    5 and 21 default bits) and merge exactly -- equal keys add (beyond int64), the
    ORDER BY of the root holds (key 1 asc, then SUM desc), and a shard's SQL-NULL
    row of an empty ungrouped aggregate is dropped (O7)."""
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.dist import merge_finalized
    root = _root([A.AGG_SUM, A.AGG_COUNT], n_keys=2, key_bits=[5, 0], order_by=[1, -101])
    big = 1 << 70
    shard0 = [(3, 1_000_000, big, 2), (1, 7, -5, 1)]
    shard1 = [(3, 1_000_000, big + 1, 3), (3, 9, 4, 1), (1, 7, 6, 2)]
    got = merge_finalized(root, [shard0, shard1]).rows
    assert got == [(1, 7, 1, 3), (3, 1_000_000, 2 * big + 1, 5), (3, 9, 4, 1)]
    ungrouped = _root([A.AGG_SUM, A.AGG_COUNT])
    assert merge_finalized(ungrouped, [[(None, 0)], [(10, 2)]]).rows == [(10, 2)]
    assert merge_finalized(ungrouped, [[(None, 0)], [(None, 0)]]).rows == [(None, 0)]
