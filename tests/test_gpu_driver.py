"""Pins of the paper's driver (SURVEY 8(c).5 "Driver"), through the C ABI on the GPU.

* Algorithm 1 (Sec. 3.2) on hand-computed cases: columns sorted by access
  count (descending), ties by column id, the greedy prefix that fits buffer_size,
  stopping at the FIRST column that does not fit (reading O16); the LRU variant
  (App. E); evict(old \\ new) deferred while a running plan references
  the column.
* The heap-contention closed form n = floor(M / (f |C|)) (Sec. 3.4): with
  P:188's numbers scaled by 1/1024 (|C| = 218 KiB, f = 3.25, M = 5 MiB) exactly 7
  operator footprints fit the fail-fast heap (the 8th fails at once); a
  chopping pool of W <= n GPU workers never aborts.
* Placement traces: Fig. 4 (Sec. 3.1) -- operators go to the GPU iff their
  input is cached; Sec. 3.3 -- the chain from the leaves stops at the first
  operator with a non-resident input, the rest runs on the CPU; Fig. 8 (P:195,
  Sec. 4.1) -- after an abort, run-time placement keeps the successor on
  the CPU (the data is there), compile-time placement sends it back to the GPU and
  pays the unplanned transfer.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

# four one-column tables: sizes 160 000, 120 000, 80 000, 40 000 bytes (int32)
ROWS = [40_000, 30_000, 20_000, 10_000]


def _db(budget, policy=0, **kw):
    from paper_conf_sigmod_bressft16_b200 import Database
    db = Database(cache_bytes=budget, heap_bytes=64 << 20, cache_policy=policy, **kw)
    rng = np.random.default_rng(3)
    for i, n in enumerate(ROWS):
        db.create_table(f"t{i}", n)
        db.load_column(f"t{i}", "c", rng.integers(0, 100, n).astype(np.int32))
    return db


def _touch(db, i, times=1):
    """`times` operator accesses of column t{i}.c (one SELECT each; P:144 access counter)."""
    for _ in range(times):
        P = db.plan()
        P.select(f"t{i}", [("c", 0, 49)])
        db.run(P)


def _cached(db):
    return {i for i in range(len(ROWS)) if db.is_cached(f"t{i}", "c")}


def test_algorithm1_greedy_prefix():
    db = _db(240_000)
    db.reset_access_counts()
    for i, k in enumerate([1, 4, 3, 2]):
        _touch(db, i, k)
    assert [db.access_count(f"t{i}", "c") for i in range(4)] == [1, 4, 3, 2]
    db.update_placement()
    # K = (t1 120K, t2 80K, t3 40K, t0 160K): 120 + 80 + 40 = 240 fits, t0 does not
    assert _cached(db) == {1, 2, 3}
    db.close()


def test_algorithm1_stops_at_first_misfit():
    """Reading O16: the loop condition `used + K_i.size <= buffer_size` ends the loop
    at the first column that does not fit -- no knapsack skip to smaller ones."""
    db = _db(240_000)
    db.reset_access_counts()
    for i, k in enumerate([4, 3, 2, 1]):
        _touch(db, i, k)
    db.update_placement()
    # t0 160K fits; t1 would make 280K > 240K: stop (t2 + t0 = 240K would have fit)
    assert _cached(db) == {0}
    db.close()


def test_algorithm1_ties_by_column_id():
    db = _db(200_000)
    db.reset_access_counts()
    for i, k in enumerate([1, 2, 2, 2]):
        _touch(db, i, k)
    db.update_placement()
    # t1, t2, t3 tie at 2: ids ascending -> t1 120K + t2 80K = 200K, then t3 misfits
    assert _cached(db) == {1, 2}
    db.close()


def test_algorithm1_lru_variant():
    """cache_policy 1 (App. E): most recently accessed first.  The same touches under
    LFU (every count 1, ties by id) choose differently."""
    order = [3, 0, 2, 1]  # t1 is the most recent
    got = {}
    for policy in (0, 1):
        db = _db(240_000, policy=policy)
        db.reset_access_counts()
        for i in order:
            _touch(db, i)
        db.update_placement()
        got[policy] = _cached(db)
        db.close()
    assert got[1] == {1, 2}      # LRU: t1 120K, t2 80K; t0 160K misfits
    assert got[0] == {0}         # LFU ties by id: t0 160K; t1 misfits


def test_algorithm1_evicts_and_defers_while_referenced():
    db = _db(240_000)
    db.reset_access_counts()
    for i, k in enumerate([1, 4, 3, 2]):
        _touch(db, i, k)
    db.update_placement()
    assert _cached(db) == {1, 2, 3}
    P = db.plan()
    P.select("t1", [("c", 0, 49)])
    prep = db.prepare(P)               # holds a cache reference on t1.c
    want = np.flatnonzero(db_col(db, 1) <= 49)
    db.reset_access_counts()
    _touch(db, 0, 5)
    db.update_placement()               # new set {t0}: t1, t2, t3 leave the cache
    assert _cached(db) == set()         # t1 is evicted (no longer placeable) ...
    assert db.stats()["cache_used_bytes"] == 120_000  # ... but its memory stays: a plan reads it
    prep.launch()                       # ... so the plan still reads the right column
    assert np.array_equal(prep.fetch().tids, want)
    prep.close()                        # last reference gone: the deferred eviction runs
    assert db.stats()["cache_used_bytes"] == 0
    db.update_placement()               # the next periodic run caches t0
    assert _cached(db) == {0} and db.stats()["cache_used_bytes"] == 160_000
    db.close()


_COLS = {}


def db_col(db, i):
    if i not in _COLS:
        rng = np.random.default_rng(3)
        cols = [rng.integers(0, 100, n).astype(np.int32) for n in ROWS]
        _COLS.update(enumerate(cols))
    return _COLS[i]


def test_heap_admission_closed_form():
    """n = |M| / (3.25 |C|) ~ 7 for M = 5 GB, |C| = 218 MB.  Scaled by 1/1024:
    the fail-fast heap admits exactly floor(M / F) footprints F = 3.25 |C|, the next
    request fails immediately (no waiting), and freeing one admits one more."""
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    C = 218 * 1024
    F = int(3.25 * C)                    # 725 504 bytes (a multiple of the heap's 256 B)
    M = 5 << 20
    n = M // F
    assert n == 7
    db = Database(cache_bytes=1 << 20, heap_bytes=M)
    L = A.lib()
    blocks = []
    while True:
        p = L.ddq_heap_try_alloc(db.h, F)
        if not p:
            break
        blocks.append(p)
    assert len(blocks) == n
    L.ddq_heap_free(db.h, blocks.pop())
    assert L.ddq_heap_try_alloc(db.h, F)
    db.close()


def _footprint_db(workers, heap, chopping=True):
    from paper_conf_sigmod_bressft16_b200 import Database
    db = Database(cache_bytes=1 << 30, heap_bytes=heap, gpu_workers=workers, chopping=chopping)
    n = 4_000_000
    db.create_table("f", n)
    db.load_column("f", "x", np.arange(n, dtype=np.int32) % 1000)
    db.cache("f", "x")
    return db


def _select_all(db):
    P = db.plan()
    P.select("f", [("x", 0, 999)])  # every row: the output TID list is the whole column
    return P


def test_chopping_bound_caps_heap_contention():
    """A query's select footprint F measured alone; with a heap of n = floor(M / F)
    footprints, a pool of W = n GPU workers runs 32 concurrent queries without a
    single abort (the bounded pull queue caps the accumulated footprint)."""
    db = _footprint_db(4, 8 << 30)
    db.reset_stats()
    db.run(_select_all(db))
    F = db.stats()["heap_peak_bytes"]
    db.close()
    assert F >= 16_000_000
    n = 3
    db = _footprint_db(n, n * F + F // 2)
    qs = [db.submit(_select_all(db)) for _ in range(32)]
    for q in qs:
        assert db.fetch(q).tids.size == 4_000_000
    st = db.stats()
    assert st["aborts"] == 0 and st["host_ops"] == 0
    assert st["heap_peak_bytes"] <= n * F
    db.close()


def test_fig4_data_driven_placement_trace():
    """Fig. 4: operators 1 and 3 read cached columns and run on the GPU, operator 2's
    column is not cached and it runs on the CPU."""
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    db = _db(1 << 30)
    db.cache("t0", "c")
    db.cache("t2", "c")
    traces = []
    for i in (0, 1, 2):
        P = db.plan()
        P.select(f"t{i}", [("c", 0, 49)])
        r = db.run(P)
        traces.append(r.placement)
        assert np.array_equal(r.tids, np.flatnonzero(db_col(db, i) <= 49))
    assert traces == [[A.RAN_GPU], [A.RAN_HOST], [A.RAN_GPU]]
    db.close()


def _chain(db):
    """op0: select over all rows of f.a; op1: select at op0's TIDs on f.b; op2: select
    at op1's TIDs on f.c (a select-* root)."""
    P = db.plan()
    t = P.select("f", [("a", 0, 59)])
    t = P.select("f", [("b", 20, 99)], input=t)
    P.select("f", [("c", 0, 79)], input=t)
    return P


def _chain_db(cache_b=True, **kw):
    from paper_conf_sigmod_bressft16_b200 import Database
    db = Database(cache_bytes=1 << 30, heap_bytes=1 << 30, **kw)
    n = 1_000_003
    rng = np.random.default_rng(8)
    cols = {c: rng.integers(0, 100, n).astype(np.int32) for c in "abc"}
    db.create_table("f", n)
    for c, v in cols.items():
        db.load_column("f", c, v)
        if c != "b" or cache_b:
            db.cache("f", c)
    want = np.flatnonzero((cols["a"] <= 59) & (cols["b"] >= 20) & (cols["c"] <= 79))
    return db, want


def test_sec33_chain_stops_at_first_uncached_input():
    """Sec. 3.3: operators are chained on the co-processor from the leaves until one
    whose input is not resident; from there the query runs on the CPU, even where a
    later operator's own column is cached."""
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    db, want = _chain_db(cache_b=False)
    r = db.run(_chain(db))
    assert r.placement == [A.RAN_GPU, A.RAN_HOST, A.RAN_HOST]
    assert np.array_equal(r.tids, want)
    db.close()


@pytest.mark.parametrize("chopping", [True, False])
def test_fig8_abort_then_successor_placement(chopping):
    """Fig. 8: op1 aborts on the GPU (fault injection) and restarts on the CPU.
    Run-time placement (chopping) keeps op2 with the data on the CPU; compile-time
    placement sends op2 back to the GPU and moves op1's output there (an unplanned
    H2D copy).  Results are the same either way."""
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    db, want = _chain_db(chopping=chopping, fault_op_mask=1 << 1)
    db.reset_stats()
    r = db.run(_chain(db))
    assert np.array_equal(r.tids, want)
    st = db.stats()
    assert r.aborts == 1 and st["aborts"] == 1 and st["wasted_ns"] > 0
    if chopping:
        assert r.placement == [A.RAN_GPU, A.RAN_ABORTED, A.RAN_HOST]
        assert st["h2d_bytes"] == 0          # every column cached; the data stays on the CPU
    else:
        assert r.placement == [A.RAN_GPU, A.RAN_ABORTED, A.RAN_GPU]
        assert st["h2d_bytes"] > 0           # op1's output copied back for op2
    assert st["d2h_bytes"] > 0               # op0's output moved to the CPU for op1's restart
    db.close()


def test_admission_control_runs_queries_one_at_a_time():
    """ddq_config.max_queries = 1 (the admission-control arm): concurrently
    submitted queries run strictly in submission order, one at a time; results are
    unchanged."""
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    db, want = _chain_db(placement=A.PLACE_GPU_ONLY, chopping=False, max_queries=1)
    qs = [db.submit(_chain(db)) for _ in range(8)]
    res = [db.fetch(q) for q in qs]
    assert all(np.array_equal(r.tids, want) for r in res)
    ms = [r.exec_ms for r in res]  # submit -> done: FIFO service makes it increase
    assert ms == sorted(ms)
    db.close()


def test_periodic_placement_job():
    """placement_period_ms: the background job runs Algorithm 1 periodically:
    columns the workload touched become resident without a call, and the next run of
    the same query is placed on the GPU (data-driven)."""
    import time
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    db = _db(1 << 30, placement_period_ms=20)
    P = db.plan()
    P.select("t2", [("c", 0, 49)])
    r = db.run(P)
    assert r.placement == [A.RAN_HOST]  # nothing cached yet
    deadline = time.time() + 5
    while not db.is_cached("t2", "c") and time.time() < deadline:
        time.sleep(0.02)
    assert db.is_cached("t2", "c")
    r = db.run(P)
    assert r.placement == [A.RAN_GPU] and np.array_equal(r.tids, np.flatnonzero(db_col(db, 2) <= 49))
    db.close()
