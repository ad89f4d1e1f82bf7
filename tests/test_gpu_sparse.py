"""Open addressing against the oracle: every SSB and TPC-H query on SPARSE primary /
foreign keys (datagen keys="sparse": keys spread over >= 16x the rows and > 2^20
values, so reading O24 sends every build except the date dimension's to the
open-addressing hash table -- hash_build_kernel and ws_kernel's WK_HT_* probes --
instead of the direct-mapped join index).  Exact equality with the oracle run on the
same sparse data (the oracle itself is pinned to SQLite on sparse keys).

Covered shapes: dense first probes (shared-memory and global tables), probes at a TID
list, probes keyed by an aligned vector (TPC-H Q5 / Q7), fetches through a hash join
(late materialisation), key-set builds with duplicate keys (TPC-H Q4), the STAR
operator, the unfused SELECT -> BUILD plans, the chopping driver and the host
executor (CPU-only placement), and a row-bitmap intermediate feeding a hash probe."""
import functools

import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu

VARIANTS = {"chain": dict(star=False), "chain_fused": dict(star=False, fuse_tail=True), "star": dict(star=True), "chain_eager": dict(star=False, late=False),
            "chain_unfused": dict(star=False, fused_build=False, late=False, fused_agg=False)}
TPCH = ["tpch1", "tpch2", "tpch3", "tpch4", "tpch5", "tpch6", "tpch7"]


@functools.lru_cache(maxsize=None)
def _ssb(sf):
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.ssb import load_ssb
    data = datagen.SSB(sf, keys="sparse")
    db = Database(cache_bytes=8 << 30, heap_bytes=8 << 30)
    load_ssb(db, data)
    return data, db


@functools.lru_cache(maxsize=None)
def _tpch(sf):
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch
    data = datagen.TPCH(sf, keys="sparse")
    db = Database(cache_bytes=8 << 30, heap_bytes=8 << 30)
    load_tpch(db, data)
    return data, db


@functools.lru_cache(maxsize=None)
def _want_ssb(sf, q):
    return oracle.run(_ssb(sf)[0], q)


@functools.lru_cache(maxsize=None)
def _want_tpch(sf, q):
    return oracle.run(_tpch(sf)[0], q)


def test_sparse_builds_take_the_hash_path():
    """The generated keys violate both O24 conditions of the join index."""
    data, db = _ssb(1)
    for t, c in (("customer", "c_custkey"), ("supplier", "s_suppkey"), ("part", "p_partkey")):
        n, lo, hi = db.column_stats(t, c)
        assert hi - lo + 1 > (1 << 20) and hi - lo + 1 > 16 * n, c


@pytest.mark.parametrize("variant", list(VARIANTS))
@pytest.mark.parametrize("q", oracle.SSB_QUERIES)
def test_ssb_sparse_prepared_equals_oracle(q, variant):
    from paper_conf_sigmod_bressft16_b200.ssb import ssb_plan
    data, db = _ssb(1)
    p = db.prepare(ssb_plan(db, q, **VARIANTS[variant]))
    for _ in range(2):
        p.launch()
        assert p.fetch().rows == _want_ssb(1, q)
    p.close()


@pytest.mark.parametrize("q", oracle.SSB_QUERIES)
def test_ssb_sparse_submit_equals_oracle(q):
    from paper_conf_sigmod_bressft16_b200.ssb import ssb_plan
    data, db = _ssb(1)
    r = db.run(ssb_plan(db, q))
    assert r.rows == _want_ssb(1, q) and r.host_ops == 0


def test_ssb_sparse_o30_orders(monkeypatch):
    """Supplier-first join orders (O30) over hash tables."""
    from paper_conf_sigmod_bressft16_b200 import ssb as S
    monkeypatch.setattr(S, "SMEM_BITMAP_KEYS", 1)
    data, db = _ssb(1)
    for q in ("ssb3.1", "ssb3.3", "ssb4.1", "ssb4.2"):
        p = db.prepare(S.ssb_plan(db, q))
        p.launch()
        assert p.fetch().rows == _want_ssb(1, q), q
        p.close()


@pytest.mark.parametrize("q", TPCH)
def test_tpch_sparse_prepared_equals_oracle(q):
    from paper_conf_sigmod_bressft16_b200.tpch import tpch_plan
    data, db = _tpch(1)
    p = db.prepare(tpch_plan(db, q))
    p.launch()
    got = p.fetch().rows
    p.close()
    assert got and got == _want_tpch(1, q)


@pytest.mark.parametrize("q", TPCH)
def test_tpch_sparse_submit_equals_oracle(q):
    from paper_conf_sigmod_bressft16_b200.tpch import tpch_plan
    data, db = _tpch(1)
    r = db.run(tpch_plan(db, q))
    assert r.rows == _want_tpch(1, q) and r.host_ops == 0


def test_sparse_host_executor_and_aborts():
    """CPU-only placement (the host executor's hash tables) and fault-injected
    aborts (GPU hash builds restarted on the host mid-query) on sparse keys."""
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.ssb import load_ssb, ssb_plan
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch, tpch_plan
    sd, td = datagen.SSB(0.05, keys="sparse"), datagen.TPCH(0.05, keys="sparse")
    for kw in (dict(placement=A.PLACE_CPU_ONLY), dict(fault_alloc_every=3)):
        for data, load, plan, qs in ((sd, load_ssb, ssb_plan, oracle.SSB_QUERIES), (td, load_tpch, tpch_plan, TPCH)):
            db = Database(cache_bytes=4 << 30, heap_bytes=2 << 30, **kw)
            load(db, data)
            hs = [(q, db.submit(plan(db, q))) for q in qs]
            for q, h in hs:
                assert db.fetch(h).rows == oracle.run(data, q), (kw, q)
            assert db.stats()["host_ops"] > 0
            db.close()
