"""TPC-H Q1/Q3/Q5/Q6 parity (BASELINE config 4): libddq through the C ABI vs the
oracle, exact (scale-2 decimals as int64, int128 sums), prepared CUDA-graph plans
and the chopping driver, plus the cold path (GPU-only placement on an empty cache:
every column copied from pinned host memory)."""
import functools

import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu

SF = 0.1


@functools.lru_cache(maxsize=None)
def _data():
    return datagen.TPCH(SF)


@functools.lru_cache(maxsize=None)
def _db():
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch
    db = Database(cache_bytes=8 << 30, heap_bytes=8 << 30)
    load_tpch(db, _data())
    return db


@functools.lru_cache(maxsize=None)
def _want(q):
    return [tuple(r) for r in oracle.run(_data(), q)]


@pytest.mark.parametrize("q", ["tpch1", "tpch3", "tpch5", "tpch6"])
def test_tpch_prepared_equals_oracle(q):
    from paper_conf_sigmod_bressft16_b200.tpch import tpch_plan
    db = _db()
    p = db.prepare(tpch_plan(db, q))
    p.launch()
    got = p.fetch().rows
    p.close()
    assert got and got == _want(q)


@pytest.mark.parametrize("q", ["tpch1", "tpch3", "tpch5", "tpch6"])
def test_tpch_submit_equals_oracle(q):
    from paper_conf_sigmod_bressft16_b200.tpch import tpch_plan
    db = _db()
    r = db.run(tpch_plan(db, q))
    assert r.rows == _want(q) and r.host_ops == 0


def test_tpch3_limit10():
    from paper_conf_sigmod_bressft16_b200.tpch import tpch_plan
    db = _db()
    r = db.run(tpch_plan(db, "tpch3", limit=10))
    assert r.rows == _want("tpch3")[:10]


def test_tpch_cold_path_gpu_only():
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch, tpch_plan
    db = Database(cache_bytes=8 << 30, heap_bytes=4 << 30, placement=A.PLACE_GPU_ONLY)
    load_tpch(db, _data(), cache=False)
    for q in ("tpch1", "tpch6", "tpch5"):
        r = db.run(tpch_plan(db, q))
        assert r.rows == _want(q) and r.host_ops == 0
    st = db.stats()
    assert st["h2d_bytes"] > 0 and st["cache_misses"] > 0
    db.close()
