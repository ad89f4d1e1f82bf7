"""Result semantics on the GPU path (S8(a7), S8(b)): decoded string keys, TPC-H Q1's
AVG columns, SQL NULL of an empty ungrouped SUM, and dictionary predicates
(ddq_dictionary_range / ddq_dictionary_like -> IN / BITSET code sets).

Pins: the oracle (AVG in long double from exact sums, rel 1e-9 per north_star);
Python's own string comparisons / fnmatch over the datagen dictionaries for the
predicates (a library routine, independent of the product)."""
import fnmatch
import functools
import math

import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu


@functools.lru_cache(maxsize=None)
def _ssb(sf):
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.ssb import load_ssb
    data = datagen.SSB(sf)
    db = Database(cache_bytes=4 << 30, heap_bytes=4 << 30)
    load_ssb(db, data)
    return data, db


@functools.lru_cache(maxsize=None)
def _tpch(sf):
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch
    data = datagen.TPCH(sf)
    db = Database(cache_bytes=4 << 30, heap_bytes=4 << 30)
    load_tpch(db, data)
    return data, db


# (query, dictionaries of its keys in order; None = integer key)
DECODE = {"ssb2.1": [None, "brand1"], "ssb3.1": ["nation", "nation", None], "ssb3.2": ["city", "city", None],
          "ssb4.1": [None, "nation"], "ssb4.2": [None, "nation", "category"], "ssb4.3": [None, "city", "brand1"]}


@pytest.mark.parametrize("q", list(DECODE))
def test_decoded_keys_equal_oracle_strings(q):
    from paper_conf_sigmod_bressft16_b200.ssb import ssb_plan
    data, db = _ssb(1)
    want = oracle.run(data, q)
    dicts = [datagen.dictionary(d) if d else None for d in DECODE[q]]
    want_dec = [tuple(dicts[k][r[k]] if dicts[k] else r[k] for k in range(len(dicts))) + tuple(r[len(dicts):])
                for r in want]
    p = db.prepare(ssb_plan(db, q))
    p.launch()
    got = p.fetch()
    p.close()
    assert got.rows == want
    assert got.decoded == want_dec
    r = db.run(ssb_plan(db, q))  # the chopping driver decodes the same way
    assert r.decoded == want_dec


@pytest.mark.parametrize("dense", [True, False])
@pytest.mark.parametrize("path", ["prepared", "submit"])
def test_tpch1_avg_columns(path, dense):
    """avg_qty / avg_price / avg_disc (reading O10) within rel 1e-9 of the oracle's
    long-double sum / count / 100; the exact sums equal too."""
    from paper_conf_sigmod_bressft16_b200.tpch import tpch_plan
    data, db = _tpch(0.1)
    want, want_avg = oracle.run_with_avgs(data, "tpch1")
    if path == "prepared":
        p = db.prepare(tpch_plan(db, "tpch1", dense=dense))
        p.launch()
        got = p.fetch()
        p.close()
    else:
        got = db.run(tpch_plan(db, "tpch1", dense=dense))
    assert got.rows == want
    assert len(got.avgs) == len(want_avg) == len(want)
    for a, b in zip(got.avgs, want_avg):
        for x, y in zip(a, b):
            assert abs(x - y) <= 1e-9 * abs(y)
    rf, ls = datagen.dictionary("returnflag"), datagen.dictionary("linestatus")
    assert [d[:2] for d in got.decoded] == [(rf[r[0]], ls[r[1]]) for r in want]


def test_ungrouped_empty_sum_is_null_row():
    """Q1.1 over a selection nothing passes: one row, SUM NULL, COUNT 0 (O7) -- the
    same row the oracle returns; prepared and submitted paths."""
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    data, db = _ssb(0.05)
    P = db.plan()
    hd = P.build("date", "d_datekey", where=[("d_year", 1993, 1993)])
    t = P.probe("lineorder", "lo_orderdate", hd)
    P.aggregate("lineorder", t, keys=[], aggs=[(A.AGG_SUM_MUL, ["lo_extendedprice", "lo_discount"]),
                                              (A.AGG_COUNT, []), (A.AGG_MIN, ["lo_revenue"])],
                max_groups=1, where=[("lo_discount", 11, 20)])  # discount is 0..10: empty
    p = db.prepare(P)
    p.launch()
    assert p.fetch().rows == [(None, 0, None)]
    p.close()
    assert db.run(P).rows == [(None, 0, None)]


@pytest.mark.parametrize("pattern", ["MFGR#12%", "MFGR#3%3", "MFGR#4_1_", "MFGR#2239", "MFGR#5%", "nothing%",
                                     "MFGR#1_1"])
def test_dictionary_like_selection(pattern):
    """p_brand1 LIKE pattern folded into a code predicate (IN for <= 8 codes, BITSET
    beyond) and evaluated by the selection kernel and the fused build: the
    survivors equal numpy over fnmatch on the decoded strings."""
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    data, db = _ssb(1)
    brands = datagen.dictionary("brand1")
    glob = pattern.replace("%", "*").replace("_", "?")
    codes = [i for i, s in enumerate(brands) if fnmatch.fnmatchcase(s, glob)]
    pred = db.like("part", "p_brand1", pattern)
    assert pred.kind == (A.PRED_RANGE if not codes else A.PRED_IN if len(codes) <= 8 else A.PRED_BITSET)
    col = data["p_brand1"]
    want = np.flatnonzero(np.isin(col, codes))
    # SELECT -> TIDs (select-* root returns sorted global row ids)
    P = db.plan()
    P.select("part", [pred])
    got = db.prepare(P)
    got.launch()
    r = got.fetch()
    got.close()
    assert np.array_equal(r.tids, want)
    # the same predicate fused into a build, probed by lineorder: semi-join count
    P = db.plan()
    hp = P.build("part", "p_partkey", where=[pred])
    t = P.probe("lineorder", "lo_partkey", hp)
    P.aggregate("lineorder", t, keys=[], aggs=[(A.AGG_COUNT, [])], max_groups=1)
    n = int(np.isin(data["lo_partkey"], data["p_partkey"][want]).sum())
    p = db.prepare(P)
    p.launch()
    assert p.fetch().rows == [(n,)]
    p.close()


def test_dictionary_api_validation():
    from paper_conf_sigmod_bressft16_b200 import DDQError
    data, db = _ssb(0.05)
    with pytest.raises(DDQError):
        db.set_dictionary("part", "p_mfgr", ["MFGR#2", "MFGR#1", "MFGR#3", "MFGR#4", "MFGR#5"])  # not sorted
    with pytest.raises(DDQError):
        db.set_dictionary("part", "p_mfgr", ["MFGR#1", "MFGR#2"])  # codes 2..4 outside it
    lo, hi = db.dictionary_range("part", "p_brand1", "MFGR#2221")
    b = datagen.dictionary("brand1")
    assert b[lo] == "MFGR#2221" and hi == lo + 1
    lo2, hi2 = db.dictionary_range("part", "p_brand1", "MFGR#2221x")  # absent: empty range
    assert lo2 == hi2 == lo + 1
    assert not math.isnan(lo)
    with pytest.raises(DDQError):  # matches spread over more than 512 codes
        db.like("part", "p_brand1", "%3")
