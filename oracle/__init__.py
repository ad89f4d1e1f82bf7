"""TEST INFRASTRUCTURE ONLY -- the CPU oracle (see oracle/oracle.cpp header).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference``) may import this package.  The product package
``paper_conf_sigmod_bressft16_b200`` never imports it and shares no code with it.

``run(db, query)`` evaluates one query on a ``datagen.SSB`` / ``datagen.TPCH``
database with the plain single-threaded column-at-a-time evaluator of
oracle/oracle.cpp and returns rows as tuples of Python ints
``(key_0, ..., key_{k-1}, agg_0, ..., agg_{m-1})`` in the query's ORDER BY order.

Parity status per function:
  ssb1.1 .. ssb4.3   pinned: SQLite 3.45 on decoded tables, nested-loop brute force
                     on planted tables, group-count / sum-conservation invariants
  listing1..8        pinned: closed form (empty by the SSB value domains), brute force
  listing2b          pinned: numpy.flatnonzero of the predicate, binomial bounds
  tpch1-7            pinned: SQLite 3.45 on decoded tables (tpch4: EXISTS subquery;
                     tpch2: the correlated MIN subquery, LIKE '%BRASS')
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

import datagen

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.cpp")


def build(force: bool = False) -> str:
    if not force and os.path.exists(_SO) and os.path.getmtime(_SO) >= os.path.getmtime(_SRC):
        return _SO
    subprocess.check_call(["g++", "-std=c++17", "-O2", "-fPIC", "-shared", "-o", _SO, _SRC])
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        L.oracle_db_new.restype = ctypes.c_void_p
        L.oracle_db_free.argtypes = [ctypes.c_void_p]
        L.oracle_db_set_col.argtypes = [ctypes.c_void_p, ctypes.c_char_p, ctypes.c_void_p,
                                        ctypes.c_int64, ctypes.c_int]
        L.oracle_db_set_dict.argtypes = [ctypes.c_void_p, ctypes.c_char_p, ctypes.c_int,
                                         ctypes.POINTER(ctypes.c_char_p)]
        L.oracle_last_error.restype = ctypes.c_char_p
        L.oracle_query.restype = ctypes.c_void_p
        L.oracle_query.argtypes = [ctypes.c_void_p, ctypes.c_char_p]
        L.oracle_result_free.argtypes = [ctypes.c_void_p]
        L.oracle_result_rows.restype = ctypes.c_int64
        L.oracle_result_rows.argtypes = [ctypes.c_void_p]
        L.oracle_result_nkeys.argtypes = [ctypes.c_void_p]
        L.oracle_result_naggs.argtypes = [ctypes.c_void_p]
        L.oracle_result_row.argtypes = [ctypes.c_void_p, ctypes.c_int64,
                                        ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]
        L.oracle_result_nulls.argtypes = [ctypes.c_void_p, ctypes.c_int64]
        L.oracle_result_navg.argtypes = [ctypes.c_void_p]
        L.oracle_result_avgs.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.POINTER(ctypes.c_double)]
        L.oracle_result_ntids.restype = ctypes.c_int64
        L.oracle_result_ntids.argtypes = [ctypes.c_void_p]
        L.oracle_result_tids.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
        _lib = L
    return _lib


# Columns each query reads (the wrapper hands exactly these to the evaluator).
_DIMS_SSB = ["d_datekey", "d_year", "d_yearmonthnum", "d_yearmonth", "d_weeknuminyear",
             "c_custkey", "c_city", "c_nation", "c_region",
             "s_suppkey", "s_city", "s_nation", "s_region",
             "p_partkey", "p_mfgr", "p_category", "p_brand1"]
SSB_QUERY_COLUMNS = {
    1: ["lo_orderdate", "lo_discount", "lo_quantity", "lo_extendedprice"],
    2: ["lo_partkey", "lo_suppkey", "lo_orderdate", "lo_revenue"],
    3: ["lo_custkey", "lo_suppkey", "lo_orderdate", "lo_revenue"],
    4: ["lo_custkey", "lo_suppkey", "lo_partkey", "lo_orderdate", "lo_revenue", "lo_supplycost"],
}
LISTING_COLUMNS = {1: "lo_quantity", 2: "lo_discount", 3: "lo_shippriority", 4: "lo_extendedprice",
                   5: "lo_ordtotalprice", 6: "lo_revenue", 7: "lo_supplycost", 8: "lo_tax"}
TPCH_QUERY_COLUMNS = {
    2: [("region", "r_regionkey"), ("region", "r_name"), ("nation", "n_nationkey"), ("nation", "n_name"),
        ("nation", "n_regionkey"), ("supplier", "s_suppkey"), ("supplier", "s_nationkey"),
        ("supplier", "s_acctbal"), ("part", "p_partkey"), ("part", "p_size"), ("part", "p_type"),
        ("part", "p_mfgr"), ("partsupp", "ps_partkey"), ("partsupp", "ps_suppkey"),
        ("partsupp", "ps_supplycost")],
    1: [("lineitem", c) for c in ["l_shipdate", "l_returnflag", "l_linestatus", "l_quantity",
                                  "l_extendedprice", "l_discount", "l_tax"]],
    3: [("customer", "c_custkey"), ("customer", "c_mktsegment"), ("orders", "o_orderkey"),
        ("orders", "o_custkey"), ("orders", "o_orderdate"), ("orders", "o_shippriority"),
        ("lineitem", "l_orderkey"), ("lineitem", "l_shipdate"), ("lineitem", "l_extendedprice"),
        ("lineitem", "l_discount")],
    5: [("region", "r_regionkey"), ("region", "r_name"), ("nation", "n_nationkey"),
        ("nation", "n_name"), ("nation", "n_regionkey"), ("supplier", "s_suppkey"),
        ("supplier", "s_nationkey"), ("customer", "c_custkey"), ("customer", "c_nationkey"),
        ("orders", "o_orderkey"), ("orders", "o_custkey"), ("orders", "o_orderdate"),
        ("lineitem", "l_orderkey"), ("lineitem", "l_suppkey"), ("lineitem", "l_extendedprice"),
        ("lineitem", "l_discount")],
    4: [("orders", "o_orderkey"), ("orders", "o_orderdate"), ("orders", "o_orderpriority"),
        ("lineitem", "l_orderkey"), ("lineitem", "l_commitdate"), ("lineitem", "l_receiptdate")],
    6: [("lineitem", c) for c in ["l_shipdate", "l_discount", "l_quantity", "l_extendedprice"]],
    7: [("nation", "n_nationkey"), ("nation", "n_name"), ("supplier", "s_suppkey"),
        ("supplier", "s_nationkey"), ("customer", "c_custkey"), ("customer", "c_nationkey"),
        ("orders", "o_orderkey"), ("orders", "o_custkey"), ("lineitem", "l_orderkey"),
        ("lineitem", "l_suppkey"), ("lineitem", "l_shipdate"), ("lineitem", "l_extendedprice"),
        ("lineitem", "l_discount")],
}


class OracleDB:
    """Column pointers + dictionaries handed to the C++ evaluator (arrays kept alive)."""

    def __init__(self):
        self._h = lib().oracle_db_new()
        self._keep: list = []

    def __del__(self):
        try:
            lib().oracle_db_free(self._h)
        except Exception:
            pass

    def set_col(self, name: str, arr: np.ndarray, n: int | None = None) -> None:
        arr = np.ascontiguousarray(arr)
        assert arr.dtype in (np.int32, np.int64)
        self._keep.append(arr)
        lib().oracle_db_set_col(self._h, name.encode(), arr.ctypes.data,
                                arr.size if n is None else n, arr.itemsize)

    def set_dict(self, name: str, strings: list[str]) -> None:
        enc = [s.encode() for s in strings]
        arr = (ctypes.c_char_p * len(enc))(*enc)
        self._keep.append((enc, arr))
        lib().oracle_db_set_dict(self._h, name.encode(), len(enc), arr)

    def query(self, name: str):
        L = lib()
        r = L.oracle_query(self._h, name.encode())
        if not r:
            raise RuntimeError("oracle: " + L.oracle_last_error().decode())
        try:
            if name.startswith("listing"):
                n = L.oracle_result_ntids(r)
                out = np.empty(n, dtype=np.int32)
                L.oracle_result_tids(r, out.ctypes.data)
                return out
            nk, na, nv = L.oracle_result_nkeys(r), L.oracle_result_naggs(r), L.oracle_result_navg(r)
            keys = (ctypes.c_int64 * 4)()
            aggs = (ctypes.c_int64 * 16)()
            av = (ctypes.c_double * 4)()
            rows, avgs = [], []
            for i in range(L.oracle_result_rows(r)):
                L.oracle_result_row(r, i, keys, aggs)
                nulls = L.oracle_result_nulls(r, i)
                vals = [int(keys[k]) for k in range(nk)]
                for a in range(na):
                    lo = aggs[2 * a] & 0xFFFFFFFFFFFFFFFF
                    hi = aggs[2 * a + 1]
                    vals.append(None if (nulls >> a) & 1 else (hi << 64) | lo)  # SQL NULL (O7)
                rows.append(tuple(vals))
                if nv:
                    L.oracle_result_avgs(r, i, av)
                    avgs.append(tuple(float(av[k]) for k in range(nv)))
            self.last_avgs = avgs
            return rows
        finally:
            L.oracle_result_free(r)


def _set_dicts(odb: OracleDB) -> None:
    for name in datagen.DICTS:
        odb.set_dict(name, datagen.dictionary(name))


def ssb_db(db: "datagen.SSB", query: str, fact_rows: int | None = None) -> OracleDB:
    """Evaluator inputs for one SSB query; fact_rows bounds lineorder to a prefix."""
    odb = OracleDB()
    _set_dicts(odb)
    if query.startswith("ssb"):
        cols = _DIMS_SSB + SSB_QUERY_COLUMNS[int(query[3])]
    elif query == "listing2b":
        cols = ["lo_discount", "lo_quantity"]
    else:
        cols = [LISTING_COLUMNS[int(query[7])]]
    for c in cols:
        a = db[c]
        n = a.size if (fact_rows is None or not c.startswith("lo_")) else min(fact_rows, a.size)
        odb.set_col(c, a, n)
    return odb


def run(db, query: str, fact_rows: int | None = None):
    """Evaluate `query` ("ssb1.1".."ssb4.3", "listing1".."listing8", "listing2b",
    "tpch1", "tpch3", "tpch4", "tpch5", "tpch6", "tpch7") on a datagen database.
    Rows are (keys..., aggregates...) with None for a SQL NULL aggregate."""
    return run_with_avgs(db, query, fact_rows)[0]


def run_with_avgs(db, query: str, fact_rows: int | None = None):
    """(rows, avgs): avgs[i] = the AVG columns of row i (TPC-H Q1: avg_qty,
    avg_price, avg_disc as sum / count / 100 in long double, reading O10)."""
    if query.startswith("tpch"):
        odb = OracleDB()
        _set_dicts(odb)
        for (t, c) in TPCH_QUERY_COLUMNS[int(query[4:])]:
            odb.set_col(c, db.col(t, c))
    else:
        odb = ssb_db(db, query, fact_rows)
    rows = odb.query(query)
    return rows, getattr(odb, "last_avgs", [])


SSB_QUERIES = ["ssb1.1", "ssb1.2", "ssb1.3", "ssb2.1", "ssb2.2", "ssb2.3", "ssb3.1", "ssb3.2",
               "ssb3.3", "ssb3.4", "ssb4.1", "ssb4.2", "ssb4.3"]
