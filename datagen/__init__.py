"""Seeded synthetic SSB / TPC-H column generator (shared input infrastructure).

Both sides of every parity test use this module: the oracle (``oracle/``) and the
product (``paper_conf_sigmod_bressft16_b200``).  It contains no arithmetic of the
paper's method (no selection, join, gather or aggregation) -- only base-table
columns and their order-preserving string dictionaries.  The recipe is
SURVEY.md 8(c).2; the readings it fixes (O2, O3, O4, O6, O12, O21) are listed in
DESIGN.md.  Workloads named by the paper: SSB [28] and
TPC-H.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libddqgen.so")
_SRC = [os.path.join(_HERE, "ssbgen.c"), os.path.join(_HERE, "tpchgen.c")]

DEFAULT_SEED = 0x5EED2016
# primary-key encodings (ssbgen.c ddqgen_key_of): "dense" keys 1..n, or "sparse" keys
# spread by a bijection over >= 16x the rows (the general open-addressing join path)
KEY_MODES = {"dense": 0, "sparse": 1}


def build(force: bool = False) -> str:
    """Compile libddqgen.so in-tree (gcc, OpenMP)."""
    srcs = [s for s in _SRC if os.path.exists(s)]
    if not force and os.path.exists(_SO) and all(
            os.path.getmtime(_SO) >= os.path.getmtime(s) for s in srcs):
        return _SO
    cmd = ["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11", "-o", _SO] + srcs + ["-lm"]
    subprocess.check_call(cmd)
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        L.ddqgen_ssb_rows.restype = ctypes.c_int64
        L.ddqgen_ssb_rows.argtypes = [ctypes.c_int, ctypes.c_double]
        L.ddqgen_ssb_width.restype = ctypes.c_int
        L.ddqgen_ssb_width.argtypes = [ctypes.c_int, ctypes.c_int]
        L.ddqgen_ssb_column.restype = ctypes.c_int
        L.ddqgen_ssb_column.argtypes = [ctypes.c_uint64, ctypes.c_double, ctypes.c_int, ctypes.c_int,
                                        ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int]
        L.ddqgen_ssb_column_k.restype = ctypes.c_int
        L.ddqgen_ssb_column_k.argtypes = L.ddqgen_ssb_column.argtypes + [ctypes.c_int]
        L.ddqgen_key_of.restype = ctypes.c_int64
        L.ddqgen_key_of.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_int64]
        L.ddqgen_dict_size.restype = ctypes.c_int
        L.ddqgen_dict_size.argtypes = [ctypes.c_int]
        L.ddqgen_dict_entry.restype = ctypes.c_char_p
        L.ddqgen_dict_entry.argtypes = [ctypes.c_int, ctypes.c_int]
        L.ddqgen_hash.restype = ctypes.c_uint64
        L.ddqgen_hash.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint64]
        L.ddqgen_datekey_of_index.restype = ctypes.c_int32
        L.ddqgen_datekey_of_index.argtypes = [ctypes.c_int64]
        if hasattr(L, "ddqgen_tpch_rows"):
            L.ddqgen_tpch_rows.restype = ctypes.c_int64
            L.ddqgen_tpch_rows.argtypes = [ctypes.c_int, ctypes.c_double]
            L.ddqgen_tpch_width.restype = ctypes.c_int
            L.ddqgen_tpch_width.argtypes = [ctypes.c_int, ctypes.c_int]
            L.ddqgen_tpch_column.restype = ctypes.c_int
            L.ddqgen_tpch_column.argtypes = [ctypes.c_uint64, ctypes.c_double, ctypes.c_int, ctypes.c_int,
                                             ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int]
            L.ddqgen_tpch_column_k.restype = ctypes.c_int
            L.ddqgen_tpch_column_k.argtypes = L.ddqgen_tpch_column.argtypes + [ctypes.c_int]
        _lib = L
    return _lib


# ----------------------------------------------------------------- SSB schema
SSB_TABLES = {"date": 1, "customer": 2, "supplier": 3, "part": 4, "lineorder": 5}
SSB_COLUMNS = {
    "date": ["d_datekey", "d_year", "d_yearmonthnum", "d_yearmonth", "d_daynuminyear",
             "d_monthnuminyear", "d_weeknuminyear"],
    "customer": ["c_custkey", "c_city", "c_nation", "c_region", "c_mktsegment"],
    "supplier": ["s_suppkey", "s_city", "s_nation", "s_region"],
    "part": ["p_partkey", "p_mfgr", "p_category", "p_brand1", "p_retailprice"],
    "lineorder": ["lo_orderkey", "lo_linenumber", "lo_custkey", "lo_partkey", "lo_suppkey",
                  "lo_orderdate", "lo_orderpriority", "lo_shippriority", "lo_quantity",
                  "lo_extendedprice", "lo_ordtotalprice", "lo_discount", "lo_revenue",
                  "lo_supplycost", "lo_tax", "lo_commitdate", "lo_shipmode"],
}
# string columns -> dictionary id
DICTS = {"nation": 0, "region": 1, "city": 2, "mfgr": 3, "category": 4, "brand1": 5,
         "yearmonth": 6, "mktsegment": 7, "orderpriority": 8, "shipmode": 9,
         "returnflag": 10, "linestatus": 11, "type": 12, "tpch_mfgr": 13}
SSB_STRING_COLUMNS = {
    "d_yearmonth": "yearmonth", "c_city": "city", "c_nation": "nation", "c_region": "region",
    "c_mktsegment": "mktsegment", "s_city": "city", "s_nation": "nation", "s_region": "region",
    "p_mfgr": "mfgr", "p_category": "category", "p_brand1": "brand1",
    "lo_orderpriority": "orderpriority", "lo_shipmode": "shipmode",
}


def dictionary(name: str) -> list[str]:
    """Bytewise-sorted distinct strings of a dictionary; code == list index."""
    L = lib()
    d = DICTS[name]
    return [L.ddqgen_dict_entry(d, i).decode() for i in range(L.ddqgen_dict_size(d))]


def ssb_table_of(col: str) -> str:
    for t, cols in SSB_COLUMNS.items():
        if col in cols:
            return t
    raise KeyError(col)


def ssb_rows(table: str, sf: float) -> int:
    return int(lib().ddqgen_ssb_rows(SSB_TABLES[table], float(sf)))


def ssb_column(col: str, sf: float, seed: int = DEFAULT_SEED, begin: int = 0, end: int | None = None,
               nthreads: int | None = None, out: np.ndarray | None = None, keys: str = "dense") -> np.ndarray:
    """Rows [begin, end) of one SSB column as a numpy array (int32 or int64)."""
    L = lib()
    table = ssb_table_of(col)
    t = SSB_TABLES[table]
    c = SSB_COLUMNS[table].index(col)
    n = ssb_rows(table, sf)
    end = n if end is None else end
    w = L.ddqgen_ssb_width(t, c)
    dt = np.int32 if w == 4 else np.int64
    if out is None:
        out = np.empty(end - begin, dtype=dt)
    assert out.dtype == dt and out.size == end - begin and out.flags.c_contiguous
    nthreads = nthreads or os.cpu_count() or 1
    rc = L.ddqgen_ssb_column_k(seed, float(sf), t, c, begin, end, out.ctypes.data, nthreads, KEY_MODES[keys])
    if rc != 0:
        raise ValueError(f"ddqgen_ssb_column({col}, sf={sf}, [{begin},{end})) failed")
    return out


class SSB:
    """Lazily generated SSB database at one scale factor (host numpy columns);
    keys: "dense" (1..n) or "sparse" primary / foreign keys (KEY_MODES)."""

    def __init__(self, sf: float, seed: int = DEFAULT_SEED, keys: str = "dense"):
        self.sf = sf
        self.seed = seed
        self.keys = keys
        self._cols: dict[str, np.ndarray] = {}

    def rows(self, table: str) -> int:
        return ssb_rows(table, self.sf)

    def __getitem__(self, col: str) -> np.ndarray:
        if col not in self._cols:
            self._cols[col] = ssb_column(col, self.sf, self.seed, keys=self.keys)
        return self._cols[col]

    def dict_for(self, col: str) -> list[str]:
        return dictionary(SSB_STRING_COLUMNS[col])

    def drop(self, col: str) -> None:
        self._cols.pop(col, None)


# --------------------------------------------------------------- TPC-H schema
TPCH_TABLES = {"nation": 11, "region": 12, "customer": 13, "supplier": 14, "part": 15,
               "orders": 16, "lineitem": 17, "calendar": 18, "partsupp": 19}
TPCH_COLUMNS = {
    "nation": ["n_nationkey", "n_name", "n_regionkey"],
    "region": ["r_regionkey", "r_name"],
    "customer": ["c_custkey", "c_nationkey", "c_mktsegment"],
    "supplier": ["s_suppkey", "s_nationkey", "s_acctbal"],
    "part": ["p_partkey", "p_retailprice", "p_mfgr", "p_type", "p_size"],
    "orders": ["o_orderkey", "o_custkey", "o_orderdate", "o_shippriority", "o_orderpriority"],
    "lineitem": ["l_orderkey", "l_partkey", "l_suppkey", "l_linenumber", "l_quantity",
                 "l_extendedprice", "l_discount", "l_tax", "l_returnflag", "l_linestatus",
                 "l_shipdate", "l_commitdate", "l_receiptdate"],
    # the date dimension over TPC-H's date domain, 1992-01-01 .. 1998-12-31 (reading O34)
    "calendar": ["d_datekey", "d_year"],
    # TPC-H Q2: 4 suppliers per part (the TPC-H supplier rule), supplycost scale 2
    "partsupp": ["ps_partkey", "ps_suppkey", "ps_supplycost"],
}
TPCH_STRING_COLUMNS = {"n_name": "nation", "r_name": "region", "c_mktsegment": "mktsegment",
                       "l_returnflag": "returnflag", "l_linestatus": "linestatus",
                       "o_orderpriority": "orderpriority", "p_type": "type", "p_mfgr": "tpch_mfgr"}


def tpch_rows(table: str, sf: float) -> int:
    return int(lib().ddqgen_tpch_rows(TPCH_TABLES[table], float(sf)))


def tpch_column(table: str, col: str, sf: float, seed: int = DEFAULT_SEED, begin: int = 0,
                end: int | None = None, nthreads: int | None = None, keys: str = "dense") -> np.ndarray:
    L = lib()
    t = TPCH_TABLES[table]
    c = TPCH_COLUMNS[table].index(col)
    n = tpch_rows(table, sf)
    end = n if end is None else end
    w = L.ddqgen_tpch_width(t, c)
    out = np.empty(end - begin, dtype=np.int32 if w == 4 else np.int64)
    rc = L.ddqgen_tpch_column_k(seed, float(sf), t, c, begin, end, out.ctypes.data,
                                nthreads or os.cpu_count() or 1, KEY_MODES[keys])
    if rc != 0:
        raise ValueError(f"ddqgen_tpch_column({table}.{col}) failed")
    return out


class TPCH:
    """Lazily generated TPC-H database; columns addressed as (table, column);
    keys: "dense" or "sparse" (KEY_MODES)."""

    def __init__(self, sf: float, seed: int = DEFAULT_SEED, keys: str = "dense"):
        self.sf = sf
        self.seed = seed
        self.keys = keys
        self._cols: dict[tuple[str, str], np.ndarray] = {}

    def rows(self, table: str) -> int:
        return tpch_rows(table, self.sf)

    def col(self, table: str, col: str) -> np.ndarray:
        if (table, col) not in self._cols:
            self._cols[(table, col)] = tpch_column(table, col, self.sf, self.seed, keys=self.keys)
        return self._cols[(table, col)]

    def dict_for(self, col: str) -> list[str]:
        return dictionary(TPCH_STRING_COLUMNS[col])
