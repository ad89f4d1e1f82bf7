"""Pin: the oracle equals a pure-Python nested-loop brute force on planted data.

The brute force is row-at-a-time over DECODED strings: for every fact row it scans
each dimension table for the row whose primary key equals the foreign key (a
nested loop, no hashing), evaluates the WHERE clause of the SQL text
(tests/golden/ssb_queries.sql) as written, groups with a Python dict and sorts per
ORDER BY (ties: remaining keys ascending, reading O8).  It is deliberately a
different algorithm from the oracle's column-at-a-time hash joins.
"""
import functools

import pytest

import datagen
import oracle

from planted import Planted
from sqlref import load_sql, ssb_sqlite
from test_oracle_sqlite import nkeys_of, to_sql_rows

N_FACT = 1200


@functools.lru_cache(maxsize=None)
def _planted():
    return Planted()


@functools.lru_cache(maxsize=None)
def _joined():
    """Nested-loop join of the first N_FACT lineorder rows with every dimension."""
    db = _planted()
    dec = {}
    for c in datagen.SSB_STRING_COLUMNS:
        d = db.dict_for(c)
        dec[c] = [d[int(v)] for v in db[c]]

    def val(c, r):
        return dec[c][r] if c in dec else int(db[c][r])

    dims = {"date": ("d_datekey", "lo_orderdate"), "customer": ("c_custkey", "lo_custkey"),
            "supplier": ("s_suppkey", "lo_suppkey"), "part": ("p_partkey", "lo_partkey")}
    rows = []
    for i in range(N_FACT):
        row = {c: val(c, i) for c in datagen.SSB_COLUMNS["lineorder"]}
        for t, (pk, fk) in dims.items():
            match = None
            for r in range(len(db[pk])):  # nested loop: scan the dimension
                if int(db[pk][r]) == row[fk]:
                    match = r
                    break
            assert match is not None
            for c in datagen.SSB_COLUMNS[t]:
                if c != "p_retailprice":
                    row[c] = val(c, match)
        rows.append(row)
    return rows


CITIES = ("UNITED KI1", "UNITED KI5")
# WHERE clauses of tests/golden/ssb_queries.sql, transcribed; select-list keys; aggregate.
Q = {
    "ssb1.1": (lambda r: r["d_year"] == 1993 and 1 <= r["lo_discount"] <= 3 and r["lo_quantity"] < 25, None),
    "ssb1.2": (lambda r: r["d_yearmonthnum"] == 199401 and 4 <= r["lo_discount"] <= 6
               and 26 <= r["lo_quantity"] <= 35, None),
    "ssb1.3": (lambda r: r["d_weeknuminyear"] == 6 and r["d_year"] == 1994 and 5 <= r["lo_discount"] <= 7
               and 26 <= r["lo_quantity"] <= 35, None),
    "ssb2.1": (lambda r: r["p_category"] == "MFGR#12" and r["s_region"] == "AMERICA", ("d_year", "p_brand1")),
    "ssb2.2": (lambda r: "MFGR#2221" <= r["p_brand1"] <= "MFGR#2228" and r["s_region"] == "ASIA",
               ("d_year", "p_brand1")),
    "ssb2.3": (lambda r: r["p_brand1"] == "MFGR#2239" and r["s_region"] == "EUROPE", ("d_year", "p_brand1")),
    "ssb3.1": (lambda r: r["c_region"] == "ASIA" and r["s_region"] == "ASIA" and 1992 <= r["d_year"] <= 1997,
               ("c_nation", "s_nation", "d_year")),
    "ssb3.2": (lambda r: r["c_nation"] == "UNITED STATES" and r["s_nation"] == "UNITED STATES"
               and 1992 <= r["d_year"] <= 1997, ("c_city", "s_city", "d_year")),
    "ssb3.3": (lambda r: r["c_city"] in CITIES and r["s_city"] in CITIES and 1992 <= r["d_year"] <= 1997,
               ("c_city", "s_city", "d_year")),
    "ssb3.4": (lambda r: r["c_city"] in CITIES and r["s_city"] in CITIES and r["d_yearmonth"] == "Dec1997",
               ("c_city", "s_city", "d_year")),
    "ssb4.1": (lambda r: r["c_region"] == "AMERICA" and r["s_region"] == "AMERICA"
               and r["p_mfgr"] in ("MFGR#1", "MFGR#2"), ("d_year", "c_nation")),
    "ssb4.2": (lambda r: r["c_region"] == "AMERICA" and r["s_region"] == "AMERICA"
               and r["d_year"] in (1997, 1998) and r["p_mfgr"] in ("MFGR#1", "MFGR#2"),
               ("d_year", "s_nation", "p_category")),
    "ssb4.3": (lambda r: r["c_region"] == "AMERICA" and r["s_nation"] == "UNITED STATES"
               and r["d_year"] in (1997, 1998) and r["p_category"] == "MFGR#14",
               ("d_year", "s_city", "p_brand1")),
}


def brute(q):
    where, keys = Q[q]
    if q.startswith("ssb1"):
        m = [r for r in _joined() if where(r)]
        return [(sum(r["lo_extendedprice"] * r["lo_discount"] for r in m) if m else None,)]
    agg = (lambda r: r["lo_revenue"]) if q.startswith(("ssb2", "ssb3")) else \
        (lambda r: r["lo_revenue"] - r["lo_supplycost"])
    g = {}
    for r in _joined():
        if where(r):
            k = tuple(r[c] for c in keys)
            g[k] = g.get(k, 0) + agg(r)
    rows = [k + (v,) for k, v in g.items()]
    if q.startswith("ssb2"):
        return [(r[2], r[0], r[1]) for r in sorted(rows)]
    if q.startswith("ssb3"):
        return sorted(rows, key=lambda r: (r[2], -r[3], r[0], r[1]))
    return sorted(rows)


@pytest.mark.parametrize("q", oracle.SSB_QUERIES)
def test_oracle_equals_bruteforce_planted(q):
    want = brute(q)
    assert want and want != [(None,)], "planting must make every query non-empty"
    got = to_sql_rows(q, oracle.run(_planted(), q, fact_rows=N_FACT), nkeys_of(q))
    assert got == want  # same rows, same order (with the O8 tie-break)


@pytest.mark.parametrize("q", oracle.SSB_QUERIES)
def test_oracle_equals_sqlite_planted(q):
    db = _planted()
    con = _sqlite_planted()
    want = [tuple(r) for r in con.execute(load_sql("ssb_queries.sql")[q]).fetchall()]
    got = to_sql_rows(q, oracle.run(db, q), nkeys_of(q))
    assert sorted(got, key=repr) == sorted(want, key=repr)


@functools.lru_cache(maxsize=None)
def _sqlite_planted():
    db = _planted()
    return ssb_sqlite(db, overrides=dict(db))
