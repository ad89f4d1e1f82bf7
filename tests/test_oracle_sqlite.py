"""Pin: the oracle equals SQLite 3.45 executing the verbatim query texts.

SQLite is an independent SQL engine; it runs on tables whose string columns are
decoded, so this pins the oracle's predicates, joins, grouping, aggregate
arithmetic and ORDER BY (first row).
"""
import functools

import pytest

import datagen
import oracle

from sqlref import load_sql, ssb_sqlite, tpch_sqlite

# Oracle output row -> SQL select-list row (strings decoded).
#   key spec: ("k", index, dict-or-None) | ("a", index) ; None dict = integer
SSB_SELECT = {
    "ssb1": [("a", 0)],
    "ssb2": [("a", 0), ("k", 0, None), ("k", 1, "brand1")],
    "ssb3.1": [("k", 0, "nation"), ("k", 1, "nation"), ("k", 2, None), ("a", 0)],
    "ssb3": [("k", 0, "city"), ("k", 1, "city"), ("k", 2, None), ("a", 0)],
    "ssb4.1": [("k", 0, None), ("k", 1, "nation"), ("a", 0)],
    "ssb4.2": [("k", 0, None), ("k", 1, "nation"), ("k", 2, "category"), ("a", 0)],
    "ssb4.3": [("k", 0, None), ("k", 1, "city"), ("k", 2, "brand1"), ("a", 0)],
}


def select_spec(q):
    for k in (q[:6], q[:4]):
        if k in SSB_SELECT:
            return SSB_SELECT[k]
    raise KeyError(q)


def to_sql_rows(q, rows, nkeys):
    spec = select_spec(q)
    dicts = {}
    out = []
    for r in rows:
        if q.startswith("ssb1"):
            out.append((r[0],))  # the oracle reports SUM over no rows as NULL (O7)
            continue
        t = []
        for s in spec:
            if s[0] == "a":
                t.append(r[nkeys + s[1]])
            else:
                v = r[s[1]]
                if s[2]:
                    d = dicts.setdefault(s[2], datagen.dictionary(s[2]))
                    v = d[v]
                t.append(v)
        out.append(tuple(t))
    return out


NKEYS = {"ssb1": 0, "ssb2": 2, "ssb3": 3, "ssb4.1": 2, "ssb4.2": 3, "ssb4.3": 3}


def nkeys_of(q):
    return NKEYS.get(q[:6], NKEYS.get(q[:4]))


@functools.lru_cache(maxsize=None)
def _ssb(sf, keys="dense"):
    db = datagen.SSB(sf, keys=keys)
    return db, ssb_sqlite(db)


@pytest.mark.parametrize("sf,keys", [(0.01, "dense"), (0.05, "dense"), (0.01, "sparse")])
@pytest.mark.parametrize("q", oracle.SSB_QUERIES)
def test_ssb_oracle_equals_sqlite(sf, keys, q):
    db, con = _ssb(sf, keys)
    sql = load_sql("ssb_queries.sql")[q]
    want = [tuple(r) for r in con.execute(sql).fetchall()]
    got = to_sql_rows(q, oracle.run(db, q), nkeys_of(q))
    assert sorted(got, key=repr) == sorted(want, key=repr)
    # the declared ORDER BY keys must agree row by row (ties may differ: O8)
    order_idx = {"ssb2": [1, 2], "ssb3": [2], "ssb4": [0, 1, 2]}.get(q[:4], [])
    if q.startswith("ssb4.1"):
        order_idx = [0, 1]
    assert [tuple(r[i] for i in order_idx) for r in got] == [tuple(r[i] for i in order_idx) for r in want]
    if q.startswith("ssb3"):  # revenue desc within a year
        assert [r[3] for r in got] == [r[3] for r in want]


class _Override:
    """A datagen.SSB view with some columns replaced (planted data)."""

    def __init__(self, db, cols):
        self.db, self.cols = db, cols

    def __getitem__(self, c):
        return self.cols[c] if c in self.cols else self.db[c]

    def rows(self, t):
        return self.db.rows(t)

    def dict_for(self, c):
        return self.db.dict_for(c)


@pytest.mark.parametrize("q", ["ssb1.1", "ssb1.2", "ssb1.3"])
def test_ungrouped_sum_over_no_rows_is_null(q):
    """Reading O7: an aggregate without GROUP BY over an empty input is one row whose
    SUM is SQL NULL (SQLite's answer) and whose COUNT is 0."""
    import numpy as np
    db = datagen.SSB(0.01)
    planted = _Override(db, {"lo_discount": np.zeros_like(db["lo_discount"])})  # no discount qualifies
    con = ssb_sqlite(db, {"lo_discount": planted["lo_discount"]})
    want = [tuple(r) for r in con.execute(load_sql("ssb_queries.sql")[q]).fetchall()]
    assert want == [(None,)]
    assert oracle.run(planted, q) == [(None, 0)]


@functools.lru_cache(maxsize=None)
def _tpch(sf, keys="dense"):
    db = datagen.TPCH(sf, keys=keys)
    return db, tpch_sqlite(db)


def tpch_to_sql(q, rows):
    if q == "tpch2":  # (p_partkey, s_suppkey, s_acctbal, n_name, p_mfgr) -> the select list
        nat, mf = datagen.dictionary("nation"), datagen.dictionary("tpch_mfgr")
        return [(r[2], r[1], nat[r[3]], r[0], mf[r[4]]) for r in rows]
    if q == "tpch1":
        rf, ls = datagen.dictionary("returnflag"), datagen.dictionary("linestatus")
        return [(rf[r[0]], ls[r[1]]) + tuple(r[2:]) for r in rows]
    if q == "tpch4":
        pr = datagen.dictionary("orderpriority")
        return [(pr[r[0]], r[1]) for r in rows]
    if q == "tpch7":
        nat = datagen.dictionary("nation")
        return [(nat[r[0]], nat[r[1]]) + tuple(r[2:]) for r in rows]
    if q == "tpch5":
        nat = datagen.dictionary("nation")
        return [(nat[r[0]], r[1]) for r in rows]
    if q == "tpch6":
        return [(r[0], r[1]) for r in rows]
    return [tuple(r) for r in rows]


@pytest.mark.parametrize("keys", ["dense", "sparse"])
@pytest.mark.parametrize("q", ["tpch1", "tpch2", "tpch3", "tpch4", "tpch5", "tpch6", "tpch7"])
def test_tpch_oracle_equals_sqlite(q, keys):
    db, con = _tpch(0.01, keys)
    want = [tuple(r) for r in con.execute(load_sql("tpch_queries.sql")[q]).fetchall()]
    got = tpch_to_sql(q, oracle.run(db, q))
    if q == "tpch1":
        # AVG columns (reading O10): the oracle's long-double sum / count / 100 against
        # SQLite's own avg() of the scale-2 integers, / 100
        _, avgs = oracle.run_with_avgs(db, q)
        assert len(avgs) == len(want) == 4
        for a, w in zip(avgs, want):
            for x, y in zip(a, w[-3:]):
                assert x == pytest.approx(y / 100.0, rel=1e-12)
        want = [w[:-3] for w in want]
    assert len(got) > 0
    assert sorted(got, key=repr) == sorted(want, key=repr)
    if q == "tpch3":  # revenue desc, o_orderdate asc
        assert [(r[3], r[1]) for r in got] == [(r[3], r[1]) for r in want]
    if q == "tpch5":
        assert [r[1] for r in got] == [r[1] for r in want]
    if q in ("tpch2", "tpch4", "tpch7"):  # fully ordered (decoded strings, keys)
        assert got == want
