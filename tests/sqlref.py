"""SQLite 3.45 reference (an independent SQL engine) for pinning the oracle.

Loads datagen tables into an in-memory SQLite database with string columns
DECODED through their dictionaries, then runs the verbatim query texts of
tests/golden/*.sql.  Nothing here shares code with oracle/ or the product.
"""
from __future__ import annotations

import os
import sqlite3

import datagen

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_sql(fname: str) -> dict[str, str]:
    out, cur, buf = {}, None, []
    for line in open(os.path.join(GOLDEN, fname)):
        if line.startswith("-- @"):
            if cur:
                out[cur] = "".join(buf)
            cur, buf = line[4:].strip(), []
        elif cur and not line.startswith("--"):
            buf.append(line)
    if cur:
        out[cur] = "".join(buf)
    return out


def _create(con, table: str, cols: dict[str, list]) -> None:
    names = list(cols)
    con.execute(f'create table "{table}" ({", ".join(names)})')
    rows = list(zip(*[cols[n] for n in names]))
    con.executemany(f'insert into "{table}" values ({", ".join("?" * len(names))})', rows)


def ssb_sqlite(db: "datagen.SSB", overrides: dict | None = None) -> sqlite3.Connection:
    """overrides: column name -> numpy array replacing the generated one."""
    overrides = overrides or {}
    con = sqlite3.connect(":memory:")
    for table, cols in datagen.SSB_COLUMNS.items():
        data = {}
        for c in cols:
            if table == "part" and c == "p_retailprice":
                continue
            a = overrides.get(c)
            a = db[c] if a is None else a
            if c in datagen.SSB_STRING_COLUMNS:
                d = db.dict_for(c)
                data[c] = [d[int(v)] for v in a]
            else:
                data[c] = [int(v) for v in a]
        _create(con, table, data)
    return con


def tpch_sqlite(db: "datagen.TPCH") -> sqlite3.Connection:
    con = sqlite3.connect(":memory:")
    for table, cols in datagen.TPCH_COLUMNS.items():
        data = {}
        for c in cols:
            a = db.col(table, c)
            if c in datagen.TPCH_STRING_COLUMNS:
                d = db.dict_for(c)
                data[c] = [d[int(v)] for v in a]
            else:
                data[c] = [int(v) for v in a]
        _create(con, table, data)
    return con
