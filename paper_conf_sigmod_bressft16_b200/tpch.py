"""TPC-H Q1, Q3, Q4, Q5, Q6, Q7 on libddq (BASELINE config 4; the paper runs TPC-H,
PAPER.md:305, App. C.2).  Decimals are scale-2 int64 (reading O5); dates
are int32 yyyymmdd with folded constants (O11).  Query texts: SURVEY.md App. A.2.
"""
from __future__ import annotations

from . import _abi as A
from .engine import Database, PlanBuilder
from .ssb import code


TPCH_QUERIES = ["tpch1", "tpch2", "tpch3", "tpch4", "tpch5", "tpch6", "tpch7"]

TABLE_COLUMNS = {
    "nation": ["n_nationkey", "n_name", "n_regionkey"],
    "region": ["r_regionkey", "r_name"],
    "customer": ["c_custkey", "c_nationkey", "c_mktsegment"],
    "supplier": ["s_suppkey", "s_nationkey", "s_acctbal"],
    "part": ["p_partkey", "p_mfgr", "p_type", "p_size"],
    "partsupp": ["ps_partkey", "ps_suppkey", "ps_supplycost"],
    "orders": ["o_orderkey", "o_custkey", "o_orderdate", "o_shippriority", "o_orderpriority"],
    "lineitem": ["l_orderkey", "l_suppkey", "l_quantity", "l_extendedprice", "l_discount", "l_tax",
                 "l_returnflag", "l_linestatus", "l_shipdate", "l_commitdate", "l_receiptdate"],
    "calendar": ["d_datekey", "d_year"],  # datagen's date dimension (reading O34)
}
STRING_DICTS = {"n_name": "nation", "r_name": "region", "c_mktsegment": "mktsegment",
                "l_returnflag": "returnflag", "l_linestatus": "linestatus",
                "o_orderpriority": "orderpriority", "p_type": "type", "p_mfgr": "tpch_mfgr"}
QUERY_TABLES = {"tpch1": ["lineitem"], "tpch6": ["lineitem"],
                "tpch2": ["region", "nation", "supplier", "part", "partsupp"],
                "tpch3": ["customer", "orders", "lineitem"],
                "tpch4": ["orders", "lineitem"],
                "tpch7": ["nation", "supplier", "customer", "orders", "lineitem", "calendar"],
                "tpch5": ["region", "nation", "supplier", "customer", "orders", "lineitem"]}


def _bits(db, table: str, col: str) -> int:
    """Bits of a non-negative key column in a packed group key (from the column's
    load-time statistics: dense and sparse key encodings need different widths)."""
    if not hasattr(db, "column_stats"):  # host-only catalogue (finalisation tests)
        return 21
    n, lo, hi = db.column_stats(table, col)
    if lo < 0:
        raise ValueError(f"{table}.{col}: negative group key")
    return max(1, int(hi).bit_length())


def _rows(db, table: str) -> int:
    return db.table_rows(table) if hasattr(db, "table_rows") else 1 << 20


def load_tpch(db: Database, data, cache: bool = True, tables=None) -> None:
    """data: ``data.col(table, col)``, ``data.rows(table)``, ``data.dict_for(col)``."""
    for t in (tables or list(TABLE_COLUMNS)):
        cols = {c: data.col(t, c) for c in TABLE_COLUMNS[t]}
        db.create_table(t, len(next(iter(cols.values()))))
        for c, v in cols.items():
            db.load_column(t, c, v)
            if cache:
                db.cache(t, c)
    for c, d in STRING_DICTS.items():
        db.dicts[d] = data.dict_for(c)
        t = next(t for t, cols in TABLE_COLUMNS.items() if c in cols)
        if tables is None or t in tables:
            db.set_dictionary(t, c, db.dicts[d])  # decode result keys (S8(a7))


def tpch_plan(db: Database, q: str, limit: int = 0, dense: bool = True, fused_agg: bool = True) -> PlanBuilder:
    """dense (Q1): one AGGREGATE over every lineitem row with the shipdate predicate
    fused (agg_dense_small_kernel, reading O26); False: select -> TID list ->
    aggregate at the TIDs (the paper's operator granularity, kept under test).
    fused_agg: Q6's discount / quantity predicates evaluated inside the aggregation
    at the shipdate selection's TIDs (reading O26, as SSB flight 1), and Q5's supplier
    semi-join first with s_nationkey fetched late; False: the chains kept under test
    (two selections at TIDs; orders first)."""
    P = db.plan()
    li = "lineitem"
    if q == "tpch1":
        # l_shipdate <= date '1998-12-01' - interval '90' day  (= 19980902, O11)
        ship = [("l_shipdate", -2**31, 19980902)]
        t = -1 if dense else P.select(li, ship)
        P.aggregate(li, t, where=ship if dense else None, keys=["l_returnflag", "l_linestatus"],
                    aggs=[(A.AGG_SUM, ["l_quantity"]), (A.AGG_SUM, ["l_extendedprice"]),
                          (A.AGG_SUM_MUL_100M, ["l_extendedprice", "l_discount"]),
                          (A.AGG_SUM_MUL_100M_100P, ["l_extendedprice", "l_discount", "l_tax"]),
                          (A.AGG_SUM, ["l_discount"]), (A.AGG_COUNT, [])],
                    order_by=[1, 2], max_groups=6,
                    key_bits=[2, 1],  # dictionary codes: returnflag A/N/R, linestatus F/O
                    # avg_qty, avg_price, avg_disc = sum / count / 10^2 at finalisation (O10)
                    avg=[(0, 2), (1, 2), (4, 2)], avg_count=5)
        return P
    if q == "tpch6":
        # shipdate in 1994 (15 %) first; discount 0.05..0.07 and quantity < 24 at its TIDs
        t = P.select(li, [("l_shipdate", 19940101, 19941231)])
        rest = [("l_discount", 5, 7), ("l_quantity", -2**62, 2399)]
        aggs = [(A.AGG_SUM_MUL, ["l_extendedprice", "l_discount"]), (A.AGG_COUNT, [])]
        if fused_agg:  # fused into the aggregate (O26, as SSB flight 1)
            P.aggregate(li, t, keys=[], aggs=aggs, max_groups=1, where=rest)
            return P
        t = P.select(li, rest[:1], input=t)
        t = P.select(li, rest[1:], input=t)
        P.aggregate(li, t, keys=[], aggs=aggs, max_groups=1)
        return P
    if q == "tpch2":
        # The correlated scalar subquery ps_supplycost = (select min(ps_supplycost) ..
        # where p_partkey = ps_partkey ..) decorrelated (reading O35): the European
        # partsupp rows of the qualifying parts build a MIN-aggregating index
        # ps_partkey -> min cost, and the same rows keep those whose cost equals it.
        eu = code(db, "region", "EUROPE")
        r = P.select("region", [("r_name", [eu])])
        hr = P.build("region", "r_regionkey", input=r)
        n = P.probe("nation", "n_regionkey", hr)                          # nations of EUROPE
        hn = P.build("nation", "n_nationkey", "n_name", input=n)
        s = P.probe("supplier", "s_nationkey", hn)                        # European suppliers
        hsn = P.build("supplier", "s_suppkey", "s_nationkey", input=s)
        hsa = P.build("supplier", "s_suppkey", "s_acctbal", input=s)      # int64 payload, fits int32
        # p_size = 15 and p_type like '%BRASS' (a dictionary code set, ddq_dictionary_like)
        hp = P.build("part", "p_partkey", "p_mfgr", where=[("p_size", 15, 15), db.like("part", "p_type", "%BRASS")])
        ps = "partsupp"
        t = P.probe(ps, "ps_partkey", hp, emit=True)                      # vec0 = p_mfgr
        t = P.probe(ps, "ps_suppkey", hsn, input=t, emit=True)            # vec1 = s_nationkey
        hm = P.build(ps, "ps_partkey", "ps_supplycost", input=t, key_set="min")
        t = P.probe(ps, "ps_partkey", hm, input=t, emit=True)             # vec2 = the part's min cost
        t = P.gather(ps, "ps_supplycost", t, narrow=True)                 # vec3 = ps_supplycost
        t = P.filter_eq(ps, t, 2, 3)                                      # ps_supplycost = min
        t = P.probe(ps, 1, hn, input=t, emit=True)                        # vec4 = n_name
        t = P.fetch(ps, "ps_suppkey", hsa, t)                             # vec5 = s_acctbal
        # one row per (part, supplier): the select list's supplier / nation / part
        # attributes are functionally dependent -> MIN; order by s_acctbal desc,
        # n_name, s_name (= s_suppkey), p_partkey
        P.aggregate(ps, t, keys=["ps_partkey", "ps_suppkey"],
                    key_bits=[_bits(db, ps, "ps_partkey"), _bits(db, ps, "ps_suppkey")],
                    aggs=[(A.AGG_MIN, [5]), (A.AGG_MIN, [4]), (A.AGG_MIN, [0])],
                    order_by=[-101, 102, 2, 1], max_groups=max(1024, _rows(db, ps)), limit=limit)
        return P
    if q == "tpch3":
        c = P.select("customer", [("c_mktsegment", [code(db, "mktsegment", "BUILDING")])])
        hc = P.build("customer", "c_custkey", input=c)
        o = P.select("orders", [("o_orderdate", -2**31, 19950314)])        # < 1995-03-15
        o = P.probe("orders", "o_custkey", hc, input=o)
        hod = P.build("orders", "o_orderkey", "o_orderdate", input=o)
        hos = P.build("orders", "o_orderkey", "o_shippriority", input=o)
        t = P.select(li, [("l_shipdate", 19950316, 2**31 - 1)])            # > 1995-03-15
        t = P.probe(li, "l_orderkey", hod, input=t, emit=True)            # vec0 = o_orderdate
        t = P.probe(li, "l_orderkey", hos, input=t, emit=True)            # vec1 = o_shippriority
        # group by l_orderkey, o_orderdate, o_shippriority; order by revenue desc,
        # o_orderdate, then l_orderkey (O9)
        P.aggregate(li, t, keys=["l_orderkey", 0, 1],
                    key_bits=[_bits(db, li, "l_orderkey"), _bits(db, "orders", "o_orderdate"),
                              _bits(db, "orders", "o_shippriority")],
                    aggs=[(A.AGG_SUM_MUL_100M, ["l_extendedprice", "l_discount"])],
                    order_by=[-101, 2, 1], max_groups=1 << 22, limit=limit)
        return P
    if q == "tpch4":
        # EXISTS (lineitem of the order with l_commitdate < l_receiptdate) is a
        # semi-join: the late lineitems of the quarter's orders build a join index
        # over l_orderkey (duplicates collapse into one bit), the orders probe it.
        o = P.select("orders", [("o_orderdate", 19930701, 19930930)])    # [1993-07-01, 1993-10-01)
        ho = P.build("orders", "o_orderkey", input=o)
        t = P.probe(li, "l_orderkey", ho)                                # lineitems of those orders
        t = P.gather(li, "l_commitdate", t)                              # vec0
        t = P.gather(li, "l_receiptdate", t)                             # vec1
        t = P.filter_lt(li, t, 0, 1)                                     # l_commitdate < l_receiptdate
        hl = P.build(li, "l_orderkey", input=t, key_set=True)           # <= 4 lines per order
        o = P.probe("orders", "o_orderkey", hl, input=o)
        P.aggregate("orders", o, keys=["o_orderpriority"], aggs=[(A.AGG_COUNT, [])],
                    order_by=[1], max_groups=5, key_bits=[3])  # codes sorted == string order (O4)
        return P
    if q == "tpch5":
        r = P.select("region", [("r_name", [code(db, "region", "ASIA")])])
        hr = P.build("region", "r_regionkey", input=r)
        n = P.probe("nation", "n_regionkey", hr)                         # nations of ASIA
        hn = P.build("nation", "n_nationkey", "n_name", input=n)
        s = P.probe("supplier", "s_nationkey", hn)                       # suppliers in ASIA
        hs = P.build("supplier", "s_suppkey", "s_nationkey", input=s)
        hc = P.build("customer", "c_custkey", "c_nationkey")
        o = P.select("orders", [("o_orderdate", 19940101, 19941231)])
        ho = P.build("orders", "o_orderkey", "o_custkey", input=o)
        if fused_agg:
            # the ASIA suppliers' semi-join first (20 % of lineitem: a row bitmap, O27),
            # the 1994 orders probed masked by it, s_nationkey fetched late at the
            # survivors (join order and late materialisation, O23)
            t = P.probe(li, "l_suppkey", hs)                                 # semi-join
            t = P.probe(li, "l_orderkey", ho, input=t, emit=True)            # vec0 = o_custkey
            t = P.fetch(li, "l_suppkey", hs, input=t)                        # vec1 = s_nationkey
        else:
            t = P.probe(li, "l_orderkey", ho, emit=True)                     # vec0 = o_custkey
            t = P.probe(li, "l_suppkey", hs, input=t, emit=True)             # vec1 = s_nationkey
        t = P.probe(li, 0, hc, input=t, emit=True)                       # vec2 = c_nationkey
        t = P.filter_eq(li, t, 1, 2)                                     # c_nationkey = s_nationkey
        t = P.probe(li, 1, hn, input=t, emit=True)                       # vec3 = n_name
        P.aggregate(li, t, keys=[3], aggs=[(A.AGG_SUM_MUL_100M, ["l_extendedprice", "l_discount"])],
                    order_by=[-101, 1], max_groups=25)
        return P
    if q == "tpch7":
        n = P.select("nation", [("n_name", [code(db, "nation", "FRANCE"), code(db, "nation", "GERMANY")])])
        hn = P.build("nation", "n_nationkey", "n_name", input=n)
        s = P.probe("supplier", "s_nationkey", hn)
        hs = P.build("supplier", "s_suppkey", "s_nationkey", input=s)
        c = P.probe("customer", "c_nationkey", hn)
        hc = P.build("customer", "c_custkey", "c_nationkey", input=c)
        o = P.probe("orders", "o_custkey", hc)                           # orders of FR/DE customers
        ho = P.build("orders", "o_orderkey", "o_custkey", input=o)
        hy = P.build("calendar", "d_datekey", "d_year")
        t = P.select(li, [("l_shipdate", 19950101, 19961231)])
        t = P.probe(li, "l_suppkey", hs, input=t, emit=True)             # vec0 = s_nationkey
        t = P.probe(li, "l_orderkey", ho, input=t, emit=True)            # vec1 = o_custkey
        t = P.probe(li, 1, hc, input=t, emit=True)                       # vec2 = c_nationkey
        # (n1 = FRANCE and n2 = GERMANY) or (n1 = GERMANY and n2 = FRANCE), both
        # nations already restricted to {FRANCE, GERMANY}: s_nationkey != c_nationkey
        t = P.filter_eq(li, t, 0, 2, A.CMP_NE)
        t = P.probe(li, 0, hn, input=t, emit=True)                       # vec3 = supp_nation
        t = P.probe(li, 2, hn, input=t, emit=True)                       # vec4 = cust_nation
        t = P.fetch(li, "l_shipdate", hy, t)                             # vec5 = l_year
        P.aggregate(li, t, keys=[3, 4, 5], key_bits=[5, 5, 12],
                    aggs=[(A.AGG_SUM_MUL_100M, ["l_extendedprice", "l_discount"])],
                    order_by=[1, 2, 3], max_groups=64)
        return P
    raise KeyError(q)
