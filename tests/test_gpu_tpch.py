"""TPC-H Q1/Q3/Q4/Q5/Q6/Q7 parity (BASELINE config 4): libddq through the C ABI vs the
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


@pytest.mark.parametrize("q", ["tpch1", "tpch2", "tpch3", "tpch4", "tpch5", "tpch6", "tpch7"])
def test_tpch_prepared_equals_oracle(q):
    from paper_conf_sigmod_bressft16_b200.tpch import tpch_plan
    db = _db()
    p = db.prepare(tpch_plan(db, q))
    p.launch()
    got = p.fetch().rows
    p.close()
    assert got and got == _want(q)


@pytest.mark.parametrize("q", ["tpch5", "tpch6"])
@pytest.mark.parametrize("fused", [True, False])
def test_tpch_plan_forms_equal_oracle(q, fused):
    """Both plan forms = oracle, prepared and through the driver: Q6's discount /
    quantity predicates inside the aggregation (O26) or as two selections at TIDs;
    Q5's supplier semi-join first (a row bitmap) with s_nationkey fetched late, or
    orders first."""
    from paper_conf_sigmod_bressft16_b200.tpch import tpch_plan
    db = _db()
    p = db.prepare(tpch_plan(db, q, fused_agg=fused))
    p.launch()
    got = p.fetch().rows
    p.close()
    assert got == _want(q)
    assert db.run(tpch_plan(db, q, fused_agg=fused)).rows == _want(q)


@pytest.mark.parametrize("q", ["tpch1", "tpch2", "tpch3", "tpch4", "tpch5", "tpch6", "tpch7"])
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


@pytest.mark.parametrize("prefetch", [False, True])
def test_tpch_cold_path_gpu_only(prefetch):
    """Cold cache, GPU-only: columns copied on demand, or streamed from submit on the
    copy thread while earlier operators compute (prefetch, S8(f) N1) -- also with
    every query submitted at once (concurrent users, cached-first pulls)."""
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch, tpch_plan
    db = Database(cache_bytes=8 << 30, heap_bytes=4 << 30, placement=A.PLACE_GPU_ONLY, prefetch=prefetch)
    load_tpch(db, _data(), cache=False)
    for q in ("tpch1", "tpch6", "tpch5", "tpch4", "tpch7"):
        r = db.run(tpch_plan(db, q))
        assert r.rows == _want(q) and r.host_ops == 0
    for (t, c) in list(db._cols):
        db.evict(t, c)
    qs = {q: db.submit(tpch_plan(db, q)) for q in ("tpch1", "tpch2", "tpch3", "tpch4", "tpch5", "tpch6", "tpch7")}
    for q, h in qs.items():
        assert db.fetch(h).rows == _want(q), q
    st = db.stats()
    assert st["h2d_bytes"] > 0 and st["cache_misses"] > 0
    db.close()


def test_tpch1_unfused_variant():
    """select -> TID list -> aggregate (the operator-at-a-time plan) = the dense
    fused aggregation = the oracle."""
    from paper_conf_sigmod_bressft16_b200.tpch import tpch_plan
    db = _db()
    p = db.prepare(tpch_plan(db, "tpch1", dense=False))
    p.launch()
    got = p.fetch().rows
    p.close()
    assert got == _want("tpch1")


@pytest.mark.parametrize("shape", ["count_only", "no_pred", "wide_domain", "seven_cols", "in_pred"])
def test_dense_aggregate_shapes(shape):
    """AGGREGATE over all rows (no input): the dense small-domain kernel and the
    fallbacks (all-rows TID list, fused selection) vs numpy on the same columns."""
    import numpy as np
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    db, d = _db(), _data()
    li = "lineitem"
    P = db.plan()
    rf, ls = d.col(li, "l_returnflag").astype(np.int64), d.col(li, "l_linestatus").astype(np.int64)
    qty, ep = d.col(li, "l_quantity").astype(np.int64), d.col(li, "l_extendedprice").astype(np.int64)
    disc, tax = d.col(li, "l_discount").astype(np.int64), d.col(li, "l_tax").astype(np.int64)
    ship = d.col(li, "l_shipdate").astype(np.int64)
    keys, bits, where = ["l_returnflag", "l_linestatus"], [2, 1], [("l_shipdate", 19950101, 19961231)]
    mask = (ship >= 19950101) & (ship <= 19961231)
    aggs = [(A.AGG_SUM, ["l_quantity"]), (A.AGG_COUNT, [])]
    vals = [qty, np.ones_like(qty)]
    if shape == "count_only":
        aggs, vals = [(A.AGG_COUNT, [])], [np.ones_like(qty)]
    elif shape == "no_pred":
        where, mask = None, np.ones_like(mask)
    elif shape == "wide_domain":  # 21-bit keys: not a small domain -> generic kernels
        bits = None
    elif shape == "seven_cols":  # > 6 distinct argument columns -> generic kernels
        aggs = [(A.AGG_SUM, ["l_quantity"]), (A.AGG_SUM, ["l_extendedprice"]), (A.AGG_SUM, ["l_discount"]),
                (A.AGG_SUM, ["l_tax"]), (A.AGG_SUM, ["l_shipdate"]), (A.AGG_SUM, ["l_orderkey"]),
                (A.AGG_SUM, ["l_suppkey"])]
        vals = [qty, ep, disc, tax, ship, d.col(li, "l_orderkey").astype(np.int64),
                d.col(li, "l_suppkey").astype(np.int64)]
    elif shape == "in_pred":
        where = [("l_discount", [1, 4, 9])]
        mask = np.isin(disc, [1, 4, 9])
        aggs = [(A.AGG_SUM_MUL_100M_100P, ["l_extendedprice", "l_discount", "l_tax"]), (A.AGG_COUNT, [])]
        vals = [ep * (100 - disc) * (100 + tax), np.ones_like(qty)]
    P.aggregate(li, -1, keys=keys, key_bits=bits, aggs=aggs, where=where, order_by=[1, 2], max_groups=64)
    r = db.run(P)
    p = db.prepare(P)
    p.launch()
    got = p.fetch().rows
    p.close()
    assert r.rows == got
    want = []
    for a in sorted(set(zip(rf[mask].tolist(), ls[mask].tolist()))):
        m = mask & (rf == a[0]) & (ls == a[1])
        want.append(a + tuple(int(v[m].sum()) for v in vals))
    assert [tuple(x) for x in got] == want


@pytest.mark.parametrize("n", [1000, 200_003])
def test_dense_aggregate_int64_overflow_is_exact(n):
    """Per-thread int64 partials overflow (values near 2^62, both signs): the
    dense kernel spills into int128 cells, the group sums stay exact."""
    import numpy as np
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    rng = np.random.default_rng(n)
    g = rng.integers(0, 3, size=n).astype(np.int32)
    x = rng.integers((1 << 62) - 1000, (1 << 62), size=n, dtype=np.int64)
    x[rng.random(n) < 0.3] *= -1
    y = rng.integers(0, 50, size=n).astype(np.int64)
    db = Database(cache_bytes=1 << 30, heap_bytes=1 << 28)
    db.create_table("t", n)
    for name, col in (("g", g), ("x", x), ("y", y)):
        db.load_column("t", name, col)
        db.cache("t", name)
    P = db.plan()
    P.aggregate("t", -1, keys=["g"], key_bits=[2], aggs=[(A.AGG_SUM, ["x"]), (A.AGG_SUM, ["y"]), (A.AGG_COUNT, [])],
                order_by=[1], max_groups=4)
    p = db.prepare(P)
    p.launch()
    got = p.fetch().rows
    p.close()
    db.close()
    want = [(k, int(sum(int(v) for v in x[g == k])), int(y[g == k].sum()), int((g == k).sum()))
            for k in sorted(set(g.tolist()))]
    assert [tuple(r) for r in got] == want


@pytest.mark.parametrize("q", ["tpch4", "tpch7"])
def test_tpch_cpu_only_host_operators(q):
    """CPU-only placement: every operator of Q4 / Q7 (incl. FILTER_EQ with CMP_LT /
    CMP_NE, the lineitem-side semi-join build, the calendar fetch) runs in the
    host executor."""
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch, tpch_plan
    db = Database(cache_bytes=1 << 30, heap_bytes=1 << 30, placement=A.PLACE_CPU_ONLY)
    load_tpch(db, _data(), cache=False)
    r = db.run(tpch_plan(db, q))
    assert r.rows == _want(q) and r.host_ops > 0
    db.close()


@pytest.mark.parametrize("cmp", ["eq", "lt", "ne"])
def test_filter_compare_vectors_at_tids(cmp):
    """FILTER_EQ over two gathered int32 vectors (CMP_EQ / CMP_LT, negative values,
    ragged tail) vs numpy: the kept TIDs and a count aggregate at them."""
    import numpy as np
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    rng = np.random.default_rng(7)
    n = 300_001
    a = rng.integers(-50, 50, size=n).astype(np.int32)
    b = rng.integers(-50, 50, size=n).astype(np.int32)
    s = rng.integers(0, 10, size=n).astype(np.int32)
    g = rng.integers(0, 4, size=n).astype(np.int32)
    db = Database(cache_bytes=1 << 30, heap_bytes=1 << 28)
    db.create_table("t", n)
    for name, col in (("a", a), ("b", b), ("s", s), ("g", g)):
        db.load_column("t", name, col)
        db.cache("t", name)
    P = db.plan()
    t = P.select("t", [("s", 0, 6)])
    t = P.gather("t", "a", t)
    t = P.gather("t", "b", t)
    t = P.filter_eq("t", t, 0, 1, {"eq": A.CMP_EQ, "lt": A.CMP_LT, "ne": A.CMP_NE}[cmp])
    P.aggregate("t", t, keys=["g"], key_bits=[2], aggs=[(A.AGG_COUNT, []), (A.AGG_SUM, ["a"])],
                order_by=[1], max_groups=4)
    m = (s <= 6) & {"eq": a == b, "lt": a < b, "ne": a != b}[cmp]
    want = [(k, int((m & (g == k)).sum()), int(a[m & (g == k)].astype(np.int64).sum())) for k in range(4)]
    r = db.run(P)
    p = db.prepare(P)
    p.launch()
    got = p.fetch().rows
    p.close()
    db.close()
    assert [tuple(x) for x in got] == want and [tuple(x) for x in r.rows] == want


@pytest.mark.parametrize("sparse", [False, True])
def test_key_set_build_semi_join(sparse):
    """HASH_BUILD with key_set (reading O32): duplicate keys collapse; a probe is the
    semi-join `exists`.  Dense keys take the direct-mapped index, sparse keys
    (range > 16x rows) the open-addressing table; a plain build of the same
    duplicates is rejected."""
    import numpy as np
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    rng = np.random.default_rng(11)
    n, m = 200_003, 50_021
    mult = 30_011 if sparse else 1  # sparse: keys up to 1.8e9, range >> 16 x rows
    bk = (rng.integers(1, 40_000, size=n) * mult).astype(np.int32)   # many duplicates
    f = rng.integers(0, 3, size=n).astype(np.int32)
    pk = (rng.integers(1, 60_000, size=m) * mult).astype(np.int32)
    g = rng.integers(0, 4, size=m).astype(np.int32)
    db = Database(cache_bytes=1 << 30, heap_bytes=1 << 28)
    db.create_table("b", n)
    db.create_table("p", m)
    for t, name, col in (("b", "k", bk), ("b", "f", f), ("p", "k", pk), ("p", "g", g)):
        db.load_column(t, name, col)
        db.cache(t, name)
    P = db.plan()
    s = P.select("b", [("f", 0, 1)])
    h = P.build("b", "k", input=s, key_set=True)
    t = P.probe("p", "k", h)
    P.aggregate("p", t, keys=["g"], key_bits=[2], aggs=[(A.AGG_COUNT, [])], order_by=[1], max_groups=4)
    keys = set(bk[f <= 1].tolist())
    hit = np.array([k in keys for k in pk.tolist()])
    want = [(k, int((hit & (g == k)).sum())) for k in range(4)]
    p = db.prepare(P)
    p.launch()
    got = [tuple(x) for x in p.fetch().rows]
    p.close()
    assert got == want and [tuple(x) for x in db.run(P).rows] == want
    P2 = db.plan()
    P2.probe("p", "k", P2.build("b", "k"))
    with pytest.raises(A.DDQError):
        db.run(P2)
    db.close()


@pytest.mark.parametrize("shape", ["tids_vec_keys", "dense_col_keys", "fused_pred", "cpu_only"])
def test_aggregate_min(shape):
    """AGG_MIN (S8(a6)) next to SUM / COUNT: group minima of int64 values of both
    signs (and int32 arguments) vs numpy, at a TID list with vector keys, over all
    rows with column keys, with a fused selection, and in the host executor."""
    import numpy as np
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    rng = np.random.default_rng(5)
    n = 250_007
    g = rng.integers(0, 37, size=n).astype(np.int32)
    x = rng.integers(-(1 << 60), 1 << 60, size=n, dtype=np.int64)
    y = rng.integers(-1000, 1000, size=n).astype(np.int32)
    s = rng.integers(0, 10, size=n).astype(np.int32)
    kw = {"placement": A.PLACE_CPU_ONLY} if shape == "cpu_only" else {}
    db = Database(cache_bytes=1 << 30, heap_bytes=1 << 28, **kw)
    db.create_table("t", n)
    for name, col in (("g", g), ("x", x), ("y", y), ("s", s)):
        db.load_column("t", name, col)
        if shape != "cpu_only":
            db.cache("t", name)
    P = db.plan()
    aggs = [(A.AGG_MIN, ["x"]), (A.AGG_SUM, ["y"]), (A.AGG_MIN, ["y"]), (A.AGG_COUNT, [])]
    m = s <= 6
    if shape in ("tids_vec_keys", "cpu_only"):
        t = P.select("t", [("s", 0, 6)])
        t = P.gather("t", "g", t)
        P.aggregate("t", t, keys=[0], key_bits=[6], aggs=aggs, order_by=[1], max_groups=64)
    elif shape == "dense_col_keys":
        m = np.ones(n, dtype=bool)
        P.aggregate("t", -1, keys=["g"], key_bits=[6], aggs=aggs, order_by=[1], max_groups=64)
    else:
        P.aggregate("t", -1, keys=["g"], key_bits=[6], aggs=aggs, where=[("s", 0, 6)], order_by=[1],
                    max_groups=64)
    want = []
    for k in sorted(set(g[m].tolist())):
        mk = m & (g == k)
        want.append((k, int(x[mk].min()), int(y[mk].astype(np.int64).sum()), int(y[mk].min()), int(mk.sum())))
    r = db.run(P)
    assert [tuple(v) for v in r.rows] == want
    if shape != "cpu_only":
        p = db.prepare(P)
        p.launch()
        assert [tuple(v) for v in p.fetch().rows] == want
        p.close()
    db.close()


class _Ties:
    """TPC-H data with every ps_supplycost equal: each qualifying part's minimum is
    reached by ALL its European suppliers, so Q2 must return every such row (SQL
    `=` against the subquery's MIN, not an arg-min)."""

    def __init__(self, d):
        import numpy as np
        self.d = d
        self.cost = np.full(d.rows("partsupp"), 50000, np.int64)

    def col(self, t, c):
        return self.cost if (t, c) == ("partsupp", "ps_supplycost") else self.d.col(t, c)

    def rows(self, t):
        return self.d.rows(t)

    def dict_for(self, c):
        return self.d.dict_for(c)


@pytest.mark.parametrize("path", ["prepared", "submit", "host"])
def test_tpch2_min_ties(path):
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch, tpch_plan
    data = _Ties(_data())
    want = [tuple(r) for r in oracle.run(data, "tpch2")]
    assert len({r[0] for r in want}) < len(want)  # several suppliers per part tie
    db = Database(cache_bytes=4 << 30, heap_bytes=2 << 30,
                  **(dict(placement=A.PLACE_CPU_ONLY) if path == "host" else {}))
    load_tpch(db, data, tables=["region", "nation", "supplier", "part", "partsupp"])
    if path == "prepared":
        p = db.prepare(tpch_plan(db, "tpch2"))
        p.launch()
        got = p.fetch().rows
        p.close()
    else:
        got = db.run(tpch_plan(db, "tpch2")).rows
    db.close()
    assert got == want


def test_tpch2_limit100():
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch, tpch_plan
    data = datagen.TPCH(1)
    want = [tuple(r) for r in oracle.run(data, "tpch2")]
    assert len(want) > 100
    db = Database(cache_bytes=4 << 30, heap_bytes=2 << 30)
    load_tpch(db, data, tables=["region", "nation", "supplier", "part", "partsupp"])
    assert db.run(tpch_plan(db, "tpch2", limit=100)).rows == want[:100]
    db.close()


@pytest.mark.parametrize("index", ["join_index", "hash"])
def test_min_build_and_narrow_gather(index):
    """A MIN-aggregating build (build_key_set = 2) over duplicate keys, read back by a
    fetch at every row, equals numpy's per-key minimum; an int64 payload is narrowed
    exactly; a narrowing GATHER of a column whose values do not fit int32 is refused."""
    import numpy as np
    from paper_conf_sigmod_bressft16_b200 import Database, DDQError
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    rng = np.random.default_rng(11)
    n = 100_003
    nk = 997
    keys = rng.integers(0, nk, n).astype(np.int32)
    if index == "hash":  # a sparse key range: open addressing (reading O24)
        keys = (keys.astype(np.int64) * 1_000_003 + 7).astype(np.int32)
    vals = rng.integers(-2**31, 2**31 - 1, n).astype(np.int64)
    big = vals.copy()
    big[5] = 2**40
    db = Database(cache_bytes=1 << 30, heap_bytes=1 << 30)
    db.create_table("t", n)
    for c, v in (("k", keys), ("v", vals), ("big", big)):
        db.load_column("t", c, v)
        db.cache("t", c)
    P = db.plan()
    hm = P.build("t", "k", "v", key_set="min")
    t = P.select("t", [("k", -2**31, 2**31 - 1)])
    t = P.fetch("t", "k", hm, t)                      # vec0 = min of the row's key
    t = P.gather("t", "v", t, narrow=True)            # vec1 = own value
    t = P.filter_eq("t", t, 0, 1)                     # rows holding their key's minimum
    P.aggregate("t", t, keys=["k"], key_bits=[32], aggs=[(A.AGG_COUNT, []), (A.AGG_MIN, [1])], max_groups=4096)
    mins = {}
    for k, v in zip(keys.tolist(), vals.tolist()):
        mins[k] = min(mins.get(k, v), v)
    cnt = {}
    for k, v in zip(keys.tolist(), vals.tolist()):
        if v == mins[k]:
            cnt[k] = cnt.get(k, 0) + 1
    want = sorted((k & 0xFFFFFFFF, cnt[k], mins[k]) for k in cnt)
    for path in ("prepared", "submit"):
        if path == "prepared":
            p = db.prepare(P)
            p.launch()
            got = p.fetch().rows
            p.close()
        else:
            got = db.run(P).rows
        assert sorted(got) == want, path
    Q = db.plan()
    t = Q.select("t", [("k", -2**31, 2**31 - 1)])
    t = Q.gather("t", "big", t, narrow=True)
    Q.aggregate("t", t, keys=[], aggs=[(A.AGG_COUNT, [])], max_groups=1)
    with pytest.raises(DDQError):
        db.prepare(Q)
    db.close()
