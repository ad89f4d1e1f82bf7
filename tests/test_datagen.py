"""Generator checks (SURVEY.md 8(c).5 "Generator"): determinism, shard
regeneration, dictionaries, FK integrity, value domains, selectivities."""
import numpy as np
import pytest

import datagen


def test_deterministic_and_thread_invariant():
    a = datagen.ssb_column("lo_revenue", 0.1, nthreads=1)
    b = datagen.ssb_column("lo_revenue", 0.1, nthreads=8)
    assert np.array_equal(a, b)
    c = datagen.ssb_column("lo_revenue", 0.1, seed=datagen.DEFAULT_SEED + 1)
    assert not np.array_equal(a, c)


@pytest.mark.parametrize("col", ["lo_custkey", "lo_orderdate", "lo_ordtotalprice", "lo_extendedprice"])
def test_row_range_regeneration_is_bit_identical(col):
    full = datagen.ssb_column(col, 0.1)
    n = full.size
    for b, e in [(0, 1), (3, 77777), (n // 3, n // 2 + 5), (n - 9, n)]:
        assert np.array_equal(datagen.ssb_column(col, 0.1, begin=b, end=e), full[b:e])


@pytest.mark.parametrize("name", list(datagen.DICTS))
def test_dictionaries_sorted_unique(name):
    d = datagen.dictionary(name)
    assert d == sorted(d, key=lambda s: s.encode())
    assert len(set(d)) == len(d)


def test_dictionary_sizes():
    assert [len(datagen.dictionary(n)) for n in ("nation", "region", "city", "mfgr", "category", "brand1",
                                                  "yearmonth")] == [25, 5, 250, 5, 25, 1000, 84]


def test_string_codes_consistent():
    db = datagen.SSB(0.1)
    nat, reg, city = datagen.dictionary("nation"), datagen.dictionary("region"), datagen.dictionary("city")
    region_of = {  # TPC-H nation -> region
        "ALGERIA": "AFRICA", "ETHIOPIA": "AFRICA", "KENYA": "AFRICA", "MOROCCO": "AFRICA",
        "MOZAMBIQUE": "AFRICA", "ARGENTINA": "AMERICA", "BRAZIL": "AMERICA", "CANADA": "AMERICA",
        "PERU": "AMERICA", "UNITED STATES": "AMERICA", "INDIA": "ASIA", "INDONESIA": "ASIA",
        "JAPAN": "ASIA", "CHINA": "ASIA", "VIETNAM": "ASIA", "FRANCE": "EUROPE", "GERMANY": "EUROPE",
        "ROMANIA": "EUROPE", "RUSSIA": "EUROPE", "UNITED KINGDOM": "EUROPE", "EGYPT": "MIDDLE EAST",
        "IRAN": "MIDDLE EAST", "IRAQ": "MIDDLE EAST", "JORDAN": "MIDDLE EAST", "SAUDI ARABIA": "MIDDLE EAST"}
    for p in ("c", "s"):
        for cc, nn, rr in zip(db[p + "_city"][:5000], db[p + "_nation"][:5000], db[p + "_region"][:5000]):
            assert city[cc][:9] == nat[nn][:9].ljust(9)
            assert reg[rr] == region_of[nat[nn]]
    brand, cat, mfgr = datagen.dictionary("brand1"), datagen.dictionary("category"), datagen.dictionary("mfgr")
    for b, c, m in zip(db["p_brand1"][:5000], db["p_category"][:5000], db["p_mfgr"][:5000]):
        assert brand[b].startswith(cat[c]) and cat[c].startswith(mfgr[m])
        assert 1 <= int(brand[b][len(cat[c]):]) <= 40


def test_date_table():
    db = datagen.SSB(1)
    dk = db["d_datekey"]
    assert dk.size == 2557 and dk[0] == 19920101 and dk[-1] == 19981231
    assert np.all(np.diff(dk) > 0)
    assert np.array_equal(db["d_year"], dk // 10000)
    assert np.array_equal(db["d_yearmonthnum"], dk // 100)
    ym = datagen.dictionary("yearmonth")
    months = ["Jan", "Feb", "Mar", "Apr", "May", "Jun", "Jul", "Aug", "Sep", "Oct", "Nov", "Dec"]
    for i in range(0, 2557, 37):
        assert ym[db["d_yearmonth"][i]] == months[dk[i] // 100 % 100 - 1] + str(dk[i] // 10000)
    # day-of-year restarts each January 1st; week = (doy-1)//7+1 (reading O12)
    doy = db["d_daynuminyear"]
    assert np.all(doy[dk % 10000 == 101] == 1) and doy.max() == 366
    assert np.array_equal(db["d_weeknuminyear"], (doy - 1) // 7 + 1)


def test_fk_integrity_and_domains():
    sf = 0.5
    db = datagen.SSB(sf)
    n = db.rows("lineorder")
    assert n == 3_000_000
    for fk, t in [("lo_custkey", "customer"), ("lo_suppkey", "supplier"), ("lo_partkey", "part")]:
        assert db[fk].min() >= 1 and db[fk].max() <= db.rows(t)
    assert np.all(np.isin(db["lo_orderdate"], db["d_datekey"]))
    assert db["lo_orderdate"].max() <= 19980802
    assert db["lo_quantity"].min() == 1 and db["lo_quantity"].max() == 50
    assert db["lo_discount"].min() == 0 and db["lo_discount"].max() == 10
    assert db["lo_tax"].min() == 0 and db["lo_tax"].max() == 8
    assert np.all(db["lo_shippriority"] == 0)
    # lines of an order share custkey and orderdate (4 lines per order, reading O2)
    assert np.all(db["lo_custkey"].reshape(-1, 4) == db["lo_custkey"][::4, None])
    assert np.all(db["lo_orderdate"].reshape(-1, 4) == db["lo_orderdate"][::4, None])


def test_selectivities_within_binomial_bounds():
    db = datagen.SSB(1)
    n = db.rows("lineorder")
    checks = [
        (np.mean((db["lo_discount"] >= 1) & (db["lo_discount"] <= 3)), 3 / 11),
        (np.mean(db["lo_quantity"] < 25), 24 / 50),
        (np.mean((db["lo_orderdate"] >= 19930101) & (db["lo_orderdate"] <= 19931231)), 365 / 2406),
        (np.mean(datagen.ssb_column("c_region", 1) == 2), 1 / 5),
    ]
    for got, p in checks:
        sigma = (p * (1 - p) / n) ** 0.5
        assert abs(got - p) < 6 * max(sigma, (p * (1 - p) / 30000) ** 0.5)


def test_sizes():
    assert datagen.ssb_rows("lineorder", 20) == 120_000_000
    assert datagen.ssb_rows("part", 20) == 1_000_000
    assert datagen.ssb_rows("part", 100) == 1_400_000
    assert datagen.ssb_rows("customer", 100) == 3_000_000
    assert datagen.ssb_rows("part", 0.001) == 200
    assert datagen.tpch_rows("lineitem", 30) == 180_000_000


def test_tpch_domains():
    db = datagen.TPCH(0.05)
    sd, rd, od = db.col("lineitem", "l_shipdate"), db.col("lineitem", "l_receiptdate"), db.col("orders", "o_orderdate")
    ok = db.col("lineitem", "l_orderkey")
    assert np.all(sd > od[ok - 1]) and np.all(rd > sd)
    rf = np.array(datagen.dictionary("returnflag"))[db.col("lineitem", "l_returnflag")]
    assert np.all((rf == "N") == (rd > 19950617))
    ls = np.array(datagen.dictionary("linestatus"))[db.col("lineitem", "l_linestatus")]
    assert np.all((ls == "O") == (sd > 19950617))
    q = db.col("lineitem", "l_quantity")
    assert q.min() == 100 and q.max() == 5000 and np.all(q % 100 == 0)
    nat = datagen.dictionary("nation")
    names = np.array(nat)[db.col("nation", "n_name")]
    assert names[24] == "UNITED STATES" and names[18] == "CHINA" and names[0] == "ALGERIA"


# ---- sparse key encoding ("the kernels must not assume dense keys")
SSB_KEYS = [("c_custkey", "lo_custkey"), ("s_suppkey", "lo_suppkey"), ("p_partkey", "lo_partkey")]
TPCH_KEYS = [(("customer", "c_custkey"), ("orders", "o_custkey")), (("orders", "o_orderkey"), ("lineitem", "l_orderkey")),
             (("supplier", "s_suppkey"), ("lineitem", "l_suppkey")), (("part", "p_partkey"), ("lineitem", "l_partkey"))]


def _takes_hash_path(keys: np.ndarray) -> bool:
    """DESIGN.md reading O24: a build key column gets the direct-mapped join index iff
    its range is <= 2^20 values or <= 16x the rows; sparse keys must exceed both."""
    rng = int(keys.max()) - int(keys.min()) + 1
    return rng > (1 << 20) and rng > 16 * keys.size


@pytest.mark.parametrize("sf", [0.01, 1.0])
def test_sparse_ssb_keys(sf):
    sp, de = datagen.SSB(sf, keys="sparse"), datagen.SSB(sf)
    for pk, fk in SSB_KEYS:
        k = sp[pk]
        assert np.unique(k).size == k.size and k.min() >= 1 and k.max() < 2**31
        assert _takes_hash_path(k), pk
        # the FK maps through the same bijection as the PK: row r of the dense FK
        # (a key 1..n) becomes the sparse key of dimension row r - 1
        assert np.array_equal(sp[fk], k[de[fk] - 1])
    for c in ("lo_revenue", "lo_extendedprice", "lo_supplycost", "lo_orderdate", "c_nation", "p_brand1"):
        assert np.array_equal(sp[c], de[c]), c  # measures and attributes unchanged


def test_sparse_tpch_keys():
    sp, de = datagen.TPCH(0.1, keys="sparse"), datagen.TPCH(0.1)
    for (pt, pk), (ft, fk) in TPCH_KEYS:
        k = sp.col(pt, pk)
        assert np.unique(k).size == k.size and _takes_hash_path(k), pk
        assert np.array_equal(sp.col(ft, fk), k[de.col(ft, fk) - 1]), fk
    assert np.array_equal(sp.col("lineitem", "l_extendedprice"), de.col("lineitem", "l_extendedprice"))
