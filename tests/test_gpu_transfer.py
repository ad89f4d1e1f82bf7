"""Cold-path transfer encoding (transfer.cu): a column cached
from its frame-of-reference bit-packed pinned copy is bit-identical to the raw
column, for bit lengths 1..32 (every byte boundary and odd lengths), negative bases,
widths 4 and 8, ragged lengths, and columns that stay raw (range >= 2^32); the bytes
sent are the packed stream's; columns with few distinct values in a wide range go
as ranks into a sorted dictionary when that is smaller (dates)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


class _Dev:  # zero-copy view of a library-owned device buffer
    def __init__(self, ptr, n, typestr):
        self.__cuda_array_interface__ = {"data": (ptr, False), "shape": (n,), "typestr": typestr, "version": 3}


def _roundtrip(values: np.ndarray, packing: bool = True):
    import torch
    from paper_conf_sigmod_bressft16_b200 import Database
    db = Database(cache_bytes=1 << 30, heap_bytes=1 << 28, transfer_packing=packing)
    db.create_table("t", len(values))
    db.load_column("t", "c", values)
    db.reset_stats()
    db.cache("t", "c")
    st = db.stats()
    ptr = db.device_ptr("t", "c")
    typestr = "<i4" if values.dtype == np.int32 else "<i8"
    got = torch.as_tensor(_Dev(ptr, len(values), typestr), device="cuda").cpu().numpy().copy() if len(values) else \
        np.empty(0, values.dtype)
    db.close()
    return got, st["h2d_bytes"]


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 7, 8, 9, 1023, 4097, 1_000_003])
@pytest.mark.parametrize("span,base,dtype", [
    (1, 0, np.int32), (10, 0, np.int32), (49, 1, np.int64), (255, -7, np.int32), (256, 19920101, np.int32),
    (60701, 19920101, np.int32), (65535, -(1 << 31), np.int32), (65536, 5, np.int64),
    (599_999, 1, np.int32), ((1 << 24) - 1, -3, np.int64), (1 << 24, 1 << 40, np.int64),
    ((1 << 31) + 12345, 7, np.int64), ((1 << 32) - 1, -(1 << 62), np.int64), (1 << 32, 0, np.int64)])
def test_packed_cache_roundtrip(n, span, base, dtype):
    rng = np.random.default_rng(n * 7919 + span)
    v = (base + rng.integers(0, span + 1, size=n, dtype=np.int64)).astype(dtype)
    if n >= 2:  # both ends of the range present
        v[0], v[-1] = base, base + span
    got, moved = _roundtrip(v)
    assert got.dtype == v.dtype and np.array_equal(got, v)
    assert moved == _expected_moved(v)


def _packed(n, bits):  # the packed stream's bytes (+ <= 63 bytes of padding)
    return (n * bits + 7) // 8 // 16 * 16 + 48


def _expected_moved(v):
    """Bytes over the link: the raw column, the range code (value - vmin in the
    range's bit length), or -- when smaller -- the dictionary code (ranks of the
    distinct values in their bit length, plus the 8-byte sorted dictionary; value
    ranges < 2^24)."""
    n, width = len(v), v.dtype.itemsize
    span = int(v.max()) - int(v.min())
    bits = max(1, span.bit_length())
    if not (bits <= 32 and bits < 8 * width):
        return n * width
    best = _packed(n, bits)
    if span < (1 << 24):
        d = len(np.unique(v))
        dbits = max(1, (d - 1).bit_length())
        if _packed(n, dbits) + 8 * d < best:
            best = _packed(n, dbits) + 8 * d
    return best


@pytest.mark.parametrize("dtype", [np.int32, np.int64])
@pytest.mark.parametrize("n", [5000, 1_000_003])
def test_dictionary_transfer_code(n, dtype):
    """yyyymmdd dates (2556 distinct days over a 69 129-wide range): 12-bit ranks into
    a sorted dictionary instead of a 17-bit range code, bit-identical after the cache;
    and a sparse domain (every 1000th value of 10^7) likewise."""
    import datetime
    days = np.array([int((datetime.date(1992, 1, 1) + datetime.timedelta(d)).strftime("%Y%m%d"))
                     for d in range(2556)], dtype=np.int64)
    rng = np.random.default_rng(n)
    for dom in (days, np.arange(0, 10_000_000, 1000, dtype=np.int64)):
        v = dom[rng.integers(0, len(dom), size=n)].astype(dtype)
        v[0], v[-1] = dom[0], dom[-1]
        got, moved = _roundtrip(v)
        assert np.array_equal(got, v)
        d = len(np.unique(v))
        if n > 100_000:  # large enough that the dictionary pays
            assert moved == _packed(n, max(1, (d - 1).bit_length())) + 8 * d
        assert moved == _expected_moved(v)


def test_packing_off_sends_raw():
    v = np.arange(100_000, dtype=np.int64)
    got, moved = _roundtrip(v, packing=False)
    assert np.array_equal(got, v) and moved == v.nbytes


def test_ssb_cold_packed_equals_raw_equals_oracle():
    import datagen
    import oracle
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES, load_ssb, ssb_plan
    data = datagen.SSB(0.05)
    moved = {}
    for packing in (True, False):
        db = Database(cache_bytes=4 << 30, heap_bytes=1 << 30, placement=A.PLACE_GPU_ONLY,
                      transfer_packing=packing)
        load_ssb(db, data, cache=False)
        for q in SSB_QUERIES:
            r = db.run(ssb_plan(db, q))
            want = [tuple(x) for x in oracle.run(data, q)]
            assert r.rows == want and r.host_ops == 0, (q, packing)
        moved[packing] = db.stats()["h2d_bytes"]
        db.close()
    assert moved[True] < 0.6 * moved[False]
