"""Cold-path transfer encoding (transfer.cu): a column cached
from its frame-of-reference bit-packed pinned copy is bit-identical to the raw
column, for bit lengths 1..32 (every byte boundary and odd lengths), negative bases,
widths 4 and 8, ragged lengths, and columns that stay raw (range >= 2^32); the bytes
sent are the packed stream's."""
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
    width = v.dtype.itemsize
    bits = max(1, (int(v.max()) - int(v.min())).bit_length())
    if bits <= 32 and bits < 8 * width:  # the packed stream (+ <= 63 bytes of padding) went over the link
        assert moved == (n * bits + 7) // 8 // 16 * 16 + 48
    else:
        assert moved == n * width


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
