"""Operator-level parity of the sm_100a kernels against library routines on
seeded random inputs (SURVEY.md 4.2 "Unit (GPU)"): select vs numpy.flatnonzero,
build/probe vs numpy.isin + a dict, gather vs numpy.take, group-by vs numpy.unique
with exact Python-int sums.  Sizes span several 4096-row tiles plus ragged tails,
and the edge cases n = 0, 1, 31, 32, 33, all-pass and none-pass."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

SIZES = [0, 1, 31, 32, 33, 4095, 4096, 4097, 100_003, 3_000_017]


def _t(a):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()



def tile_order(tids, *vecs, check_tiles=True):
    """Scans emit their survivors as a multiset (reading O14': the order
    of a TID list is unspecified; every consumer is order-free).  Over an input
    without repeated rows no row may appear twice: check that, then return
    everything sorted by TID (vectors permuted alike) for comparison."""
    tids = np.asarray(tids)
    if tids.size and check_tiles:
        assert np.unique(tids).size == tids.size, "a row was emitted twice"
    order = np.argsort(tids, kind="stable")
    return (tids[order],) + tuple(np.asarray(v)[order] for v in vecs)


@pytest.fixture(scope="module")
def ops():
    from paper_conf_sigmod_bressft16_b200 import ops
    return ops


@pytest.mark.parametrize("n", SIZES)
def test_select_dense_int64_range(ops, n):
    rng = np.random.default_rng(n)
    a = rng.integers(0, 11, n, dtype=np.int64)
    b = rng.integers(1, 51, n, dtype=np.int64)
    tids, cnt, _ = ops.select([(_t(a), 4, 6), (_t(b), 26, 35)], n)
    want = np.flatnonzero((a >= 4) & (a <= 6) & (b >= 26) & (b <= 35))
    c = int(cnt[0].item())
    assert c == want.size
    assert np.array_equal(tile_order(tids[:c].cpu().numpy())[0], want)


@pytest.mark.parametrize("n", [0, 5, 4097, 1_000_001])
def test_select_int32_in_set_and_all_none(ops, n):
    rng = np.random.default_rng(7 + n)
    a = rng.integers(0, 250, n, dtype=np.int32)
    tids, cnt, _ = ops.select([(_t(a), [3, 17, 249, 0])], n)
    want = np.flatnonzero(np.isin(a, [3, 17, 249, 0]))
    c = int(cnt[0].item())
    assert np.array_equal(tile_order(tids[:c].cpu().numpy())[0], want)
    _, cnt_all, _ = ops.select([(_t(a), -1, 1000)], n)
    _, cnt_none, _ = ops.select([(_t(a), 1000, 2000)], n)
    assert int(cnt_all[0].item()) == n and int(cnt_none[0].item()) == 0


@pytest.mark.parametrize("n", [0, 33, 4097, 777_777])
def test_select_at_tids_with_carry(ops, n):
    import torch
    rng = np.random.default_rng(11 + n)
    N = max(n * 3, 1)
    col = rng.integers(0, 100, N, dtype=np.int64)
    tids_in = np.sort(rng.choice(N, size=n, replace=False)).astype(np.int32)
    carry = rng.integers(-5, 5, n, dtype=np.int32)
    cnt_in = ops.count_cell(n)
    out, cnt, couts = ops.select([(_t(col), 10, 40)], n, in_tids=_t(tids_in) if n else
                                 torch.empty(1, dtype=torch.int32, device="cuda"), in_count=cnt_in,
                                 carry=[_t(carry) if n else torch.empty(1, dtype=torch.int32, device="cuda")])
    keep = (col[tids_in] >= 10) & (col[tids_in] <= 40)
    c = int(cnt[0].item())
    assert c == int(keep.sum())
    o, cv = tile_order(out[:c].cpu().numpy(), couts[0][:c].cpu().numpy(), check_tiles=False)
    assert np.array_equal(o, tids_in[keep])
    assert np.array_equal(cv, carry[keep])


@pytest.mark.parametrize("ndim,nfact", [(2557, 4097), (40_000, 1_000_003), (600_000, 3_000_000), (1, 100)])
def test_build_probe_semijoin_payload(ops, ndim, nfact):
    rng = np.random.default_rng(ndim)
    keys = rng.permutation(np.arange(1, 3 * ndim + 1, dtype=np.int32))[:ndim]  # sparse unique keys
    payload = rng.integers(0, 1000, ndim, dtype=np.int32)
    sel = np.flatnonzero(rng.random(ndim) < 0.3).astype(np.int32)
    cap = 16
    while cap < 2 * max(sel.size, 1):
        cap *= 2
    table, err = ops.hash_build(_t(keys), cap, payload=_t(payload), in_tids=_t(sel) if sel.size else None,
                                in_count=ops.count_cell(sel.size) if sel.size else None, n=sel.size)
    assert int(err[0].item()) == 0
    fk = rng.integers(1, 3 * ndim + 1, nfact, dtype=np.int32)
    out, pay, cnt, _ = ops.hash_probe(table, _t(fk), nfact, emit_payload=True)
    m = dict(zip(keys[sel].tolist(), payload[sel].tolist()))
    want = np.flatnonzero(np.isin(fk, keys[sel]))
    c = int(cnt[0].item())
    assert c == want.size
    o, p = tile_order(out[:c].cpu().numpy(), pay[:c].cpu().numpy())
    assert np.array_equal(o, want)
    assert p.tolist() == [m[int(k)] for k in fk[want]]


@pytest.mark.parametrize("ndim,nfact,smem", [(2557, 4097, True), (40_000, 1_000_003, True),
                                             (1_000_000, 3_000_000, False), (1, 100, True)])
def test_join_index_semijoin_payload(ops, ndim, nfact, smem):
    """Direct-mapped join index: dense probe (bitmap staged in smem when <= 96 KB)
    and the same probe at a TID list, vs numpy.isin + a dict."""
    rng = np.random.default_rng(ndim + 1)
    kmin = 1000
    keys = (kmin + rng.permutation(ndim)).astype(np.int32)          # unique keys in the range
    payload = rng.integers(0, 1 << 20, ndim, dtype=np.int32)
    sel = np.flatnonzero(rng.random(ndim) < 0.2).astype(np.int32)
    idx, err = ops.join_index_build(_t(keys), kmin, ndim, payload=_t(payload),
                                    in_tids=_t(sel) if sel.size else None,
                                    in_count=ops.count_cell(sel.size) if sel.size else None, n=sel.size)
    assert int(err[0].item()) == 0
    assert (((ndim + 31) // 32) * 4 <= 96 * 1024) == smem
    fk = rng.integers(kmin - 50, kmin + ndim + 50, nfact, dtype=np.int32)  # includes out-of-range keys
    m = dict(zip(keys[sel].tolist(), payload[sel].tolist()))
    want = np.flatnonzero(np.isin(fk, keys[sel]))
    out, pay, cnt, _ = ops.join_index_probe(idx, kmin, ndim, _t(fk), nfact, emit_payload=True)
    c = int(cnt[0].item())
    o, p = tile_order(out[:c].cpu().numpy(), pay[:c].cpu().numpy())
    assert np.array_equal(o, want)
    assert p.tolist() == [m[int(k)] for k in fk[want]]
    # at TIDs (every other row), carrying a vector
    tin = np.arange(0, nfact, 2, dtype=np.int32)
    carry = (tin * 3).astype(np.int32)
    out2, pay2, cnt2, cv = ops.join_index_probe(idx, kmin, ndim, _t(fk), tin.size, in_tids=_t(tin),
                                                in_count=ops.count_cell(tin.size), carry=[_t(carry)],
                                                emit_payload=True)
    c2 = int(cnt2[0].item())
    keep = np.isin(fk[tin], keys[sel])
    o2, c2v, p2 = tile_order(out2[:c2].cpu().numpy(), cv[0][:c2].cpu().numpy(), pay2[:c2].cpu().numpy(),
                             check_tiles=False)
    assert np.array_equal(o2, tin[keep])
    assert np.array_equal(c2v, carry[keep])
    assert p2.tolist() == [m[int(k)] for k in fk[tin[keep]]]


def test_join_index_rejects_duplicates_and_out_of_range(ops):
    _, err = ops.join_index_build(_t(np.array([5, 9, 5], dtype=np.int32)), 0, 16)
    assert int(err[0].item()) == 1
    _, err = ops.join_index_build(_t(np.array([5, 99], dtype=np.int32)), 0, 16)
    assert int(err[0].item()) == 3


@pytest.mark.parametrize("keys", [
    [3, 4, 3], [7] * 32, list(range(40)) + [17], [1, 2, 33, 34, 1], list(range(0, 64, 2)) + [62],
    [5] + list(range(100, 131)) + [5]])
def test_join_index_warp_build_detects_duplicates(ops, keys):
    """Duplicate build keys are reported wherever they sit: adjacent rows, far
    apart in one warp, across warps."""
    _, err = ops.join_index_build(_t(np.array(keys, dtype=np.int32)), 0, 256)
    assert int(err[0].item()) == 1


@pytest.mark.parametrize("keys", [[0, 40, 1, 2], [0, 64, 1, 65, 2, 66], [3, 100, 4, 101, 5] * 1 + [200, 6]])
def test_join_index_warp_build_interleaved_words_no_false_duplicates(ops, keys):
    """Unique keys whose bitmap words interleave inside a warp (separate runs of one
    word): no duplicate reported, every key present."""
    idx, err = ops.join_index_build(_t(np.array(keys, dtype=np.int32)), 0, 256)
    assert int(err[0].item()) == 0
    bits = np.unpackbits(idx[:32].cpu().numpy().view(np.uint8), bitorder="little")[:256].astype(bool)
    assert np.flatnonzero(bits).tolist() == sorted(keys)


@pytest.mark.parametrize("n_keys,order", [(3_000_000, "sorted"), (3_000_000, "random"), (1_600_000, "sorted"),
                                          (20_000_000, "sorted")])
def test_join_index_bitmaps_and_coarse_bits(ops, n_keys, order):
    """Membership bitmap, payloads and (range > 1.5 M) the coarse bitmap of a build
    over a selected subset of keys (sorted rows: one atomic per word; random order)
    equal numpy's; no false errors."""
    rng = np.random.default_rng(n_keys)
    rows = np.arange(n_keys, dtype=np.int32)
    keys = rows + 1 if order == "sorted" else (rng.permutation(n_keys) + 1).astype(np.int32)
    sel = np.flatnonzero(rng.random(n_keys) < 0.3).astype(np.int32)
    payload = (rows * 7).astype(np.int32)
    idx, err = ops.join_index_build(_t(keys), 1, n_keys, payload=_t(payload), in_tids=_t(sel),
                                    in_count=ops.count_cell(sel.size), n=sel.size)
    assert int(err[0].item()) == 0
    raw = idx.cpu().numpy()
    fine_bytes = ((n_keys + 31) // 32 * 4 + 15) // 16 * 16
    member = np.zeros(n_keys, dtype=bool)
    member[keys[sel] - 1] = True
    bits = np.unpackbits(raw[:fine_bytes].view(np.uint8), bitorder="little")[:n_keys].astype(bool)
    assert np.array_equal(bits, member)
    pay = raw[fine_bytes:fine_bytes + n_keys * 4].view(np.int32)
    assert np.array_equal(pay[keys[sel] - 1], payload[sel])
    coarse_off = fine_bytes + (n_keys * 4 + 15) // 16 * 16
    if n_keys <= 1_500_000:
        assert raw.size == coarse_off
        return
    cg = 1
    while (((n_keys >> cg) + 1 + 31) // 32 * 4 + 15) // 16 * 16 > 160 * 1024:
        cg += 1
    if cg > 3:  # too coarse to filter: no coarse bitmap
        assert raw.size == coarse_off
        return
    ncb = (n_keys >> cg) + 1
    want = np.zeros(ncb, dtype=bool)
    want[np.flatnonzero(member) >> cg] = True
    got = np.unpackbits(raw[coarse_off:].view(np.uint8), bitorder="little")[:ncb].astype(bool)
    assert np.array_equal(got, want)


def test_build_rejects_duplicate_keys(ops):
    keys = np.array([5, 9, 5, 1], dtype=np.int32)
    _, err = ops.hash_build(_t(keys), 16)
    assert int(err[0].item()) == 1


def test_probe_chain_at_tids_carries_payload(ops):
    rng = np.random.default_rng(3)
    n = 200_000
    fk1 = rng.integers(1, 1001, n, dtype=np.int32)
    fk2 = rng.integers(1, 101, n, dtype=np.int32)
    t1, _ = ops.hash_build(_t(np.arange(1, 501, dtype=np.int32)), 1024,
                           payload=_t(np.arange(1, 501, dtype=np.int32) * 7))
    t2, _ = ops.hash_build(_t(np.arange(1, 101, 3, dtype=np.int32)), 128)
    o1, p1, c1, _ = ops.hash_probe(t1, _t(fk1), n, emit_payload=True)
    n1 = int(c1[0].item())
    o2, _, c2, carried = ops.hash_probe(t2, _t(fk2), n1, in_tids=o1, in_count=c1, carry=[p1])
    n2 = int(c2[0].item())
    m = (fk1 <= 500) & np.isin(fk2, np.arange(1, 101, 3))
    want = np.flatnonzero(m)
    o, cv = tile_order(o2[:n2].cpu().numpy(), carried[0][:n2].cpu().numpy(), check_tiles=False)
    assert np.array_equal(o, want)
    assert np.array_equal(cv, fk1[want] * 7)


@pytest.mark.parametrize("dtype", [np.int32, np.int64])
def test_gather(ops, dtype):
    rng = np.random.default_rng(5)
    col = rng.integers(-2**30, 2**30, 1_000_003).astype(dtype)
    tids = np.sort(rng.choice(col.size, 123_457, replace=False)).astype(np.int32)
    out = ops.gather(_t(col), _t(tids), ops.count_cell(tids.size), tids.size)
    assert np.array_equal(out[:tids.size].cpu().numpy(), col[tids])


def _acc_to_int(accs):
    a = accs.cpu().numpy()
    lo = a[..., 0].astype(np.uint64).astype(object)
    hi = a[..., 1].astype(object)
    return hi * (1 << 64) + lo


@pytest.mark.parametrize("ngroups,n", [(1, 1_000_000), (7, 33), (800, 2_000_003), (50_000, 1_500_000)])
def test_groupby_exact(ops, ngroups, n):
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    rng = np.random.default_rng(ngroups)
    N = n + 1000
    tids = np.sort(rng.choice(N, n, replace=False)).astype(np.int32)
    k0 = rng.integers(0, ngroups, n, dtype=np.int32)             # aligned vector key
    kc = rng.integers(0, 3, N, dtype=np.int32)                   # column key at tid
    ep = rng.integers(90_000 * 1, 209_900 * 50, N, dtype=np.int64)
    d = rng.integers(0, 11, N, dtype=np.int64)
    t = rng.integers(0, 9, N, dtype=np.int64)
    sc = rng.integers(0, 10**7, N, dtype=np.int64) * 3
    aggs = [(A.AGG_SUM_MUL, [_t(ep), _t(d)]), (A.AGG_COUNT, []), (A.AGG_SUM_SUB, [_t(d), _t(sc)]),
            (A.AGG_SUM_MUL_100M_100P, [_t(ep), _t(d), _t(t)]), (A.AGG_SUM_MUL_100M, [_t(ep), _t(d)]),
            (A.AGG_SUM, [_t(sc)])]
    cap = 64
    while cap < 2 * ngroups * 3:
        cap *= 2
    keys, accs, err = ops.groupby(_t(tids), ops.count_cell(n), n, key_vecs=[_t(k0), None],
                                  key_cols=[None, _t(kc)], aggs=aggs, capacity=cap)
    assert err == 0
    keys = keys.cpu().numpy()
    got = _acc_to_int(accs)
    r = tids
    key = k0.astype(np.int64) | (kc[r].astype(np.int64) << 21)
    vals = [ep[r].astype(object) * d[r], np.ones(n, dtype=object), d[r].astype(object) - sc[r],
            ep[r].astype(object) * (100 - d[r]) * (100 + t[r]), ep[r].astype(object) * (100 - d[r]),
            sc[r].astype(object)]
    uk = np.unique(key)
    assert sorted(keys.tolist()) == uk.tolist()
    pos = {int(k): i for i, k in enumerate(keys)}
    for a, v in enumerate(vals):
        want = {}
        for kk, vv in zip(key.tolist(), v.tolist()):
            want[kk] = want.get(kk, 0) + vv
        for kk, vv in want.items():
            assert got[pos[kk], a] == vv, (a, kk)


@pytest.mark.parametrize("nkeys", [0, 1])
def test_groupby_few_groups_int128_exact(ops, nkeys):
    """Register-accumulating few-group kernel: per-thread int64 partial sums that
    would overflow must spill exactly into the int128 table."""
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    rng = np.random.default_rng(9)
    n = 300_000
    big = rng.integers(2**60, 2**62, n, dtype=np.int64) * rng.choice([-1, 1], n)
    tids = np.arange(n, dtype=np.int32)
    k = rng.integers(0, 3, n, dtype=np.int32)
    keys, accs, err = ops.groupby(_t(tids), ops.count_cell(n), n, key_vecs=[_t(k)] if nkeys else [],
                                  aggs=[(A.AGG_SUM, [_t(big)]), (A.AGG_COUNT, [])], capacity=64)
    assert err == 0
    got = _acc_to_int(accs)
    keys = keys.cpu().numpy()
    for i, kk in enumerate(keys):
        m = (k == kk) if nkeys else np.ones(n, bool)
        assert got[i, 0] == sum(int(x) for x in big[m])
        assert got[i, 1] == int(m.sum())


@pytest.mark.parametrize("n", [1, 517, 2_000_003])
@pytest.mark.parametrize("bits", [(1,), (2, 1), (3, 2, 1)])
def test_groupby_small_domain_exact(ops, n, bits):
    """Dictionary-coded keys with sum(key_bits) <= 6: the small-domain kernel
    (thread-private int64 partials in smem, overflow spills to int128) must give
    the exact per-group sums, only for groups that occur (tids: every 3rd row)."""
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    rng = np.random.default_rng(n + len(bits))
    N = 3 * n + 7
    tids = np.arange(0, 3 * n, 3, dtype=np.int32)
    nk = len(bits)
    codes = [rng.integers(0, max(1, (1 << b) - 1), N if k else n, dtype=np.int32) for k, b in enumerate(bits)]
    big = rng.integers(2**61, 2**62, N, dtype=np.int64) * rng.choice([-1, 1], N)
    ep = rng.integers(1, 10**7, N, dtype=np.int64)
    d = rng.integers(0, 11, N, dtype=np.int64)
    t = rng.integers(0, 9, N, dtype=np.int64)
    aggs = [(A.AGG_SUM, [_t(big)]), (A.AGG_COUNT, []), (A.AGG_SUM_MUL_100M_100P, [_t(ep), _t(d), _t(t)])]
    keys, accs, err = ops.groupby(_t(tids), ops.count_cell(n), n, key_vecs=[_t(codes[0])] + [None] * (nk - 1),
                                  key_cols=[None] + [_t(c) for c in codes[1:]], aggs=aggs, capacity=128,
                                  key_bits=list(bits))
    assert err == 0
    r = tids
    key = codes[0].astype(np.int64)
    sh = bits[0]
    for k in range(1, nk):
        key = key | (codes[k][r].astype(np.int64) << sh)
        sh += bits[k]
    got = _acc_to_int(accs)
    keys = keys.cpu().numpy()
    assert sorted(keys.tolist()) == sorted(set(key.tolist()))
    vals = [big[r].astype(object), np.ones(n, dtype=object), ep[r].astype(object) * (100 - d[r]) * (100 + t[r])]
    for i, kk in enumerate(keys):
        m = key == kk
        for a, v in enumerate(vals):
            assert got[i, a] == sum(v[m]), (kk, a)


def test_groupby_overflow_flagged(ops):
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    n = 10_000
    tids = np.arange(n, dtype=np.int32)
    k = np.arange(n, dtype=np.int32)
    _, _, err = ops.groupby(_t(tids), ops.count_cell(n), n, key_vecs=[_t(k)],
                            aggs=[(A.AGG_COUNT, [])], capacity=1024)
    assert err == 2
