"""Operator-level binding (include/ddq.h section 1) over torch CUDA tensors.

torch provides device memory and the current stream; every operator is one or
more libddq kernels.  Counts produced on the device stay there (uint32 cells) so
operator chains do not synchronise with the host.  No CPU fallback exists.
"""
from __future__ import annotations

import ctypes

import torch

from . import _abi as A
from ._abi import check, lib


def _stream() -> ctypes.c_void_p:
    return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)


def _ptr(t) -> int | None:
    return None if t is None else t.data_ptr()


def _require_cuda(*ts) -> None:
    for t in ts:
        if t is not None and not t.is_cuda:
            raise ValueError("libddq operators take CUDA tensors (no CPU fallback)")


def _ptr_array(ts):
    arr = (ctypes.c_void_p * max(1, len(ts)))(*[t.data_ptr() for t in ts])
    return arr


def count_cell(n: int | None = None) -> torch.Tensor:
    c = torch.zeros(16, dtype=torch.int32, device="cuda")
    if n is not None:
        c[0] = n
    return c


def _dev_preds(preds):
    """preds: list of (column tensor, lo, hi) or (column tensor, [values])."""
    arr = (A.DevPred * max(1, len(preds)))()
    for i, p in enumerate(preds):
        col = p[0]
        _require_cuda(col)
        arr[i].col = col.data_ptr()
        arr[i].width = col.element_size()
        if len(p) == 3:
            arr[i].kind, arr[i].lo, arr[i].hi = A.PRED_RANGE, int(p[1]), int(p[2])
        else:
            arr[i].kind, arr[i].n_in = A.PRED_IN, len(p[1])
            for j, v in enumerate(p[1]):
                arr[i].in_vals[j] = int(v)
    return arr


def select(preds, n: int, in_tids=None, in_count=None, carry=()):
    """Stable selection.  Returns (out_tids, count_cell, carried outputs)."""
    out = torch.empty(max(n, 1), dtype=torch.int32, device="cuda")
    cnt = count_cell()
    scratch = torch.empty(lib().ddq_op_scratch_bytes(n), dtype=torch.uint8, device="cuda")
    cout = [torch.empty(max(n, 1), dtype=torch.int32, device="cuda") for _ in carry]
    dp = _dev_preds(preds)
    check(lib().ddq_op_select(dp, len(preds), _ptr(in_tids), _ptr(in_count), n, _ptr_array(list(carry)),
                              _ptr_array(cout), len(carry), out.data_ptr(), cnt.data_ptr(),
                              scratch.data_ptr(), scratch.numel(), _stream()))
    return out, cnt, cout


def hash_build(keys, capacity: int, payload=None, in_tids=None, in_count=None, n: int | None = None):
    n = keys.numel() if n is None else n
    table = torch.empty(capacity, dtype=torch.int64, device="cuda")
    err = count_cell()
    check(lib().ddq_op_hash_init(table.data_ptr(), capacity, _stream()))
    check(lib().ddq_op_hash_build(keys.data_ptr(), _ptr(payload), _ptr(in_tids), _ptr(in_count), n,
                                  table.data_ptr(), capacity, err.data_ptr(), _stream()))
    return table, err


def hash_probe(table, fk, n: int, in_tids=None, in_count=None, carry=(), emit_payload: bool = False):
    out = torch.empty(max(n, 1), dtype=torch.int32, device="cuda")
    pay = torch.empty(max(n, 1), dtype=torch.int32, device="cuda") if emit_payload else None
    cnt = count_cell()
    scratch = torch.empty(lib().ddq_op_scratch_bytes(n), dtype=torch.uint8, device="cuda")
    cout = [torch.empty(max(n, 1), dtype=torch.int32, device="cuda") for _ in carry]
    check(lib().ddq_op_hash_probe(table.data_ptr(), table.numel(), fk.data_ptr(), _ptr(in_tids), _ptr(in_count),
                                  n, _ptr_array(list(carry)), _ptr_array(cout), len(carry), out.data_ptr(),
                                  _ptr(pay), cnt.data_ptr(), scratch.data_ptr(), scratch.numel(), _stream()))
    return out, pay, cnt, cout


def join_index_build(keys, key_min: int, key_range: int, payload=None, in_tids=None, in_count=None,
                     n: int | None = None):
    """Direct-mapped join index over [key_min, key_min + key_range)."""
    n = keys.numel() if n is None else n
    idx = torch.empty(lib().ddq_op_join_index_bytes(key_range), dtype=torch.uint8, device="cuda")
    err = count_cell()
    check(lib().ddq_op_join_index_init(idx.data_ptr(), key_range, _stream()))
    check(lib().ddq_op_join_index_build(keys.data_ptr(), _ptr(payload), _ptr(in_tids), _ptr(in_count), n, key_min,
                                        key_range, idx.data_ptr(), err.data_ptr(), _stream()))
    return idx, err


def join_index_probe(idx, key_min: int, key_range: int, fk, n: int, in_tids=None, in_count=None, carry=(),
                     emit_payload: bool = False):
    out = torch.empty(max(n, 1), dtype=torch.int32, device="cuda")
    pay = torch.empty(max(n, 1), dtype=torch.int32, device="cuda") if emit_payload else None
    cnt = count_cell()
    scratch = torch.empty(lib().ddq_op_scratch_bytes(n), dtype=torch.uint8, device="cuda")
    cout = [torch.empty(max(n, 1), dtype=torch.int32, device="cuda") for _ in carry]
    check(lib().ddq_op_join_index_probe(idx.data_ptr(), key_min, key_range, fk.data_ptr(), _ptr(in_tids),
                                        _ptr(in_count), n, _ptr_array(list(carry)), _ptr_array(cout), len(carry),
                                        out.data_ptr(), _ptr(pay), cnt.data_ptr(), scratch.data_ptr(),
                                        scratch.numel(), _stream()))
    return out, pay, cnt, cout


def gather(col, tids, count, n: int):
    out = torch.empty(max(n, 1), dtype=col.dtype, device="cuda")
    check(lib().ddq_op_gather(col.data_ptr(), col.element_size(), tids.data_ptr(), _ptr(count), n,
                              out.data_ptr(), _stream()))
    return out


def groupby(tids, count, n: int, key_vecs=(), key_cols=(), aggs=(), capacity: int = 1024, key_bits=None):
    """aggs: list of (kind, [arg column tensors]).  Returns (keys[g], accs[g, n_aggs, 2], g)."""
    nk = max(len(key_vecs), len(key_cols))
    kv = (ctypes.c_void_p * 3)(*[(key_vecs[k].data_ptr() if k < len(key_vecs) and key_vecs[k] is not None
                                  else None) for k in range(3)])
    kc = (ctypes.c_void_p * 3)(*[(key_cols[k].data_ptr() if k < len(key_cols) and key_cols[k] is not None
                                  else None) for k in range(3)])
    da = (A.DevAgg * max(1, len(aggs)))()
    for a, (kind, args) in enumerate(aggs):
        da[a].kind = kind
        for j, t in enumerate(args):
            da[a].arg[j] = t.data_ptr()
            da[a].width[j] = t.element_size()
    na = len(aggs)
    table = torch.empty(lib().ddq_op_groupby_table_bytes(capacity, na), dtype=torch.uint8, device="cuda")
    err = count_cell()
    check(lib().ddq_op_groupby_init(table.data_ptr(), capacity, na, _stream()))
    kb = (ctypes.c_int32 * 3)(*(list(key_bits or []) + [0, 0, 0])[:3])
    check(lib().ddq_op_groupby(tids.data_ptr(), _ptr(count), n, kv, kc, nk, kb, da, na, table.data_ptr(), capacity,
                               err.data_ptr(), _stream()))
    keys = torch.empty(capacity, dtype=torch.int64, device="cuda")
    accs = torch.empty(capacity * max(na, 1) * 2, dtype=torch.int64, device="cuda")
    g = count_cell()
    check(lib().ddq_op_groupby_compact(table.data_ptr(), capacity, na, keys.data_ptr(), accs.data_ptr(),
                                       g.data_ptr(), _stream()))
    ng = int(g[0].item())
    return keys[:ng], accs[:ng * na * 2].view(ng, na, 2), int(err[0].item())
