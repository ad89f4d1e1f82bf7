"""Python binding of the libddq database layer (include/ddq.h section 2).

Argument marshalling only: plans are built here as C structs, every operator runs
in libddq (sm_100a kernels or the C++ host executor the driver falls back to on an
aborted GPU operator).  Names follow the paper: data cache + heap,
data-driven placement, query chopping, Algorithm 1.
"""
from __future__ import annotations

import ctypes
import weakref
from dataclasses import dataclass, field

import numpy as np

from . import _abi as A
from ._abi import check, lib


@dataclass
class QueryResult:
    """Rows (keys..., aggregates...) as Python ints (None = SQL NULL, reading O7), in
    ORDER BY order, or TIDs.  avgs: per row the AVG columns (reading O10); decoded:
    rows with dictionary-coded keys replaced by their strings (S8(a7))."""
    rows: list = field(default_factory=list)
    tids: np.ndarray | None = None
    avgs: list = field(default_factory=list)
    decoded: list = field(default_factory=list)
    placement: list = field(default_factory=list)  # per plan op: A.RAN_GPU / RAN_HOST / RAN_ABORTED
    op_ms: list = field(default_factory=list)      # per plan op: wall ms (driver results)
    n_keys: int = 0
    n_aggs: int = 0
    gpu_ops: int = 0
    host_ops: int = 0
    aborts: int = 0
    exec_ms: float = 0.0


def _convert(res_ptr) -> QueryResult:
    r = res_ptr.contents
    out = QueryResult(n_keys=r.n_keys, n_aggs=r.n_aggs, gpu_ops=r.gpu_ops, host_ops=r.host_ops,
                      aborts=r.aborts, exec_ms=r.exec_ms)
    if r.n_tids > 0 or (r.n_rows == 0 and r.n_keys == 0 and r.n_aggs == 0):
        out.tids = np.ctypeslib.as_array(r.tids, shape=(r.n_tids,)).copy() if r.n_tids else \
            np.empty(0, np.int32)
    nk, na = r.n_keys, r.n_aggs
    if r.op_place:
        out.placement = [int(r.op_place[i]) for i in range(r.n_ops)]
    if r.op_ms:
        out.op_ms = [float(r.op_ms[i]) for i in range(r.n_ops)]
    n = r.n_rows
    # whole-array slices of the ctypes pointers (one C-level copy each; indexing the
    # pointer element by element cost ~2 us per value: 26 ms for TPC-H Q2's 14 K rows)
    keys = r.keys[:n * nk] if n * nk else []
    aggs = r.aggs[:n * na * 2] if n * na else []
    nul = r.agg_null[:n * na] if (r.agg_null and n * na) else None
    avgs = r.avgs[:n * r.n_avg] if r.n_avg > 0 and n else None
    kstr = r.key_str[:n * nk] if (r.key_str and n * nk) else None
    for i in range(n):
        vals = keys[i * nk:(i + 1) * nk]
        for a in range(na):
            j = i * na + a
            if nul is not None and nul[j]:
                vals.append(None)
                continue
            vals.append((aggs[2 * j + 1] << 64) | (aggs[2 * j] & 0xFFFFFFFFFFFFFFFF))
        out.rows.append(tuple(vals))
        if avgs is not None:
            out.avgs.append(tuple(float(x) for x in avgs[i * r.n_avg:(i + 1) * r.n_avg]))
        if kstr is not None:
            ks = kstr[i * nk:(i + 1) * nk]
            out.decoded.append(tuple(ks[k].decode() if ks[k] is not None else vals[k] for k in range(nk))
                               + tuple(vals[nk:]))
    lib().ddq_result_free(res_ptr)
    return out


class PlanBuilder:
    """Builds a ddq_plan (operator DAG, children before parents; last op = root)."""

    def __init__(self, db: "Database"):
        self.db = db
        self.plan = A.Plan()
        self.n = 0

    def _op(self, kind: int, table: str, input: int = -1) -> tuple[int, A.Op]:
        if self.n >= A.MAX_OPS:
            raise ValueError("plan too long")
        op = self.plan.ops[self.n]
        ctypes.memset(ctypes.addressof(op), 0, ctypes.sizeof(op))
        op.kind = kind
        op.input = input
        op.table = self.db.table_id(table)
        op.build = -1
        op.payload_col = -1
        op.fk_col = -1
        op.key_col = -1
        op.gather_col = -1
        idx = self.n
        self.n += 1
        self.plan.n_ops = self.n
        return idx, op

    def select(self, table: str, preds: list, input: int = -1) -> int:
        """preds: list of (column, lo, hi) ranges or (column, [values]) IN-sets."""
        idx, op = self._op(A.OP_SELECT, table, input)
        self._preds(op, table, preds)
        return idx

    def _preds(self, op, table: str, preds: list):
        if len(preds) > A.MAX_PREDS:
            raise ValueError("too many predicates")
        op.n_preds = len(preds)
        for i, p in enumerate(preds):
            pr = op.preds[i]
            if isinstance(p, A.Pred):  # a predicate built by the library (Database.like)
                ctypes.memmove(ctypes.byref(pr), ctypes.byref(p), ctypes.sizeof(A.Pred))
                continue
            pr.column = self.db.col(table, p[0])
            if len(p) == 3:
                pr.kind, pr.lo, pr.hi = A.PRED_RANGE, int(p[1]), int(p[2])
            else:
                vals = list(p[1])
                if not 1 <= len(vals) <= A.MAX_IN:
                    raise ValueError("IN list must have 1..8 values")
                pr.kind, pr.n_in = A.PRED_IN, len(vals)
                for j, v in enumerate(vals):
                    pr.in_vals[j] = int(v)

    def build(self, table: str, key: str, payload: str | None = None, input: int = -1,
              where: list | None = None, key_set: bool | str = False) -> int:
        """where: predicates evaluated on the input rows inside the build (a fused
        selection: no intermediate TID list), same forms as select().  key_set:
        True = the key set of a semi-join (EXISTS / IN), duplicate keys allowed
        (reading O32); "min" = duplicate keys keep the smallest payload (a
        decorrelated MIN subquery, reading O35)."""
        idx, op = self._op(A.OP_HASH_BUILD, table, input)
        op.build_key_set = 2 if key_set == "min" else 1 if key_set else 0
        op.key_col = self.db.col(table, key)
        op.payload_col = self.db.col(table, payload) if payload else -1
        if where:
            self._preds(op, table, where)
        return idx

    def probe(self, table: str, fk, build: int, input: int = -1, emit: bool = False) -> int:
        """fk: a column of `table`, or an int = index of an aligned input vector."""
        idx, op = self._op(A.OP_HASH_PROBE, table, input)
        if isinstance(fk, int):
            op.fk_vec = fk + 1
        else:
            op.fk_col = self.db.col(table, fk)
        op.build = build
        op.emit_payload = 1 if emit else 0
        return idx

    def star(self, table: str, terms: list) -> int:
        """n-ary semi-join over all rows of `table` in one pass.  terms (evaluated in
        order, most selective first): ("pred", (col, lo, hi)) | ("pred", (col, [vals]))
        | ("probe", fk_col, build_op, emit).  Emitted payloads become aligned vectors
        in term order -- the same output as the equivalent SELECT/HASH_PROBE chain."""
        idx, op = self._op(A.OP_STAR, table, -1)
        if not 1 <= len(terms) <= 4:
            raise ValueError("STAR takes 1..4 terms")
        op.n_terms = len(terms)
        for j, term in enumerate(terms):
            if term[0] == "pred":
                p = term[1]
                pr = op.preds[j]
                pr.column = self.db.col(table, p[0])
                if len(p) == 3:
                    pr.kind, pr.lo, pr.hi = A.PRED_RANGE, int(p[1]), int(p[2])
                else:
                    pr.kind, pr.n_in = A.PRED_IN, len(p[1])
                    for i, v in enumerate(p[1]):
                        pr.in_vals[i] = int(v)
                op.term_kind[j] = A.TERM_PRED
            else:
                _, fk, build, emit = term
                op.term_kind[j] = A.TERM_PROBE
                op.term_fk[j] = self.db.col(table, fk)
                op.term_build[j] = build
                op.term_emit[j] = 1 if emit else 0
        op.n_preds = 0
        return idx

    def filter_eq(self, table: str, input: int, vec_a: int, vec_b: int, cmp: int = A.CMP_EQ) -> int:
        """Keep rows whose aligned vectors satisfy vec_a == vec_b (cmp=CMP_EQ) or
        vec_a < vec_b (cmp=CMP_LT)."""
        idx, op = self._op(A.OP_FILTER_EQ, table, input)
        op.eq_vec[0], op.eq_vec[1] = vec_a + 1, vec_b + 1
        op.eq_cmp = cmp
        return idx

    def filter_lt(self, table: str, input: int, vec_a: int, vec_b: int) -> int:
        """Keep rows whose aligned vectors satisfy vec_a < vec_b (column-column
        comparison, e.g. TPC-H Q4's l_commitdate < l_receiptdate)."""
        return self.filter_eq(table, input, vec_a, vec_b, A.CMP_LT)

    def gather(self, table: str, col: str, input: int, narrow: bool = False) -> int:
        """narrow: an int64 column whose values fit int32 becomes an int32 vector."""
        idx, op = self._op(A.OP_GATHER, table, input)
        op.gather_col = self.db.col(table, col)
        op.gather_narrow = 1 if narrow else 0
        return idx

    def fetch(self, table: str, fk: str, build: int, input: int) -> int:
        """Dimension attribute fetch (a GATHER through a join): appends the payload of
        `build` matched by fk[r] for every input row r as an aligned vector (late
        materialisation after a semi-join probe of the same build)."""
        idx, op = self._op(A.OP_GATHER, table, input)
        op.gather_col = self.db.col(table, fk)
        op.fetch_build = build + 1
        return idx

    def aggregate(self, table: str, input: int, keys: list, aggs: list, order_by: list | None = None,
                  max_groups: int = 0, limit: int = 0, key_bits: list | None = None,
                  where: list | None = None, avg: list | None = None, avg_count: int = -1,
                  terms: list | None = None) -> int:
        """keys: int (aligned vector index) or str (column of `table`).
        aggs: (kind, [cols]).  order_by: ints per include/ddq.h (+/-(1+k), +/-(101+a)).
        key_bits: bits per key in the packed group key (default 21 each, sum <= 63).
        where: predicates on the input rows evaluated inside the aggregation (a fused
        selection, reading O26), same forms as select().
        terms: fused probe / fetch terms evaluated at the input rows after `where`
        (reading O37): ("probe", fk_col, build_op, emit) | ("fetch", fk_col, build_op);
        emitted payloads are numbered after the input's aligned vectors."""
        idx, op = self._op(A.OP_AGGREGATE, table, input)
        if where:
            self._preds(op, table, where)
        terms = terms or []
        if len(terms) > 4:
            raise ValueError("at most 4 aggregate terms")
        op.n_terms = len(terms)
        for j, t in enumerate(terms):
            op.term_kind[j] = A.TERM_FETCH if t[0] == "fetch" else A.TERM_PROBE
            op.term_fk[j] = self.db.col(table, t[1])
            op.term_build[j] = t[2]
            op.term_emit[j] = 1 if (t[0] == "fetch" or t[3]) else 0
        for k, b in enumerate(key_bits or []):
            op.key_bits[k] = b
        op.n_keys = len(keys)
        for k, src in enumerate(keys):
            op.key_src[k] = src if isinstance(src, int) else -2 - self.db.col(table, src)
        op.n_aggs = len(aggs)
        for a, (kind, cols) in enumerate(aggs):
            op.agg_kind[a] = kind
            for j in range(3):  # an int operand = aligned vector index (MIN only): -2 - v
                c = cols[j] if j < len(cols) else None
                op.agg_col[a][j] = -1 if c is None else (-2 - c if isinstance(c, int) else self.db.col(table, c))
        order_by = order_by or []
        op.n_order = len(order_by)
        for i, o in enumerate(order_by):
            op.order_by[i] = o
        op.max_groups = max_groups
        op.limit = limit
        # AVG columns computed at finalisation: (index of the SUM aggregate, decimal scale)
        # over the COUNT aggregate avg_count (reading O10)
        avg = avg or []
        if len(avg) > 4:
            raise ValueError("at most 4 AVG columns")
        op.n_avg = len(avg)
        op.avg_count = avg_count
        for k, (a, scale) in enumerate(avg):
            op.avg_sum[k], op.avg_scale[k] = a, scale
        return idx


def nccl_unique_id() -> bytes:
    """128-byte NCCL unique id (rank 0 creates it; the bootstrap sends it to the others)."""
    buf = ctypes.create_string_buffer(128)
    check(lib().ddq_dist_nccl_unique_id(buf))
    return buf.raw


def finalize_partials(root: A.Op, keys: np.ndarray, accs: np.ndarray) -> QueryResult:
    """Host finalisation of (possibly duplicated) partial groups: exact merge of equal
    packed keys, ORDER BY / LIMIT of the root AGGREGATE (no GPU needed)."""
    keys = np.ascontiguousarray(keys, np.int64)
    accs = np.ascontiguousarray(accs, np.int64)
    p = ctypes.POINTER(A.Result)()
    check(lib().ddq_finalize_partials(ctypes.byref(root), keys.size, keys.ctypes.data, accs.ctypes.data,
                                      ctypes.byref(p)))
    return _convert(p)


class Catalog:
    """Name -> id catalogue without a device (plans for host-only finalisation)."""

    def __init__(self, dicts: dict[str, list[str]], rows: dict[str, int] | None = None):
        self.dicts = dicts
        self._ids: dict = {}
        self._rows = rows or {}  # table sizes the plans' join orders depend on (reading O30)

    def table_rows(self, table: str) -> int:
        return self._rows.get(table, 0)

    def _id(self, key) -> int:
        return self._ids.setdefault(key, len(self._ids))

    def table_id(self, table: str) -> int:
        return self._id(("t", table))

    def col(self, table: str, name: str) -> int:
        return self._id(("c", table, name))

    def plan(self) -> "PlanBuilder":
        return PlanBuilder(self)


class Prepared:
    """A plan placed entirely on the GPU and captured into one CUDA graph."""

    def __init__(self, db: "Database", plan: A.Plan, use_graph: bool = True):
        self.db = db
        self.h = None
        h = ctypes.c_void_p()
        check(lib().ddq_prepare(db.h, ctypes.byref(plan), 1 if use_graph else 0, ctypes.byref(h)))
        self.h = h
        self.kernels = lib().ddq_prepared_kernel_count(h)
        db._prepared.add(self)

    def launch(self, stream: int = 0) -> None:
        check(lib().ddq_prepared_launch(self.h, ctypes.c_void_p(stream)))

    def fetch(self, stream: int = 0) -> QueryResult:
        p = ctypes.POINTER(A.Result)()
        check(lib().ddq_prepared_fetch(self.h, ctypes.c_void_p(stream), ctypes.byref(p)))
        return _convert(p)

    def profile(self, stream: int = 0):
        """Per-operator (ms, algorithmic bytes, class) from an event-timed replay."""
        n = 64
        ms = (ctypes.c_float * n)()
        by = (ctypes.c_double * n)()
        cl = (ctypes.c_int32 * n)()
        k = lib().ddq_prepared_profile(self.h, ctypes.c_void_p(stream), n, ms, by, cl)
        if k < 0:
            check(k)
        return [(float(ms[i]), float(by[i]), int(cl[i])) for i in range(k)]

    def partials(self, stream: int = 0):
        """Compacted partial group table (keys int64[g], accs int64[g, n_aggs, 2])."""
        cap = lib().ddq_prepared_group_capacity(self.h)
        keys = np.empty(max(cap, 1), np.int64)
        na = self.db._root_aggs.get(id(self), 1)
        accs = np.empty(max(cap, 1) * 16, np.int64)
        g = ctypes.c_int64()
        check(lib().ddq_prepared_partials(self.h, ctypes.c_void_p(stream), ctypes.byref(g),
                                          keys.ctypes.data, accs.ctypes.data, cap))
        return keys[:g.value], accs[:g.value * na * 2].reshape(g.value, na, 2)

    def partials_device(self):
        """(keys_ptr, accs_ptr, count_ptr, capacity) of the device partial table."""
        k, a, c = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_void_p()
        cap = ctypes.c_int64()
        check(lib().ddq_prepared_partials_device(self.h, ctypes.byref(k), ctypes.byref(a), ctypes.byref(c),
                                                 ctypes.byref(cap)))
        return k.value, a.value, c.value, cap.value

    def finalize(self, keys: np.ndarray, accs: np.ndarray) -> QueryResult:
        keys = np.ascontiguousarray(keys, np.int64)
        accs = np.ascontiguousarray(accs, np.int64)
        p = ctypes.POINTER(A.Result)()
        check(lib().ddq_prepared_finalize(self.h, keys.size, keys.ctypes.data, accs.ctypes.data, ctypes.byref(p)))
        return _convert(p)

    def close(self) -> None:
        # a prepared plan belongs to its database: freed before it (Database.close)
        if self.h and self.db.h:
            lib().ddq_prepared_free(self.h)
        self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Database:
    """A libddq database on one GPU: pinned host columns + device cache + heap."""

    def __init__(self, device: int = 0, cache_bytes: int = 64 << 30, heap_bytes: int = 32 << 30,
                 gpu_workers: int = 4, host_workers: int = 4, placement: int = A.PLACE_DATA_DRIVEN,
                 chopping: bool = True, cache_policy: int = 0, fault_alloc_every: int = 0,
                 rank: int = 0, world: int = 1, transfer_packing: bool = True, fault_op_mask: int = 0,
                 max_queries: int = 0, prefetch: bool = False, placement_period_ms: int = 0,
                 _handle: int | None = None):
        cfg = A.Config()
        lib().ddq_config_default(ctypes.byref(cfg))
        cfg.device, cfg.rank, cfg.world = device, rank, world
        cfg.cache_bytes, cfg.heap_bytes = cache_bytes, heap_bytes
        cfg.gpu_workers, cfg.host_workers = gpu_workers, host_workers
        cfg.placement, cfg.chopping = placement, 1 if chopping else 0
        cfg.cache_policy, cfg.fault_alloc_every = cache_policy, fault_alloc_every
        cfg.transfer_packing = 1 if transfer_packing else 0
        cfg.fault_op_mask = fault_op_mask
        cfg.max_queries = max_queries
        cfg.prefetch = 1 if prefetch else 0
        cfg.placement_period_ms = placement_period_ms
        self._owner = _handle is None
        if _handle is None:
            h = ctypes.c_void_p()
            check(lib().ddq_open(ctypes.byref(cfg), ctypes.byref(h)))
        else:  # a member of a Cluster (owned by the cluster)
            h = ctypes.c_void_p(_handle)
        self.h = h
        self._tables: dict[str, int] = {}
        self._rows: dict[str, int] = {}
        self._cols: dict[tuple[str, str], int] = {}
        self.dicts: dict[str, list[str]] = {}
        self._root_aggs: dict = {}
        self._prepared = weakref.WeakSet()

    def close(self) -> None:
        if self.h:
            for p in list(self._prepared):  # prepared plans hold cache references and heap blocks
                p.close()
            if self._owner:
                lib().ddq_close(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ---- catalog -------------------------------------------------------------
    def create_table(self, name: str, n_rows: int, row_begin: int = 0) -> int:
        t = ctypes.c_int32()
        check(lib().ddq_create_table(self.h, name.encode(), n_rows, row_begin, ctypes.byref(t)))
        self._tables[name] = t.value
        self._rows[name] = n_rows
        return t.value

    def table_rows(self, table: str) -> int:
        """Rows of `table` in this process (a shard's rows for row-sharded tables)."""
        return self._rows[table]

    def load_column(self, table: str, name: str, data: np.ndarray) -> int:
        data = np.ascontiguousarray(data)
        if data.dtype == np.int32:
            ty = A.I32
        elif data.dtype == np.int64:
            ty = A.I64
        else:
            raise TypeError("columns are int32 or int64")
        c = ctypes.c_int32()
        check(lib().ddq_load_column(self.h, self._tables[table], name.encode(), ty, data.ctypes.data,
                                    data.size, ctypes.byref(c)))
        self._cols[(table, name)] = c.value
        return c.value

    def column_stats(self, table: str, name: str) -> tuple[int, int, int]:
        """(rows, min, max) of a loaded column (recorded by the library at load)."""
        n, lo, hi = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        check(lib().ddq_column_stats(self.h, self.col(table, name), ctypes.byref(n), ctypes.byref(lo),
                                     ctypes.byref(hi)))
        return n.value, lo.value, hi.value

    def set_dictionary(self, table: str, name: str, strings: list[str]) -> None:
        """Order-preserving dictionary of a string column (codes = ranks, reading O4)."""
        enc = [x.encode() for x in strings]
        arr = (ctypes.c_char_p * max(len(enc), 1))(*enc)
        check(lib().ddq_set_dictionary(self.h, self.col(table, name), arr, len(enc)))

    def dictionary_range(self, table: str, name: str, s: str) -> tuple[int, int]:
        """[lower, upper) codes of string s in the column's dictionary."""
        lo, hi = ctypes.c_int32(), ctypes.c_int32()
        check(lib().ddq_dictionary_range(self.h, self.col(table, name), s.encode(), ctypes.byref(lo),
                                         ctypes.byref(hi)))
        return lo.value, hi.value

    def like(self, table: str, name: str, pattern: str) -> A.Pred:
        """SQL `name LIKE pattern` folded over the dictionary into a code predicate."""
        pr = A.Pred()
        check(lib().ddq_dictionary_like(self.h, self.col(table, name), pattern.encode(), ctypes.byref(pr)))
        return pr

    def table_id(self, table: str) -> int:
        return self._tables[table]

    def col(self, table: str, name: str) -> int:
        return self._cols[(table, name)]

    def has_col(self, table: str, name: str) -> bool:
        return (table, name) in self._cols

    def cache(self, table: str, name: str) -> None:
        check(lib().ddq_cache_column(self.h, self.col(table, name)))

    def evict(self, table: str, name: str) -> None:
        check(lib().ddq_evict_column(self.h, self.col(table, name)))

    def is_cached(self, table: str, name: str) -> bool:
        return bool(lib().ddq_column_is_cached(self.h, self.col(table, name)))

    def device_ptr(self, table: str, name: str) -> int:
        return lib().ddq_column_device_ptr(self.h, self.col(table, name)) or 0

    def access_count(self, table: str, name: str) -> int:
        return int(lib().ddq_column_access_count(self.h, self.col(table, name)))

    def update_placement(self) -> None:
        """Algorithm 1."""
        check(lib().ddq_update_placement(self.h))

    def reset_access_counts(self) -> None:
        check(lib().ddq_reset_access_counts(self.h))

    # ---- multi-GPU (include/ddq.h "multi-GPU"; S8(e)) -----------------------
    def set_partitioned(self, table: str, partitioned: bool = True) -> None:
        check(lib().ddq_table_set_partitioned(self.h, self._tables[table], 1 if partitioned else 0))

    def dist_init_nccl(self, unique_id: bytes, rank: int, world: int, build_once: bool = True) -> None:
        """NCCL communicator of this database (unique_id from nccl_unique_id() on rank 0)."""
        buf = ctypes.create_string_buffer(bytes(unique_id), 128)
        check(lib().ddq_dist_init_nccl(self.h, buf, rank, world, 1 if build_once else 0))

    def dist_init_host(self, rank: int, world: int, allgather) -> None:
        """Exchange through a host all-gather: allgather(send: bytes) -> bytes (rank-major)."""
        def cb(send, recv, nbytes, user):
            try:
                out = allgather(ctypes.string_at(send, nbytes))
                ctypes.memmove(recv, out, len(out))
                return 0
            except Exception:  # an exception must not cross the C ABI
                return -1
        self._allgather_cb = A.ALLGATHER_FN(cb)  # kept alive with the database
        check(lib().ddq_dist_init_host(self.h, rank, world, ctypes.cast(self._allgather_cb, ctypes.c_void_p), None))

    def dist_exchange(self, preps: list, stream: int = 0) -> None:
        """All-gather the partial group tables of the prepared plans (after their launches)."""
        arr = (ctypes.c_void_p * len(preps))(*[p.h.value if hasattr(p.h, "value") else p.h for p in preps])
        check(lib().ddq_dist_exchange(self.h, arr, len(preps), ctypes.c_void_p(stream)))

    def dist_result(self, i: int) -> QueryResult:
        """The result of plan i of the last exchange over every rank's rows."""
        p = ctypes.POINTER(A.Result)()
        check(lib().ddq_dist_result(self.h, i, ctypes.byref(p)))
        return _convert(p)

    # ---- plans -----------------------------------------------------------------
    def plan(self) -> PlanBuilder:
        return PlanBuilder(self)

    def submit(self, plan: PlanBuilder | A.Plan) -> int:
        p = plan.plan if isinstance(plan, PlanBuilder) else plan
        q = ctypes.c_int64()
        check(lib().ddq_submit(self.h, ctypes.byref(p), ctypes.byref(q)))
        return q.value

    def wait(self, q: int, timeout_s: float | None = None) -> None:
        check(lib().ddq_wait(self.h, q, -1 if timeout_s is None else int(timeout_s * 1e9)))

    def fetch(self, q: int) -> QueryResult:
        p = ctypes.POINTER(A.Result)()
        check(lib().ddq_fetch(self.h, q, ctypes.byref(p)))
        return _convert(p)

    def run(self, plan: PlanBuilder | A.Plan) -> QueryResult:
        return self.fetch(self.submit(plan))

    def prepare(self, plan: PlanBuilder | A.Plan, use_graph: bool = True) -> Prepared:
        p = plan.plan if isinstance(plan, PlanBuilder) else plan
        pr = Prepared(self, p, use_graph)
        self._root_aggs[id(pr)] = p.ops[p.n_ops - 1].n_aggs
        return pr

    # ---- statistics -----------------------------------------------------------
    def stats(self) -> dict:
        s = A.Stats()
        check(lib().ddq_get_stats(self.h, ctypes.byref(s)))
        return {n: int(getattr(s, n)) for n, _ in A.Stats._fields_}

    def reset_stats(self) -> None:
        check(lib().ddq_reset_stats(self.h))


class Cluster:
    """Multi-GPU data-driven placement (include/ddq.h "cluster"): one
    database per device; load the same tables into every member (`members`), then
    submit: each query goes to the member whose cache holds most of its input bytes."""

    def __init__(self, devices: list[int], **kw):
        cfg = A.Config()
        lib().ddq_config_default(ctypes.byref(cfg))
        for k, v in {"cache_bytes": 64 << 30, "heap_bytes": 32 << 30, **kw}.items():
            setattr(cfg, k, int(v))
        devs = (ctypes.c_int32 * len(devices))(*devices)
        h = ctypes.c_void_p()
        check(lib().ddq_cluster_open(ctypes.byref(cfg), devs, len(devices), ctypes.byref(h)))
        self.h = h
        self.members = [Database(_handle=lib().ddq_cluster_db(h, i)) for i in range(len(devices))]

    def submit(self, plan) -> tuple[int, int]:
        p = plan.plan if isinstance(plan, PlanBuilder) else plan
        m, q = ctypes.c_int32(), ctypes.c_int64()
        check(lib().ddq_cluster_submit(self.h, ctypes.byref(p), ctypes.byref(m), ctypes.byref(q)))
        return m.value, q.value

    def fetch(self, member: int, q: int) -> QueryResult:
        p = ctypes.POINTER(A.Result)()
        check(lib().ddq_cluster_fetch(self.h, member, q, ctypes.byref(p)))
        return _convert(p)

    def update_placement(self) -> None:
        check(lib().ddq_cluster_update_placement(self.h))

    def close(self) -> None:
        if self.h:
            for m in self.members:
                m.close()
            lib().ddq_cluster_close(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
