/*
 * ddq.h -- C ABI of libddq, the B200-native hot path of Bress, Funke & Teubner,
 * "Robust Query Processing in Co-Processor-accelerated Databases" (SIGMOD'16).
 *
 * Citations "P:n" are /root/reference/PAPER.md line n (section named alongside);
 * "S8(x)" is SURVEY.md section 8(x).  No torch or CUDA types appear here: device
 * memory is passed as plain pointers, CUDA streams as `void*` (a cudaStream_t),
 * sizes as integers.  Every call returns a ddq_status; nothing throws across the
 * ABI.  On error, ddq_last_error() returns a thread-local message.
 *
 * Two layers:
 *   1. Operator calls (ddq_op_*): the data-parallel kernels of S8(a1)-(a6) on
 *      device buffers, stream-ordered, asynchronous.  Element counts that are
 *      produced on the device stay on the device (a uint32 in device memory) so
 *      operator chains never synchronise with the host.
 *   2. The database (ddq_open .. ddq_fetch): a column store with a per-GPU column
 *      cache and a heap-budget allocator (device memory = data cache + heap, P:62
 *      Sec. 2.1), physical plans executed operator-at-a-time (Sec. 2.5) under
 *      data-driven placement (Sec. 3.1, Sec. 3.3) and query chopping
 *      (Sec. 5.1-5.2, Sec. 5.4), with abort-and-restart of a failed
 *      operator on the host (Sec. 2.5.1, Sec. 4.1).
 */
#ifndef DDQ_H
#define DDQ_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ------------------------------------------------------------------ status */
typedef int32_t ddq_status;
enum {
  DDQ_OK = 0,
  DDQ_EINVAL = -1,        /* invalid argument / plan / duplicate build key */
  DDQ_ENOTFOUND = -2,     /* unknown table, column or query handle */
  DDQ_ENOMEM_HOST = -3,   /* host allocation failed */
  DDQ_ENOMEM_DEVICE = -4, /* device heap exhausted (op layer / prepared plans only;
                             inside ddq_submit an OOM aborts the operator and it is
                             restarted on the host, P:111 -- never surfaced) */
  DDQ_ECUDA = -5,         /* CUDA error (sticky) */
  DDQ_ENCCL = -6,
  DDQ_ESTATE = -7,        /* call not valid in the current state */
  DDQ_ETIMEOUT = -8,
  DDQ_EOVERFLOW = -9      /* a device hash table overflowed its capacity */
};
const char* ddq_last_error(void);
const char* ddq_version(void);

/* ========================================================================
 * 1. Operator calls (device buffers; all pointers below are DEVICE pointers
 *    unless named h_*).  TIDs are int32 row ids (< 2^31).  A TID list is a
 *    MULTISET (reading O14'): the operators emit survivors in an
 *    unspecified order (per-CTA write-combined blocks), each input item at most
 *    once; every consumer (probe, select, gather, aggregate) is order-free and
 *    all aggregates are exact integer sums, so query results are bit-identical.
 *    "count" arguments are device uint32 cells: an input count is read by the
 *    kernel; an output count is written by it.  `n_cap` is a HOST upper bound on
 *    the input count (sizes grids and scratch).  Outputs must hold n_cap items.
 *    `scratch` is device memory of ddq_op_scratch_bytes(n_cap) bytes, owned by
 *    the caller, reused freely after the call's stream work completes.
 *    Errors: DDQ_EINVAL for bad widths / null required pointers / n_cap > 2^31;
 *    DDQ_ECUDA if a launch fails.  Kernel-side overflow is reported through the
 *    d_error cell where one exists.
 * ====================================================================== */

/* Predicate kinds (S8(a1)-(a2)).  RANGE covers =, <, <=, >, >=, BETWEEN on integer
 * columns (constants folded into an inclusive [lo, hi]); IN holds up to 8 values
 * (string IN/= become dictionary-code sets, reading O4). */
enum { DDQ_PRED_RANGE = 1, DDQ_PRED_IN = 2, DDQ_PRED_BITSET = 3 };
/* DDQ_PRED_BITSET: a dictionary-code set too large for IN (e.g. TPC-H Q2's
 * p_type LIKE '%BRASS', 30 of 150 codes; reading O35): v holds iff
 * 0 <= v - lo < 512 and bit (v - lo) of the 512-bit mask in_vals[0..7] is set
 * (bit b of word b / 64).  hi and n_in are ignored.  ddq_dictionary_like builds one. */
#define DDQ_MAX_IN 8
#define DDQ_MAX_PREDS 4
#define DDQ_MAX_CARRY 4

typedef struct {
  const void* col; /* device column, indexed by row id */
  int32_t width;   /* 4 (int32) or 8 (int64) */
  int32_t kind;    /* DDQ_PRED_RANGE | DDQ_PRED_IN */
  int64_t lo, hi;  /* RANGE: lo <= v <= hi */
  int32_t n_in;    /* IN: number of values in in_vals */
  int32_t _pad;
  int64_t in_vals[DDQ_MAX_IN];
} ddq_dev_pred;

/* Scratch bytes needed by select / probe / build / groupby for n_cap inputs. */
size_t ddq_op_scratch_bytes(int64_t n_cap);

/* Selection (S8(a1) dimension, S8(a2) fact; App. B):
 * out_tids = the row ids r of the input (all rows [0, n_cap) when in_tids ==
 * NULL, else r = in_tids[i] for i < *d_in_count) for which EVERY predicate
 * holds, as a multiset (order unspecified).  Carried vectors (aligned with the
 * input, int32; 16-byte aligned) are compacted alongside: carry_out[c][j] =
 * carry_in[c][i] where out_tids[j] came from input item i.  *d_out_count
 * receives the survivor count. */
ddq_status ddq_op_select(const ddq_dev_pred* preds, int32_t n_preds,
                         const int32_t* in_tids, const uint32_t* d_in_count, int64_t n_cap,
                         const int32_t* const* carry_in, int32_t* const* carry_out, int32_t n_carry,
                         int32_t* out_tids, uint32_t* d_out_count,
                         void* scratch, size_t scratch_bytes, void* stream);

/* Hash build (S8(a3); join memory): insert (key = keys[r], payload =
 * payload ? payload[r] : r) for every input row r into an open-addressing table
 * of `capacity` 8-byte slots (power of two, >= 2x the number of keys, load <= 0.5;
 * reading O13).  The table must be initialised with ddq_op_hash_init.  Keys must
 * be unique and != INT32_MIN; a duplicate or a full table sets *d_error != 0
 * (1 = duplicate key, 2 = table full). */
ddq_status ddq_op_hash_init(uint64_t* table, uint32_t capacity, void* stream);
ddq_status ddq_op_hash_build(const int32_t* keys, const int32_t* payload,
                             const int32_t* in_tids, const uint32_t* d_in_count, int64_t n_cap,
                             uint64_t* table, uint32_t capacity, uint32_t* d_error, void* stream);

/* Hash probe = semi-join + payload (S8(a4)): for each input row r
 * (all rows or in_tids[i]), look up fk[r]; survivors are compacted into
 * out_tids (a multiset, as in ddq_op_select), with the matched payload into
 * out_payload (may be NULL) aligned with them and carried vectors compacted
 * alongside (as in ddq_op_select). */
ddq_status ddq_op_hash_probe(const uint64_t* table, uint32_t capacity, const int32_t* fk,
                             const int32_t* in_tids, const uint32_t* d_in_count, int64_t n_cap,
                             const int32_t* const* carry_in, int32_t* const* carry_out, int32_t n_carry,
                             int32_t* out_tids, int32_t* out_payload, uint32_t* d_out_count,
                             void* scratch, size_t scratch_bytes, void* stream);

/* Direct-mapped join index (S8(a3)/(a4), the build/probe used when the build key
 * column spans a compact range [key_min, key_min + range)): a membership bitmap of
 * `range` bits followed (16-byte aligned) by an int32 payload array of `range`
 * entries and, when range > 1.5 M keys (a bitmap too large for one SM's shared
 * memory), a coarse bitmap (1 bit per 2^cg keys, set by the build; probes filter
 * with it in shared memory and read exact bits from L2 only for its hits);
 * ddq_op_join_index_bytes(range) bytes, zero the bitmaps with
 * ddq_op_join_index_init.  Same semantics as hash build / probe: unique keys
 * (duplicate -> *d_error = 1; key outside the range -> *d_error = 3), probe =
 * semi-join + payload of survivors.  Chosen by the engine when range <= 16 x the
 * dimension's rows (dimension primary keys); hash tables remain the general path. */
size_t ddq_op_join_index_bytes(uint32_t range);
ddq_status ddq_op_join_index_init(void* index, uint32_t range, void* stream);
ddq_status ddq_op_join_index_build(const int32_t* keys, const int32_t* payload,
                                   const int32_t* in_tids, const uint32_t* d_in_count, int64_t n_cap,
                                   int32_t key_min, uint32_t range, void* index, uint32_t* d_error,
                                   void* stream);
ddq_status ddq_op_join_index_probe(const void* index, int32_t key_min, uint32_t range, const int32_t* fk,
                                   const int32_t* in_tids, const uint32_t* d_in_count, int64_t n_cap,
                                   const int32_t* const* carry_in, int32_t* const* carry_out, int32_t n_carry,
                                   int32_t* out_tids, int32_t* out_payload, uint32_t* d_out_count,
                                   void* scratch, size_t scratch_bytes, void* stream);

/* Star semi-join (S8(a2)+(a4) in one pass; the n-ary operator behind DDQ_OP_STAR):
 * rows r in [0, n_rows) of a fact table survive iff every term holds -- a predicate
 * on its column, or membership of its int32 fk column value in a join index
 * (index != NULL: bitmap + payload over [key_min, key_min+range), see
 * ddq_op_join_index_*) or hash table (table/capacity).  Probe terms with
 * out_payload != NULL write the matched payload aligned with out_tids.  All term
 * columns are streamed once (TMA); terms are evaluated in order.  Output order:
 * ascending within 2048-row tiles, tiles in reservation order (a multiset).
 * Columns must be 16-byte aligned and readable up to the next 16-byte boundary.
 * *d_out_count uses 2 words (count, CTA counter); overflow of out_cap sets
 * *d_overflow = 4 (if non-NULL). */
enum { DDQ_TERM_PRED = 1, DDQ_TERM_PROBE = 2, DDQ_TERM_FETCH = 3 /* AGGREGATE terms only, see ddq_op */ };
typedef struct {
  int32_t kind;          /* DDQ_TERM_PRED | DDQ_TERM_PROBE */
  int32_t width;         /* column width (4 or 8; probes: 4) */
  const void* col;       /* streamed column */
  int32_t pred_kind;     /* DDQ_PRED_RANGE | DDQ_PRED_IN */
  int32_t n_in;
  int64_t lo, hi;
  int64_t in_vals[DDQ_MAX_IN];
  const void* index;     /* join index, or NULL */
  int32_t key_min;
  uint32_t range;
  const uint64_t* table; /* hash table when index == NULL */
  uint32_t capacity;
  int32_t _pad;
  int32_t* out_payload;  /* probe payload output or NULL */
} ddq_dev_term;
ddq_status ddq_op_star(const ddq_dev_term* terms, int32_t n_terms, int64_t n_rows, int32_t* out_tids,
                       uint32_t* d_out_count, int64_t out_cap, uint32_t* d_overflow, void* stream);

/* Positional gather (S8(a5); P:107 materialisation): out[i] = col[tids[i]] for
 * i < *d_count; width 4 or 8. */
ddq_status ddq_op_gather(const void* col, int32_t width, const int32_t* tids,
                         const uint32_t* d_count, int64_t n_cap, void* out, void* stream);

/* Group-by aggregation (S8(a6)).  For each input position i < *d_count with
 * row r = tids[i]: group key = k0 | k1 << b0 | k2 << (b0 + b1) (bj = key_bits[j],
 * key_bits NULL or 0 -> 21) where kj is either the aligned vector key_vec[j][i] or
 * the column key_col[j][r] (int32, 0 <= kj < 2^bj, sum of bits <= 63);
 * aggregate a adds expr_a(r) to the group's exact int128 accumulator.  The result
 * is an open-addressing table of `capacity` slots (power of two, >= 2x groups):
 *   keys  int64[capacity]           (empty = -1)
 *   accs  int64[n_aggs][capacity][2] (lo, hi words of an int128)
 * Init with ddq_op_groupby_init; read it back with ddq_op_groupby_compact.
 * Overflow of the table sets *d_error = 2. */
enum {
  DDQ_AGG_COUNT = 1,          /* 1 */
  DDQ_AGG_SUM = 2,            /* a */
  DDQ_AGG_SUM_MUL = 3,        /* a * b */
  DDQ_AGG_SUM_SUB = 4,        /* a - b */
  DDQ_AGG_SUM_MUL_100M = 5,   /* a * (100 - b)            (TPC-H scale-2 decimals) */
  DDQ_AGG_SUM_MUL_100M_100P = 6, /* a * (100 - b) * (100 + c) */
  DDQ_AGG_MIN = 7             /* min(a) (S8(a6); TPC-H Q2's min(ps_supplycost)): the group's
                                 smallest int64 value, returned sign-extended in the
                                 int128 cell; aggregations carrying a MIN run the
                                 generic one-row-per-thread kernel on the global table */
};
#define DDQ_MAX_AGGS 8
#define DDQ_MAX_KEYS 3
typedef struct {
  int32_t kind;            /* DDQ_AGG_* */
  int32_t width[3];        /* widths of the argument columns (4 or 8) */
  const void* arg[3];      /* argument columns (device, indexed by row id) */
} ddq_dev_agg;

size_t ddq_op_groupby_table_bytes(uint32_t capacity, int32_t n_aggs);
ddq_status ddq_op_groupby_init(void* table, uint32_t capacity, int32_t n_aggs, void* stream);
ddq_status ddq_op_groupby(const int32_t* tids, const uint32_t* d_count, int64_t n_cap,
                          const int32_t* const* key_vec, const int32_t* const* key_col, int32_t n_keys,
                          const int32_t* key_bits, const ddq_dev_agg* aggs, int32_t n_aggs,
                          void* table, uint32_t capacity, uint32_t* d_error, void* stream);
/* Compact the non-empty groups: out_keys int64[capacity], out_accs int64[n_aggs *
 * capacity * 2] (group-major: accs of group g at [(g * n_aggs + a) * 2]),
 * *d_out_groups = number of groups.  Group order is unspecified. */
ddq_status ddq_op_groupby_compact(const void* table, uint32_t capacity, int32_t n_aggs,
                                  int64_t* out_keys, int64_t* out_accs, uint32_t* d_out_groups,
                                  void* stream);

/* ========================================================================
 * 2. The database: column store, device cache + heap, plans, chopping.
 * ====================================================================== */
typedef struct ddq_db ddq_db;
typedef int32_t ddq_table;
typedef int32_t ddq_column;
typedef int64_t ddq_query;

typedef enum { DDQ_I32 = 1, DDQ_I64 = 2 } ddq_type;

/* Placement strategies (Sec. 6.2 and Sec. 3-5). */
typedef enum {
  DDQ_PLACE_DATA_DRIVEN = 0, /* GPU iff all inputs are cached there */
  DDQ_PLACE_GPU_ONLY = 1,    /* "GPU Preferred": everything on the GPU; inputs that are
                                not cached are copied on demand (operator-driven data
                                placement with LRU caching) */
  DDQ_PLACE_CPU_ONLY = 2
} ddq_placement;

typedef struct {
  int32_t device;                /* CUDA device ordinal (one process per GPU) */
  int32_t rank, world;           /* this process's rank / the ranks of a row-sharded multi-GPU run
                                    (P:407); informational until ddq_dist_init_nccl / _host,
                                    which set them and create the exchange (multi-GPU, below) */
  uint64_t cache_bytes;          /* device column cache budget */
  uint64_t heap_bytes;           /* device heap for intermediates */
  int32_t gpu_workers;           /* chopping bound: GPU worker threads, O17 */
  int32_t host_workers;          /* host executor threads */
  int32_t placement;             /* ddq_placement */
  int32_t chopping;              /* 1: run-time placement + bounded pull queues (Sec. 5.2);
                                    0: compile-time placement, one thread per operator */
  int32_t cache_policy;          /* 0 = LFU (Alg. 1), 1 = LRU (App. E) */
  uint32_t fault_alloc_every;    /* fault injection: fail every Nth device heap alloc (0=off) */
  int32_t transfer_packing;      /* 1 (default): ddq_load_column also keeps a frame-of-reference
                                    byte-packed pinned copy (value - min in 1..4 bytes) and a
                                    cold cache load copies that and widens it on the device
                                    (fewer bytes over PCIe);
                                    0: copy the raw column */
  int32_t prefetch;              /* 1: streamed cold path (S8(f) N1, "overlap data transfer and
                                    computation"): at submit, every column the plan reads that is not
                                    resident is queued for an asynchronous H2D copy in plan order on
                                    the copy stream (a background copy thread), so operator k computes
                                    while the columns of operators k+1.. stream in; GPU workers pull
                                    ready operators whose columns are resident first (cached-first
                                    schedule).  0 (default): columns are copied when an operator
                                    needs them (the paper's operator-driven placement) */
  int32_t placement_period_ms;   /* > 0: a background job runs Algorithm 1 (ddq_update_placement)
                                    every this many ms while the database is open -- the paper's
                                    periodic data placement; 0 (default): only when
                                    the caller invokes ddq_update_placement */
  int32_t max_queries;           /* query-level admission control (the comparison arm of P:371,
                                    P:445, Wang et al.): at most this many submitted queries run at
                                    once, later ones wait in submission order until one finishes;
                                    0 (default) = no admission control */
  uint32_t fault_op_mask;        /* fault injection: the GPU attempt of plan op i (i < 32) aborts as if
                                    its heap allocation failed when bit i is set (deterministic
                                    abort -> host restart traces, Fig. 8); 0 = off */
} ddq_config;

void ddq_config_default(ddq_config* cfg);
ddq_status ddq_open(const ddq_config* cfg, ddq_db** out);
void ddq_close(ddq_db* db);

/* Tables and columns.  ddq_load_column copies host_data (n_rows values of the
 * given type) into library-owned pinned host memory (Sec. 2.5.3); the caller
 * keeps ownership of host_data.  shard_row_begin = global row id of local row 0. */
ddq_status ddq_create_table(ddq_db* db, const char* name, int64_t n_rows, int64_t shard_row_begin,
                            ddq_table* out);
ddq_status ddq_load_column(ddq_db* db, ddq_table t, const char* name, ddq_type type,
                           const void* host_data, int64_t n_rows, ddq_column* out);
ddq_status ddq_find_column(ddq_db* db, const char* table, const char* name, ddq_column* out);
/* Column statistics recorded at load (the strategic optimiser's input):
 * row count and value range [vmin, vmax] (vmin > vmax for an empty column).  Plans
 * size packed group keys from them (e.g. bits of a key column = bit length of vmax). */
ddq_status ddq_column_stats(ddq_db* db, ddq_column c, int64_t* n, int64_t* vmin, int64_t* vmax);

/* Storage adviser: pin a column into the device cache (H2D copy on the
 * library's copy stream, counted in stats) / evict it (freed once no running
 * operator references it).  Fails with DDQ_ENOMEM_DEVICE if it does not
 * fit the cache budget. */
ddq_status ddq_cache_column(ddq_db* db, ddq_column c);
ddq_status ddq_evict_column(ddq_db* db, ddq_column c);
int32_t ddq_column_is_cached(ddq_db* db, ddq_column c);
/* Device pointer of a cached column (for the operator layer), or NULL. */
const void* ddq_column_device_ptr(ddq_db* db, ddq_column c);
/* Run Algorithm 1 once (Sec. 3.2): sort columns by access count
 * (descending; ties by column id, O16), keep the greedy prefix that fits the cache
 * budget (stop at the first that does not fit), evict old\new, cache new\old. */
ddq_status ddq_update_placement(ddq_db* db);
/* Access counters (incremented per operator access) */
uint64_t ddq_column_access_count(ddq_db* db, ddq_column c);
ddq_status ddq_reset_access_counts(ddq_db* db);

/* ---- physical plans (S8(b) plan IR) ----------------------------------------
 * A plan is an array of operators; op i's children have indices < i; the last
 * op is the root and must be an AGGREGATE (or a SELECT/GATHER for select-*).
 * Every op produces a materialised intermediate: a TID list over a table's
 * row space plus aligned int32/int64 vectors. */
enum {
  DDQ_OP_SELECT = 1,     /* preds over `table` at input TIDs (or all rows) */
  DDQ_OP_HASH_BUILD = 2, /* hash table over input TIDs of `table` (key_col, payload_col) */
  DDQ_OP_HASH_PROBE = 3, /* semi-join input TIDs of `table` via fk_col against op `build` */
  DDQ_OP_GATHER = 4,     /* append vector col[tid] to the input's aligned vectors */
  DDQ_OP_AGGREGATE = 5,  /* group-by at input TIDs; root; finalised on the host */
  DDQ_OP_FILTER_EQ = 6,  /* keep input rows whose two aligned vectors compare true under
                            eq_cmp: equal (TPC-H Q5's c_nationkey = s_nationkey), less
                            (Q4's l_commitdate < l_receiptdate) or not equal (Q7's
                            n1 <> n2); vectors carried */
  DDQ_OP_STAR = 7        /* conjunction of predicates and probes over all rows of a fact
                            table in one pass (all term columns streamed once); output as
                            a chain of SELECT/HASH_PROBE ops would produce it */
};

typedef struct {
  ddq_column column;
  int32_t kind;   /* DDQ_PRED_RANGE | DDQ_PRED_IN */
  int64_t lo, hi;
  int32_t n_in;
  int32_t _pad;
  int64_t in_vals[DDQ_MAX_IN];
} ddq_pred;

typedef struct {
  int32_t kind;            /* DDQ_OP_* */
  int32_t input;           /* child op index whose output TIDs are consumed, or -1 = all rows */
  ddq_table table;         /* row space of input and output TIDs */
  /* SELECT; also HASH_BUILD and AGGREGATE, where they are a fused selection of the
     op's input rows (readings O25, O26) */
  int32_t n_preds;
  ddq_pred preds[DDQ_MAX_PREDS];
  /* HASH_BUILD */
  ddq_column key_col;
  ddq_column payload_col;  /* -1: payload = dimension row id */
  /* HASH_PROBE */
  int32_t build;           /* op index of the HASH_BUILD */
  ddq_column fk_col;
  int32_t emit_payload;    /* append matched payload as an aligned vector */
  /* GATHER */
  ddq_column gather_col;
  /* AGGREGATE: keys are aligned vectors (index >= 0) or columns (-2 - column id).
     agg_col[a][j] is a column id (>= 0), -1 = none, or, for DDQ_AGG_MIN only, an
     aligned int32 vector v of the input encoded as -2 - v (a functionally dependent
     dimension attribute fetched through a join, TPC-H Q2); not with fused predicates. */
  int32_t n_keys;
  int32_t key_src[DDQ_MAX_KEYS];
  int32_t n_aggs;
  int32_t agg_kind[DDQ_MAX_AGGS];
  ddq_column agg_col[DDQ_MAX_AGGS][3];
  int64_t max_groups;      /* upper bound on the number of groups (sizes the table) */
  /* finalisation (S8(a7)): ORDER BY entries: +(1+k) key k asc, -(1+k) key k desc,
     +(101+a) aggregate a asc, -(101+a) desc; codes are order-preserving (O4). */
  int32_t n_order;
  int32_t order_by[8];
  int64_t limit;           /* <= 0: no limit */
  /* extensions (zero = default) */
  int32_t key_bits[DDQ_MAX_KEYS]; /* AGGREGATE: bits of key k in the packed group key
                                     (0 = 21); keys are packed low to high; sum <= 63 */
  int32_t fk_vec;          /* HASH_PROBE: 1 + index of an aligned input vector holding the
                              probe keys (instead of fk_col); 0 = use fk_col */
  int32_t eq_vec[2];       /* FILTER_EQ: 1 + indexes of the two aligned vectors compared */
  /* STAR (n-ary semi-join over all rows of `table`, evaluated in one pass): term j is
     a predicate (preds[j]) or a probe of fk column term_fk[j] against HASH_BUILD op
     term_build[j], emitting its payload as the next aligned vector if term_emit[j].
     AGGREGATE (reading O37, the fused late-materialised tail): terms evaluated at the
     input TIDs after the fused predicates, in order -- DDQ_TERM_PROBE (a semi-join:
     rows whose fk misses the build are dropped; payload emitted if term_emit[j]) or
     DDQ_TERM_FETCH (the build's payload of fk, INT32_MIN on a miss, the row kept, as
     a GATHER with fetch_build); emitted payloads are appended, in term order, after
     the input's aligned vectors, so key_src may name them.  GPU: <= 2 aggregates, no
     MIN, group table <= 2048 slots (the warp-autonomous aggregation), else EINVAL. */
  int32_t n_terms;
  int32_t term_kind[4];    /* DDQ_TERM_PRED | DDQ_TERM_PROBE */
  int32_t term_build[4];
  ddq_column term_fk[4];
  int32_t term_emit[4];
  /* GATHER through a join (dimension attribute fetch): 1 + index of a HASH_BUILD op;
     0 = plain column gather.  The new vector is then payload(build, gather_col[r])
     for every input row r (gather_col = the fact FK column), INT32_MIN where r's key
     has no match -- a fetch after a semi-join probe of the same build (late
     materialisation) never has one.  int32 output. */
  int32_t fetch_build;
  /* FILTER_EQ comparison: DDQ_CMP_EQ (0, default) keeps rows with vec_a == vec_b,
     DDQ_CMP_LT keeps rows with vec_a < vec_b (signed int32; TPC-H Q4's
     l_commitdate < l_receiptdate), DDQ_CMP_NE keeps vec_a != vec_b (TPC-H Q7's
     pair of distinct nations).  Other values: DDQ_EINVAL. */
  int32_t eq_cmp;
  /* HASH_BUILD: 1 = the build is a key SET for a semi-join (EXISTS / IN subquery,
     TPC-H Q4): duplicate keys are allowed and collapse into one entry whose
     payload is any one of their rows; 2 = a MIN-aggregating build (a decorrelated
     scalar subquery `= (select min(x) ... where key = outer.key)`, TPC-H Q2, reading
     O35): duplicate keys collapse into one entry whose payload is the SMALLEST payload
     value among them; 0 (default) = unique keys, a duplicate is DDQ_EINVAL (reading
     O13).  Any build's payload column may be int64 when its load-time range fits
     int32 (it is narrowed exactly; else DDQ_EINVAL). */
  int32_t build_key_set;
  /* AGGREGATE finalisation (S8(a7), reading O10): n_avg derived double columns,
     avg k = (double)acc[avg_sum[k]] / (double)acc[avg_count] / 10^avg_scale[k] (SQL AVG
     of a scale-s decimal; TPC-H Q1's avg_qty / avg_price / avg_disc).  NULL when the
     count is 0.  Computed on the host after the exact int128 merge. */
  int32_t n_avg;
  int32_t avg_sum[4];
  int32_t avg_count;
  int32_t avg_scale[4];
  /* GATHER: 1 = gather an int64 column into an int32 vector (exact: allowed only when
     the column's load-time range fits int32, else DDQ_EINVAL), so it can be compared
     with FILTER_EQ or carried (TPC-H Q2's ps_supplycost = min cost) */
  int32_t gather_narrow;
} ddq_op;

#define DDQ_CMP_EQ 0
#define DDQ_CMP_LT 1
#define DDQ_CMP_NE 2

#define DDQ_MAX_OPS 32
typedef struct {
  int32_t n_ops;
  ddq_op ops[DDQ_MAX_OPS];
} ddq_plan;

/* Order-preserving dictionary of a string column (reading O4; S8(b)): the column's
 * int32 values are codes = ranks in `sorted_strings` (n distinct strings, strictly
 * ascending in bytewise (C-locale) order; DDQ_EINVAL otherwise).  The strings are
 * copied; the library decodes result keys through them (ddq_result.key_str) and
 * folds string predicates into code predicates (below).  Plan-time host work only. */
ddq_status ddq_set_dictionary(ddq_db* db, ddq_column c, const char* const* sorted_strings, int32_t n);
/* Code range of a string constant: *lower = first code whose string >= s, *upper =
 * first code whose string > s (so s is present iff lower < upper; BETWEEN a AND b
 * is [lower(a), upper(b)) ).  DDQ_ENOTFOUND if the column has no dictionary. */
ddq_status ddq_dictionary_range(ddq_db* db, ddq_column c, const char* s, int32_t* lower, int32_t* upper);
/* SQL LIKE over the dictionary (TPC-H Q2's p_type like '%BRASS'; reading O35):
 * fills *out with a predicate on column c that holds exactly for the codes whose
 * string matches `pattern` ('%' = any run, '_' = any one byte, no escapes):
 * DDQ_PRED_IN when <= 8 codes match, else DDQ_PRED_BITSET when they lie within
 * 512 consecutive codes, else DDQ_EINVAL.  No match: an empty RANGE (lo > hi). */
ddq_status ddq_dictionary_like(ddq_db* db, ddq_column c, const char* pattern, ddq_pred* out);

/* Result of a query: rows of (n_keys int32-code keys, n_aggs int128 aggregates)
 * in ORDER BY order, or, for a select-* root, the TID list. Owned by the library. */
typedef struct {
  int64_t n_rows;
  int32_t n_keys, n_aggs;
  const int64_t* keys;   /* n_rows * n_keys (decoded from the packed group key) */
  const int64_t* aggs;   /* n_rows * n_aggs * 2: (lo, hi) words of each int128 */
  int64_t n_tids;        /* select-* roots: surviving TIDs (global row ids) */
  const int32_t* tids;
  int32_t gpu_ops, host_ops, aborts;
  double exec_ms;        /* submit -> root finished */
  /* SQL NULLs (reading O7): agg_null[i * n_aggs + a] = 1 when aggregate a of row i
     is NULL -- SUM / MIN over an empty input.  An AGGREGATE without keys always
     returns exactly one row (count 0, SUMs NULL, when nothing qualified); grouped
     queries return no row for an empty input. */
  const uint8_t* agg_null;
  /* root->n_avg finalisation doubles per row (avgs[i * n_avg + k]); NaN when NULL */
  int32_t n_avg;
  int32_t _pad;
  const double* avgs;
  /* decoded group keys: key_str[i * n_keys + k] = the dictionary string of key k of
     row i when its source column has a dictionary (ddq_set_dictionary), else NULL.
     The key source is the column behind the key: a key column, or the column an
     aligned vector was gathered from / a build emitted as payload.  Strings are
     owned by the database (valid until ddq_close); the pointer array by the result. */
  const char* const* key_str;
  /* placement trace (driver results only; prepared plans: NULL): op_place[i] for plan
     op i = DDQ_RAN_GPU, DDQ_RAN_HOST, or DDQ_RAN_ABORTED (started on the GPU, aborted
     on allocation failure, restarted on the host) */
  int32_t n_ops;
  int32_t _pad2;
  const uint8_t* op_place;
  const float* op_ms;    /* driver results: per op, host wall time from its pull by a worker to its
                            completion (incl. transfers and synchronisation), ms; else NULL */
} ddq_result;
enum { DDQ_RAN_GPU = 1, DDQ_RAN_HOST = 2, DDQ_RAN_ABORTED = 3 };

/* Submit a plan (copied; thread-safe; many user threads may submit). */
ddq_status ddq_submit(ddq_db* db, const ddq_plan* plan, ddq_query* out);
ddq_status ddq_wait(ddq_db* db, ddq_query q, int64_t timeout_ns);
ddq_status ddq_fetch(ddq_db* db, ddq_query q, ddq_result** out);
void ddq_result_free(ddq_result* r);

/* Prepared plans: the hot path for resident data (configs 1-3).  All operators
 * are placed on the GPU (every input must be cached: data-driven placement,
 * P:140), intermediates are allocated from the heap once (fail-fast), and
 * the operator sequence is captured into one CUDA graph.  ddq_prepared_launch
 * enqueues one execution on `stream` with no host synchronisation;
 * ddq_prepared_fetch synchronises and finalises. */
typedef struct ddq_prepared ddq_prepared;
ddq_status ddq_prepare(ddq_db* db, const ddq_plan* plan, int32_t use_graph, ddq_prepared** out);
ddq_status ddq_prepared_launch(ddq_prepared* p, void* stream);
ddq_status ddq_prepared_fetch(ddq_prepared* p, void* stream, ddq_result** out);
/* Partial aggregate access for multi-GPU merges (S8(e)): after a launch, copy the
 * compacted group table (keys int64[cap], accs int64[cap*n_aggs*2]) to host. */
ddq_status ddq_prepared_partials(ddq_prepared* p, void* stream, int64_t* h_n_groups,
                                 int64_t* h_keys, int64_t* h_accs, int64_t cap);
int64_t ddq_prepared_group_capacity(ddq_prepared* p);
/* Per-op kernel timing of the last launch is not tracked in graph mode; this
 * returns the number of kernels one launch enqueues. */
int32_t ddq_prepared_kernel_count(ddq_prepared* p);
/* Profiling pass (no graph): replays the plan on `stream` with a CUDA event
 * before and after every operator, then reports per operator (up to max_ops):
 * op_ms = event-timed duration, op_bytes = algorithmic HBM bytes of the SURVEY
 * 8(d) model computed from the actual cardinalities (columns read once; TID-driven
 * reads at 32-byte-sector granularity: N*w*(1-(1-m/N)^(32/w)); TID / vector /
 * payload reads and writes; hash tables 0 bytes except their build writes),
 * op_class = 0 dense scan (select/probe over all rows), 1 select/probe/fetch at
 * TIDs, 2 hash build, 3 gather, 4 aggregate, 5 probe masked by a row bitmap (the
 * key column streamed for every row).  Returns the number of operators. */
int32_t ddq_prepared_profile(ddq_prepared* p, void* stream, int32_t max_ops, float* op_ms, double* op_bytes,
                             int32_t* op_class);
/* Device views of the compacted partial group table of the last launch (for an
 * NCCL exchange without host copies): keys int64[cap], accs int64[cap*n_aggs*2],
 * *count = number of valid groups (device uint32).  Library-owned; valid until
 * ddq_prepared_free. */
ddq_status ddq_prepared_partials_device(ddq_prepared* p, int64_t** keys, int64_t** accs, uint32_t** count,
                                        int64_t* cap);
/* Finalise partial group tables on the host, no GPU needed (S8(a7) + the S8(e)
 * merge): rows with equal packed keys (e.g. the same group from several shards)
 * are merged by exact int128 addition, then ORDER BY / LIMIT of `root` apply.
 * keys: int64[n] packed group keys; accs: int64[n * root->n_aggs * 2]. */
ddq_status ddq_finalize_partials(const ddq_op* root, int64_t n, const int64_t* keys, const int64_t* accs,
                                 ddq_result** out);
/* Finalise externally merged partials (keys/accs as returned above) into a result. */
ddq_status ddq_prepared_finalize(ddq_prepared* p, int64_t n_groups, const int64_t* h_keys,
                                 const int64_t* h_accs, ddq_result** out);
void ddq_prepared_free(ddq_prepared* p);

/* ---- multi-GPU: row-sharded fact table, one process per GPU (S8(e); Sec. 6.3
 * "Our Data-Driven strategy can support multiple co-processors by performing
 * horizontal partitioning").  Each rank loads its row range of the partitioned table
 * (ddq_create_table's shard_row_begin = global row id of its first row) and the whole
 * replicated (dimension) tables.
 *
 * ddq_dist_nccl_unique_id: 128 bytes for ncclCommInitRank (rank 0 creates it; the
 * caller's bootstrap -- e.g. a torch.distributed process group -- sends it to the
 * other ranks).  ddq_dist_init_nccl: the NCCL communicator of this database (NCCL is
 * loaded at run time: DDQ_ENCCL if libnccl.so.2 is missing); build_once = 1: a
 * prepared plan's HASH_BUILD over a replicated table runs on rank 0 only and its
 * index is broadcast (ncclBroadcast on the plan's stream, inside its CUDA graph,
 * which is then captured serially so every rank issues its collectives in one order;
 * every rank must prepare the same plans in the same order).  ddq_dist_init_host:
 * the same exchange through a caller-provided host all-gather (fn gathers `bytes` of
 * `send` from every rank into `recv`, rank-major, returns 0 on success) -- e.g. a
 * gloo process group; no build broadcast.
 *
 * ddq_table_set_partitioned: mark the row-sharded table (builds over it are never
 * broadcast; its rows differ per rank).
 *
 * ddq_dist_exchange: after the plans' launches on `stream`, pack each plan's compacted
 * partial group table ([count, keys[cap], accs[cap * n_aggs * 2]] int64 words) into a
 * library-owned device buffer and all-gather it across the ranks (ncclAllGather on
 * `stream`, asynchronous; host transport: synchronous).  Every rank calls it with the
 * same plans in the same order.  ddq_dist_result(i): the result of plans[i] over ALL
 * ranks' rows -- partial groups merged exactly (SUM / COUNT by int128 addition, MIN
 * by minimum; the same result as one GPU) and finalised (S8(a7)); synchronises
 * the exchange stream.  Owned by the caller (ddq_result_free). */
typedef int32_t (*ddq_allgather_fn)(const void* send, void* recv, size_t bytes, void* user);
ddq_status ddq_dist_nccl_unique_id(void* out128);
ddq_status ddq_dist_init_nccl(ddq_db* db, const void* id128, int32_t rank, int32_t world, int32_t build_once);
ddq_status ddq_dist_init_host(ddq_db* db, int32_t rank, int32_t world, ddq_allgather_fn fn, void* user);
ddq_status ddq_table_set_partitioned(ddq_db* db, ddq_table t, int32_t partitioned);
ddq_status ddq_dist_exchange(ddq_db* db, ddq_prepared* const* plans, int32_t n, void* stream);
ddq_status ddq_dist_result(ddq_db* db, int32_t i, ddq_result** out);

/* ---- multi-GPU data-driven placement (Sec. 6.3) ---------
 * A cluster is one database per GPU (ddq_cluster_open: cfg copied, device taken from
 * devices[i]); the caller loads the SAME tables and columns, in the same order, into
 * every member (ddq_cluster_db), so column ids agree.  Each member's cache is filled by
 * Algorithm 1 over the access counts of the queries it ran (ddq_cluster_update_
 * placement runs ddq_update_placement on every member).  ddq_cluster_submit is
 * data-driven placement of the query: the member whose cache holds the most of the
 * plan's input bytes (ties: fewest queries in flight, then round robin); inside the
 * member every operator is placed as in ddq_submit.  *member receives the member;
 * fetch with ddq_cluster_fetch(member, query).  A single process drives all members
 * (devices may repeat: several members on one GPU are valid, e.g. for tests). */
typedef struct ddq_cluster ddq_cluster;
ddq_status ddq_cluster_open(const ddq_config* cfg, const int32_t* devices, int32_t n, ddq_cluster** out);
void ddq_cluster_close(ddq_cluster* c);
int32_t ddq_cluster_size(ddq_cluster* c);
ddq_db* ddq_cluster_db(ddq_cluster* c, int32_t i);
ddq_status ddq_cluster_submit(ddq_cluster* c, const ddq_plan* plan, int32_t* member, ddq_query* out);
ddq_status ddq_cluster_fetch(ddq_cluster* c, int32_t member, ddq_query q, ddq_result** out);
ddq_status ddq_cluster_update_placement(ddq_cluster* c);

/* ---- statistics (paper's counters, D10: P:330) ---- */
typedef struct {
  uint64_t h2d_bytes, d2h_bytes;
  uint64_t h2d_ns, d2h_ns;
  uint64_t gpu_ops, host_ops;
  uint64_t aborts;          /* GPU operators aborted on allocation failure */
  uint64_t wasted_ns;       /* begin->abort time of aborted GPU operators */
  uint64_t heap_peak_bytes, heap_used_bytes, cache_used_bytes;
  uint64_t cache_hits, cache_misses;
  uint64_t queries_done;
} ddq_stats;
ddq_status ddq_get_stats(ddq_db* db, ddq_stats* out);
ddq_status ddq_reset_stats(ddq_db* db);

/* Device heap (for the operator layer / tests): fail-fast sub-allocation. */
void* ddq_heap_try_alloc(ddq_db* db, uint64_t bytes);
void ddq_heap_free(ddq_db* db, void* p);

#ifdef __cplusplus
}
#endif
#endif /* DDQ_H */
