// ops.cu -- the operator layer of the C ABI (include/ddq.h, section 1).
#include <cstdio>
#include <cstring>
#include <string>

#include "ops_internal.h"

namespace ddq {
thread_local std::string g_last_error;
ddq_status set_error(ddq_status s, const std::string& msg) {
  g_last_error = msg;
  return s;
}
ddq_status cuda_status(cudaError_t e, const char* where) {
  if (e == cudaSuccess) return DDQ_OK;
  return set_error(DDQ_ECUDA, std::string(where) + ": " + cudaGetErrorString(e));
}
}  // namespace ddq

using namespace ddq;

extern "C" {

const char* ddq_last_error(void) { return g_last_error.c_str(); }
const char* ddq_version(void) { return "libddq 0.1 (sm_100a)"; }

size_t ddq_op_scratch_bytes(int64_t n_cap) { return filter_scratch_bytes(n_cap); }

static ddq_status check_cap(int64_t n_cap) {
  if (n_cap < 0 || n_cap > INT32_MAX) return set_error(DDQ_EINVAL, "n_cap out of range [0, 2^31)");
  return DDQ_OK;
}

ddq_status ddq_op_select(const ddq_dev_pred* preds, int32_t n_preds, const int32_t* in_tids,
                         const uint32_t* d_in_count, int64_t n_cap, const int32_t* const* carry_in,
                         int32_t* const* carry_out, int32_t n_carry, int32_t* out_tids, uint32_t* d_out_count,
                         void* scratch, size_t scratch_bytes, void* stream) {
  if (ddq_status s = check_cap(n_cap)) return s;
  if (n_preds < 0 || n_preds > DDQ_MAX_PREDS || (n_preds > 0 && !preds))
    return set_error(DDQ_EINVAL, "select: bad predicate list");
  if (n_carry < 0 || n_carry > DDQ_MAX_CARRY) return set_error(DDQ_EINVAL, "select: bad carry count");
  for (int i = 0; i < n_preds; i++) {
    if ((n_cap > 0 && !preds[i].col) || (preds[i].width != 4 && preds[i].width != 8))
      return set_error(DDQ_EINVAL, "select: predicate column must be non-null int32/int64");
    if (preds[i].kind != DDQ_PRED_RANGE && preds[i].kind != DDQ_PRED_IN && preds[i].kind != DDQ_PRED_BITSET)
      return set_error(DDQ_EINVAL, "select: bad predicate kind");
    if (preds[i].kind == DDQ_PRED_IN && (preds[i].n_in < 0 || preds[i].n_in > DDQ_MAX_IN))
      return set_error(DDQ_EINVAL, "select: IN list too long");
  }
  if (!out_tids || !d_out_count || !scratch) return set_error(DDQ_EINVAL, "select: null output");
  if (scratch_bytes < filter_scratch_bytes(n_cap)) return set_error(DDQ_EINVAL, "select: scratch too small");
  if (in_tids && !d_in_count) return set_error(DDQ_EINVAL, "select: TID input needs a device count");
  FilterArgs a;
  a.preds = preds;
  a.n_preds = n_preds;
  a.in_tids = in_tids;
  a.d_in_count = d_in_count;
  a.n_cap = n_cap;
  a.carry_in = carry_in;
  a.carry_out = carry_out;
  a.n_carry = n_carry;
  a.out_tids = out_tids;
  a.d_out_count = d_out_count;
  a.scratch = scratch;
  return cuda_status(launch_filter(a, (cudaStream_t)stream), "ddq_op_select");
}

ddq_status ddq_op_hash_init(uint64_t* table, uint32_t capacity, void* stream) {
  if (!table || capacity < 2 || (capacity & (capacity - 1)))
    return set_error(DDQ_EINVAL, "hash_init: capacity must be a power of two >= 2");
  return cuda_status(launch_hash_init(table, capacity, (cudaStream_t)stream), "ddq_op_hash_init");
}

ddq_status ddq_op_hash_build(const int32_t* keys, const int32_t* payload, const int32_t* in_tids,
                             const uint32_t* d_in_count, int64_t n_cap, uint64_t* table, uint32_t capacity,
                             uint32_t* d_error, void* stream) {
  if (ddq_status s = check_cap(n_cap)) return s;
  if (!keys || !table || !d_error || capacity < 2 || (capacity & (capacity - 1)))
    return set_error(DDQ_EINVAL, "hash_build: bad arguments");
  if (in_tids && !d_in_count) return set_error(DDQ_EINVAL, "hash_build: TID input needs a device count");
  return cuda_status(launch_hash_build(keys, payload, in_tids, d_in_count, n_cap, table, capacity, d_error,
                                       (cudaStream_t)stream),
                     "ddq_op_hash_build");
}

ddq_status ddq_op_hash_probe(const uint64_t* table, uint32_t capacity, const int32_t* fk, const int32_t* in_tids,
                             const uint32_t* d_in_count, int64_t n_cap, const int32_t* const* carry_in,
                             int32_t* const* carry_out, int32_t n_carry, int32_t* out_tids, int32_t* out_payload,
                             uint32_t* d_out_count, void* scratch, size_t scratch_bytes, void* stream) {
  if (ddq_status s = check_cap(n_cap)) return s;
  if (!table || (n_cap > 0 && !fk) || capacity < 2 || (capacity & (capacity - 1)))
    return set_error(DDQ_EINVAL, "hash_probe: bad table / fk");
  if (n_carry < 0 || n_carry > DDQ_MAX_CARRY) return set_error(DDQ_EINVAL, "hash_probe: bad carry count");
  if (!out_tids || !d_out_count || !scratch) return set_error(DDQ_EINVAL, "hash_probe: null output");
  if (scratch_bytes < filter_scratch_bytes(n_cap)) return set_error(DDQ_EINVAL, "hash_probe: scratch too small");
  if (in_tids && !d_in_count) return set_error(DDQ_EINVAL, "hash_probe: TID input needs a device count");
  FilterArgs a;
  a.probe = true;
  a.table = table;
  a.capacity = capacity;
  a.fk = fk;
  a.out_payload = out_payload;
  a.in_tids = in_tids;
  a.d_in_count = d_in_count;
  a.n_cap = n_cap;
  a.carry_in = carry_in;
  a.carry_out = carry_out;
  a.n_carry = n_carry;
  a.out_tids = out_tids;
  a.d_out_count = d_out_count;
  a.scratch = scratch;
  return cuda_status(launch_filter(a, (cudaStream_t)stream), "ddq_op_hash_probe");
}

ddq_status ddq_op_star(const ddq_dev_term* terms, int32_t n_terms, int64_t n_rows, int32_t* out_tids,
                       uint32_t* d_out_count, int64_t out_cap, uint32_t* d_overflow, void* stream) {
  if (ddq_status s = check_cap(n_rows)) return s;
  if (!terms || n_terms < 1 || n_terms > 4) return set_error(DDQ_EINVAL, "star: 1..4 terms");
  if (!out_tids || !d_out_count) return set_error(DDQ_EINVAL, "star: null output");
  for (int j = 0; j < n_terms; j++) {
    const ddq_dev_term& t = terms[j];
    if (t.kind != DDQ_TERM_PRED && t.kind != DDQ_TERM_PROBE) return set_error(DDQ_EINVAL, "star: bad term kind");
    if ((n_rows > 0 && !t.col) || ((uintptr_t)t.col & 15)) return set_error(DDQ_EINVAL, "star: column must be 16-byte aligned");
    if (t.width != 4 && t.width != 8) return set_error(DDQ_EINVAL, "star: bad width");
    if (t.kind == DDQ_TERM_PRED) {
      if (t.pred_kind != DDQ_PRED_RANGE && t.pred_kind != DDQ_PRED_IN && t.pred_kind != DDQ_PRED_BITSET) return set_error(DDQ_EINVAL, "star: bad predicate");
      if (t.pred_kind == DDQ_PRED_IN && (t.n_in < 0 || t.n_in > DDQ_MAX_IN)) return set_error(DDQ_EINVAL, "star: IN list too long");
    } else {
      if (t.width != 4) return set_error(DDQ_EINVAL, "star: probe keys are int32");
      if (!t.index && (!t.table || t.capacity < 2 || (t.capacity & (t.capacity - 1))))
        return set_error(DDQ_EINVAL, "star: probe needs a join index or a hash table");
      if (t.index && t.range == 0) return set_error(DDQ_EINVAL, "star: empty join index range");
    }
  }
  return cuda_status(launch_star(terms, n_terms, n_rows, out_tids, d_out_count, out_cap, d_overflow, (cudaStream_t)stream),
                     "ddq_op_star");
}

size_t ddq_op_join_index_bytes(uint32_t range) { return join_index_bytes(range); }

ddq_status ddq_op_join_index_init(void* index, uint32_t range, void* stream) {
  if (!index || range == 0) return set_error(DDQ_EINVAL, "join_index_init: bad arguments");
  return cuda_status(join_index_init(index, range, (cudaStream_t)stream), "ddq_op_join_index_init");
}

ddq_status ddq_op_join_index_build(const int32_t* keys, const int32_t* payload, const int32_t* in_tids,
                                   const uint32_t* d_in_count, int64_t n_cap, int32_t key_min, uint32_t range,
                                   void* index, uint32_t* d_error, void* stream) {
  if (ddq_status s = check_cap(n_cap)) return s;
  if ((n_cap > 0 && !keys) || !index || !d_error || range == 0)
    return set_error(DDQ_EINVAL, "join_index_build: bad arguments");
  if (in_tids && !d_in_count) return set_error(DDQ_EINVAL, "join_index_build: TID input needs a device count");
  return cuda_status(launch_join_index_build(keys, payload, in_tids, d_in_count, n_cap, key_min, range, index, d_error,
                                             (cudaStream_t)stream),
                     "ddq_op_join_index_build");
}

ddq_status ddq_op_join_index_probe(const void* index, int32_t key_min, uint32_t range, const int32_t* fk,
                                   const int32_t* in_tids, const uint32_t* d_in_count, int64_t n_cap,
                                   const int32_t* const* carry_in, int32_t* const* carry_out, int32_t n_carry,
                                   int32_t* out_tids, int32_t* out_payload, uint32_t* d_out_count, void* scratch,
                                   size_t scratch_bytes, void* stream) {
  if (ddq_status s = check_cap(n_cap)) return s;
  if (!index || range == 0 || (n_cap > 0 && !fk)) return set_error(DDQ_EINVAL, "join_index_probe: bad index / fk");
  if (n_carry < 0 || n_carry > DDQ_MAX_CARRY) return set_error(DDQ_EINVAL, "join_index_probe: bad carry count");
  if (!out_tids || !d_out_count || !scratch) return set_error(DDQ_EINVAL, "join_index_probe: null output");
  if (scratch_bytes < filter_scratch_bytes(n_cap)) return set_error(DDQ_EINVAL, "join_index_probe: scratch too small");
  if (in_tids && !d_in_count) return set_error(DDQ_EINVAL, "join_index_probe: TID input needs a device count");
  FilterArgs a;
  a.probe = true;
  a.bitmap = join_index_bitmap(const_cast<void*>(index));
  a.payarr = join_index_payload(const_cast<void*>(index), range);
  a.coarse = join_index_coarse(const_cast<void*>(index), range);
  a.key_min = key_min;
  a.range = range;
  a.fk = fk;
  a.out_payload = out_payload;
  a.in_tids = in_tids;
  a.d_in_count = d_in_count;
  a.n_cap = n_cap;
  a.carry_in = carry_in;
  a.carry_out = carry_out;
  a.n_carry = n_carry;
  a.out_tids = out_tids;
  a.d_out_count = d_out_count;
  a.scratch = scratch;
  return cuda_status(launch_filter(a, (cudaStream_t)stream), "ddq_op_join_index_probe");
}

ddq_status ddq_op_gather(const void* col, int32_t width, const int32_t* tids, const uint32_t* d_count,
                         int64_t n_cap, void* out, void* stream) {
  if (ddq_status s = check_cap(n_cap)) return s;
  if ((n_cap > 0 && (!col || !tids || !out)) || (width != 4 && width != 8)) return set_error(DDQ_EINVAL, "gather: bad arguments");
  return cuda_status(launch_gather(col, width, tids, d_count, n_cap, out, (cudaStream_t)stream), "ddq_op_gather");
}

size_t ddq_op_groupby_table_bytes(uint32_t capacity, int32_t n_aggs) { return groupby_table_bytes(capacity, n_aggs); }

ddq_status ddq_op_groupby_init(void* table, uint32_t capacity, int32_t n_aggs, void* stream) {
  if (!table || capacity < 2 || (capacity & (capacity - 1)) || n_aggs < 0 || n_aggs > DDQ_MAX_AGGS)
    return set_error(DDQ_EINVAL, "groupby_init: bad arguments");
  return cuda_status(launch_groupby_init(table, capacity, n_aggs, (cudaStream_t)stream), "ddq_op_groupby_init");
}

ddq_status ddq_op_groupby(const int32_t* tids, const uint32_t* d_count, int64_t n_cap, const int32_t* const* key_vec,
                          const int32_t* const* key_col, int32_t n_keys, const int32_t* key_bits,
                          const ddq_dev_agg* aggs, int32_t n_aggs, void* table, uint32_t capacity, uint32_t* d_error,
                          void* stream) {
  if (ddq_status s = check_cap(n_cap)) return s;
  {
    int bits = 0;
    for (int k = 0; k < n_keys && k < DDQ_MAX_KEYS; k++) bits += (key_bits && key_bits[k] > 0) ? key_bits[k] : 21;
    if (bits > 63) return set_error(DDQ_EINVAL, "groupby: packed key wider than 63 bits");
  }
  if (!tids || !table || !d_error || capacity < 2 || (capacity & (capacity - 1)))
    return set_error(DDQ_EINVAL, "groupby: bad arguments");
  if (n_keys < 0 || n_keys > DDQ_MAX_KEYS || n_aggs < 1 || n_aggs > DDQ_MAX_AGGS || !aggs)
    return set_error(DDQ_EINVAL, "groupby: bad key/aggregate count");
  for (int k = 0; k < n_keys; k++)
    if (!((key_vec && key_vec[k]) || (key_col && key_col[k]))) return set_error(DDQ_EINVAL, "groupby: null key");
  for (int a = 0; a < n_aggs; a++) {
    int need = aggs[a].kind == DDQ_AGG_COUNT ? 0 : (aggs[a].kind == DDQ_AGG_SUM || aggs[a].kind == DDQ_AGG_MIN) ? 1
             : aggs[a].kind == DDQ_AGG_SUM_MUL_100M_100P ? 3 : 2;
    if (aggs[a].kind < DDQ_AGG_COUNT || aggs[a].kind > DDQ_AGG_MIN)
      return set_error(DDQ_EINVAL, "groupby: bad aggregate kind");
    for (int j = 0; j < need; j++)
      if (!aggs[a].arg[j] || (aggs[a].width[j] != 4 && aggs[a].width[j] != 8))
        return set_error(DDQ_EINVAL, "groupby: bad aggregate argument");
  }
  return cuda_status(launch_groupby(tids, d_count, n_cap, key_vec, key_col, n_keys, key_bits, aggs, n_aggs, table,
                                    capacity,
                                    d_error, (cudaStream_t)stream),
                     "ddq_op_groupby");
}

ddq_status ddq_op_groupby_compact(const void* table, uint32_t capacity, int32_t n_aggs, int64_t* out_keys,
                                  int64_t* out_accs, uint32_t* d_out_groups, void* stream) {
  if (!table || !out_keys || !out_accs || !d_out_groups || capacity < 2 || (capacity & (capacity - 1)))
    return set_error(DDQ_EINVAL, "groupby_compact: bad arguments");
  return cuda_status(launch_groupby_compact(table, capacity, n_aggs, out_keys, out_accs, d_out_groups,
                                            (cudaStream_t)stream),
                     "ddq_op_groupby_compact");
}

}  // extern "C"
