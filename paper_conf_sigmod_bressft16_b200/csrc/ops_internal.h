// ops_internal.h -- host-side launch interfaces of the libddq kernels.
#pragma once
#include <cstddef>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#include "../../include/ddq.h"

namespace ddq {

// ---- buffer initialisation (counters, error cells, bitmaps, empty tables) ----
// Every operator's "zero this / fill that before the kernel" goes through
// init_fill.  A prepared plan records them in its eager run and captures ONE
// multi-range fill kernel at the root of its graph instead (fill_hoist().skip
// during capture), so no memset node sits on the operator chain.
struct FillRec {
  void* ptr;
  uint64_t n64;      // 8-byte words
  uint64_t pattern;  // 64-bit fill value
};
struct FillHoist {
  std::vector<FillRec>* rec = nullptr;  // record (and still perform) every fill
  bool skip = false;                    // fills were hoisted: do nothing
};
FillHoist& fill_hoist();  // per host thread
// bytes are rounded up to a multiple of 8 (every target allocation is padded)
// cold-path transfer encoding (transfer.cu): frame-of-reference byte packing
size_t packed_bytes(int64_t n, int tw);
// dict: null = frame of reference (value = base + code), else the sorted distinct
// values (int64, device) the codes rank into
cudaError_t launch_unpack(const void* packed, int tw, int64_t base, void* out, int width, int64_t n, cudaStream_t st,
                          const void* dict = nullptr);
cudaError_t init_fill(void* ptr, size_t bytes, uint64_t pattern, cudaStream_t st);
cudaError_t launch_delay(uint64_t ns, cudaStream_t st);  // profiling: hold the stream
bool ws_masked_probe_smem(bool join_index, uint32_t range_or_capacity, int64_t n_rows, bool pay);
cudaError_t launch_multi_fill(const std::vector<FillRec>& recs, cudaStream_t st);

struct FilterArgs {
  const ddq_dev_pred* preds = nullptr;
  int n_preds = 0;
  bool probe = false;
  bool no_smem = false;
  bool stable = false;  // dense inputs: force the single-pass look-back kernel (ascending TIDs)
  bool fk_by_pos = false;          // probe keys from an aligned vector (TID inputs)
  const int32_t* eq_a = nullptr;   // FILTER_EQ positional vectors (TID inputs)
  const int32_t* eq_b = nullptr;
  int eq_cmp = 0;                  // FILTER_EQ comparison: DDQ_CMP_EQ / _LT / _NE
  const uint64_t* table = nullptr;
  uint32_t capacity = 0;
  // direct-mapped join index (probe): bitmap + payload array over [key_min, key_min+range)
  const uint32_t* bitmap = nullptr;
  const int32_t* payarr = nullptr;
  const uint32_t* coarse = nullptr;  // the index's coarse bitmap (join_index_coarse), or null
  int32_t key_min = 0;
  uint32_t range = 0;
  const int32_t* fk = nullptr;
  int32_t* out_payload = nullptr;
  const int32_t* in_tids = nullptr;
  const uint32_t* d_in_count = nullptr;
  // row bitmap input (instead of in_tids; n_cap = the table's rows): 16 words per
  // 512-row tile; row bitmap output of a dense probe (instead of out_tids); see dense.cu
  const uint32_t* in_bits = nullptr;
  uint32_t* out_bits = nullptr;
  int64_t n_cap = 0;
  const int32_t* const* carry_in = nullptr;
  int32_t* const* carry_out = nullptr;
  int n_carry = 0;
  int32_t* out_tids = nullptr;
  uint32_t* d_out_count = nullptr;
  int64_t out_cap = 0;            // 0: n_cap
  uint32_t* d_overflow = nullptr; // set to 4 when survivors exceed out_cap
  void* scratch = nullptr;
};

size_t filter_scratch_bytes(int64_t n_cap);
bool scan_supported(const FilterArgs& a);
cudaError_t launch_scan(const FilterArgs& a, cudaStream_t st);
cudaError_t launch_filter(const FilterArgs& a, cudaStream_t st);
// warp-autonomous filter kernels (dense.cu): dense probes and every TID-input operator
bool ws_supported(const FilterArgs& a);
inline size_t row_bitmap_bytes(int64_t rows) { return (size_t)((rows + 511) / 512) * 64; }
cudaError_t launch_ws(const FilterArgs& a, cudaStream_t st);

// HASH_BUILD with a fused selection (a BUILD op carrying predicates): rows that
// fail any predicate are not inserted -- the select -> build pair of a dimension
// table in one kernel, without the intermediate TID list.
struct BuildPreds {
  int32_t key_set = 0;  // 1: duplicate build keys allowed (semi-join key set, ddq_op.build_key_set);
                        // 2: duplicates allowed, the payload is their MINIMUM (a MIN-aggregating
                        //    build: TPC-H Q2's decorrelated min(ps_supplycost) per part)
  int32_t n = 0;
  ddq_dev_pred p[DDQ_MAX_PREDS];
  const long long* payload64 = nullptr;  // int64 payload column whose values fit int32 (checked
                                         // from the column's load-time range), narrowed exactly
};

cudaError_t launch_hash_init(uint64_t* table, uint32_t capacity, cudaStream_t st);
cudaError_t launch_hash_build(const int32_t* keys, const int32_t* payload, const int32_t* in_tids,
                              const uint32_t* d_in_count, int64_t n_cap, uint64_t* table, uint32_t capacity,
                              uint32_t* d_error, cudaStream_t st, const BuildPreds* preds = nullptr);
cudaError_t launch_star(const ddq_dev_term* terms, int n_terms, int64_t n_rows, int32_t* out_tids,
                        uint32_t* d_out_count, int64_t out_cap, uint32_t* d_overflow, cudaStream_t st);

// Direct-mapped join index over [key_min, key_min + range):
//   [membership bitmap, range bits][payload int32 x range][coarse bitmap]
// The coarse bitmap (1 bit per 2^cg keys, OR of the group; set by the build) exists
// only when the bitmap is too large for one SM's shared memory next to a probe's
// compaction ring (range > JI_SMEM_KEYS); probes then filter with the coarse bitmap
// in shared memory and read exact bits from L2 for coarse hits only (dense.cu).
// thresholds (defaults 1.5 M keys, 160 KB; env DDQ_JI_SMEM_KEYS / DDQ_JI_COARSE_MAX
// override them for tests that force coarse bitmaps on small data)
uint32_t ji_smem_keys();
size_t ji_coarse_max();
inline size_t ji_fine_bytes(uint32_t range) { return ((((size_t)range + 31) / 32 * 4 + 15) / 16) * 16; }
inline size_t ji_coarse_bytes_cg(uint32_t range, uint32_t cg) {
  return (((size_t)(range >> cg) + 1 + 31) / 32 * 4 + 15) / 16 * 16;
}
inline uint32_t join_index_cg(uint32_t range) {
  if (range <= ji_smem_keys()) return 0;
  uint32_t cg = 1;
  while (cg < 16 && ji_coarse_bytes_cg(range, cg) > ji_coarse_max()) cg++;
  // > 8 keys per coarse bit filters little (TPC-H orders, 45 M keys at 3 %
  // selected: 86 % of the coarse bits set) and costs build atomics: no coarse bitmap
  return cg <= 3 ? cg : 0;
}
inline size_t join_index_coarse_bytes(uint32_t range) {
  const uint32_t cg = join_index_cg(range);
  return cg ? ji_coarse_bytes_cg(range, cg) : 0;
}
size_t join_index_bytes(uint32_t range);
inline uint32_t* join_index_bitmap(void* idx) { return reinterpret_cast<uint32_t*>(idx); }
inline int32_t* join_index_payload(void* idx, uint32_t range) {
  return reinterpret_cast<int32_t*>(reinterpret_cast<char*>(idx) + ji_fine_bytes(range));
}
inline uint32_t* join_index_coarse(void* idx, uint32_t range) {
  return join_index_cg(range) ? reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(idx) + ji_fine_bytes(range) +
                                                            ((size_t)range * 4 + 15) / 16 * 16)
                              : nullptr;
}
// zero the membership and coarse bitmaps of an index (the payload needs no init)
cudaError_t join_index_init(void* idx, uint32_t range, cudaStream_t st);
// the coarse words of a host-side membership bitmap (a host-built index moving to the GPU)
void join_index_coarse_host(const uint32_t* bitmap, uint32_t range, uint32_t* coarse);
cudaError_t launch_join_index_build(const int32_t* keys, const int32_t* payload, const int32_t* in_tids,
                                    const uint32_t* d_in_count, int64_t n_cap, int32_t key_min, uint32_t range,
                                    void* index, uint32_t* d_error, cudaStream_t st,
                                    const BuildPreds* preds = nullptr);
// dimension attribute fetch (GATHER through a join): join index (bitmap != NULL) or hash table
cudaError_t launch_fetch(const int32_t* tids, const uint32_t* d_count, int64_t n_cap, const int32_t* fk,
                         const uint32_t* bitmap, const int32_t* payarr, int32_t key_min, uint32_t range,
                         const uint64_t* table, uint32_t capacity, int32_t* out, cudaStream_t st);
cudaError_t launch_gather(const void* col, int width, const int32_t* tids, const uint32_t* d_count,
                          int64_t n_cap, void* out, cudaStream_t st);

size_t groupby_table_bytes(uint32_t capacity, int n_aggs);
cudaError_t launch_groupby_init(void* table, uint32_t capacity, int n_aggs, cudaStream_t st);
cudaError_t launch_groupby(const int32_t* tids, const uint32_t* d_count, int64_t n_cap,
                           const int32_t* const* key_vec, const int32_t* const* key_col, int n_keys,
                           const int32_t* key_bits,
                           const ddq_dev_agg* aggs, int n_aggs, void* table, uint32_t capacity,
                           uint32_t* d_error, cudaStream_t st);
// AGGREGATE with fused predicates (reading O26): only input rows passing every
// predicate contribute; *d_rows (optional) += the number that did.
// warp-autonomous aggregation for <= 2 aggregates and small group counts (agg.cu)
// dense small-domain aggregation over every row of a table (agg.cu)
bool agg_dense_supported(int64_t n_rows, const struct BuildPreds* preds, const int32_t* const* key_col, int n_keys,
                         const int32_t* key_bits, const ddq_dev_agg* aggs, int n_aggs);
cudaError_t launch_agg_dense(int64_t n_rows, const int32_t* const* key_col, int n_keys, const int32_t* key_bits,
                             const ddq_dev_agg* aggs, int n_aggs, void* table, uint32_t capacity, uint32_t* d_error,
                             cudaStream_t st, const struct BuildPreds* preds, uint32_t* d_rows, double max_row_abs = -1);
cudaError_t launch_iota(int32_t* out, int64_t n, uint32_t* d_count, cudaStream_t st);
// A probe / fetch term fused into the aggregation at TIDs (reading O37):
// the fk column is gathered at the row, looked up in a join index (bitmap +
// payload array) or an open-addressing hash table; a PROBE drops rows whose key
// misses, a FETCH keeps them with payload INT32_MIN; `emit` >= 0 stores the payload
// in slot `emit` (0..2) for use as a group key (AggKeys::pay).
struct AggTerm {
  int32_t kind = 0;  // DDQ_TERM_PROBE | DDQ_TERM_FETCH
  int32_t emit = -1;
  const int32_t* fk = nullptr;
  const uint32_t* bitmap = nullptr;  // join index (or null: hash table)
  const int32_t* payarr = nullptr;
  int32_t key_min = 0;
  uint32_t range = 0;
  const uint64_t* table = nullptr;
  uint32_t capacity = 0;
};
struct AggTerms {
  int32_t n = 0;
  AggTerm t[4];
  int32_t key_pay[3] = {-1, -1, -1};  // key k = payload slot key_pay[k] (>= 0) instead of a vector / column
};
bool agg_ws_supported(const int32_t* tids, const int32_t* const* key_vec, int n_keys, int n_aggs,
                      uint32_t capacity);
cudaError_t launch_agg_ws(const int32_t* tids, const uint32_t* d_count, int64_t n_cap,
                          const int32_t* const* key_vec, const int32_t* const* key_col, int n_keys,
                          const int32_t* key_bits, const ddq_dev_agg* aggs, int n_aggs, void* table,
                          uint32_t capacity, uint32_t* d_error, cudaStream_t st,
                          const BuildPreds* preds = nullptr, uint32_t* d_rows = nullptr,
                          const AggTerms* terms = nullptr);
cudaError_t launch_groupby_compact(const void* table, uint32_t capacity, int n_aggs, int64_t* out_keys,
                                   int64_t* out_accs, uint32_t* d_out_groups, cudaStream_t st);

int num_sms();

}  // namespace ddq
