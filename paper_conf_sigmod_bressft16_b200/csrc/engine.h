// engine.h -- internal structures of the libddq database (column store, device
// cache, heap-budget allocator, operator runners).
#pragma once
#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include <cuda_runtime.h>

#include "../../include/ddq.h"

namespace ddq {

ddq_status set_error(ddq_status s, const std::string& msg);
ddq_status cuda_status(cudaError_t e, const char* where);
uint64_t now_ns();

// ---- heap-budget allocator (P:62 heap; P:113 fail fast, never wait) --------
class Heap {
 public:
  ddq_status init(uint64_t bytes, uint32_t fault_every);
  ~Heap();
  void* try_alloc(uint64_t bytes);  // nullptr on failure (no waiting)
  void free(void* p);
  uint64_t used() const { return used_; }
  uint64_t peak() const { return peak_; }
  uint64_t capacity() const { return cap_; }
  void reset_peak() { peak_ = used_; }

 private:
  std::mutex mu_;
  char* base_ = nullptr;
  uint64_t cap_ = 0, used_ = 0, peak_ = 0;
  uint32_t fault_every_ = 0;
  uint64_t n_allocs_ = 0;
  std::map<uint64_t, uint64_t> free_;   // offset -> size
  std::map<uint64_t, uint64_t> alloc_;  // offset -> size
};

struct Column {
  std::string name;
  int table = -1;
  int type = DDQ_I32;
  int width = 4;
  int64_t n = 0;
  int64_t vmin = 0, vmax = -1;  // value range (computed at load; sizes join indexes)
  void* host = nullptr;   // pinned host copy
  void* host_packed = nullptr;  // frame-of-reference bit-packed pinned copy (transfer.cu)
  int tw = 0;                   // its bits per value (1..32); 0 = none, the raw copy is sent
  // dictionary transfer code: the packed values are ranks into this sorted pinned
  // int64 array of the column's distinct values (sent with them), instead of
  // value - vmin, when that is fewer bytes (e.g. yyyymmdd dates: 12 bits, not 17)
  int64_t* host_tdict = nullptr;
  int64_t tdict_n = 0;
  void* dev = nullptr;    // device cache copy or nullptr
  std::atomic<uint64_t> access{0};
  std::atomic<uint64_t> last_access{0};
  int refs = 0;             // running operators using `dev`
  bool evict_pending = false;
  bool on_demand = false;   // cached by operator-driven placement (GPU-only arm)
  bool loading = false;     // H2D copy in flight (db->mu released; waiters use cache_cv)
  // order-preserving dictionary (reading O4): code = index; set once, read-only after
  std::vector<std::string> dict;
};

struct Table {
  std::string name;
  int64_t n_rows = 0;
  int64_t row_begin = 0;
  bool partitioned = false;  // row-sharded across ranks (ddq_table_set_partitioned)
  std::vector<int> cols;
};

struct Vec {
  void* ptr = nullptr;  // device or host, aligned with the TID list
  int width = 4;
  bool host = false;
};

// A materialised intermediate: TIDs + aligned vectors, on one processor.
struct Inter {
  bool on_host = false;
  bool all_rows = false;   // implicit TIDs 0..cap-1
  int table = -1;
  int32_t* tids = nullptr;
  uint32_t* bits = nullptr;     // row bitmap instead of a TID list (prepared plans, see bits_out)
  uint32_t* d_count = nullptr;  // device count cell (GPU)
  int64_t cap = 0;              // capacity (upper bound on count)
  int64_t count = -1;           // exact count when known on the host
  std::vector<Vec> vecs;
  // hash build output
  uint64_t* table_ptr = nullptr;
  uint32_t table_cap = 0;
  uint32_t* d_error = nullptr;
  // host-side hash table (host build)
  std::shared_ptr<std::vector<uint64_t>> host_table;
  // direct-mapped join index (device: jidx; host copy: h_bitmap/h_payarr)
  void* jidx = nullptr;
  int32_t jmin = 0;
  uint32_t jrange = 0;
  std::shared_ptr<std::vector<uint32_t>> h_bitmap;
  std::shared_ptr<std::vector<int32_t>> h_payarr;
  // aggregate output
  void* gb_table = nullptr;
  uint32_t gb_cap = 0;
  int64_t* gb_keys = nullptr;
  int64_t* gb_accs = nullptr;
  uint32_t* gb_groups = nullptr;
  uint32_t* d_rows = nullptr;  // AGGREGATE with fused predicates: rows that passed (profile)
  // host aggregate result (host executor)
  std::shared_ptr<std::vector<int64_t>> h_keys, h_accs;
  int64_t h_groups = 0;
  // allocations owned by this intermediate (heap or host)
  std::vector<void*> heap_blocks;
  std::vector<void*> host_blocks;
};

struct Stats {
  std::atomic<uint64_t> h2d_bytes{0}, d2h_bytes{0}, h2d_ns{0}, d2h_ns{0}, gpu_ops{0}, host_ops{0}, aborts{0},
      wasted_ns{0}, cache_hits{0}, cache_misses{0}, queries_done{0};
};

struct QueryState;

}  // namespace ddq

struct ddq_db {
  ddq_config cfg{};
  int device = 0;
  cudaStream_t copy_stream = nullptr;
  // device column cache: a stream-ordered pool that keeps freed blocks (release
  // threshold = max), so evict + re-cache reuses device memory without a
  // cudaMalloc/cudaFree round trip through the driver per column
  cudaMemPool_t cache_pool = nullptr;
  // freed cache blocks by exact size (evict + re-cache of the same columns reuses
  // them without the pool allocator; db->mu guards it)
  std::multimap<size_t, void*> cache_free;
  ddq::Heap heap;
  std::mutex mu;  // catalog + cache
  std::condition_variable cache_cv;
  std::vector<ddq::Table> tables;
  std::vector<std::unique_ptr<ddq::Column>> cols;
  uint64_t cache_used = 0;
  std::atomic<uint64_t> clock{0};
  ddq::Stats stats;
  // chopping executor
  std::mutex qmu;
  std::condition_variable qcv;
  std::deque<std::pair<std::shared_ptr<ddq::QueryState>, int>> gpu_ready, host_ready;
  std::map<int64_t, std::shared_ptr<ddq::QueryState>> queries;
  int64_t next_query = 1;
  bool stopping = false;
  std::vector<std::thread> workers;
  int busy_gpu = 0;
  // admission control (ddq_config.max_queries): queries running / waiting (qmu)
  int running_queries = 0;
  std::deque<std::shared_ptr<ddq::QueryState>> admit_queue;
  // streamed cold path (ddq_config.prefetch): columns queued for H2D (qmu), copy thread
  std::deque<int> prefetch_queue;
  std::thread prefetcher;
  std::thread placer;  // periodic Algorithm 1 (ddq_config.placement_period_ms)
  void* dist = nullptr;  // multi-GPU state (dist.cpp), or null
};

namespace ddq {

// Runs one operator on the GPU, allocating outputs from the heap (fail fast).
// exact_caps: if non-null, output capacities to use (prepared plans), else the
// input capacity.  Returns DDQ_ENOMEM_DEVICE when an allocation fails.
struct GpuOpCtx {
  ddq_db* db;
  cudaStream_t stream;
  const std::vector<Inter>* inters;  // outputs of earlier ops (same plan)
  int64_t forced_cap = -1;           // output capacity override
  bool count_column_access = true;
  const std::vector<void*>* reuse = nullptr;  // replay on existing buffers
  // a dense semi-join probe writes its survivors as a row bitmap (1 bit per row)
  // instead of a TID list: set by ddq_prepare when every consumer reads bitmaps
  bool bits_out = false;
  // prepared plans on a multi-GPU database: builds over replicated tables run once and
  // are broadcast (dist.cpp); off for calibration runs and the chopping driver
  bool dist = false;
};
// dist.cpp
void dist_free(ddq_db* db);
bool dist_build_receives(ddq_db* db, const ddq_op& op);
ddq_status dist_build_broadcast(ddq_db* db, const ddq_op& op, void* buf, size_t bytes, cudaStream_t st);
bool dist_serial_capture(ddq_db* db);
void count_accesses(ddq_db* db, const ddq_op& op);
void driver_start(ddq_db* db);
void driver_stop(ddq_db* db);
ddq_status run_gpu_op(GpuOpCtx& ctx, const ddq_op& op, Inter& out);
// Host executor (CPU fallback handler for every operator).
ddq_status run_host_op(ddq_db* db, const ddq_op& op, const std::vector<Inter>& inters, Inter& out);
void release_inter(ddq_db* db, Inter& x);
ddq_status inter_to_host(ddq_db* db, Inter& x, cudaStream_t st);
// unique_keys: the groups come from ONE group table (a prepared plan, a driver
// query), so equal packed keys cannot occur and the merge step is skipped
ddq_status finalize_result(const ddq_op& root, int64_t n_groups, const int64_t* keys, const int64_t* accs,
                           ddq_result** out, bool unique_keys = false);
// S8(a7) decode: attach the dictionary strings of the result's keys (key_str)
void decode_result_keys(ddq_db* db, const ddq_plan& plan, ddq_result* r);
int64_t pow2_at_least(int64_t x);
const ddq::Column* col_of(ddq_db* db, int c);
bool fits_int32(const ddq::Column& c);
// columns an operator reads (driver.cpp): placement checks and cache references
std::vector<int> op_columns(const ddq_op& op);
void evict_column_locked(ddq_db* db, int c);
void release_column_refs(ddq_db* db, const std::vector<int>& cols);

}  // namespace ddq
