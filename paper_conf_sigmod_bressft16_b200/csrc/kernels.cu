// kernels.cu -- hash build (S8(a3)), positional gather (S8(a5)) and group-by
// aggregation (S8(a6)) for sm_100a.
//
// Group-by design: every warp aggregates its 32 rows per
// distinct key first (__match_any_sync + a log-step peer reduction), the lowest
// lane of each key group then updates a per-CTA shared-memory hash table, and each
// CTA merges its table into the global open-addressing table once at the end.
// Accumulators are exact int128 (two 64-bit atomics with carry), so results are
// bit-identical whatever the scheduling (integer addition is associative).
#include <algorithm>
#include <climits>
#include <cstdint>
#include <cstring>
#include <cstdlib>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "ops_internal.h"

namespace ddq {

int num_sms() {
  static const int sms = [] {
    int dev = 0, v = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    return v <= 0 ? 1 : v;
  }();
  return sms;
}

static inline uint32_t read_count_host_cap(int64_t n_cap) { return (uint32_t)n_cap; }

// ----------------------------------------------------------------- hash build
__device__ __forceinline__ bool build_row_passes(const BuildPreds& bp, int32_t r) {
  for (int i = 0; i < bp.n; i++) {
    const ddq_dev_pred& p = bp.p[i];
    const int64_t v = col_at(p.col, p.width, r);
    bool m = false;
    if (p.kind == DDQ_PRED_RANGE) {
      m = v >= p.lo && v <= p.hi;
    } else if (p.kind == DDQ_PRED_BITSET) {
      m = bitset_hit(p.in_vals, p.lo, v);
    } else {
#pragma unroll
      for (int j = 0; j < DDQ_MAX_IN; j++) m |= j < p.n_in && v == p.in_vals[j];
    }
    if (!m) return false;
  }
  return true;
}

__global__ void hash_init_kernel(uint64_t* table, uint32_t capacity) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < capacity; i += gridDim.x * blockDim.x)
    table[i] = HT_EMPTY;
}

__global__ void hash_build_kernel(const int32_t* __restrict__ keys, const int32_t* __restrict__ payload,
                                  const int32_t* __restrict__ in_tids, const uint32_t* d_in_count,
                                  uint32_t n_static, uint64_t* table, uint32_t capacity, int shift,
                                  uint32_t* d_error, const __grid_constant__ BuildPreds bp) {
  const uint32_t n = d_in_count ? ld_relaxed_u32(d_in_count) : n_static;
  const uint32_t mask = capacity - 1;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t r = in_tids ? in_tids[i] : (int32_t)i;
    if (bp.n && !build_row_passes(bp, r)) continue;
    const int32_t k = keys[r];
    const int32_t v = bp.payload64 ? (int32_t)bp.payload64[r] : payload ? payload[r] : r;
    if (k == INT32_MIN) {
      atomicMax(d_error, 3u);
      continue;
    }
    const uint64_t slot = ((uint64_t)(uint32_t)k << 32) | (uint32_t)v;
    uint32_t h = ht_hash(k, shift);
    uint32_t probes = 0;
    while (true) {
      unsigned long long old = atomicCAS(reinterpret_cast<unsigned long long*>(table + h),
                                         (unsigned long long)HT_EMPTY, (unsigned long long)slot);
      if (old == HT_EMPTY) break;
      if (ht_key(old) == k) {  // PKs must be unique (reading O13) unless a key set
        if (!bp.key_set) atomicMax(d_error, 1u);
        // MIN build: lower the slot's payload until it holds the smallest value
        while (bp.key_set == 2 && v < ht_val(old)) {
          const unsigned long long seen = atomicCAS(reinterpret_cast<unsigned long long*>(table + h), old,
                                                    (unsigned long long)slot);
          if (seen == old) break;
          old = seen;
        }
        break;
      }
      h = (h + 1) & mask;
      if (++probes >= capacity) {
        atomicMax(d_error, 2u);
        break;
      }
    }
  }
}

cudaError_t launch_hash_init(uint64_t* table, uint32_t capacity, cudaStream_t st) {
  return init_fill(table, (size_t)capacity * 8, HT_EMPTY, st);
}

// ---- buffer initialisation -------------------------------------------------
constexpr int MF_MAX = 48;
struct MultiFill {
  int32_t n;
  FillRec r[MF_MAX];
};

__global__ void multi_fill_kernel(const __grid_constant__ MultiFill M) {
  const FillRec& f = M.r[blockIdx.y];
  uint64_t* p = reinterpret_cast<uint64_t*>(f.ptr);
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < f.n64; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = f.pattern;
}

FillHoist& fill_hoist() {
  static thread_local FillHoist h;
  return h;
}

cudaError_t launch_multi_fill(const std::vector<FillRec>& recs, cudaStream_t st) {
  for (size_t b = 0; b < recs.size(); b += MF_MAX) {
    MultiFill M{};
    M.n = (int32_t)std::min<size_t>(MF_MAX, recs.size() - b);
    uint64_t mx = 1;
    for (int i = 0; i < M.n; i++) {
      M.r[i] = recs[b + (size_t)i];
      mx = std::max<uint64_t>(mx, M.r[i].n64);
    }
    uint64_t gx = (mx + 255) / 256;
    if (gx > (uint64_t)num_sms() * 2) gx = (uint64_t)num_sms() * 2;
    multi_fill_kernel<<<dim3((unsigned)gx, (unsigned)M.n), 256, 0, st>>>(M);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// One thread that holds the stream for `ns` nanoseconds (%globaltimer): a profiling
// replay enqueues its operators behind it, so their event-to-event times are device
// time, not the host's launch and set-up latency between small operators.
__global__ void delay_kernel(uint64_t ns) {
  uint64_t t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  do {
    __nanosleep(1000);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  } while (t - t0 < ns);
}

cudaError_t launch_delay(uint64_t ns, cudaStream_t st) {
  delay_kernel<<<1, 1, 0, st>>>(ns);
  return cudaGetLastError();
}

cudaError_t init_fill(void* ptr, size_t bytes, uint64_t pattern, cudaStream_t st) {
  if (bytes == 0) return cudaSuccess;
  FillHoist& h = fill_hoist();
  if (h.skip) return cudaSuccess;
  const uint64_t n64 = (bytes + 7) / 8;
  if (h.rec) h.rec->push_back(FillRec{ptr, n64, pattern});
  if (pattern == 0) return cudaMemsetAsync(ptr, 0, n64 * 8, st);
  std::vector<FillRec> one{FillRec{ptr, n64, pattern}};
  return launch_multi_fill(one, st);
}

cudaError_t launch_hash_build(const int32_t* keys, const int32_t* payload, const int32_t* in_tids,
                              const uint32_t* d_in_count, int64_t n_cap, uint64_t* table, uint32_t capacity,
                              uint32_t* d_error, cudaStream_t st, const BuildPreds* preds) {
  int lg = 0;
  while ((1u << lg) < capacity) lg++;
  int64_t g = (n_cap + 255) / 256;
  int grid = (int)(g > num_sms() * 8 ? num_sms() * 8 : (g < 1 ? 1 : g));
  const BuildPreds bp = preds ? *preds : BuildPreds{};
  hash_build_kernel<<<grid, 256, 0, st>>>(keys, payload, in_tids, d_in_count, read_count_host_cap(n_cap), table,
                                          capacity, 32 - lg, d_error, bp);
  return cudaGetLastError();
}

// ------------------------------------------------------- direct-mapped join index
uint32_t ji_smem_keys() {
  static const uint32_t v = [] {
    const char* e = getenv("DDQ_JI_SMEM_KEYS");
    return e ? (uint32_t)strtoul(e, nullptr, 10) : 1500000u;
  }();
  return v;
}
size_t ji_coarse_max() {
  static const size_t v = [] {
    const char* e = getenv("DDQ_JI_COARSE_MAX");
    return e ? (size_t)strtoull(e, nullptr, 10) : (size_t)160 * 1024;
  }();
  return v;
}

size_t join_index_bytes(uint32_t range) {
  return ji_fine_bytes(range) + ((size_t)range * 4 + 15) / 16 * 16 + join_index_coarse_bytes(range);
}

cudaError_t join_index_init(void* idx, uint32_t range, cudaStream_t st) {
  cudaError_t e = init_fill(idx, ((size_t)range + 31) / 32 * 4, 0, st);
  if (e == cudaSuccess && join_index_cg(range))
    e = init_fill(join_index_coarse(idx, range), join_index_coarse_bytes(range), 0, st);
  return e;
}

void join_index_coarse_host(const uint32_t* bitmap, uint32_t range, uint32_t* coarse) {
  const uint32_t cg = join_index_cg(range);
  if (!cg) return;
  std::memset(coarse, 0, join_index_coarse_bytes(range));
  for (uint32_t o = 0; o < range; o++)
    if ((bitmap[o >> 5] >> (o & 31)) & 1u) coarse[(o >> cg) >> 5] |= 1u << ((o >> cg) & 31);
}

// One thread per build row: atomicOr of its bit (an old bit = a duplicate key),
// the coarse bit when the index has a coarse bitmap, the payload.  (A warp-
// aggregated variant -- one atomic per run of equal words -- measured no faster:
// SSB builds 531 -> 571 us per step, TPC-H Q3's orders builds 174 -> 155 us.)
__global__ void join_index_build_kernel(const int32_t* __restrict__ keys, const int32_t* __restrict__ payload,
                                        const int32_t* __restrict__ in_tids, const uint32_t* d_in_count,
                                        uint32_t n_static, int32_t key_min, uint32_t range, uint32_t* bitmap,
                                        int32_t* payarr, uint32_t* coarse, uint32_t cg, uint32_t* d_error,
                                        const __grid_constant__ BuildPreds bp) {
  const uint32_t n = d_in_count ? ld_relaxed_u32(d_in_count) : n_static;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t r = in_tids ? in_tids[i] : (int32_t)i;
    if (bp.n && !build_row_passes(bp, r)) continue;
    const uint32_t o = (uint32_t)(keys[r] - key_min);
    if (o >= range) {
      atomicMax(d_error, 3u);
      continue;
    }
    const uint32_t old = atomicOr(bitmap + (o >> 5), 1u << (o & 31));
    if ((old & (1u << (o & 31))) && !bp.key_set) atomicMax(d_error, 1u);  // PKs are unique (O13)
    const int32_t v = bp.payload64 ? (int32_t)bp.payload64[r] : payload ? payload[r] : r;
    if (bp.key_set == 2) {  // MIN build: payload array pre-filled with INT32_MAX
      atomicMin(payarr + o, v);
      if (coarse) {
        uint32_t* cw = coarse + ((o >> cg) >> 5);
        const uint32_t cb = 1u << ((o >> cg) & 31);
        if (!(*reinterpret_cast<volatile uint32_t*>(cw) & cb)) atomicOr(cw, cb);
      }
      continue;
    }
    if (coarse) {  // most coarse bits are set early: test before the atomic
      uint32_t* cw = coarse + ((o >> cg) >> 5);
      const uint32_t cb = 1u << ((o >> cg) & 31);
      if (!(*reinterpret_cast<volatile uint32_t*>(cw) & cb)) atomicOr(cw, cb);
    }
    // only the row that set the bit writes the payload: a key set's duplicates
    // (O32; ~3 of 4 late lineitems of TPC-H Q4) skip their random 4-byte store
    // (measured neutral on B200: Q4's key-set build stays at 100 us, atomic-bound)
    if (!(old & (1u << (o & 31)))) payarr[o] = v;
  }
}

cudaError_t launch_join_index_build(const int32_t* keys, const int32_t* payload, const int32_t* in_tids,
                                    const uint32_t* d_in_count, int64_t n_cap, int32_t key_min, uint32_t range,
                                    void* index, uint32_t* d_error, cudaStream_t st, const BuildPreds* preds) {
  const BuildPreds bp = preds ? *preds : BuildPreds{};
  int64_t g = (n_cap + 255) / 256;
  int grid = (int)(g > num_sms() * 8 ? num_sms() * 8 : (g < 1 ? 1 : g));
  join_index_build_kernel<<<grid, 256, 0, st>>>(keys, payload, in_tids, d_in_count, (uint32_t)n_cap, key_min, range,
                                                join_index_bitmap(index), join_index_payload(index, range),
                                                join_index_coarse(index, range), join_index_cg(range), d_error, bp);
  return cudaGetLastError();
}

// --------------------------------------------------------------------- gather
// W = 8 / 4: copy; W = -8: an int64 column narrowed to an int32 vector (the caller
// checked from the column's load-time range that every value fits)
template <int W>
__global__ void gather_kernel(const void* __restrict__ col, const int32_t* __restrict__ tids,
                              const uint32_t* d_count, uint32_t n_static, void* __restrict__ out) {
  const uint32_t n = d_count ? ld_relaxed_u32(d_count) : n_static;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t r = tids[i];
    if (W == 8)
      reinterpret_cast<long long*>(out)[i] = ldg_gather(reinterpret_cast<const long long*>(col) + r);
    else if (W == -8)
      reinterpret_cast<int*>(out)[i] = (int)ldg_gather(reinterpret_cast<const long long*>(col) + r);
    else
      reinterpret_cast<int*>(out)[i] = ldg_gather(reinterpret_cast<const int32_t*>(col) + r);
  }
}

// Dimension attribute fetch (GATHER through a join index / hash table): for every
// input TID r, out[i] = payload of fk[r] (INT32_MIN if fk[r] has no match).  Pure
// streaming -- TIDs and out coalesced, fk gathered (64 B chunks), the index L2-
// resident -- no compaction: a late-materialisation fetch after a semi-join of the
// same build passes every row, so a probe's ring, reservation and TID copy would be
// wasted work (opprofile SF20 Q3.1: 119 us as an emitting probe).
constexpr int FT_PER = 8;  // items per thread (independent gathers in flight)
__global__ void __launch_bounds__(256) fetch_kernel(const int32_t* __restrict__ tids, const uint32_t* d_count,
                                                    const int32_t* __restrict__ fk, const uint32_t* __restrict__ bitmap,
                                                    const int32_t* __restrict__ payarr, int32_t key_min, uint32_t range,
                                                    const uint64_t* __restrict__ table, uint32_t cap_mask, int shift,
                                                    int32_t* __restrict__ out) {
  const uint32_t n = ld_relaxed_u32(d_count);
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t i0 = blockIdx.x * blockDim.x + threadIdx.x; i0 < n; i0 += FT_PER * stride) {
    int32_t k[FT_PER];
#pragma unroll
    for (int u = 0; u < FT_PER; u++) {
      const uint32_t i = i0 + u * stride;
      k[u] = i < n ? ldg_gather(fk + (uint32_t)tids[i]) : 0;
    }
    if (bitmap) {  // join index: every item's bitmap word, then the payloads of the hits
      // (two rounds of independent L2 loads instead of FT_PER dependent pairs: ncu
      // showed the fetch stalled on long scoreboard 167 cycles per issue)
      uint32_t w[FT_PER];
#pragma unroll
      for (int u = 0; u < FT_PER; u++) {
        const uint32_t o = (uint32_t)(k[u] - key_min);
        w[u] = (i0 + u * stride < n && o < range) ? __ldg(bitmap + (o >> 5)) : 0u;
      }
      int32_t v[FT_PER];
#pragma unroll
      for (int u = 0; u < FT_PER; u++) {
        const uint32_t o = (uint32_t)(k[u] - key_min);
        v[u] = ((w[u] >> (o & 31)) & 1u) ? __ldg(payarr + o) : INT32_MIN;
      }
#pragma unroll
      for (int u = 0; u < FT_PER; u++)
        if (i0 + u * stride < n) out[i0 + u * stride] = v[u];
      continue;
    }
#pragma unroll
    for (int u = 0; u < FT_PER; u++) {
      const uint32_t i = i0 + u * stride;
      if (i >= n) continue;
      int32_t v = INT32_MIN;
      {
        uint32_t h = ht_hash(k[u], shift);
        uint64_t sl = __ldg(table + h);
        while (sl != HT_EMPTY && ht_key(sl) != k[u]) {
          h = (h + 1) & cap_mask;
          sl = __ldg(table + h);
        }
        if (sl != HT_EMPTY) v = ht_val(sl);
      }
      out[i] = v;
    }
  }
}

cudaError_t launch_fetch(const int32_t* tids, const uint32_t* d_count, int64_t n_cap, const int32_t* fk,
                         const uint32_t* bitmap, const int32_t* payarr, int32_t key_min, uint32_t range,
                         const uint64_t* table, uint32_t capacity, int32_t* out, cudaStream_t st) {
  int lg = 0;
  while (capacity && (1u << lg) < capacity) lg++;
  int64_t g = (n_cap + 256 * FT_PER - 1) / (256 * FT_PER);
  int grid = (int)(g > num_sms() * 8 ? num_sms() * 8 : (g < 1 ? 1 : g));
  fetch_kernel<<<grid, 256, 0, st>>>(tids, d_count, fk, bitmap, payarr, key_min, range, table,
                                     capacity ? capacity - 1 : 0, 32 - lg, out);
  return cudaGetLastError();
}

cudaError_t launch_gather(const void* col, int width, const int32_t* tids, const uint32_t* d_count,
                          int64_t n_cap, void* out, cudaStream_t st) {
  int64_t g = (n_cap + 255) / 256;
  int grid = (int)(g > num_sms() * 16 ? num_sms() * 16 : (g < 1 ? 1 : g));
  if (width == 8)
    gather_kernel<8><<<grid, 256, 0, st>>>(col, tids, d_count, (uint32_t)n_cap, out);
  else if (width == -8)
    gather_kernel<-8><<<grid, 256, 0, st>>>(col, tids, d_count, (uint32_t)n_cap, out);
  else
    gather_kernel<4><<<grid, 256, 0, st>>>(col, tids, d_count, (uint32_t)n_cap, out);
  return cudaGetLastError();
}

// -------------------------------------------------------------------- groupby
constexpr int GB_THREADS = 256;
constexpr int GB_SMEM_BUDGET = 32 * 1024;

struct GroupbyParams {
  const int32_t* tids;
  const uint32_t* d_count;
  uint32_t n_static;
  int32_t n_keys;
  const int32_t* key_vec[3];
  const int32_t* key_col[3];
  int32_t key_shift[3];
  int32_t n_aggs;
  int32_t kind[8];
  int32_t width[8][3];
  const void* arg[8][3];
  long long* g_keys;
  unsigned long long* g_accs;  // [(a * cap + slot) * 2 + {0: lo, 1: hi}]
  uint32_t cap_mask;
  int32_t shift;
  uint32_t* d_error;
  uint32_t s_slots;
  int32_t s_shift;
  // small-domain kernel: the distinct argument columns, loaded once per row, and
  // each aggregate's arguments as indices into them
  int32_t n_ucols;
  const void* ucol[8];
  int32_t uwidth[8];
  int32_t uidx[8][3];
};

__device__ __forceinline__ long long agg_value(const GroupbyParams& P, int a, int32_t r) {
  const int k = P.kind[a];
  if (k == DDQ_AGG_COUNT) return 1;
  const long long x = col_at(P.arg[a][0], P.width[a][0], r);
  if (k == DDQ_AGG_SUM) return x;
  const long long y = col_at(P.arg[a][1], P.width[a][1], r);
  if (k == DDQ_AGG_SUM_MUL) return x * y;
  if (k == DDQ_AGG_SUM_SUB) return x - y;
  if (k == DDQ_AGG_SUM_MUL_100M) return x * (100 - y);
  const long long z = col_at(P.arg[a][2], P.width[a][2], r);
  return x * (100 - y) * (100 + z);  // DDQ_AGG_SUM_MUL_100M_100P
}

// Exact int128 sum (lo, hi) of x over the lanes of `peers` (log-step peer
// reduction: each round a lane adds the value of its next remaining peer and the
// odd-ranked lanes retire); the total lands in the lowest peer lane.
__device__ __forceinline__ void peer_reduce128(unsigned peers, long long x, int lane, unsigned long long& lo,
                                               long long& hi) {
  lo = (unsigned long long)x;
  hi = x < 0 ? -1 : 0;
  unsigned rest = peers & (0xfffffffeu << lane);
  unsigned rank = __popc(peers & ((1u << lane) - 1u));
  while (__any_sync(FULL, rest != 0)) {
    const int next = __ffs(rest);
    const int src = next ? next - 1 : lane;
    const unsigned long long tlo = __shfl_sync(FULL, lo, src);
    const long long thi = __shfl_sync(FULL, hi, src);
    if (next) {
      const unsigned long long s = lo + tlo;
      hi += thi + (s < lo ? 1 : 0);
      lo = s;
    }
    rest &= ~__ballot_sync(FULL, rank & 1u);
    rank >>= 1;
  }
}

// exact int128 accumulation of an int128 (lo, hi) addend
__device__ __forceinline__ void atomic_add_i128_pair(unsigned long long* plo, unsigned long long* phi,
                                                     unsigned long long lo, long long hi) {
  const unsigned long long old = atomicAdd(plo, lo);
  const long long h = hi + ((old + lo < old) ? 1 : 0);
  if (h) atomicAdd(phi, (unsigned long long)h);
}

// find-or-insert `key` into an open-addressing table of int64 keys; -1 if full
__device__ __forceinline__ int64_t table_slot(long long* keys, uint32_t mask, uint32_t h, long long key) {
  for (uint32_t probes = 0; probes <= mask; probes++) {
    long long cur = keys[h];
    if (cur == key) return h;
    if (cur == GB_EMPTY) {
      long long old = (long long)atomicCAS(reinterpret_cast<unsigned long long*>(keys + h),
                                           (unsigned long long)GB_EMPTY, (unsigned long long)key);
      if (old == GB_EMPTY || old == key) return h;
    }
    h = (h + 1) & mask;
  }
  return -1;
}

__global__ void __launch_bounds__(GB_THREADS) groupby_kernel(const __grid_constant__ GroupbyParams P) {
  extern __shared__ unsigned long long s_mem[];
  long long* s_keys = reinterpret_cast<long long*>(s_mem);
  unsigned long long* s_accs = s_mem + P.s_slots;  // [(a * S + slot) * 2 + w]
  const uint32_t S = P.s_slots, smask = S - 1;
  for (uint32_t i = threadIdx.x; i < S; i += GB_THREADS) s_keys[i] = GB_EMPTY;
  for (uint32_t i = threadIdx.x; i < S * 2 * P.n_aggs; i += GB_THREADS) s_accs[i] = 0;
  __syncthreads();

  const int lane = threadIdx.x & 31;
  const uint32_t n = P.d_count ? ld_relaxed_u32(P.d_count) : P.n_static;
  const uint32_t warps_total = gridDim.x * (GB_THREADS / 32);
  const uint32_t gw = blockIdx.x * (GB_THREADS / 32) + (threadIdx.x >> 5);
  for (uint32_t base = gw * 32; base < n; base += warps_total * 32) {
    const uint32_t i = base + lane;
    const bool valid = i < n;
    int32_t r = 0;
    long long key = LLONG_MIN;
    if (valid) {
      r = P.tids[i];
      key = 0;
      for (int k = 0; k < P.n_keys; k++) {
        const int32_t c = P.key_vec[k] ? P.key_vec[k][i] : ldg_gather(P.key_col[k] + r);
        key |= (long long)(uint32_t)c << P.key_shift[k];
      }
    }
    const unsigned peers = __match_any_sync(FULL, key);
    const bool leader = (peers & ((1u << lane) - 1u)) == 0;
    long long slot = -1;
    bool global = false;
    if (valid && leader) {
      slot = table_slot(s_keys, smask, gb_hash(key, P.s_shift), key);
      if (slot < 0) {
        global = true;
        slot = table_slot(P.g_keys, P.cap_mask, gb_hash(key, P.shift), key);
        if (slot < 0) atomicMax(P.d_error, 2u);
      }
    }
    for (int a = 0; a < P.n_aggs; a++) {
      const long long v = valid ? agg_value(P, a, r) : 0;
      unsigned long long lo;
      long long hi;
      peer_reduce128(peers, v, lane, lo, hi);  // exact: 32 int64 values can exceed int64
      if (valid && leader && slot >= 0) {
        if (!global)
          atomic_add_i128_pair(&s_accs[((size_t)a * S + slot) * 2], &s_accs[((size_t)a * S + slot) * 2 + 1], lo, hi);
        else
          atomic_add_i128_pair(&P.g_accs[((size_t)a * (P.cap_mask + 1) + slot) * 2],
                               &P.g_accs[((size_t)a * (P.cap_mask + 1) + slot) * 2 + 1], lo, hi);
      }
    }
  }
  __syncthreads();
  // merge this CTA's table into the global one
  for (uint32_t s = threadIdx.x; s < S; s += GB_THREADS) {
    const long long key = s_keys[s];
    if (key == GB_EMPTY) continue;
    const long long g = table_slot(P.g_keys, P.cap_mask, gb_hash(key, P.shift), key);
    if (g < 0) {
      atomicMax(P.d_error, 2u);
      continue;
    }
    for (int a = 0; a < P.n_aggs; a++) {
      const unsigned long long lo = s_accs[((size_t)a * S + s) * 2], hi = s_accs[((size_t)a * S + s) * 2 + 1];
      unsigned long long* glo = &P.g_accs[((size_t)a * (P.cap_mask + 1) + g) * 2];
      const unsigned long long old = atomicAdd(glo, lo);
      const unsigned long long carry = (old + lo < old) ? 1ull : 0ull;
      if (hi + carry) atomicAdd(glo + 1, hi + carry);
    }
  }
}

// ---- small key domain (every key dictionary-coded in key_bits, D = 2^sum(bits)
// groups, D * n_aggs <= GBS_MAX_DA): no warp reduction and no atomics per row.
// Every thread owns D x n_aggs int64 partial sums in shared memory ([entry][thread],
// conflict-free) updated with a plain read-modify-write; a signed-overflow test
// per add spills the partial into a per-CTA int128 accumulator (exact for any
// data).  At the end one warp per entry sums the CTA's partials in int128 and adds
// them to the global table -- only for groups some row hit (`present` mask).
constexpr int GBS_THREADS = 128;
constexpr int GBS_ROWS = 4;  // rows per thread per iteration (independent gathers in flight)
constexpr int GBS_MAX_DA = 64;

__global__ void __launch_bounds__(GBS_THREADS) groupby_small_kernel(const __grid_constant__ GroupbyParams P,
                                                                     uint32_t D) {
  extern __shared__ unsigned long long s_mem[];
  const int A = P.n_aggs;
  const uint32_t DA = D * (uint32_t)A;
  long long* part = reinterpret_cast<long long*>(s_mem);       // [DA][GBS_THREADS]
  unsigned long long* spill = s_mem + (size_t)DA * GBS_THREADS;  // [DA][2] int128
  uint32_t* present = reinterpret_cast<uint32_t*>(spill + (size_t)DA * 2);
  const int tid = threadIdx.x;
  for (uint32_t e = 0; e < DA; e++) part[(size_t)e * GBS_THREADS + tid] = 0;
  for (uint32_t i = tid; i < DA * 2; i += GBS_THREADS) spill[i] = 0;
  if (tid == 0) *present = 0;
  __syncthreads();

  const uint32_t n = P.d_count ? ld_relaxed_u32(P.d_count) : P.n_static;
  uint32_t pm = 0;  // groups this thread hit
  for (uint32_t base = blockIdx.x * (GBS_THREADS * GBS_ROWS); base < n;
       base += gridDim.x * (GBS_THREADS * GBS_ROWS)) {
    int32_t r[GBS_ROWS];
    uint32_t d[GBS_ROWS];
#pragma unroll
    for (int j = 0; j < GBS_ROWS; j++) {
      const uint32_t i = base + j * GBS_THREADS + tid;
      r[j] = i < n ? P.tids[i] : -1;
    }
#pragma unroll
    for (int j = 0; j < GBS_ROWS; j++) {
      const uint32_t i = base + j * GBS_THREADS + tid;
      uint32_t key = 0;
      if (r[j] >= 0)
        for (int k = 0; k < P.n_keys; k++) {
          const int32_t c = P.key_vec[k] ? P.key_vec[k][i] : ldg_gather(P.key_col[k] + r[j]);
          key |= (uint32_t)c << P.key_shift[k];
        }
      d[j] = key & (D - 1);
      if (r[j] >= 0) pm |= 1u << d[j];
    }
    // every distinct argument column of the GBS_ROWS rows: independent loads in flight
    long long val[8][GBS_ROWS];
#pragma unroll
    for (int c = 0; c < 8; c++)
      if (c < P.n_ucols)
#pragma unroll
        for (int j = 0; j < GBS_ROWS; j++) val[c][j] = col_at(P.ucol[c], P.uwidth[c], r[j] < 0 ? 0 : r[j]);
#pragma unroll
    for (int a = 0; a < 8; a++) {
      if (a >= A) break;
      const int kind = P.kind[a], i0 = P.uidx[a][0], i1 = P.uidx[a][1], i2 = P.uidx[a][2];
#pragma unroll
      for (int j = 0; j < GBS_ROWS; j++) {
        if (r[j] < 0) continue;
        long long x = 0, y = 0, z = 0;
#pragma unroll
        for (int c = 0; c < 8; c++) {  // register selects, no dynamic indexing
          x = c == i0 ? val[c][j] : x;
          y = c == i1 ? val[c][j] : y;
          z = c == i2 ? val[c][j] : z;
        }
        const long long v = kind == DDQ_AGG_COUNT ? 1
                          : kind == DDQ_AGG_SUM ? x
                          : kind == DDQ_AGG_SUM_MUL ? x * y
                          : kind == DDQ_AGG_SUM_SUB ? x - y
                          : kind == DDQ_AGG_SUM_MUL_100M ? x * (100 - y)
                          : x * (100 - y) * (100 + z);
        long long* slot = part + (size_t)(d[j] * A + a) * GBS_THREADS + tid;
        const long long old = *slot;
        const long long sum = (long long)((unsigned long long)old + (unsigned long long)v);
        if (((old ^ sum) & (v ^ sum)) < 0) {  // signed overflow: spill the partial exactly
          unsigned long long* sp = spill + (size_t)(d[j] * A + a) * 2;
          atomic_add_i128_pair(sp, sp + 1, (unsigned long long)old, old < 0 ? -1 : 0);
          *slot = v;
        } else {
          *slot = sum;
        }
      }
    }
  }
  if (pm) atomicOr(present, pm);
  __syncthreads();
  // one warp per entry: int128 sum of the CTA's partials, then into the global table
  const int lane = tid & 31, warp = tid >> 5;
  const uint32_t pres = *present;
  for (uint32_t e = warp; e < DA; e += GBS_THREADS / 32) {
    const uint32_t g = e / A;
    const int a = (int)(e % A);
    if (!((pres >> g) & 1u)) continue;
    unsigned long long lo = 0;
    long long hi = 0;
    for (int t = lane; t < GBS_THREADS; t += 32) {
      const long long x = part[(size_t)e * GBS_THREADS + t];
      const unsigned long long s2 = lo + (unsigned long long)x;
      hi += (x < 0 ? -1 : 0) + (s2 < lo ? 1 : 0);
      lo = s2;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const unsigned long long tlo = __shfl_down_sync(FULL, lo, o);
      const long long thi = __shfl_down_sync(FULL, hi, o);
      const unsigned long long s2 = lo + tlo;
      hi += thi + (s2 < lo ? 1 : 0);
      lo = s2;
    }
    if (lane == 0) {
      const unsigned long long slo = spill[(size_t)e * 2], shi = spill[(size_t)e * 2 + 1];
      const unsigned long long s2 = lo + slo;
      hi += (long long)shi + (s2 < lo ? 1 : 0);
      lo = s2;
      const long long key = (long long)g;
      const int64_t slot = table_slot(P.g_keys, P.cap_mask, gb_hash(key, P.shift), key);
      if (slot < 0) {
        atomicMax(P.d_error, 2u);
      } else {
        unsigned long long* glo = &P.g_accs[((size_t)a * (P.cap_mask + 1) + slot) * 2];
        atomic_add_i128_pair(glo, glo + 1, lo, hi);
      }
    }
  }
}

// Aggregations carrying a MIN (DDQ_AGG_MIN, S8(a6)): one row per thread straight
// into the global table.  SUM kinds add exactly into the int128 cell; MIN takes
// atomicMin of the cell's int64 lo word, which groupby_min_init_kernel set to
// INT64_MAX and groupby_min_fix_kernel sign-extends into hi before compaction.
__global__ void groupby_generic_kernel(const __grid_constant__ GroupbyParams P) {
  const uint32_t n = P.d_count ? ld_relaxed_u32(P.d_count) : P.n_static;
  const size_t cap = (size_t)P.cap_mask + 1;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t r = P.tids[i];
    long long key = 0;
    for (int k = 0; k < P.n_keys; k++) {
      const int32_t c = P.key_vec[k] ? P.key_vec[k][i] : ldg_gather(P.key_col[k] + r);
      key |= (long long)(uint32_t)c << P.key_shift[k];
    }
    const int64_t slot = table_slot(P.g_keys, P.cap_mask, gb_hash(key, P.shift), key);
    if (slot < 0) {
      atomicMax(P.d_error, 2u);
      continue;
    }
    for (int a = 0; a < P.n_aggs; a++) {
      unsigned long long* cell = &P.g_accs[((size_t)a * cap + slot) * 2];
      if (P.kind[a] == DDQ_AGG_MIN) {  // width < 0: an aligned vector, indexed by position
        const int w = P.width[a][0];
        atomicMin(reinterpret_cast<long long*>(cell), w < 0 ? col_at(P.arg[a][0], -w, i) : col_at(P.arg[a][0], w, r));
      } else {
        const long long v = agg_value(P, a, r);
        atomic_add_i128_pair(cell, cell + 1, (unsigned long long)v, v < 0 ? -1 : 0);
      }
    }
  }
}

__global__ void groupby_min_init_kernel(unsigned long long* accs, uint32_t capacity, int n_aggs, uint32_t min_mask) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < (size_t)capacity * n_aggs;
       i += (size_t)gridDim.x * blockDim.x)
    if ((min_mask >> (i / capacity)) & 1u) accs[i * 2] = (unsigned long long)LLONG_MAX;
}

__global__ void groupby_min_fix_kernel(unsigned long long* accs, uint32_t capacity, int n_aggs, uint32_t min_mask) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < (size_t)capacity * n_aggs;
       i += (size_t)gridDim.x * blockDim.x)
    if ((min_mask >> (i / capacity)) & 1u) accs[i * 2 + 1] = (long long)accs[i * 2] < 0 ? ~0ull : 0ull;
}

size_t groupby_table_bytes(uint32_t capacity, int n_aggs) {
  return (size_t)capacity * 8 + (size_t)capacity * n_aggs * 16;
}

__global__ void groupby_init_kernel(long long* keys, unsigned long long* accs, uint32_t capacity, int n_aggs) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < capacity; i += gridDim.x * blockDim.x) {
    keys[i] = GB_EMPTY;
    for (int a = 0; a < n_aggs; a++) {
      accs[((size_t)a * capacity + i) * 2] = 0;
      accs[((size_t)a * capacity + i) * 2 + 1] = 0;
    }
  }
}

cudaError_t launch_groupby_init(void* table, uint32_t capacity, int n_aggs, cudaStream_t st) {
  cudaError_t e = init_fill(table, (size_t)capacity * 8, (uint64_t)GB_EMPTY, st);  // keys
  if (e != cudaSuccess) return e;
  return init_fill((char*)table + (size_t)capacity * 8, (size_t)capacity * n_aggs * 16, 0, st);  // accs
}

cudaError_t launch_groupby(const int32_t* tids, const uint32_t* d_count, int64_t n_cap,
                           const int32_t* const* key_vec, const int32_t* const* key_col, int n_keys,
                           const int32_t* key_bits,
                           const ddq_dev_agg* aggs, int n_aggs, void* table, uint32_t capacity,
                           uint32_t* d_error, cudaStream_t st) {
  uint32_t min_mask = 0;
  for (int a = 0; a < n_aggs; a++)
    if (aggs[a].kind == DDQ_AGG_MIN) min_mask |= 1u << a;
  if (!min_mask && agg_ws_supported(tids, key_vec, n_keys, n_aggs, capacity) && d_count) {
    static const char* env = getenv("DDQ_AGG_WS");  // "0": the warp-match kernels below
    if (!env || env[0] != '0')
      return launch_agg_ws(tids, d_count, n_cap, key_vec, key_col, n_keys, key_bits, aggs, n_aggs, table, capacity,
                           d_error, st);
  }
  GroupbyParams p{};
  p.tids = tids;
  p.d_count = d_count;
  p.n_static = (uint32_t)n_cap;
  p.n_keys = n_keys;
  for (int k = 0, sh = 0; k < 3; k++) {
    p.key_shift[k] = sh;
    sh += (key_bits && key_bits[k] > 0) ? key_bits[k] : 21;
  }
  for (int k = 0; k < n_keys; k++) {
    p.key_vec[k] = key_vec ? key_vec[k] : nullptr;
    p.key_col[k] = key_col ? key_col[k] : nullptr;
  }
  p.n_aggs = n_aggs;
  for (int a = 0; a < n_aggs; a++) {
    p.kind[a] = aggs[a].kind;
    for (int j = 0; j < 3; j++) {
      p.width[a][j] = aggs[a].width[j];
      p.arg[a][j] = aggs[a].arg[j];
    }
  }
  p.g_keys = reinterpret_cast<long long*>(table);
  p.g_accs = reinterpret_cast<unsigned long long*>((char*)table + (size_t)capacity * 8);
  p.cap_mask = capacity - 1;
  int lg = 0;
  while ((1u << lg) < capacity) lg++;
  p.shift = 64 - lg;
  p.d_error = d_error;
  if (min_mask) {  // MIN: the generic kernel on the global table (init / fix the MIN cells)
    const int64_t cells = (int64_t)capacity * n_aggs;
    const int gi = (int)std::min<int64_t>((cells + 255) / 256, (int64_t)num_sms() * 8);
    groupby_min_init_kernel<<<gi, 256, 0, st>>>(p.g_accs, capacity, n_aggs, min_mask);
    const int64_t g = (n_cap + 255) / 256;
    const int grid = (int)(g < 1 ? 1 : (g > (int64_t)num_sms() * 8 ? (int64_t)num_sms() * 8 : g));
    groupby_generic_kernel<<<grid, 256, 0, st>>>(p);
    groupby_min_fix_kernel<<<gi, 256, 0, st>>>(p.g_accs, capacity, n_aggs, min_mask);
    return cudaGetLastError();
  }
  // small key domain: every key dictionary-coded (key_bits), D * n_aggs <= 64
  int total_bits = 0;
  bool coded = n_keys == 0 || key_bits != nullptr;
  for (int k = 0; k < n_keys && coded; k++) {
    coded = key_bits[k] > 0;
    total_bits += coded ? key_bits[k] : 0;
  }
  bool ucols_ok = true;  // the small kernel loads at most 8 distinct argument columns
  p.n_ucols = 0;
  for (int a = 0; a < n_aggs; a++)
    for (int j = 0; j < 3; j++) {
      p.uidx[a][j] = -1;
      const int need = aggs[a].kind == DDQ_AGG_COUNT ? 0 : (aggs[a].kind == DDQ_AGG_SUM || aggs[a].kind == DDQ_AGG_MIN) ? 1
                     : aggs[a].kind == DDQ_AGG_SUM_MUL_100M_100P ? 3 : 2;
      if (j >= need) continue;
      int c = 0;
      while (c < p.n_ucols && !(p.ucol[c] == aggs[a].arg[j] && p.uwidth[c] == aggs[a].width[j])) c++;
      if (c == p.n_ucols) {
        if (c == 8) {
          ucols_ok = false;
          continue;
        }
        p.ucol[c] = aggs[a].arg[j];
        p.uwidth[c] = aggs[a].width[j];
        p.n_ucols++;
      }
      p.uidx[a][j] = c;
    }
  if (ucols_ok && coded && total_bits <= 6 && (n_aggs << total_bits) <= GBS_MAX_DA && p.tids != nullptr) {
    const uint32_t D = 1u << total_bits;
    const size_t smem = (size_t)D * n_aggs * (GBS_THREADS * 8 + 16) + 16;
    static const int occs = [] {  // thread-safe one-time opt-in
      int o = 0;
      cudaFuncSetAttribute(groupby_small_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           GBS_MAX_DA * (GBS_THREADS * 8 + 16) + 16);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, groupby_small_kernel, GBS_THREADS,
                                                    GBS_MAX_DA * (GBS_THREADS * 8 + 16) + 16);
      return o < 1 ? 1 : o;
    }();
    const int64_t want = (n_cap + GBS_THREADS * GBS_ROWS - 1) / (GBS_THREADS * GBS_ROWS);
    const int64_t maxb = (int64_t)num_sms() * occs;
    const int grid = (int)(want < 1 ? 1 : (want > maxb ? maxb : want));
    groupby_small_kernel<<<grid, GBS_THREADS, smem, st>>>(p, D);
    return cudaGetLastError();
  }
  uint32_t S = 1u << 12;
  while (S > 64 && (size_t)S * (8 + 16 * (size_t)n_aggs) > GB_SMEM_BUDGET) S >>= 1;
  // no point in a CTA table larger than the global one
  while (S > 64 && S > capacity) S >>= 1;
  int slg = 0;
  while ((1u << slg) < S) slg++;
  p.s_slots = S;
  p.s_shift = 64 - slg;
  const size_t smem = (size_t)S * (8 + 16 * (size_t)n_aggs);
  static const int occ = [] {  // thread-safe one-time opt-in
    int o = 0;
    cudaFuncSetAttribute(groupby_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, groupby_kernel, GB_THREADS, GB_SMEM_BUDGET);
    return o < 1 ? 1 : o;
  }();
  int64_t want = (n_cap + GB_THREADS - 1) / GB_THREADS;
  int64_t maxb = (int64_t)num_sms() * occ;
  int grid = (int)(want < 1 ? 1 : (want > maxb ? maxb : want));
  groupby_kernel<<<grid, GB_THREADS, smem, st>>>(p);
  return cudaGetLastError();
}

__global__ void groupby_compact_kernel(const long long* keys, const unsigned long long* accs, uint32_t capacity,
                                       int n_aggs, int64_t* out_keys, int64_t* out_accs, uint32_t* d_out) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < capacity; i += gridDim.x * blockDim.x) {
    const long long k = keys[i];
    if (k == GB_EMPTY) continue;
    const uint32_t pos = atomicAdd(d_out, 1u);
    out_keys[pos] = k;
    for (int a = 0; a < n_aggs; a++) {
      out_accs[((size_t)pos * n_aggs + a) * 2] = (int64_t)accs[((size_t)a * capacity + i) * 2];
      out_accs[((size_t)pos * n_aggs + a) * 2 + 1] = (int64_t)accs[((size_t)a * capacity + i) * 2 + 1];
    }
  }
}

cudaError_t launch_groupby_compact(const void* table, uint32_t capacity, int n_aggs, int64_t* out_keys,
                                   int64_t* out_accs, uint32_t* d_out_groups, cudaStream_t st) {
  cudaError_t e = init_fill(d_out_groups, sizeof(uint32_t), 0, st);
  if (e != cudaSuccess) return e;
  int grid = (int)((capacity + 255) / 256);
  if (grid > num_sms() * 8) grid = num_sms() * 8;
  groupby_compact_kernel<<<grid < 1 ? 1 : grid, 256, 0, st>>>(
      reinterpret_cast<const long long*>(table),
      reinterpret_cast<const unsigned long long*>((const char*)table + (size_t)capacity * 8), capacity, n_aggs,
      out_keys, out_accs, d_out_groups);
  return cudaGetLastError();
}

}  // namespace ddq
