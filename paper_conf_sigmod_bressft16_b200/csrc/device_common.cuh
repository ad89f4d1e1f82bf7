// device_common.cuh -- small device helpers shared by the libddq kernels
// (vector loads, warp scans, decoupled look-back, hashing, int128 atomics).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace ddq {

constexpr unsigned FULL = 0xffffffffu;

// ---- loads ---------------------------------------------------------------
// Streaming 128-bit loads that do not allocate in L1 (each column byte is read once).
// FILTER_EQ comparison of two aligned int32 vector entries (ddq_op.eq_cmp:
// DDQ_CMP_EQ 0, DDQ_CMP_LT 1, DDQ_CMP_NE 2).
__device__ __forceinline__ bool vec_cmp(int cmp, int32_t a, int32_t b) {
  return cmp == 1 ? a < b : cmp == 2 ? a != b : a == b;
}

// DDQ_PRED_BITSET membership (include/ddq.h): bit (v - lo) of a 512-bit mask
__device__ __forceinline__ bool bitset_hit(const int64_t* words, int64_t lo, int64_t v) {
  const uint64_t o = (uint64_t)(v - lo);
  return o < 512 && ((uint64_t)words[o >> 6] >> (o & 63)) & 1;
}

__device__ __forceinline__ int4 ld_stream_i4(const void* p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ longlong2 ld_stream_l2(const void* p) {
  longlong2 r;
  asm volatile("ld.global.nc.L1::no_allocate.v2.s64 {%0,%1}, [%2];"
               : "=l"(r.x), "=l"(r.y) : "l"(p));
  return r;
}
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// Sparse gathers (one value per selected row): the L2 otherwise fetches 128 B
// from HBM per miss; the .L2::64B size hint halves that (tools/cuda/gather_probe:
// int64 at 2 % TID density 275 -> 153 MB of DRAM reads, 46 -> 33 us).
__device__ __forceinline__ int32_t ldg_gather(const int32_t* p) {
  int32_t v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.s32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ long long ldg_gather(const long long* p) {
  long long v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.s64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint32_t ldg_gather(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint64_t ldg_gather(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}

// Scalar read of column element r (width 4 or 8) widened to int64.
__device__ __forceinline__ int64_t col_at(const void* col, int width, int64_t r) {
  return width == 8 ? ldg_gather(reinterpret_cast<const long long*>(col) + r)
                    : (int64_t)ldg_gather(reinterpret_cast<const int32_t*>(col) + r);
}

// ---- TMA bulk copies (cp.async.bulk) completing on an mbarrier ---------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
        : "=r"(done) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  }
}
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
// Stage `bytes` (multiple of 16, both addresses 16-byte aligned) from global into
// shared memory with TMA bulk copies; called by ALL threads of the CTA (thread 0
// issues, everyone waits on the mbarrier).  One round trip instead of a
// load->store loop whose per-iteration latency serialises (a 75 KB bitmap staged by
// 512 threads with scalar loads took ~40 us).
__device__ __forceinline__ void stage_bulk(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  if (threadIdx.x == 0) {
    mbar_init(bar, 1);
    fence_mbar_init();
    mbar_arrive_expect_tx(bar, bytes);
    constexpr uint32_t kChunk = 32768;
    for (uint32_t o = 0; o < bytes; o += kChunk)
      tma_load_1d(reinterpret_cast<uint8_t*>(dst) + o, reinterpret_cast<const uint8_t*>(src) + o,
                  bytes - o < kChunk ? bytes - o : kChunk, bar);
  }
  __syncthreads();  // the barrier is initialised before anyone waits on it
  mbar_wait(bar, 0);
}

// ---- warp scan -----------------------------------------------------------
__device__ __forceinline__ uint32_t warp_incl_scan(uint32_t v, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t t = __shfl_up_sync(FULL, v, o);
    if (lane >= o) v += t;
  }
  return v;
}

// ---- decoupled look-back (single-pass prefix over tiles) -------------------
// status word: [63:62] flag (0 invalid, 1 aggregate, 2 inclusive prefix), [31:0] value
constexpr uint64_t LB_AGG = 1ull << 62;
constexpr uint64_t LB_INC = 2ull << 62;

// Called by one full warp.  Returns the exclusive prefix of `tile` (all lanes).
__device__ __forceinline__ uint32_t lookback(uint64_t* status, uint32_t tile, uint32_t total, int lane) {
  if (tile == 0) {
    if (lane == 0) st_relaxed_u64(&status[0], LB_INC | total);
    return 0;
  }
  if (lane == 0) st_relaxed_u64(&status[tile], LB_AGG | total);
  uint32_t excl = 0;
  int64_t pred = (int64_t)tile - 1 - lane;
  while (true) {
    uint64_t s;
    unsigned spins = 0;
    while (true) {
      s = pred >= 0 ? ld_relaxed_u64(&status[pred]) : (LB_INC | 0ull);
      if (__ballot_sync(FULL, (s >> 62) == 0) == 0) break;
      if (++spins > 8) __nanosleep(32);
    }
    unsigned inc = __ballot_sync(FULL, (s >> 62) == 2);
    uint32_t v = (uint32_t)s;
    if (inc) {
      int k = __ffs(inc) - 1;
      if (lane > k) v = 0;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
      excl += v;
      break;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    excl += v;
    pred -= 32;
  }
  if (lane == 0) st_relaxed_u64(&status[tile], LB_INC | (uint64_t)(excl + total));
  return excl;
}

// ---- hashing ---------------------------------------------------------------
constexpr uint64_t HT_EMPTY = 0x8000000000000000ull;  // key INT32_MIN, payload 0
__device__ __forceinline__ uint32_t ht_hash(int32_t k, int shift) {
  return ((uint32_t)k * 0x9E3779B1u) >> shift;  // shift = 32 - log2(capacity)
}
__device__ __forceinline__ int32_t ht_key(uint64_t s) { return (int32_t)(s >> 32); }
__device__ __forceinline__ int32_t ht_val(uint64_t s) { return (int32_t)(uint32_t)s; }

constexpr int64_t GB_EMPTY = -1;
__device__ __forceinline__ uint32_t gb_hash(int64_t k, int shift) {
  return (uint32_t)(((uint64_t)k * 0x9E3779B97F4A7C15ull) >> shift);  // shift = 64 - log2(cap)
}

// exact int128 accumulation with two 64-bit atomics (lo unsigned, hi signed)
__device__ __forceinline__ void atomic_add_i128(unsigned long long* lo, unsigned long long* hi, long long v) {
  unsigned long long old = atomicAdd(lo, (unsigned long long)v);
  unsigned long long sum = old + (unsigned long long)v;
  long long hadd = (v < 0 ? -1ll : 0ll) + (sum < old ? 1ll : 0ll);
  if (hadd) atomicAdd(hi, (unsigned long long)hadd);
}

}  // namespace ddq
