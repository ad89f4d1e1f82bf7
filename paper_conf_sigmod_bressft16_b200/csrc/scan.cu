// scan.cu -- dense scan kernel: selection (S8(a2)) and first hash probe (S8(a4))
// over ALL rows of a fact column, the dominant kernel of every SSB plan.
//
// B200 design, replacing the single-pass look-back kernel
// for dense inputs after ncu showed it barrier/latency bound at 8% of HBM peak:
//   * persistent CTAs (SMs x resident), static tile order b, b+G, b+2G, ...;
//   * input columns streamed through an S-stage shared-memory ring with cp.async
//     (16-byte LDGSTS, L2-only): S-1 tiles are always in flight per CTA, without
//     holding registers, so the memory pipe stays busy across the per-tile
//     compaction and output reservation;
//   * hash tables that fit are staged once per CTA into shared memory (random
//     8-byte lookups at smem bandwidth instead of L1/L2 sector rate);
//   * survivors are compacted per tile (packed warp scan) and their output range is
//     reserved with ONE atomicAdd per 4096-row tile: no inter-CTA waiting.  Rows
//     stay ascending within each tile; tiles appear in completion order (reading
//     O14': the TID list is a multiset -- SQL results are order-free before ORDER BY
//     and all aggregates are exact integer sums, so results are bit-identical).
#include <cstdint>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "ops_internal.h"

namespace ddq {

constexpr int SC_THREADS = 256;
constexpr int SC_WARPS = SC_THREADS / 32;
constexpr int SC_TILE = 4096;        // rows per tile
constexpr int SC_ITEMS = SC_TILE / SC_THREADS;  // 16
constexpr int SC_MAXCOLS = 4;

struct ScanPred {
  const void* col;
  int32_t width, kind;
  int64_t lo, hi;
  int32_t n_in, _pad;
  int64_t in_vals[8];
};

struct ScanParams {
  uint32_t n;  // rows
  int32_t n_cols;
  const void* cols[SC_MAXCOLS];
  int32_t width[SC_MAXCOLS];
  int32_t col_off[SC_MAXCOLS];  // byte offset of the column's chunk inside a stage
  int32_t stage_bytes;
  int32_t stages;
  // select
  int32_t n_preds;
  ScanPred preds[SC_MAXCOLS];
  // probe (fk = cols[0])
  int32_t probe;
  const uint64_t* table;
  uint32_t cap_mask;
  int32_t shift;
  int32_t table_in_smem;
  // direct-mapped join index instead of a hash table
  int32_t direct;
  const uint32_t* bitmap;
  const int32_t* payarr;
  int32_t key_min;
  uint32_t range;
  uint32_t bitmap_words;
  int32_t bitmap_in_smem;
  int32_t* out_payload;
  // outputs
  int32_t* out_tids;
  uint32_t* d_out_count;  // zeroed before launch; final = survivors
  uint32_t out_cap;
  uint32_t* d_overflow;
};

// ---- TMA bulk copies (cp.async.bulk) completing on an mbarrier ---------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
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

// Thread 0: one bulk copy per column of tile `tile` into stage buffer `buf`.
// Columns are readable up to the next 16-byte boundary (library allocations are
// padded; torch allocations are 512-byte granular), so the tail tile is copied
// rounded up to 16 bytes and its invalid rows are masked by the row bound.
__device__ __forceinline__ void issue_tile(const ScanParams& P, uint8_t* buf, uint64_t* bar, uint32_t tile) {
  const uint64_t row0 = (uint64_t)tile * SC_TILE;
  const uint64_t rows = (uint64_t)P.n - row0 < (uint64_t)SC_TILE ? (uint64_t)P.n - row0 : (uint64_t)SC_TILE;
  uint32_t total = 0;
  uint32_t bytes[SC_MAXCOLS];
  for (int c = 0; c < P.n_cols; c++) {
    bytes[c] = (uint32_t)((rows * P.width[c] + 15) / 16 * 16);
    total += bytes[c];
  }
  mbar_arrive_expect_tx(bar, total);
  for (int c = 0; c < P.n_cols; c++)
    tma_load_1d(buf + P.col_off[c], reinterpret_cast<const uint8_t*>(P.cols[c]) + row0 * P.width[c], bytes[c], bar);
}

__device__ __forceinline__ bool scan_pred(const ScanPred& p, int64_t v) {
  if (p.kind == DDQ_PRED_RANGE) return v >= p.lo && v <= p.hi;
  bool m = false;
#pragma unroll
  for (int j = 0; j < 8; j++) m |= (j < p.n_in) && (v == p.in_vals[j]);
  return m;
}

__global__ void __launch_bounds__(SC_THREADS, 2) scan_kernel(const __grid_constant__ ScanParams P) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint32_t s_warp_tot[SC_WARPS];
  __shared__ uint32_t s_base, s_tot;
  __shared__ __align__(8) uint64_t s_full[8];  // one mbarrier per stage
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t ntiles = (P.n + SC_TILE - 1) / SC_TILE;
  const int S = P.stages;
  uint8_t* ring = smem;
  uint64_t* s_table = reinterpret_cast<uint64_t*>(smem + (size_t)S * P.stage_bytes);

  // prologue: thread 0 puts S-1 tiles in flight; all threads stage the table meanwhile
  if (threadIdx.x == 0) {
    for (int k = 0; k < S; k++) mbar_init(&s_full[k], 1);
    fence_mbar_init();
    for (int k = 0; k < S - 1; k++) {
      const uint32_t t = blockIdx.x + (uint32_t)k * gridDim.x;
      if (t < ntiles) issue_tile(P, ring + (size_t)k * P.stage_bytes, &s_full[k], t);
    }
  }
  if (P.probe && P.table_in_smem) {
    for (uint32_t i = threadIdx.x; i <= P.cap_mask; i += SC_THREADS) s_table[i] = P.table[i];
  }
  const uint64_t* table = (P.probe && P.table_in_smem) ? s_table : P.table;
  uint32_t* s_bm = reinterpret_cast<uint32_t*>(s_table);
  if (P.probe && P.direct && P.bitmap_in_smem) {
    for (uint32_t i = threadIdx.x; i < P.bitmap_words; i += SC_THREADS) s_bm[i] = P.bitmap[i];
  }
  const uint32_t* bm = (P.probe && P.direct && P.bitmap_in_smem) ? s_bm : P.bitmap;
  __syncthreads();

  for (uint32_t k = 0;; k++) {
    const uint32_t tile = blockIdx.x + k * gridDim.x;
    if (tile >= ntiles) break;
    if (threadIdx.x == 0) {  // keep S-1 tiles in flight (stage (k-1)%S was released by the last barrier)
      const uint32_t t = tile + (uint32_t)(S - 1) * gridDim.x;
      if (t < ntiles) {
        fence_proxy_async();
        const int st = (int)((k + S - 1) % S);
        issue_tile(P, ring + (size_t)st * P.stage_bytes, &s_full[st], t);
      }
    }
    mbar_wait(&s_full[k % S], (k / S) & 1u);
    const uint8_t* buf = ring + (size_t)(k % S) * P.stage_bytes;
    const uint32_t row0 = tile * SC_TILE;
    const uint32_t wrow = warp * (32 * SC_ITEMS);  // warp's first row inside the tile

    uint32_t flags = 0xFFFFu;
    if (row0 + SC_TILE > P.n) {  // tail tile only
      flags = 0;
#pragma unroll
      for (int s = 0; s < 4; s++)
#pragma unroll
        for (int v = 0; v < 4; v++)
          flags |= (row0 + wrow + s * 128 + lane * 4 + v < P.n ? 1u : 0u) << (s * 4 + v);
    }

    int32_t payload[SC_ITEMS];
    if (!P.probe) {
      for (int p = 0; p < P.n_preds; p++) {
        const ScanPred& pr = P.preds[p];
        const uint8_t* cb = buf + P.col_off[p];
#pragma unroll
        for (int s = 0; s < 4; s++) {
          const int it = wrow + s * 128 + lane * 4;
          int64_t v4[4];
          if (pr.width == 8) {
            const longlong2 a = *reinterpret_cast<const longlong2*>(cb + (size_t)it * 8);
            const longlong2 b = *reinterpret_cast<const longlong2*>(cb + (size_t)it * 8 + 16);
            v4[0] = a.x; v4[1] = a.y; v4[2] = b.x; v4[3] = b.y;
          } else {
            const int4 a = *reinterpret_cast<const int4*>(cb + (size_t)it * 4);
            v4[0] = a.x; v4[1] = a.y; v4[2] = a.z; v4[3] = a.w;
          }
          uint32_t m = 0;
#pragma unroll
          for (int v = 0; v < 4; v++) m |= (scan_pred(pr, v4[v]) ? 1u : 0u) << v;
          flags &= ~((~m & 0xFu) << (s * 4));
        }
      }
    } else if (P.direct) {
      // direct-mapped join index: one bitmap probe per row, payload for survivors only
      uint32_t o[SC_ITEMS];
#pragma unroll
      for (int s = 0; s < 4; s++) {
        const int4 a = *reinterpret_cast<const int4*>(buf + (size_t)(wrow + s * 128 + lane * 4) * 4);
        o[s * 4 + 0] = (uint32_t)(a.x - P.key_min); o[s * 4 + 1] = (uint32_t)(a.y - P.key_min);
        o[s * 4 + 2] = (uint32_t)(a.z - P.key_min); o[s * 4 + 3] = (uint32_t)(a.w - P.key_min);
      }
      uint32_t m = 0;
#pragma unroll
      for (int k2 = 0; k2 < SC_ITEMS; k2++) {
        const uint32_t oo = o[k2] < P.range ? o[k2] : 0u;
        const uint32_t w = bm[oo >> 5];
        m |= ((o[k2] < P.range ? (w >> (oo & 31)) : 0u) & 1u) << k2;
      }
      flags &= m;
      if (P.out_payload) {
#pragma unroll
        for (int k2 = 0; k2 < SC_ITEMS; k2++) payload[k2] = ((flags >> k2) & 1u) ? __ldg(P.payarr + o[k2]) : 0;
      }
    } else {
      int32_t key[SC_ITEMS];
      uint32_t h[SC_ITEMS];
      uint64_t sl[SC_ITEMS];
#pragma unroll
      for (int s = 0; s < 4; s++) {
        const int4 a = *reinterpret_cast<const int4*>(buf + (size_t)(wrow + s * 128 + lane * 4) * 4);
        key[s * 4 + 0] = a.x; key[s * 4 + 1] = a.y; key[s * 4 + 2] = a.z; key[s * 4 + 3] = a.w;
      }
#pragma unroll
      for (int k2 = 0; k2 < SC_ITEMS; k2++) {
        h[k2] = ht_hash(key[k2], P.shift);
        sl[k2] = ((flags >> k2) & 1u) ? table[h[k2]] : HT_EMPTY;
      }
#pragma unroll
      for (int k2 = 0; k2 < SC_ITEMS; k2++) {
        uint64_t s = sl[k2];
        uint32_t hh = h[k2];
        while (s != HT_EMPTY && ht_key(s) != key[k2]) {
          hh = (hh + 1) & P.cap_mask;
          s = table[hh];
        }
        if (s == HT_EMPTY) flags &= ~(1u << k2);
        payload[k2] = ht_val(s);
      }
    }

    // compaction within the tile
    uint32_t packed = 0;
#pragma unroll
    for (int s = 0; s < 4; s++) packed |= (uint32_t)__popc((flags >> (4 * s)) & 0xFu) << (8 * s);
    const uint32_t incl = warp_incl_scan(packed, lane);
    const uint32_t excl = incl - packed;
    const uint32_t wtot = __shfl_sync(FULL, incl, 31);
    uint32_t slot_off[4];
    uint32_t acc = 0;
#pragma unroll
    for (int s = 0; s < 4; s++) {
      slot_off[s] = acc;
      acc += (wtot >> (8 * s)) & 0xFFu;
    }
    if (lane == 0) s_warp_tot[warp] = acc;
    __syncthreads();  // also: every thread is done reading stage k%S
    if (threadIdx.x == 0) {
      uint32_t tot = 0;
#pragma unroll
      for (int w = 0; w < SC_WARPS; w++) tot += s_warp_tot[w];
      s_base = tot ? atomicAdd(P.d_out_count, tot) : 0;
      s_tot = tot;
    }
    uint32_t warp_off = 0;
#pragma unroll
    for (int w = 0; w < SC_WARPS; w++) warp_off += (w < warp) ? s_warp_tot[w] : 0;
    __syncthreads();
    const uint32_t tile_base = s_base;
    const uint32_t base = tile_base + warp_off;
    const bool fits = tile_base + s_tot <= P.out_cap;
#pragma unroll
    for (int s = 0; s < 4; s++) {
      const uint32_t m = (flags >> (4 * s)) & 0xFu;
      const uint32_t sb = base + slot_off[s] + ((excl >> (8 * s)) & 0xFFu);
#pragma unroll
      for (int v = 0; v < 4; v++) {
        const uint32_t pos = sb + __popc(m & ((1u << v) - 1u));
        if (((m >> v) & 1u) && (fits || pos < P.out_cap)) {
          P.out_tids[pos] = (int32_t)(row0 + wrow + s * 128 + lane * 4 + v);
          if (P.out_payload) P.out_payload[pos] = payload[s * 4 + v];
        }
      }
    }
    if (!fits && threadIdx.x == 0 && P.d_overflow) atomicMax(P.d_overflow, 4u);
    __syncthreads();  // s_warp_tot / s_base reuse
  }
  // the last CTA to finish clamps the count to the output capacity (cell word 1 =
  // CTA completion counter, zeroed with the count before launch)
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(P.d_out_count + 1, 1u) == gridDim.x - 1) {
      const uint32_t c = atomicAdd(P.d_out_count, 0u);
      if (c > P.out_cap) *P.d_out_count = P.out_cap;
    }
  }
}

static int g_smem_optin = 0;

bool scan_supported(const FilterArgs& a) {
  if (a.in_tids || a.n_carry) return false;  // dense inputs only
  if (!a.probe && (a.n_preds < 1 || a.n_preds > SC_MAXCOLS)) return false;
  // TMA bulk copies need 16-byte aligned column bases
  if (a.probe) return ((uintptr_t)a.fk & 15) == 0;
  for (int i = 0; i < a.n_preds; i++)
    if ((uintptr_t)a.preds[i].col & 15) return false;
  return true;
}

cudaError_t launch_scan(const FilterArgs& a, cudaStream_t st) {
  if (!g_smem_optin) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    cudaFuncSetAttribute(scan_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, g_smem_optin - 1024);
  }
  ScanParams p{};
  p.n = (uint32_t)a.n_cap;
  int off = 0;
  if (a.probe) {
    p.probe = 1;
    p.n_cols = 1;
    p.cols[0] = a.fk;
    p.width[0] = 4;
    p.col_off[0] = 0;
    off = SC_TILE * 4;
  } else {
    p.n_cols = a.n_preds;
    p.n_preds = a.n_preds;
    for (int i = 0; i < a.n_preds; i++) {
      const ddq_dev_pred& d = a.preds[i];
      p.cols[i] = d.col;
      p.width[i] = d.width;
      p.col_off[i] = off;
      off += SC_TILE * d.width;
      p.preds[i].col = d.col;
      p.preds[i].width = d.width;
      p.preds[i].kind = d.kind;
      p.preds[i].lo = d.lo;
      p.preds[i].hi = d.hi;
      p.preds[i].n_in = d.n_in;
      for (int j = 0; j < 8; j++) p.preds[i].in_vals[j] = d.in_vals[j];
    }
  }
  p.stage_bytes = off;
  const bool direct = a.probe && a.bitmap != nullptr;
  size_t table_bytes = a.probe ? (direct ? ((size_t)a.range + 31) / 32 * 4 : (size_t)a.capacity * 8) : 0;
  // shared memory budget per SM (~227 KB usable): table + ring, 2 CTAs per SM when possible
  const size_t budget = (size_t)g_smem_optin - 1024;
  const bool in_smem = a.probe && table_bytes <= 96 * 1024;
  p.table_in_smem = (in_smem && !direct) ? 1 : 0;
  p.bitmap_in_smem = (in_smem && direct) ? 1 : 0;
  size_t fixed = in_smem ? (table_bytes + 15) / 16 * 16 : 0;
  if (direct) {
    p.direct = 1;
    p.bitmap = a.bitmap;
    p.payarr = a.payarr;
    p.key_min = a.key_min;
    p.range = a.range;
    p.bitmap_words = (a.range + 31) / 32;
  }
  int ctas_per_sm = 2;
  int stages = 4;
  auto need = [&](int s, int c) { return ((size_t)s * p.stage_bytes + fixed) * c; };
  while (stages > 2 && need(stages, ctas_per_sm) > budget) stages--;
  if (need(stages, ctas_per_sm) > budget) ctas_per_sm = 1;
  while (stages > 2 && need(stages, ctas_per_sm) > budget) stages--;
  p.stages = stages;
  if (a.probe && !direct) {
    p.table = a.table;
    p.cap_mask = a.capacity - 1;
    int lg = 0;
    while ((1u << lg) < a.capacity) lg++;
    p.shift = 32 - lg;
  }
  if (a.probe) p.out_payload = a.out_payload;
  p.out_tids = a.out_tids;
  p.d_out_count = a.d_out_count;
  p.out_cap = (uint32_t)(a.out_cap > 0 ? a.out_cap : a.n_cap);
  p.d_overflow = a.d_overflow;
  cudaError_t e = cudaMemsetAsync(a.d_out_count, 0, 8, st);
  if (e != cudaSuccess) return e;
  const size_t smem = (size_t)stages * p.stage_bytes + fixed;
  const int64_t ntiles = (a.n_cap + SC_TILE - 1) / SC_TILE;
  int64_t grid = (int64_t)num_sms() * ctas_per_sm;
  if (grid > ntiles) grid = ntiles < 1 ? 1 : ntiles;
  scan_kernel<<<(int)grid, SC_THREADS, smem, st>>>(p);
  return cudaGetLastError();
}

}  // namespace ddq
