// filter.cu -- selection (S8(a1)/(a2)) and hash probe (S8(a4)) as one stable
// stream-compaction kernel family.
//
// Both operators map an input (all rows of a table, or a TID list) to the ascending
// list of surviving row ids (operators materialise their output; P:188 the
// paper's selection is He et al.'s [13]).  B200 design:
//   * persistent grid (SMs x resident CTAs) pulling 4096-item tiles from an atomic
//     tile counter, so tiles are acquired in order;
//   * each warp owns 512 consecutive items as 4 slots x (32 lanes x 4 items), so
//     every column access of a slot is one coalesced 128-bit (int32) or 2x128-bit
//     (int64) load per lane, all issued before any predicate is evaluated;
//   * the 4 per-slot survivor counts are packed into one 32-bit word and scanned
//     with a single warp shuffle scan; warps are combined through shared memory;
//   * the tile's output offset comes from a decoupled look-back over the previous
//     tiles (single pass over the input, stable, deterministic);
//   * probes read an open-addressing table staged in shared memory when it fits,
//     else from global memory (L2-resident), with all first probes issued together.
#include <cstdint>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "ops_internal.h"

namespace ddq {

constexpr int FT_THREADS = 256;
constexpr int FT_WARPS = FT_THREADS / 32;
constexpr int FT_SLOTS = 4;
constexpr int FT_ITEMS = FT_SLOTS * 4;              // items per thread
constexpr int FT_WARP_ITEMS = 32 * FT_ITEMS;        // 512
constexpr int FT_TILE = FT_THREADS * FT_ITEMS;      // 4096

struct DevPredK {
  const void* col;
  int32_t width, kind;
  int64_t lo, hi;
  int32_t n_in, _pad;
  int64_t in_vals[8];
};

struct FilterParams {
  const int32_t* in_tids;
  const uint32_t* d_in_count;
  uint32_t n_static;  // used when d_in_count == nullptr
  int32_t n_preds;
  DevPredK preds[4];
  // probe
  const uint64_t* table;
  uint32_t cap_mask;
  int32_t shift;
  const int32_t* fk;
  int32_t* out_payload;
  int32_t fk_by_pos;    // probe keys are an aligned vector (fk[i]), not a column (fk[row])
  const int32_t* eq_a;  // FILTER_EQ vectors (positional), or null
  const int32_t* eq_b;
  int eq_cmp;  // FILTER_EQ comparison: 0 a == b, 1 a < b, 2 a != b (DDQ_CMP_*)
  int32_t direct;  // direct-mapped join index instead of the hash table
  const uint32_t* bitmap;
  const int32_t* payarr;
  int32_t key_min;
  uint32_t range;
  // carries
  int32_t n_carry;
  const int32_t* carry_in[4];
  int32_t* carry_out[4];
  // outputs
  int32_t* out_tids;
  uint32_t* d_out_count;
  uint32_t out_cap;      // survivors beyond out_cap are dropped and flagged
  uint32_t* d_overflow;  // nullable
  uint64_t* tile_status;
  uint32_t* tile_counter;
};

__device__ __forceinline__ bool eval_pred(const DevPredK& p, int64_t v) {
  if (p.kind == 1) return v >= p.lo && v <= p.hi;
  if (p.kind == DDQ_PRED_BITSET) return bitset_hit(p.in_vals, p.lo, v);
  bool m = false;
#pragma unroll
  for (int j = 0; j < 8; j++) m |= (j < p.n_in) && (v == p.in_vals[j]);
  return m;
}

// Load the 4 values of column `col` for items base..base+3 (dense rows, aligned).
__device__ __forceinline__ void load4(const void* col, int width, int64_t base, int64_t v[4]) {
  if (width == 8) {
    longlong2 a = ld_stream_l2(reinterpret_cast<const long long*>(col) + base);
    longlong2 b = ld_stream_l2(reinterpret_cast<const long long*>(col) + base + 2);
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  } else {
    int4 a = ld_stream_i4(reinterpret_cast<const int*>(col) + base);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
  }
}

template <bool kTids, bool kProbe, bool kSmemTable>
__global__ void __launch_bounds__(FT_THREADS)
filter_kernel(const __grid_constant__ FilterParams P) {
  extern __shared__ uint64_t s_table[];
  __shared__ uint32_t s_warp_tot[FT_WARPS];
  __shared__ uint32_t s_tile, s_excl;

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t n = P.d_in_count ? ld_relaxed_u32(P.d_in_count) : P.n_static;
  const uint32_t ntiles = (n + FT_TILE - 1) / FT_TILE;
  if (ntiles == 0) {
    if (blockIdx.x == 0 && threadIdx.x == 0) *P.d_out_count = 0;
    return;
  }
  if (kProbe && kSmemTable) {
    for (uint32_t i = threadIdx.x; i <= P.cap_mask; i += FT_THREADS) s_table[i] = P.table[i];
    __syncthreads();
  }
  const uint64_t* table = kSmemTable ? s_table : P.table;

  while (true) {
    if (threadIdx.x == 0) s_tile = atomicAdd(P.tile_counter, 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    if (tile >= ntiles) break;
    const int64_t wbase = (int64_t)tile * FT_TILE + warp * FT_WARP_ITEMS;

    int32_t rows[FT_ITEMS];
    uint32_t flags = 0;
    int32_t payload[kProbe ? FT_ITEMS : 1];

    // ---- 1. rows of this thread's items --------------------------------
#pragma unroll
    for (int s = 0; s < FT_SLOTS; s++) {
      const int64_t i0 = wbase + s * 128 + lane * 4;
      if (kTids) {
        if (i0 + 3 < n) {
          int4 t = ld_stream_i4(P.in_tids + i0);
          rows[s * 4 + 0] = t.x; rows[s * 4 + 1] = t.y; rows[s * 4 + 2] = t.z; rows[s * 4 + 3] = t.w;
        } else {
#pragma unroll
          for (int v = 0; v < 4; v++) rows[s * 4 + v] = (i0 + v < n) ? P.in_tids[i0 + v] : 0;
        }
      } else {
#pragma unroll
        for (int v = 0; v < 4; v++) rows[s * 4 + v] = (int32_t)(i0 + v);
      }
#pragma unroll
      for (int v = 0; v < 4; v++) flags |= (i0 + v < n ? 1u : 0u) << (s * 4 + v);
    }

    // ---- 2. predicates / probe ------------------------------------------
    if (!kProbe) {
      for (int p = 0; p < P.n_preds; p++) {
        const DevPredK& pr = P.preds[p];
        int64_t vals[FT_ITEMS];
        if (!kTids) {
#pragma unroll
          for (int s = 0; s < FT_SLOTS; s++) {
            const int64_t i0 = wbase + s * 128 + lane * 4;
            if (i0 + 3 < n) {
              load4(pr.col, pr.width, i0, &vals[s * 4]);
            } else {
#pragma unroll
              for (int v = 0; v < 4; v++) vals[s * 4 + v] = (i0 + v < n) ? col_at(pr.col, pr.width, i0 + v) : 0;
            }
          }
        } else {
#pragma unroll
          for (int k = 0; k < FT_ITEMS; k++)
            vals[k] = ((flags >> k) & 1u) ? col_at(pr.col, pr.width, rows[k]) : 0;
        }
#pragma unroll
        for (int k = 0; k < FT_ITEMS; k++)
          if (!eval_pred(pr, vals[k])) flags &= ~(1u << k);
      }
      if (P.eq_a) {  // FILTER_EQ: two aligned (positional) vectors must be equal
#pragma unroll
        for (int k = 0; k < FT_ITEMS; k++) {
          const int64_t pos = wbase + (k >> 2) * 128 + lane * 4 + (k & 3);
          if ((flags >> k) & 1u) {
            const int32_t va = __ldg(P.eq_a + pos), vb = __ldg(P.eq_b + pos);
            if (!vec_cmp(P.eq_cmp, va, vb)) flags &= ~(1u << k);
          }
        }
      }
    } else {
      int32_t keys[FT_ITEMS];
      if (!kTids) {
#pragma unroll
        for (int s = 0; s < FT_SLOTS; s++) {
          const int64_t i0 = wbase + s * 128 + lane * 4;
          if (i0 + 3 < n) {
            int4 t = ld_stream_i4(P.fk + i0);
            keys[s * 4 + 0] = t.x; keys[s * 4 + 1] = t.y; keys[s * 4 + 2] = t.z; keys[s * 4 + 3] = t.w;
          } else {
#pragma unroll
            for (int v = 0; v < 4; v++) keys[s * 4 + v] = (i0 + v < n) ? __ldg(P.fk + i0 + v) : 0;
          }
        }
      } else {
#pragma unroll
        for (int k = 0; k < FT_ITEMS; k++) {
          const int64_t pos = wbase + (k >> 2) * 128 + lane * 4 + (k & 3);
          keys[k] = ((flags >> k) & 1u) ? __ldg(P.fk + (P.fk_by_pos ? pos : (int64_t)rows[k])) : 0;
        }
      }
      if (P.direct) {
        uint32_t w[FT_ITEMS];
#pragma unroll
        for (int k = 0; k < FT_ITEMS; k++) {
          const uint32_t o = (uint32_t)(keys[k] - P.key_min);
          w[k] = (((flags >> k) & 1u) && o < P.range) ? __ldg(P.bitmap + (o >> 5)) : 0u;
        }
#pragma unroll
        for (int k = 0; k < FT_ITEMS; k++) {
          const uint32_t o = (uint32_t)(keys[k] - P.key_min);
          if (!((w[k] >> (o & 31)) & 1u)) flags &= ~(1u << k);
        }
        if (P.out_payload) {
#pragma unroll
          for (int k = 0; k < FT_ITEMS; k++)
            payload[k] = ((flags >> k) & 1u) ? __ldg(P.payarr + (uint32_t)(keys[k] - P.key_min)) : 0;
        }
      } else {
        uint32_t h[FT_ITEMS];
        uint64_t sl[FT_ITEMS];
#pragma unroll
        for (int k = 0; k < FT_ITEMS; k++) {
          h[k] = ht_hash(keys[k], P.shift);
          sl[k] = ((flags >> k) & 1u) ? table[h[k]] : HT_EMPTY;
        }
#pragma unroll
        for (int k = 0; k < FT_ITEMS; k++) {
          uint64_t s = sl[k];
          uint32_t hh = h[k];
          while (s != HT_EMPTY && ht_key(s) != keys[k]) {
            hh = (hh + 1) & P.cap_mask;
            s = table[hh];
          }
          if (s == HT_EMPTY) flags &= ~(1u << k);
          payload[k] = ht_val(s);
        }
      }
    }

    // ---- 3. stable compaction: warp scan of packed per-slot counts -------
    uint32_t packed = 0;
#pragma unroll
    for (int s = 0; s < FT_SLOTS; s++) packed |= (uint32_t)__popc((flags >> (4 * s)) & 0xFu) << (8 * s);
    const uint32_t incl = warp_incl_scan(packed, lane);
    const uint32_t excl = incl - packed;
    const uint32_t wtot = __shfl_sync(FULL, incl, 31);
    uint32_t slot_off[FT_SLOTS];
    uint32_t acc = 0;
#pragma unroll
    for (int s = 0; s < FT_SLOTS; s++) {
      slot_off[s] = acc;
      acc += (wtot >> (8 * s)) & 0xFFu;
    }
    if (lane == 0) s_warp_tot[warp] = acc;
    __syncthreads();
    uint32_t warp_off = 0, block_tot = 0;
#pragma unroll
    for (int w = 0; w < FT_WARPS; w++) {
      uint32_t t = s_warp_tot[w];
      warp_off += (w < warp) ? t : 0;
      block_tot += t;
    }
    if (warp == 0) {
      uint32_t e = lookback(P.tile_status, tile, block_tot, lane);
      if (lane == 0) {
        s_excl = e;
        if (tile == ntiles - 1) {
          const uint32_t tot = e + block_tot;
          *P.d_out_count = tot < P.out_cap ? tot : P.out_cap;
          if (tot > P.out_cap && P.d_overflow) atomicMax(P.d_overflow, 4u);
        }
      }
    }
    __syncthreads();
    const uint32_t base_out = s_excl + warp_off;

    // ---- 4. write survivors (each warp slot is a contiguous output run) ---
#pragma unroll
    for (int s = 0; s < FT_SLOTS; s++) {
      uint32_t pos = base_out + slot_off[s] + ((excl >> (8 * s)) & 0xFFu);
      const int64_t i0 = wbase + s * 128 + lane * 4;
#pragma unroll
      for (int v = 0; v < 4; v++) {
        const int k = s * 4 + v;
        if (((flags >> k) & 1u) && pos < P.out_cap) {
          P.out_tids[pos] = rows[k];
          if (kProbe && P.out_payload) P.out_payload[pos] = payload[k];
          for (int c = 0; c < P.n_carry; c++) P.carry_out[c][pos] = __ldg(P.carry_in[c] + i0 + v);
          pos++;
        }
      }
    }
    __syncthreads();  // s_tile / s_warp_tot reuse
  }
}

// ---------------------------------------------------------------------------
template <bool kTids, bool kProbe, bool kSmem>
static int occupancy_of(size_t smem) {
  int dev = 0, sms = 0, occ = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (smem > 48 * 1024)
    cudaFuncSetAttribute(filter_kernel<kTids, kProbe, kSmem>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)smem);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, filter_kernel<kTids, kProbe, kSmem>, FT_THREADS, smem);
  if (occ < 1) occ = 1;
  return sms * occ;
}

template <bool kTids, bool kProbe, bool kSmem>
static cudaError_t launch_t(const FilterParams& p, int64_t n_cap, size_t smem, cudaStream_t st) {
  int max_blocks = occupancy_of<kTids, kProbe, kSmem>(smem);
  int64_t ntiles = (n_cap + FT_TILE - 1) / FT_TILE;
  int grid = (int)(ntiles < max_blocks ? (ntiles < 1 ? 1 : ntiles) : max_blocks);
  filter_kernel<kTids, kProbe, kSmem><<<grid, FT_THREADS, smem, st>>>(p);
  return cudaGetLastError();
}

size_t filter_scratch_bytes(int64_t n_cap) {
  int64_t ntiles = (n_cap + FT_TILE - 1) / FT_TILE;
  return (size_t)(ntiles + 1) * 8 + 256;
}

constexpr size_t kSmemTableMax = 96 * 1024;

cudaError_t launch_filter(const FilterArgs& a, cudaStream_t st) {
  if (a.in_bits || a.out_bits) {  // row bitmaps exist only for the warp-autonomous kernels
    if (!ws_supported(a)) return cudaErrorInvalidValue;
    return launch_ws(a, st);
  }
  if (!a.stable && ws_supported(a)) {
    static const char* env = getenv("DDQ_WS");  // "0": the group-pipelined scan kernel (scan.cu)
    if (!env || env[0] != '0') return launch_ws(a, st);
  }
  if (!a.stable && scan_supported(a)) return launch_scan(a, st);
  FilterParams p{};
  p.in_tids = a.in_tids;
  p.d_in_count = a.d_in_count;
  p.n_static = (uint32_t)a.n_cap;
  p.n_preds = a.n_preds;
  for (int i = 0; i < a.n_preds && i < 4; i++) {
    p.preds[i].col = a.preds[i].col;
    p.preds[i].width = a.preds[i].width;
    p.preds[i].kind = a.preds[i].kind;
    p.preds[i].lo = a.preds[i].lo;
    p.preds[i].hi = a.preds[i].hi;
    p.preds[i].n_in = a.preds[i].n_in;
    for (int j = 0; j < 8; j++) p.preds[i].in_vals[j] = a.preds[i].in_vals[j];
  }
  p.table = a.table;
  p.cap_mask = a.capacity ? a.capacity - 1 : 0;
  int lg = 0;
  while ((1u << lg) < a.capacity) lg++;
  p.shift = 32 - lg;
  p.fk = a.fk;
  p.out_payload = a.out_payload;
  p.fk_by_pos = a.fk_by_pos ? 1 : 0;
  p.eq_a = a.eq_a;
  p.eq_b = a.eq_b;
  p.eq_cmp = a.eq_cmp;
  p.direct = a.bitmap != nullptr;
  p.bitmap = a.bitmap;
  p.payarr = a.payarr;
  p.key_min = a.key_min;
  p.range = a.range;
  p.n_carry = a.n_carry;
  for (int c = 0; c < a.n_carry && c < 4; c++) {
    p.carry_in[c] = a.carry_in[c];
    p.carry_out[c] = a.carry_out[c];
  }
  p.out_tids = a.out_tids;
  p.d_out_count = a.d_out_count;
  p.out_cap = (uint32_t)(a.out_cap > 0 ? a.out_cap : a.n_cap);
  p.d_overflow = a.d_overflow;
  uint8_t* sc = reinterpret_cast<uint8_t*>(a.scratch);
  p.tile_counter = reinterpret_cast<uint32_t*>(sc);
  p.tile_status = reinterpret_cast<uint64_t*>(sc + 256);
  cudaError_t e = init_fill(a.scratch, filter_scratch_bytes(a.n_cap), 0, st);
  if (e != cudaSuccess) return e;
  const bool tids = a.in_tids != nullptr;
  if (!a.probe) {
    return tids ? launch_t<true, false, false>(p, a.n_cap, 0, st) : launch_t<false, false, false>(p, a.n_cap, 0, st);
  }
  size_t tbytes = (size_t)a.capacity * 8;
  if (!p.direct && tbytes <= kSmemTableMax && !a.no_smem) {
    return tids ? launch_t<true, true, true>(p, a.n_cap, tbytes, st)
                : launch_t<false, true, true>(p, a.n_cap, tbytes, st);
  }
  return tids ? launch_t<true, true, false>(p, a.n_cap, 0, st) : launch_t<false, true, false>(p, a.n_cap, 0, st);
}

}  // namespace ddq
