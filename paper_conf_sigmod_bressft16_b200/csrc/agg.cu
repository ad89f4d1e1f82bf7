// agg.cu -- group-by aggregation over a TID list for small group counts
// (S8(a6): SSB 1..800 groups, TPC-H Q5/Q6), the last operator of every plan.
//
// B200 design ("aggregate"): the predecessor groupby_kernel handled
// one row per lane per iteration (TID -> key -> argument gathers -> warp match ->
// peer reduction -> atomics: a dependent chain of global round trips, ILP 1) and
// ran at ~1 TB/s of its sector bytes.  Here
//   * one persistent CTA of 16 warps per SM; every warp walks its own 256-item
//     tiles (8 items per lane, TIDs and positional key vectors read with 16-byte
//     loads, the next tile's TIDs prefetched); every argument column is gathered
//     for the lane's 8 items at once (8 independent loads in flight);
//   * every lane keeps a running (group key, int128 partial sums) in registers and
//     touches the shared-memory table only when its key changes -- a single-group
//     query (Q1.x, Q6) never does until the end, a 150-group one does per row but
//     with conflict-free random slots (no warp match / shuffle reduction);
//   * the shared-memory table accumulates every aggregate as a 128-bit two's
//     complement number in FOUR 32-bit limbs updated with native 32-bit shared
//     atomics (sm_100a has no 64-bit shared atomicAdd: it compiles to a CAS spin
//     loop, which ncu showed at 45 % of the kernel's instructions); a limb is only
//     touched when its addend or the carry into it is non-zero, so a small
//     positive partial sum costs one returning atomic; the table is merged into
//     the global int128 table (two 64-bit atomics with carry) once per CTA.
// Sums are exact int128 whatever the order (integer addition is associative).
#include <climits>
#include <cstdint>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "ops_internal.h"

namespace ddq {

namespace {

constexpr int AG_NW = 16;                // warps per CTA
constexpr int AG_ITEMS = 8;              // items per lane per tile
constexpr int AG_TILE = 32 * AG_ITEMS;   // items per warp tile
constexpr uint32_t AG_MAX_SLOTS = 2048;  // shared-memory table slots

struct AggParams {
  const int32_t* tids;
  const uint32_t* d_count;
  int32_t n_keys;
  const int32_t* key_vec[3];  // positional (aligned with the TIDs), or
  const int32_t* key_col[3];  // a column gathered at the TIDs
  int32_t key_shift[3];
  int32_t kind[2];
  const void* arg[2][3];
  int32_t width[2][3];
  long long* g_keys;
  unsigned long long* g_accs;  // [(a * cap + slot) * 2 + {0: lo, 1: hi}]
  uint32_t cap_mask;
  int32_t shift;
  uint32_t* d_error;
  uint32_t s_slots;
  int32_t s_shift;
  // fused predicates (reading O26): conjunction evaluated at the TIDs first
  int32_t n_preds;
  struct Pred {
    const void* col;
    int32_t width, kind;
    int64_t lo;
    uint64_t d64;  // RANGE: (u64)(v - lo) <= d64
    int32_t empty, n_in;
    int64_t in_vals[8];
  } preds[4];
  uint32_t* d_rows;
};

__device__ __forceinline__ int64_t find_or_insert(long long* keys, uint32_t mask, uint32_t h, long long key) {
  for (uint32_t probes = 0; probes <= mask; probes++) {
    const long long cur = keys[h];
    if (cur == key) return h;
    if (cur == GB_EMPTY) {
      const long long old = (long long)atomicCAS(reinterpret_cast<unsigned long long*>(keys + h),
                                                 (unsigned long long)GB_EMPTY, (unsigned long long)key);
      if (old == GB_EMPTY || old == key) return h;
    }
    h = (h + 1) & mask;
  }
  return -1;
}

__device__ __forceinline__ void add_i128(unsigned long long* plo, unsigned long long* phi, unsigned long long lo,
                                         long long hi) {
  const unsigned long long old = atomicAdd(plo, lo);
  const long long h = hi + ((old + lo < old) ? 1 : 0);
  if (h) atomicAdd(phi, (unsigned long long)h);
}

// the lane's 8 values of an argument column at its TIDs (independent loads)
__device__ __forceinline__ void gather8(const void* col, int width, const int32_t (&tid)[AG_ITEMS], uint32_t valid,
                                        long long (&v)[AG_ITEMS]) {
  if (width == 8) {
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++)
      v[j] = ((valid >> j) & 1u) ? ldg_gather(reinterpret_cast<const long long*>(col) + (uint32_t)tid[j]) : 0;
  } else {
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++)
      v[j] = ((valid >> j) & 1u) ? (long long)ldg_gather(reinterpret_cast<const int32_t*>(col) + (uint32_t)tid[j]) : 0;
  }
}

// aggregate a's per-item value (the fixed expression set of include/ddq.h)
__device__ __forceinline__ void agg_values(const AggParams& P, int a, const int32_t (&tid)[AG_ITEMS], uint32_t valid,
                                           long long (&v)[AG_ITEMS]) {
  const int k = P.kind[a];
  if (k == DDQ_AGG_COUNT) {
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++) v[j] = 1;
    return;
  }
  gather8(P.arg[a][0], P.width[a][0], tid, valid, v);
  if (k == DDQ_AGG_SUM) return;
  long long y[AG_ITEMS];
  gather8(P.arg[a][1], P.width[a][1], tid, valid, y);
  if (k == DDQ_AGG_SUM_MUL) {
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++) v[j] *= y[j];
  } else if (k == DDQ_AGG_SUM_SUB) {
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++) v[j] -= y[j];
  } else if (k == DDQ_AGG_SUM_MUL_100M) {
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++) v[j] *= 100 - y[j];
  } else {  // DDQ_AGG_SUM_MUL_100M_100P
    long long z[AG_ITEMS];
    gather8(P.arg[a][2], P.width[a][2], tid, valid, z);
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++) v[j] = v[j] * (100 - y[j]) * (100 + z[j]);
  }
}

__device__ __forceinline__ uint32_t hash32(long long k, int shift) {
  const uint32_t x = (uint32_t)k ^ (uint32_t)((unsigned long long)k >> 32);
  return (x * 0x9E3779B1u) >> shift;  // shift = 32 - log2(slots)
}

template <int NA>
__global__ void __launch_bounds__(AG_NW * 32, 1) agg_ws_kernel(const __grid_constant__ AggParams P) {
  extern __shared__ __align__(16) unsigned long long ag_smem[];
  long long* s_keys = reinterpret_cast<long long*>(ag_smem);
  uint32_t* s_acc = reinterpret_cast<uint32_t*>(ag_smem + P.s_slots);  // [(a * S + slot) * 4 + limb]
  const uint32_t S = P.s_slots, smask = S - 1;
  for (uint32_t i = threadIdx.x; i < S; i += blockDim.x) s_keys[i] = GB_EMPTY;
  for (uint32_t i = threadIdx.x; i < S * 4 * NA; i += blockDim.x) s_acc[i] = 0;
  __syncthreads();

  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t n = ld_relaxed_u32(P.d_count);
  const uint32_t ntiles = (n + AG_TILE - 1) / AG_TILE;
  const uint32_t W = gridDim.x * AG_NW;
  const uint32_t lofs = lane * 4;  // item (s, v) of lane l sits at tile*256 + s*128 + l*4 + v

  long long cur = GB_EMPTY;  // the lane's running group and its int128 partial sums
  unsigned long long lo[NA];
  long long hi[NA];
#pragma unroll
  for (int a = 0; a < NA; a++) lo[a] = 0, hi[a] = 0;
  auto flush = [&]() {
    if (cur == GB_EMPTY) return;
    uint32_t h = hash32(cur, P.s_shift);
    int64_t slot = -1;
    for (uint32_t probes = 0; probes <= smask; probes++) {
      const long long k = s_keys[h];
      if (k == cur) {
        slot = h;
        break;
      }
      if (k == GB_EMPTY) {
        const long long old = (long long)atomicCAS(reinterpret_cast<unsigned long long*>(s_keys + h),
                                                   (unsigned long long)GB_EMPTY, (unsigned long long)cur);
        if (old == GB_EMPTY || old == cur) {
          slot = h;
          break;
        }
      }
      h = (h + 1) & smask;
    }
    if (slot >= 0) {
#pragma unroll
      for (int a = 0; a < NA; a++) {  // 128-bit add in 32-bit limbs, carries rippled
        uint32_t* w = s_acc + ((size_t)a * S + slot) * 4;
        const uint32_t limb[4] = {(uint32_t)lo[a], (uint32_t)(lo[a] >> 32), (uint32_t)hi[a],
                                  (uint32_t)((unsigned long long)hi[a] >> 32)};
        uint32_t c = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) {
          const uint32_t x = limb[k] + c;
          const uint32_t cx = (c && x == 0u) ? 1u : 0u;  // limb + carry wrapped
          if (x == 0u) {
            c = cx;
          } else if (k == 3) {
            atomicAdd(w + 3, x);  // top limb: carry out of 128 bits is discarded
          } else {
            const uint32_t old = atomicAdd(w + k, x);
            c = (old + x < old) ? 1u : 0u;
          }
        }
      }
    } else {  // CTA table full: straight into the global table
      slot = find_or_insert(P.g_keys, P.cap_mask, gb_hash(cur, P.shift), cur);
      if (slot < 0) {
        atomicMax(P.d_error, 2u);
      } else {
#pragma unroll
        for (int a = 0; a < NA; a++)
          add_i128(&P.g_accs[((size_t)a * (P.cap_mask + 1) + slot) * 2],
                   &P.g_accs[((size_t)a * (P.cap_mask + 1) + slot) * 2 + 1], lo[a], hi[a]);
      }
    }
  };

  auto load8 = [&](const int32_t* base_ptr, uint32_t t0, int4 (&r)[2]) {
    if (t0 + AG_TILE <= n) {
      r[0] = ld_stream_i4(base_ptr + t0 + lofs);
      r[1] = ld_stream_i4(base_ptr + t0 + 128 + lofs);
    } else {
#pragma unroll
      for (int s2 = 0; s2 < 2; s2++) {
        const uint32_t i = t0 + s2 * 128 + lofs;
        r[s2].x = i < n ? base_ptr[i] : 0;
        r[s2].y = i + 1 < n ? base_ptr[i + 1] : 0;
        r[s2].z = i + 2 < n ? base_ptr[i + 2] : 0;
        r[s2].w = i + 3 < n ? base_ptr[i + 3] : 0;
      }
    }
  };
  uint32_t tile = blockIdx.x * AG_NW + warp;
  uint32_t rows = 0;  // rows passing the fused predicates (d_rows)
  int4 nt[2];
  if (tile < ntiles) load8(P.tids, tile * AG_TILE, nt);
  for (; tile < ntiles; tile += W) {
    const uint32_t t0 = tile * AG_TILE;
    int32_t tid[AG_ITEMS] = {nt[0].x, nt[0].y, nt[0].z, nt[0].w, nt[1].x, nt[1].y, nt[1].z, nt[1].w};
    if (tile + W < ntiles) load8(P.tids, (tile + W) * AG_TILE, nt);
    uint32_t valid = 0xFFu;
    if (t0 + AG_TILE > n) {
      valid = 0;
#pragma unroll
      for (int j = 0; j < AG_ITEMS; j++) valid |= (t0 + (j >> 2) * 128 + lofs + (j & 3) < n ? 1u : 0u) << j;
    }
    for (int p = 0; p < P.n_preds; p++) {  // fused selection: later columns only for live rows
      const AggParams::Pred& pr = P.preds[p];
      long long x[AG_ITEMS];
      gather8(pr.col, pr.width, tid, valid, x);
      uint32_t m = 0;
      if (pr.kind == DDQ_PRED_RANGE) {
#pragma unroll
        for (int j = 0; j < AG_ITEMS; j++) m |= ((uint64_t)(x[j] - pr.lo) <= pr.d64 ? 1u : 0u) << j;
        if (pr.empty) m = 0;
      } else {
#pragma unroll
        for (int j = 0; j < AG_ITEMS; j++) {
          bool hit = false;
#pragma unroll
          for (int q = 0; q < 8; q++) hit |= (q < pr.n_in) && (x[j] == pr.in_vals[q]);
          m |= (hit ? 1u : 0u) << j;
        }
      }
      valid &= m;
    }
    if (P.d_rows) rows += __popc(valid);
    long long key[AG_ITEMS];
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++) key[j] = 0;
    for (int k = 0; k < P.n_keys; k++) {
      int32_t c[AG_ITEMS];
      if (P.key_vec[k]) {
        int4 r[2];
        load8(P.key_vec[k], t0, r);
        c[0] = r[0].x; c[1] = r[0].y; c[2] = r[0].z; c[3] = r[0].w;
        c[4] = r[1].x; c[5] = r[1].y; c[6] = r[1].z; c[7] = r[1].w;
      } else {
#pragma unroll
        for (int j = 0; j < AG_ITEMS; j++) c[j] = ((valid >> j) & 1u) ? ldg_gather(P.key_col[k] + (uint32_t)tid[j]) : 0;
      }
#pragma unroll
      for (int j = 0; j < AG_ITEMS; j++) key[j] |= (long long)(uint32_t)c[j] << P.key_shift[k];
    }
    long long v[NA][AG_ITEMS];
#pragma unroll
    for (int a = 0; a < NA; a++) agg_values(P, a, tid, valid, v[a]);
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++) {
      if (!((valid >> j) & 1u)) continue;
      if (key[j] != cur) {
        flush();
        cur = key[j];
#pragma unroll
        for (int a = 0; a < NA; a++) lo[a] = 0, hi[a] = 0;
      }
#pragma unroll
      for (int a = 0; a < NA; a++) {  // exact int128 running sum
        const unsigned long long s2 = lo[a] + (unsigned long long)v[a][j];
        hi[a] += (v[a][j] < 0 ? -1 : 0) + (s2 < lo[a] ? 1 : 0);
        lo[a] = s2;
      }
    }
  }
  flush();
  if (P.d_rows) {
    rows = __reduce_add_sync(FULL, rows);
    if (lane == 0 && rows) atomicAdd(P.d_rows, rows);
  }
  __syncthreads();
  // merge this CTA's table into the global one: int128 = H * 2^32 + L
  for (uint32_t s2 = threadIdx.x; s2 < S; s2 += blockDim.x) {
    const long long key = s_keys[s2];
    if (key == GB_EMPTY) continue;
    const int64_t g = find_or_insert(P.g_keys, P.cap_mask, gb_hash(key, P.shift), key);
    if (g < 0) {
      atomicMax(P.d_error, 2u);
      continue;
    }
#pragma unroll
    for (int a = 0; a < NA; a++) {
      const uint32_t* w = s_acc + ((size_t)a * S + s2) * 4;
      const unsigned long long lo2 = (unsigned long long)w[0] | ((unsigned long long)w[1] << 32);
      const long long hi2 = (long long)((unsigned long long)w[2] | ((unsigned long long)w[3] << 32));
      add_i128(&P.g_accs[((size_t)a * (P.cap_mask + 1) + g) * 2], &P.g_accs[((size_t)a * (P.cap_mask + 1) + g) * 2 + 1],
               lo2, hi2);
    }
  }
}

}  // namespace

bool agg_ws_supported(const int32_t* tids, const int32_t* const* key_vec, int n_keys, int n_aggs,
                      uint32_t capacity) {
  if (!tids || ((uintptr_t)tids & 15) || n_aggs < 1 || n_aggs > 2 || capacity > AG_MAX_SLOTS) return false;
  for (int k = 0; k < n_keys; k++)
    if (key_vec && key_vec[k] && ((uintptr_t)key_vec[k] & 15)) return false;
  return true;
}

cudaError_t launch_agg_ws(const int32_t* tids, const uint32_t* d_count, int64_t n_cap,
                          const int32_t* const* key_vec, const int32_t* const* key_col, int n_keys,
                          const int32_t* key_bits, const ddq_dev_agg* aggs, int n_aggs, void* table,
                          uint32_t capacity, uint32_t* d_error, cudaStream_t st, const BuildPreds* preds,
                          uint32_t* d_rows) {
  AggParams p{};
  p.d_rows = d_rows;
  if (preds) {
    p.n_preds = preds->n;
    for (int i = 0; i < preds->n && i < 4; i++) {
      const ddq_dev_pred& d = preds->p[i];
      AggParams::Pred& q = p.preds[i];
      q.col = d.col;
      q.width = d.width;
      q.kind = d.kind;
      q.lo = d.lo;
      q.empty = d.hi < d.lo;
      q.d64 = q.empty ? 0 : (uint64_t)d.hi - (uint64_t)d.lo;
      q.n_in = d.n_in;
      for (int j = 0; j < 8; j++) q.in_vals[j] = d.in_vals[j];
    }
  }
  p.tids = tids;
  p.d_count = d_count;
  p.n_keys = n_keys;
  for (int k = 0, sh = 0; k < 3; k++) {
    p.key_shift[k] = sh;
    sh += (key_bits && key_bits[k] > 0) ? key_bits[k] : 21;
  }
  for (int k = 0; k < n_keys; k++) {
    p.key_vec[k] = key_vec ? key_vec[k] : nullptr;
    p.key_col[k] = key_col ? key_col[k] : nullptr;
  }
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
  uint32_t S = capacity < 64 ? 64 : capacity;  // capacity >= 2x the group bound (load <= 0.5)
  int slg = 0;
  while ((1u << slg) < S) slg++;
  p.s_slots = S;
  p.s_shift = 32 - slg;
  const size_t smem = (size_t)S * (8 + 16 * (size_t)n_aggs);
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(agg_ws_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, AG_MAX_SLOTS * (8 + 16));
    cudaFuncSetAttribute(agg_ws_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, AG_MAX_SLOTS * (8 + 32));
    attr = true;
  }
  const int64_t ntiles = (n_cap + AG_TILE - 1) / AG_TILE;  // upper bound
  int64_t grid = num_sms();
  const int64_t need = (ntiles + AG_NW - 1) / AG_NW;
  if (grid > need) grid = need < 1 ? 1 : need;
  if (n_aggs == 1) agg_ws_kernel<1><<<(int)grid, AG_NW * 32, smem, st>>>(p);
  else agg_ws_kernel<2><<<(int)grid, AG_NW * 32, smem, st>>>(p);
  return cudaGetLastError();
}

}  // namespace ddq
