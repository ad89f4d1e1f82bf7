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
#include <algorithm>
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
  // fused probe / fetch terms (reading O37), evaluated after the predicates
  int32_t n_terms;
  struct Term {
    int32_t kind, emit;
    const int32_t* fk;
    const uint32_t* bitmap;
    const int32_t* payarr;
    int32_t key_min;
    uint32_t range;
    const uint64_t* table;
    uint32_t cap_mask;
    int32_t shift;
    int32_t key_shift;  // the payload is group key bits at this shift (-1: not a key)
  } terms[4];
  int32_t key_pay[3];  // key k from payload slot key_pay[k] (>= 0): packed by its term
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
      } else if (pr.kind == DDQ_PRED_BITSET) {
#pragma unroll
        for (int j = 0; j < AG_ITEMS; j++) m |= (bitset_hit(pr.in_vals, pr.lo, x[j]) ? 1u : 0u) << j;
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
    // fused probe / fetch terms (O37): gather the fk at the live rows, look it up; an
    // emitted payload that is a group key is packed into the key right away
    long long key[AG_ITEMS];
#pragma unroll
    for (int j = 0; j < AG_ITEMS; j++) key[j] = 0;
    for (int t = 0; t < P.n_terms; t++) {
      const AggParams::Term& T = P.terms[t];
      int32_t fk[AG_ITEMS];
#pragma unroll
      for (int j = 0; j < AG_ITEMS; j++) fk[j] = ((valid >> j) & 1u) ? ldg_gather(T.fk + (uint32_t)tid[j]) : 0;
      uint32_t hit = 0;
      int32_t v[AG_ITEMS];
      if (T.bitmap) {  // join index: the bits first (independent loads), payloads of the hits
        uint32_t w[AG_ITEMS];
#pragma unroll
        for (int j = 0; j < AG_ITEMS; j++) {
          const uint32_t o = (uint32_t)(fk[j] - T.key_min);
          w[j] = ((valid >> j) & 1u) && o < T.range ? __ldg(T.bitmap + (o >> 5)) : 0u;
        }
#pragma unroll
        for (int j = 0; j < AG_ITEMS; j++)
          hit |= ((w[j] >> ((uint32_t)(fk[j] - T.key_min) & 31u)) & 1u) << j;
        if (T.emit >= 0) {
#pragma unroll
          for (int j = 0; j < AG_ITEMS; j++)
            v[j] = ((hit >> j) & 1u) ? __ldg(T.payarr + (uint32_t)(fk[j] - T.key_min)) : INT32_MIN;
        }
      } else {  // open addressing
#pragma unroll
        for (int j = 0; j < AG_ITEMS; j++) {
          v[j] = INT32_MIN;
          if (!((valid >> j) & 1u)) continue;
          uint32_t h = ht_hash(fk[j], T.shift);
          uint64_t sl = __ldg(T.table + h);
          while (sl != HT_EMPTY && ht_key(sl) != fk[j]) {
            h = (h + 1) & T.cap_mask;
            sl = __ldg(T.table + h);
          }
          if (sl != HT_EMPTY) {
            hit |= 1u << j;
            v[j] = ht_val(sl);
          }
        }
      }
      if (T.kind == DDQ_TERM_PROBE) valid &= hit;
      if (T.key_shift >= 0) {
#pragma unroll
        for (int j = 0; j < AG_ITEMS; j++) key[j] |= (long long)(uint32_t)v[j] << T.key_shift;
      }
    }
    if (P.d_rows) rows += __popc(valid);
    for (int k = 0; k < P.n_keys; k++) {
      if (P.key_pay[k] >= 0) continue;  // packed by its term
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


// ---- dense small-domain aggregation (TPC-H Q1 shape): every row of the table,
// fused range / IN predicates (reading O26), every key a dictionary code with
// key_bits (D = 2^bits <= 32 groups), <= 8 aggregates.  Replaces select -> TID
// list -> gather-based aggregation (for Q1: 177 M TIDs written and re-read, the
// operand mapping interpreted per row, 8.9 ms at SF30).
//   * the columns are streamed by TMA: one CTA per SM, a ring of DS_S stages of
//     DS_SR rows; thread 0 issues one cp.async.bulk per column per stage onto the
//     stage's mbarrier, so the whole ring (~70 KB per SM) is in flight while the
//     CTA computes on the oldest stage (a register-staged version with predicated
//     loads serialised three DRAM round trips per row batch: 1.6 TB/s);
//   * every thread owns D x A int64 partials in shared memory, [entry][thread]
//     (conflict-free), updated with a plain read-modify-write; a signed-overflow
//     test spills a partial into a per-CTA int128 cell (exact for any data);
//   * at the end one warp per (group, aggregate) entry sums the CTA's partials in
//     int128 and adds them to the global table -- only for groups some row hit.
constexpr int DS_T = 256;             // threads per CTA
constexpr int DS_R = 4;               // rows per thread per stage
constexpr int DS_SR = DS_T * DS_R;    // rows per ring stage
constexpr int DS_MAXC = 12;           // distinct columns streamed
constexpr int DS_MAX_DA = 64;
constexpr int DS_SMAX = 8;            // ring stages at most
static_assert(4 /*DS_R*/ * 8 <= 32, "overflow mask: DS_R x A bits");
constexpr size_t DS_SMEM_MAX = 227 * 1024 - 1024;

struct DenseAggParams {
  uint32_t n;
  int32_t n_cols;
  const void* col[DS_MAXC];
  int32_t width[DS_MAXC];
  int32_t off[DS_MAXC];  // byte offset of the column's segment inside a stage
  uint32_t stage_bytes;
  int32_t n_stages;
  int32_t n_preds;
  AggParams::Pred preds[4];
  int32_t pcol[4];
  int32_t n_keys;
  int32_t kcol[3];
  int32_t key_shift[3];
  uint32_t D;
  int32_t n_aggs;
  int32_t kind[8];
  int32_t acol[8][3];
  long long* g_keys;
  unsigned long long* g_accs;
  uint32_t cap_mask;
  int32_t shift;
  uint32_t* d_error;
  uint32_t* d_rows;
};

__device__ __forceinline__ bool pred_ok(const AggParams::Pred& p, long long v) {
  if (p.kind == DDQ_PRED_RANGE) return !p.empty && (uint64_t)(v - p.lo) <= p.d64;
  if (p.kind == DDQ_PRED_BITSET) return bitset_hit(p.in_vals, p.lo, v);
  bool m = false;
#pragma unroll
  for (int j = 0; j < 8; j++) m |= (j < p.n_in) && (v == p.in_vals[j]);
  return m;
}

// KINDS: the aggregate kinds, 3 bits each (compile-time straight-line code for the
// plan shapes of the workload, e.g. TPC-H Q1's), or DS_RUNTIME (kinds read per stage)
constexpr uint32_t DS_RUNTIME = 0xFFFFFFFFu;
constexpr uint32_t ds_kinds(int k0, int k1 = 0, int k2 = 0, int k3 = 0, int k4 = 0, int k5 = 0, int k6 = 0, int k7 = 0) {
  return (uint32_t)k0 | (uint32_t)k1 << 3 | (uint32_t)k2 << 6 | (uint32_t)k3 << 9 | (uint32_t)k4 << 12 |
         (uint32_t)k5 << 15 | (uint32_t)k6 << 18 | (uint32_t)k7 << 21;
}
// TPC-H Q1: sum_qty, sum_base_price, sum_disc_price, sum_charge, sum(l_discount), count(*)
constexpr uint32_t DS_Q1 = ds_kinds(DDQ_AGG_SUM, DDQ_AGG_SUM, DDQ_AGG_SUM_MUL_100M, DDQ_AGG_SUM_MUL_100M_100P,
                                    DDQ_AGG_SUM, DDQ_AGG_COUNT);

// kOvf: test every partial add for signed overflow (wrap-and-count).  The host drops
// the test when the columns' value ranges prove that no thread partial can reach
// 2^62 (|row value| x rows per thread), which holds for TPC-H / SSB measures.
template <int NA, uint32_t KINDS, bool kOvf>
__global__ void __launch_bounds__(DS_T + 32, 1) agg_dense_small_kernel(const __grid_constant__ DenseAggParams P) {
  extern __shared__ __align__(128) uint8_t ds_smem[];
  __shared__ __align__(8) uint64_t full[DS_SMAX], empty[DS_SMAX];
  __shared__ uint32_t s_present, s_rows;
  constexpr int A = NA;
  const uint32_t DA = P.D * (uint32_t)A;
  uint8_t* ring = ds_smem;  // [n_stages][stage_bytes]
  long long* part = reinterpret_cast<long long*>(ds_smem + (size_t)P.n_stages * P.stage_bytes);  // [DA][DS_T]
  unsigned long long* spill = reinterpret_cast<unsigned long long*>(part + (size_t)DA * DS_T);      // [DA][2]
  const int tid = threadIdx.x;
  const uint32_t n = P.n;
  const uint32_t nch = (n + DS_SR - 1) / DS_SR;
  const int S = P.n_stages;

  auto issue = [&](uint32_t k) {  // thread 0: stage k of this CTA -> slot k % S
    const uint32_t ci = blockIdx.x + k * gridDim.x;
    const uint32_t row0 = ci * DS_SR;
    const uint32_t rows = min((uint32_t)DS_SR, n - row0);
    uint8_t* dst = ring + (size_t)(k % S) * P.stage_bytes;
    uint32_t bytes = 0;
    for (int c = 0; c < P.n_cols; c++) bytes += (rows * P.width[c] + 15) & ~15u;
    mbar_arrive_expect_tx(&full[k % S], bytes);
    for (int c = 0; c < P.n_cols; c++)
      tma_load_1d(dst + P.off[c], reinterpret_cast<const uint8_t*>(P.col[c]) + (size_t)row0 * P.width[c],
                  (rows * P.width[c] + 15) & ~15u, &full[k % S]);
  };
  if (tid == 0) {
    for (int s = 0; s < S; s++) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], DS_T / 32);  // one arrival per consumer warp
    }
    fence_mbar_init();
    s_present = 0;
    s_rows = 0;
  }
  if (tid < DS_T) {
    for (uint32_t e = 0; e < DA; e++) part[(size_t)e * DS_T + tid] = 0;
    for (uint32_t i = tid; i < DA * 2; i += DS_T) spill[i] = 0;
  }
  __syncthreads();
  uint32_t pm = 0, nrows = 0;
  if (tid >= DS_T) {
    // the producer warp: refills a slot as soon as every consumer warp released it
    // (no CTA-wide barrier per stage: consumer warps drift up to S stages apart)
    if (tid == DS_T)
      for (uint32_t k = 0; blockIdx.x + k * gridDim.x < nch; k++) {
        if (k >= (uint32_t)S) mbar_wait(&empty[k % S], (k / S - 1) & 1u);
        issue(k);
      }
  } else
  for (uint32_t k = 0; blockIdx.x + k * gridDim.x < nch; k++) {
    const uint32_t row0 = (blockIdx.x + k * gridDim.x) * DS_SR;
    const uint8_t* stage = ring + (size_t)(k % S) * P.stage_bytes;
    mbar_wait(&full[k % S], (k / S) & 1u);
    // vector-at-a-time: every per-operator decision (predicate width and kind,
    // aggregate kind, operand columns) is taken once per stage for the thread's
    // DS_R rows; dead rows add 0 (no per-row branches)
    uint32_t livem = 0;
#pragma unroll
    for (int j = 0; j < DS_R; j++) livem |= (row0 + j * DS_T + tid < n ? 1u : 0u) << j;
    for (int p = 0; p < P.n_preds; p++) {
      const AggParams::Pred& pr = P.preds[p];
      const uint8_t* b = stage + P.off[P.pcol[p]];
      long long v[DS_R];
      if (P.width[P.pcol[p]] == 8) {
#pragma unroll
        for (int j = 0; j < DS_R; j++) v[j] = reinterpret_cast<const long long*>(b)[j * DS_T + tid];
      } else {
#pragma unroll
        for (int j = 0; j < DS_R; j++) v[j] = reinterpret_cast<const int32_t*>(b)[j * DS_T + tid];
      }
      uint32_t m = 0;
      if (pr.kind == DDQ_PRED_RANGE) {
#pragma unroll
        for (int j = 0; j < DS_R; j++) m |= ((uint64_t)(v[j] - pr.lo) <= pr.d64 ? 1u : 0u) << j;
        if (pr.empty) m = 0;
      } else {
#pragma unroll
        for (int j = 0; j < DS_R; j++) m |= (pred_ok(pr, v[j]) ? 1u : 0u) << j;
      }
      livem &= m;
    }
    uint32_t idx[DS_R];  // partial index of (group, aggregate 0) for row j
#pragma unroll
    for (int j = 0; j < DS_R; j++) idx[j] = 0;
#pragma unroll
    for (int kk = 0; kk < 3; kk++) {
      if (kk >= P.n_keys) break;
      const int32_t* kc = reinterpret_cast<const int32_t*>(stage + P.off[P.kcol[kk]]);
#pragma unroll
      for (int j = 0; j < DS_R; j++) idx[j] |= (uint32_t)kc[j * DS_T + tid] << P.key_shift[kk];
    }
#pragma unroll
    for (int j = 0; j < DS_R; j++) {
      const uint32_t d = idx[j] & (P.D - 1);
      pm |= ((livem >> j) & 1u) << d;
      idx[j] = d * (uint32_t)(A * DS_T) + tid;
    }
    nrows += __popc(livem);
    long long v[A][DS_R];  // every aggregate's value for the thread's rows (dead rows: 0)
#pragma unroll
    for (int a = 0; a < A; a++) {
      const int kind = KINDS == DS_RUNTIME ? P.kind[a] : (int)((KINDS >> (3 * a)) & 7u);
      const long long* xs = reinterpret_cast<const long long*>(stage + P.off[P.acol[a][0]]) + tid;
      const long long* ys = reinterpret_cast<const long long*>(stage + P.off[P.acol[a][1]]) + tid;
      const long long* zs = reinterpret_cast<const long long*>(stage + P.off[P.acol[a][2]]) + tid;
      if (kind == DDQ_AGG_COUNT) {
#pragma unroll
        for (int j = 0; j < DS_R; j++) v[a][j] = 1;
      } else if (kind == DDQ_AGG_SUM) {
#pragma unroll
        for (int j = 0; j < DS_R; j++) v[a][j] = xs[j * DS_T];
      } else if (kind == DDQ_AGG_SUM_MUL) {
#pragma unroll
        for (int j = 0; j < DS_R; j++) v[a][j] = xs[j * DS_T] * ys[j * DS_T];
      } else if (kind == DDQ_AGG_SUM_SUB) {
#pragma unroll
        for (int j = 0; j < DS_R; j++) v[a][j] = xs[j * DS_T] - ys[j * DS_T];
      } else if (kind == DDQ_AGG_SUM_MUL_100M) {
#pragma unroll
        for (int j = 0; j < DS_R; j++) v[a][j] = xs[j * DS_T] * (100 - ys[j * DS_T]);
      } else {
#pragma unroll
        for (int j = 0; j < DS_R; j++) v[a][j] = xs[j * DS_T] * (100 - ys[j * DS_T]) * (100 + zs[j * DS_T]);
      }
      if (livem != (1u << DS_R) - 1u) {
#pragma unroll
        for (int j = 0; j < DS_R; j++) v[a][j] = ((livem >> j) & 1u) ? v[a][j] : 0;
      }
    }
    // row-major read-modify-writes: the A partials of one row are distinct slots
    // (independent loads, one shared-memory latency per row); consecutive rows of a
    // thread may hit the same group, which the in-order LSU keeps correct
    // partials wrap modulo 2^64; a signed overflow (never for SSB/TPC-H data) adds
    // +-2^64 to the entry's int128 cell, so slot + cell stays exact
    uint32_t omask = 0;
#pragma unroll
    for (int j = 0; j < DS_R; j++) {
      long long* row = part + idx[j];
      long long old[A];
#pragma unroll
      for (int a = 0; a < A; a++) old[a] = row[a * DS_T];
#pragma unroll
      for (int a = 0; a < A; a++) {
        const long long sum = (long long)((unsigned long long)old[a] + (unsigned long long)v[a][j]);
        row[a * DS_T] = sum;
        if (kOvf) omask |= (((old[a] ^ sum) & (v[a][j] ^ sum)) < 0 ? 1u : 0u) << (j * A + a);
      }
    }
    if (__builtin_expect(omask != 0, 0)) {
#pragma unroll
      for (int j = 0; j < DS_R; j++)
#pragma unroll
        for (int a = 0; a < A; a++)
          if ((omask >> (j * A + a)) & 1u) {
            unsigned long long* sp = spill + (size_t)(idx[j] - tid + (uint32_t)a * DS_T) / DS_T * 2;
            add_i128(sp, sp + 1, 0ull, v[a][j] > 0 ? 1 : -1);
          }
    }
    __syncwarp();  // this warp is done with the slot
    if ((tid & 31) == 0) mbar_arrive(&empty[k % S]);
  }
  pm = __reduce_or_sync(FULL, pm);
  nrows = __reduce_add_sync(FULL, nrows);
  if ((tid & 31) == 0) {
    if (pm) atomicOr(&s_present, pm);
    if (nrows) atomicAdd(&s_rows, nrows);
  }
  __syncthreads();
  if (tid == 0 && P.d_rows && s_rows) atomicAdd(P.d_rows, s_rows);
  const int lane = tid & 31, warp = tid >> 5;
  const uint32_t pres = s_present;
  if (tid < DS_T)
  for (uint32_t e = warp; e < DA; e += DS_T / 32) {
    const uint32_t g = e / A;
    const int a = (int)(e % A);
    if (!((pres >> g) & 1u)) continue;
    unsigned long long lo = 0;
    long long hi = 0;
    for (int t = lane; t < DS_T; t += 32) {
      const long long x = part[(size_t)e * DS_T + t];
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
      const int64_t slot = find_or_insert(P.g_keys, P.cap_mask, gb_hash(key, P.shift), key);
      if (slot < 0) {
        atomicMax(P.d_error, 2u);
      } else {
        unsigned long long* glo = &P.g_accs[((size_t)a * (P.cap_mask + 1) + slot) * 2];
        add_i128(glo, glo + 1, lo, hi);
      }
    }
  }
}

__global__ void iota_kernel(int32_t* out, uint32_t n, uint32_t* d_count) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) out[i] = (int32_t)i;
  if (blockIdx.x == 0 && threadIdx.x == 0) *d_count = n;
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
                          uint32_t* d_rows, const AggTerms* terms) {
  AggParams p{};
  p.d_rows = d_rows;
  p.key_pay[0] = p.key_pay[1] = p.key_pay[2] = -1;
  if (terms) {
    p.n_terms = terms->n;
    for (int t = 0; t < terms->n && t < 4; t++) {
      const AggTerm& a = terms->t[t];
      AggParams::Term& q = p.terms[t];
      q.kind = a.kind;
      q.emit = a.emit;
      q.fk = a.fk;
      q.bitmap = a.bitmap;
      q.payarr = a.payarr;
      q.key_min = a.key_min;
      q.range = a.range;
      q.table = a.table;
      q.cap_mask = a.capacity ? a.capacity - 1 : 0;
      int lg = 0;
      while (a.capacity && (1u << lg) < a.capacity) lg++;
      q.shift = 32 - lg;
      q.key_shift = -1;
    }
    for (int k = 0; k < 3; k++) p.key_pay[k] = terms->key_pay[k];
  }
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
  for (int k = 0; k < n_keys && k < 3; k++)  // a term's payload used as key k
    for (int t = 0; t < p.n_terms; t++)
      if (p.key_pay[k] >= 0 && p.terms[t].emit == p.key_pay[k]) p.terms[t].key_shift = p.key_shift[k];
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
  static const bool attr = [] {  // thread-safe one-time opt-in
    cudaFuncSetAttribute(agg_ws_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, AG_MAX_SLOTS * (8 + 16));
    cudaFuncSetAttribute(agg_ws_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, AG_MAX_SLOTS * (8 + 32));
    return true;
  }();
  (void)attr;
  const int64_t ntiles = (n_cap + AG_TILE - 1) / AG_TILE;  // upper bound
  int64_t grid = num_sms();
  const int64_t need = (ntiles + AG_NW - 1) / AG_NW;
  if (grid > need) grid = need < 1 ? 1 : need;
  if (n_aggs == 1) agg_ws_kernel<1><<<(int)grid, AG_NW * 32, smem, st>>>(p);
  else agg_ws_kernel<2><<<(int)grid, AG_NW * 32, smem, st>>>(p);
  return cudaGetLastError();
}

// Dense small-domain plan: the distinct streamed columns and the ring layout;
// false if the shape does not fit (the caller takes the generic path).
static bool dense_plan(int64_t n_rows, const BuildPreds* preds, const int32_t* const* key_col, int n_keys,
                       const int32_t* key_bits, const ddq_dev_agg* aggs, int n_aggs, DenseAggParams* p) {
  if (n_rows > 0x7FFFFFFF || n_aggs < 1 || n_aggs > 8) return false;
  int bits = 0;
  for (int k = 0; k < n_keys; k++) {
    if (!key_bits || key_bits[k] <= 0 || !key_col || !key_col[k]) return false;
    bits += key_bits[k];
  }
  if (bits > 5 || ((uint32_t)n_aggs << bits) > (uint32_t)DS_MAX_DA) return false;
  p->D = 1u << bits;
  auto col_id = [&](const void* c, int w) -> int {
    for (int i = 0; i < p->n_cols; i++)
      if (p->col[i] == c && p->width[i] == w) return i;
    if (p->n_cols == DS_MAXC || !c || ((uintptr_t)c & 15)) return -1;
    p->col[p->n_cols] = c;
    p->width[p->n_cols] = w;
    return p->n_cols++;
  };
  const int np = preds ? preds->n : 0;
  if (np > 4) return false;
  for (int i = 0; i < np; i++)
    if ((p->pcol[i] = col_id(preds->p[i].col, preds->p[i].width)) < 0) return false;
  for (int k = 0; k < n_keys; k++)
    if ((p->kcol[k] = col_id(key_col[k], 4)) < 0) return false;
  for (int a = 0; a < n_aggs; a++) {
    const int need = aggs[a].kind == DDQ_AGG_COUNT ? 0 : (aggs[a].kind == DDQ_AGG_SUM || aggs[a].kind == DDQ_AGG_MIN) ? 1
                   : aggs[a].kind == DDQ_AGG_SUM_MUL_100M_100P ? 3 : 2;
    for (int j = 0; j < 3; j++) {
      p->acol[a][j] = 0;
      if (j < need && (aggs[a].width[j] != 8 || (p->acol[a][j] = col_id(aggs[a].arg[j], 8)) < 0)) return false;
    }
  }
  uint32_t sb = 0;
  for (int c = 0; c < p->n_cols; c++) {
    p->off[c] = (int32_t)sb;
    sb += DS_SR * p->width[c];
  }
  p->stage_bytes = sb < 16 ? 16 : sb;
  const size_t fixed = ((size_t)p->D * n_aggs) * (DS_T * 8 + 16);
  int S = DS_SMAX;
  while (S > 2 && fixed + (size_t)S * p->stage_bytes > DS_SMEM_MAX) S--;
  if (fixed + (size_t)S * p->stage_bytes > DS_SMEM_MAX) return false;
  p->n_stages = S;
  return true;
}

bool agg_dense_supported(int64_t n_rows, const BuildPreds* preds, const int32_t* const* key_col, int n_keys,
                         const int32_t* key_bits, const ddq_dev_agg* aggs, int n_aggs) {
  for (int a = 0; a < n_aggs; a++)
    if (aggs[a].kind == DDQ_AGG_MIN) return false;  // MIN: generic kernel (launch_groupby)
  DenseAggParams p{};
  return dense_plan(n_rows, preds, key_col, n_keys, key_bits, aggs, n_aggs, &p);
}

cudaError_t launch_agg_dense(int64_t n_rows, const int32_t* const* key_col, int n_keys, const int32_t* key_bits,
                             const ddq_dev_agg* aggs, int n_aggs, void* table, uint32_t capacity, uint32_t* d_error,
                             cudaStream_t st, const BuildPreds* preds, uint32_t* d_rows, double max_row_abs) {
  DenseAggParams p{};
  if (!dense_plan(n_rows, preds, key_col, n_keys, key_bits, aggs, n_aggs, &p)) return cudaErrorInvalidValue;
  p.n = (uint32_t)n_rows;
  p.d_rows = d_rows;
  p.n_preds = preds ? preds->n : 0;
  for (int i = 0; i < p.n_preds; i++) {
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
  p.n_keys = n_keys;
  for (int k = 0, sh = 0; k < 3; k++) {
    p.key_shift[k] = sh;
    sh += (key_bits && key_bits[k] > 0) ? key_bits[k] : 21;
  }
  p.n_aggs = n_aggs;
  for (int a = 0; a < n_aggs; a++) p.kind[a] = aggs[a].kind;
  p.g_keys = reinterpret_cast<long long*>(table);
  p.g_accs = reinterpret_cast<unsigned long long*>((char*)table + (size_t)capacity * 8);
  p.cap_mask = capacity - 1;
  int lg = 0;
  while ((1u << lg) < capacity) lg++;
  p.shift = 64 - lg;
  p.d_error = d_error;
  const size_t smem = (size_t)p.n_stages * p.stage_bytes + ((size_t)p.D * n_aggs) * (DS_T * 8 + 16);
  static const bool attr = [] {  // thread-safe one-time opt-in
    const int mx = (int)DS_SMEM_MAX;
    cudaFuncSetAttribute(agg_dense_small_kernel<6, DS_Q1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    cudaFuncSetAttribute(agg_dense_small_kernel<6, DS_Q1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    cudaFuncSetAttribute(agg_dense_small_kernel<1, DS_RUNTIME, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    cudaFuncSetAttribute(agg_dense_small_kernel<2, DS_RUNTIME, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    cudaFuncSetAttribute(agg_dense_small_kernel<3, DS_RUNTIME, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    cudaFuncSetAttribute(agg_dense_small_kernel<4, DS_RUNTIME, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    cudaFuncSetAttribute(agg_dense_small_kernel<5, DS_RUNTIME, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    cudaFuncSetAttribute(agg_dense_small_kernel<6, DS_RUNTIME, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    cudaFuncSetAttribute(agg_dense_small_kernel<7, DS_RUNTIME, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    cudaFuncSetAttribute(agg_dense_small_kernel<8, DS_RUNTIME, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    return true;
  }();
  (void)attr;
  if (n_rows == 0) return cudaSuccess;
  const int64_t nch = (n_rows + DS_SR - 1) / DS_SR;
  int64_t grid = num_sms();
  if (grid > nch) grid = nch;
  uint32_t kinds = 0;
  for (int a = 0; a < n_aggs; a++) kinds |= (uint32_t)aggs[a].kind << (3 * a);
  // rows one thread adds into one partial at most: its CTA's stages x DS_R
  const double rows_per_thread = (double)((nch + grid - 1) / grid) * DS_R;
  const bool ovf = !(max_row_abs >= 0 && max_row_abs * rows_per_thread < 4.6e18);  // < 2^62
  const dim3 blk(DS_T + 32);
  if (n_aggs == 6 && kinds == DS_Q1) {
    if (ovf) agg_dense_small_kernel<6, DS_Q1, true><<<(int)grid, blk, smem, st>>>(p);
    else agg_dense_small_kernel<6, DS_Q1, false><<<(int)grid, blk, smem, st>>>(p);
  } else switch (n_aggs) {
      case 1: agg_dense_small_kernel<1, DS_RUNTIME, true><<<(int)grid, blk, smem, st>>>(p); break;
      case 2: agg_dense_small_kernel<2, DS_RUNTIME, true><<<(int)grid, blk, smem, st>>>(p); break;
      case 3: agg_dense_small_kernel<3, DS_RUNTIME, true><<<(int)grid, blk, smem, st>>>(p); break;
      case 4: agg_dense_small_kernel<4, DS_RUNTIME, true><<<(int)grid, blk, smem, st>>>(p); break;
      case 5: agg_dense_small_kernel<5, DS_RUNTIME, true><<<(int)grid, blk, smem, st>>>(p); break;
      case 6: agg_dense_small_kernel<6, DS_RUNTIME, true><<<(int)grid, blk, smem, st>>>(p); break;
      case 7: agg_dense_small_kernel<7, DS_RUNTIME, true><<<(int)grid, blk, smem, st>>>(p); break;
      default: agg_dense_small_kernel<8, DS_RUNTIME, true><<<(int)grid, blk, smem, st>>>(p); break;
    }
  return cudaGetLastError();
}

cudaError_t launch_iota(int32_t* out, int64_t n, uint32_t* d_count, cudaStream_t st) {
  int64_t grid = (n + 255) / 256;
  if (grid > (int64_t)num_sms() * 8) grid = (int64_t)num_sms() * 8;
  iota_kernel<<<(int)(grid < 1 ? 1 : grid), 256, 0, st>>>(out, (uint32_t)n, d_count);
  return cudaGetLastError();
}

}  // namespace ddq
