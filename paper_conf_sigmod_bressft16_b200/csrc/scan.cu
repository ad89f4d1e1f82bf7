// scan.cu -- the filter kernel of the hot path: selection (S8(a1)/(a2)), hash /
// join-index probe (S8(a4)) and FILTER_EQ, over ALL rows of a column ("dense") or
// over a TID list ("gather"), emitting the compacted survivors.
//
// B200 design; each choice answers an ncu finding:
//   * one persistent CTA per SM holding G independent 256-thread "groups".  Each
//     group is a complete pipeline (own TMA ring, mbarriers, named barrier, survivor
//     lists), so one group's barrier / atomic / TMA wait overlaps the others'
//     compute, while the dimension table or bitmap is staged ONCE per SM in shared
//     memory for all groups (random lookups at smem bandwidth, not L1/L2 sectors);
//   * the streamed input (fact columns, or the TID list) goes through an S-stage
//     smem ring filled by one thread with TMA bulk copies (cp.async.bulk + mbarrier
//     complete_tx): no per-thread copy instructions, tiles in flight per group;
//     gathered columns (TID mode) are 16 independent loads per thread;
//   * full tiles need no row-bound checks; survivors are compacted with a packed
//     warp scan, staged in smem and copied out coalesced, survivors only;
//   * the output range of a 4096-item tile is reserved with ONE atomicAdd whose
//     latency is hidden: tile k is copied out in iteration k+1 (the survivor list is
//     staged after barrier (B)).  Items stay in input order within a tile; tiles appear in reservation
//     order (reading O14': a TID list is a multiset; aggregates are exact integer
//     sums, so query results are bit-identical whatever the order);
//   * compact-range dimension keys use a direct-mapped join index (membership
//     bitmap + payload array): one lookup per row, no collision chains.
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "ops_internal.h"

namespace ddq {

constexpr int SC_GT = 256;                 // threads per group
constexpr int SC_GW = SC_GT / 32;          // warps per group
constexpr int SC_TILE = 4096;              // items per tile
constexpr int SC_ITEMS = SC_TILE / SC_GT;  // 16 items per thread
constexpr int SC_SLOTS = SC_ITEMS / 4;     // 4 x (one 16-byte vector of int32)
constexpr int SC_MAXCOLS = 4;
constexpr int SC_MAXG = 4;
constexpr int SC_MAXS = 4;

struct ScanPred {
  const void* col;
  int32_t width, kind;
  int64_t lo, hi;
  int32_t n_in, _pad;
  int64_t in_vals[8];
  // RANGE, precomputed on the host: lo <= v <= hi  <=>  (unsigned)(v - lo) <= d
  // (one subtract + one compare per value); `empty` when no int32 value qualifies
  int32_t lo32;
  uint32_t d32;
  uint64_t d64;
  int32_t empty32, empty64;
};

// Kernel variants: the predicate / probe code is specialised at compile time so a
// tile costs only the instructions its operator needs (ncu: the generic path was
// issue-bound -- math-pipe throttle + not-selected stalls).
// The *_R probe variants stream the key column through registers (coalesced 16-byte
// loads one tile ahead) instead of the TMA ring: no ring in shared memory, so a
// large smem bitmap / table leaves room for 4 groups.
enum ScanMode : int {
  SM_SEL_GENERIC = 0, SM_SEL_RANGE = 1, SM_PROBE_DIRECT = 2, SM_PROBE_HASH = 3, SM_PROBE_DIRECT_R = 4,
  SM_PROBE_HASH_R = 5
};

struct ScanParams {
  uint32_t n;                  // items (dense: rows); TID mode: read from d_in_count
  const uint32_t* d_in_count;  // TID mode
  int32_t n_cols;              // streamed columns (dense: predicate / fk columns; TID mode: the TIDs)
  const void* cols[SC_MAXCOLS];
  int32_t width[SC_MAXCOLS];
  int32_t col_off[SC_MAXCOLS];  // byte offset of the column's chunk inside a stage
  int32_t stage_bytes;
  int32_t stages;
  int32_t group_bytes;  // ring + lists of one group
  int32_t list_off;     // offset of the lists inside a group's area
  int32_t shared_off;   // offset of the shared table / bitmap
  // select
  int32_t n_preds;
  ScanPred preds[SC_MAXCOLS];
  const int32_t* eq_a;  // FILTER_EQ (positional vectors)
  const int32_t* eq_b;
  int eq_cmp;  // FILTER_EQ comparison: 0 a == b, 1 a < b, 2 a != b (DDQ_CMP_*)
  // probe
  int32_t probe;
  const int32_t* fk;  // probe keys: column (indexed by row) or vector (by position)
  int32_t fk_by_pos;
  const uint64_t* table;
  uint32_t cap_mask;
  int32_t shift;
  int32_t table_in_smem;
  int32_t direct;  // direct-mapped join index instead of a hash table
  const uint32_t* bitmap;
  const int32_t* payarr;
  int32_t key_min;
  uint32_t range;
  uint32_t bitmap_words;
  int32_t bitmap_in_smem;
  int32_t payarr_in_smem;  // payload array staged after the bitmap (at payarr_off)
  int32_t payarr_off;
  int32_t tid_off;  // TID mode: survivor TID list, offset inside a group's area
  int32_t* out_payload;
  // carried vectors (TID mode)
  int32_t n_carry;
  const int32_t* carry_in[4];
  int32_t* carry_out[4];
  // outputs
  int32_t* out_tids;
  uint32_t* d_out_count;  // [0] survivors, [1] CTA completion counter; zeroed before launch
  uint32_t out_cap;
  uint32_t* d_overflow;
};

__device__ __forceinline__ void group_sync(int g) {
  asm volatile("bar.sync %0, %1;" ::"r"(g + 1), "r"(SC_GT) : "memory");
}

// Group leader: one bulk copy per streamed column of tile `tile` into `buf`.
// Buffers are readable up to the next 16-byte boundary (library allocations are
// padded; torch allocations are 512-byte granular), so the tail tile is copied
// rounded up to 16 bytes and its invalid items are masked by the item bound.
__device__ __forceinline__ void issue_tile(const ScanParams& P, uint32_t n, uint8_t* buf, uint64_t* bar,
                                           uint32_t tile) {
  const uint64_t row0 = (uint64_t)tile * SC_TILE;
  const uint64_t rows = (uint64_t)n - row0 < (uint64_t)SC_TILE ? (uint64_t)n - row0 : (uint64_t)SC_TILE;
  uint32_t total = 0;
  for (int c = 0; c < P.n_cols; c++) total += (uint32_t)((rows * P.width[c] + 15) / 16 * 16);
  mbar_arrive_expect_tx(bar, total);
  for (int c = 0; c < P.n_cols; c++)
    tma_load_1d(buf + P.col_off[c], reinterpret_cast<const uint8_t*>(P.cols[c]) + row0 * P.width[c],
                (uint32_t)((rows * P.width[c] + 15) / 16 * 16), bar);
}

__device__ __forceinline__ bool scan_pred(const ScanPred& p, int64_t v) {
  if (p.kind == DDQ_PRED_RANGE) return v >= p.lo && v <= p.hi;
  if (p.kind == DDQ_PRED_BITSET) return bitset_hit(p.in_vals, p.lo, v);
  bool m = false;
#pragma unroll
  for (int j = 0; j < 8; j++) m |= (j < p.n_in) && (v == p.in_vals[j]);
  return m;
}

// Membership of 16 keys; clears the flag bits of misses.  kPay: hash probes return
// the payloads (read with the slot); join-index probes return the payload-array
// offsets, looked up at copy-out for the survivors only (batched loads).
template <int kMode, bool kPay>
__device__ __forceinline__ void probe16(const ScanParams& P, const uint64_t* table, const uint32_t* bm,
                                        const int32_t* pa, bool bm_padded, const int32_t (&key)[SC_ITEMS],
                                        uint32_t& flags, int32_t (&payload)[SC_ITEMS]) {
  if (kMode == SM_PROBE_DIRECT) {
    uint32_t m = 0;
    if (bm_padded) {  // smem bitmap with a zero word past its end: clamp instead of test
#pragma unroll
      for (int k = 0; k < SC_ITEMS; k++) {
        const uint32_t oo = min((uint32_t)(key[k] - P.key_min), P.range);
        m |= ((bm[oo >> 5] >> (oo & 31)) & 1u) << k;
      }
    } else {
#pragma unroll
      for (int k = 0; k < SC_ITEMS; k++) {
        const uint32_t o = (uint32_t)(key[k] - P.key_min);
        const uint32_t oo = o < P.range ? o : 0u;
        const uint32_t w = bm[oo >> 5];
        m |= ((o < P.range ? (w >> (oo & 31)) : 0u) & 1u) << k;
      }
    }
    flags &= m;
    if (kPay) {  // the hits' offsets; their payloads are fetched at copy-out (survivors only)
#pragma unroll
      for (int k = 0; k < SC_ITEMS; k++) payload[k] = (int32_t)(key[k] - P.key_min);
    }
  } else {
    uint32_t h[SC_ITEMS];
    uint64_t sl[SC_ITEMS];
#pragma unroll
    for (int k = 0; k < SC_ITEMS; k++) {
      h[k] = ht_hash(key[k], P.shift);
      sl[k] = ((flags >> k) & 1u) ? table[h[k]] : HT_EMPTY;
    }
#pragma unroll
    for (int k = 0; k < SC_ITEMS; k++) {
      uint64_t s = sl[k];
      uint32_t hh = h[k];
      while (s != HT_EMPTY && ht_key(s) != key[k]) {
        hh = (hh + 1) & P.cap_mask;
        s = table[hh];
      }
      if (s == HT_EMPTY) flags &= ~(1u << k);
      if (kPay) payload[k] = ht_val(s);
    }
  }
}

// Gathered values (TID mode) against predicate p.
template <int kMode>
__device__ __forceinline__ void pred16_gathered(const ScanPred& pr, const int32_t (&row)[SC_ITEMS], uint32_t& flags) {
  int64_t v[SC_ITEMS];
#pragma unroll
  for (int k = 0; k < SC_ITEMS; k++) v[k] = ((flags >> k) & 1u) ? col_at(pr.col, pr.width, row[k]) : 0;
  if (kMode == SM_SEL_RANGE) {
    if (pr.empty64) flags = 0;
#pragma unroll
    for (int k = 0; k < SC_ITEMS; k++)
      if ((uint64_t)(v[k] - pr.lo) > pr.d64) flags &= ~(1u << k);
  } else {
    uint32_t m = 0;
#pragma unroll
    for (int k = 0; k < SC_ITEMS; k++) m |= (scan_pred(pr, v[k]) ? 1u : 0u) << k;
    flags &= m;
  }
}

// Staged (dense) column chunk against predicate p.
template <int kMode>
__device__ __forceinline__ void pred16_staged(const ScanPred& pr, const uint8_t* cb, int wrow, int lane,
                                              uint32_t& flags) {
#pragma unroll
  for (int s = 0; s < SC_SLOTS; s++) {
    const int it = wrow + s * 128 + lane * 4;
    if (kMode == SM_SEL_RANGE && pr.width == 4) {
      const int4 a = *reinterpret_cast<const int4*>(cb + (size_t)it * 4);
      const int32_t v4[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
      for (int v = 0; v < 4; v++)
        if ((uint32_t)(v4[v] - pr.lo32) > pr.d32) flags &= ~(1u << (s * 4 + v));
      continue;
    }
    int64_t v4[4];
    if (pr.width == 8) {
      const longlong2 a = *reinterpret_cast<const longlong2*>(cb + (size_t)it * 8);
      const longlong2 b = *reinterpret_cast<const longlong2*>(cb + (size_t)it * 8 + 16);
      v4[0] = a.x; v4[1] = a.y; v4[2] = b.x; v4[3] = b.y;
    } else {
      const int4 a = *reinterpret_cast<const int4*>(cb + (size_t)it * 4);
      v4[0] = a.x; v4[1] = a.y; v4[2] = a.z; v4[3] = a.w;
    }
    if (kMode == SM_SEL_RANGE) {
#pragma unroll
      for (int v = 0; v < 4; v++)
        if ((uint64_t)(v4[v] - pr.lo) > pr.d64) flags &= ~(1u << (s * 4 + v));
    } else {
      uint32_t m = 0;
#pragma unroll
      for (int v = 0; v < 4; v++) m |= (scan_pred(pr, v4[v]) ? 1u : 0u) << v;
      flags &= ~((~m & 0xFu) << (s * 4));
    }
  }
}

// One tile's keys (dense probe, register-streamed): 4 x 16-byte loads per thread.
__device__ __forceinline__ void load_keys(const int32_t* fk, uint32_t n, uint32_t row0, uint32_t wrow, int lane,
                                          int4 (&r)[SC_SLOTS]) {
  if (row0 + SC_TILE <= n) {
#pragma unroll
    for (int s = 0; s < SC_SLOTS; s++) r[s] = ld_stream_i4(fk + (size_t)row0 + wrow + s * 128 + lane * 4);
  } else {
#pragma unroll
    for (int s = 0; s < SC_SLOTS; s++) {
      const uint32_t i = row0 + wrow + s * 128 + lane * 4;
      r[s].x = i < n ? fk[i] : 0;
      r[s].y = i + 1 < n ? fk[i + 1] : 0;
      r[s].z = i + 2 < n ? fk[i + 2] : 0;
      r[s].w = i + 3 < n ? fk[i + 3] : 0;
    }
  }
}

template <int G, bool kTids, int kMode>
__global__ void __launch_bounds__(SC_GT* G, 1) scan_kernel(const __grid_constant__ ScanParams P) {
  constexpr bool kProbe = kMode >= SM_PROBE_DIRECT;
  constexpr bool kDirect = kMode == SM_PROBE_DIRECT || kMode == SM_PROBE_DIRECT_R;
  constexpr bool kHash = kProbe && !kDirect;
  // register-streamed input: dense probe keys (*_R variants) or the TID list (TID
  // mode: no ring; the TIDs of the survivors are staged with the survivor list)
  constexpr bool kReg = kMode >= SM_PROBE_DIRECT_R || kTids;
  constexpr int kPM = kDirect ? SM_PROBE_DIRECT : SM_PROBE_HASH;
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint32_t s_warp_tot[SC_MAXG][SC_GW];
  __shared__ uint32_t s_base[SC_MAXG];
  __shared__ __align__(8) uint64_t s_full[SC_MAXG][SC_MAXS];
  const int g = threadIdx.x / SC_GT;     // group
  const int t = threadIdx.x % SC_GT;     // thread within the group
  const int lane = t & 31, warp = t >> 5;
  const uint32_t n = kTids ? ld_relaxed_u32(P.d_in_count) : P.n;
  const uint32_t ntiles = (n + SC_TILE - 1) / SC_TILE;
  const int S = P.stages;
  // ring mode: S-1 tiles in flight ahead of the current one; stage (k-1)%S is
  // refilled with tile k+S-1 right after (A)
  const int ahead = S - 1;
  const uint32_t vb = blockIdx.x * G + g, vgrid = gridDim.x * G;  // virtual CTA id / count
  uint8_t* ring = smem + (size_t)g * P.group_bytes;
  uint16_t* s_list = reinterpret_cast<uint16_t*>(ring + P.list_off);             // TILE
  int32_t* s_pay = reinterpret_cast<int32_t*>(ring + P.list_off + SC_TILE * 2);  // TILE
  int32_t* s_tid = reinterpret_cast<int32_t*>(ring + P.tid_off);                   // TILE (TID mode)
  const int32_t* scol = kTids ? reinterpret_cast<const int32_t*>(P.cols[0]) : P.fk;  // streamed column
  uint64_t* s_table = reinterpret_cast<uint64_t*>(smem + P.shared_off);

  const uint32_t wrow = warp * (32 * SC_ITEMS);  // warp's first item inside a tile
  int4 nk[SC_SLOTS];                             // register-streamed keys of the next tile
  if (kReg && vb < ntiles) load_keys(scol, n, vb * SC_TILE, wrow, lane, nk);
  if (t == 0 && !kReg) {  // group leader: barriers, then the first tiles in flight
    for (int k = 0; k < S; k++) mbar_init(&s_full[g][k], 1);
    fence_mbar_init();
    for (int k = 0; k < ahead; k++) {
      const uint32_t tl = vb + (uint32_t)k * vgrid;
      if (tl < ntiles) issue_tile(P, n, ring + (size_t)k * P.stage_bytes, &s_full[g][k], tl);
    }
  }
  // all groups stage the shared table / bitmap (+ payload array) once per SM
  // (overlaps the first loads); the smem bitmap gets one zero word past its end
  uint32_t* s_bm = reinterpret_cast<uint32_t*>(s_table);
  int32_t* s_pa = reinterpret_cast<int32_t*>(smem + P.shared_off + P.payarr_off);
  if (kHash && P.table_in_smem)
    for (uint32_t i = threadIdx.x; i <= P.cap_mask; i += SC_GT * G) s_table[i] = P.table[i];
  if (kDirect && P.bitmap_in_smem) {
    for (uint32_t i = threadIdx.x; i <= P.bitmap_words; i += SC_GT * G)
      s_bm[i] = i < P.bitmap_words ? P.bitmap[i] : 0u;
    if (P.payarr_in_smem)
      for (uint32_t i = threadIdx.x; i < P.range; i += SC_GT * G) s_pa[i] = P.payarr[i];
  }
  const uint64_t* table = (kHash && P.table_in_smem) ? s_table : P.table;
  const uint32_t* bm = (kDirect && P.bitmap_in_smem) ? s_bm : P.bitmap;
  const int32_t* pa = (kDirect && P.payarr_in_smem) ? s_pa : P.payarr;
  const bool bm_padded = P.bitmap_in_smem != 0;
  const bool want_pay = kProbe && P.out_payload != nullptr;  // payloads staged with the list
  __syncthreads();

  // Software pipeline over the group's tiles: iteration k evaluates tile k, then
  // (while its output reservation -- one atomic -- is in flight) copies out tile
  // k-1, whose range was reserved last iteration, from the survivor list; after (B)
  // it stages tile k's survivors in that list (one buffer: half the smem of two).
  uint32_t prev_tot = 0, prev_base = 0;
  int stg = 0;        // ring stage of tile k (k % S)
  uint32_t ph = 0;    // its mbarrier phase parity ((k / S) & 1)
  for (uint32_t k = 0;; k++) {
    const uint32_t tile = vb + k * vgrid;
    const bool have = tile < ntiles;
    const uint32_t row0 = tile * SC_TILE;  // first item of the tile
    uint32_t flags = 0;
    int32_t payload[SC_ITEMS];
    int32_t row[SC_ITEMS];  // TID mode: the tile's TIDs
    if (have) {
      if (!kReg) mbar_wait(&s_full[g][stg], ph);
      const uint8_t* buf = ring + (size_t)stg * P.stage_bytes;
      flags = 0xFFFFu;
      if (row0 + SC_TILE > n) {  // tail tile only
        flags = 0;
#pragma unroll
        for (int s = 0; s < SC_SLOTS; s++)
#pragma unroll
          for (int v = 0; v < 4; v++)
            flags |= (row0 + wrow + s * 128 + lane * 4 + v < n ? 1u : 0u) << (s * 4 + v);
      }
      if (kTids) {
        // ---- TID mode: rows from the staged TID list, values gathered ----------
#pragma unroll
        for (int s = 0; s < SC_SLOTS; s++) {
          row[s * 4 + 0] = nk[s].x; row[s * 4 + 1] = nk[s].y; row[s * 4 + 2] = nk[s].z; row[s * 4 + 3] = nk[s].w;
        }
        if (tile + vgrid < ntiles) load_keys(scol, n, (tile + vgrid) * SC_TILE, wrow, lane, nk);
        if (!kProbe) {
          for (int p = 0; p < P.n_preds; p++) pred16_gathered<kMode>(P.preds[p], row, flags);
          if (P.eq_a) {
            uint32_t m = 0;
#pragma unroll
            for (int k2 = 0; k2 < SC_ITEMS; k2++) {
              const uint32_t pos = row0 + wrow + (k2 >> 2) * 128 + lane * 4 + (k2 & 3);
              const int32_t va = __ldg(P.eq_a + pos), vb = __ldg(P.eq_b + pos);
              m |= (((flags >> k2) & 1u) && vec_cmp(P.eq_cmp, va, vb) ? 1u : 0u) << k2;
            }
            flags &= m;
          }
        } else {
          int32_t key[SC_ITEMS];
          if (P.fk_by_pos) {  // positional key vector: coalesced
#pragma unroll
            for (int k2 = 0; k2 < SC_ITEMS; k2++) {
              const uint32_t pos = row0 + wrow + (k2 >> 2) * 128 + lane * 4 + (k2 & 3);
              key[k2] = ((flags >> k2) & 1u) ? __ldg(P.fk + pos) : 0;
            }
          } else {  // key column gathered at the TIDs
#pragma unroll
            for (int k2 = 0; k2 < SC_ITEMS; k2++) key[k2] = ((flags >> k2) & 1u) ? __ldg(P.fk + (uint32_t)row[k2]) : 0;
          }
          if (want_pay) probe16<kPM, true>(P, table, bm, pa, bm_padded, key, flags, payload);
          else probe16<kPM, false>(P, table, bm, pa, bm_padded, key, flags, payload);
        }
      } else if (!kProbe) {
        // ---- dense select: values from the staged columns ----------------------
        for (int p = 0; p < P.n_preds; p++) {
          const ScanPred& pr = P.preds[p];
          if (kMode == SM_SEL_RANGE && (pr.width == 4 ? pr.empty32 : pr.empty64)) flags = 0;
          pred16_staged<kMode>(pr, buf + P.col_off[p], wrow, lane, flags);
        }
      } else {
        // ---- dense probe: keys from the staged fk column -------------------------
        int32_t key[SC_ITEMS];
#pragma unroll
        for (int s = 0; s < SC_SLOTS; s++) {
          const int4 a = kReg ? nk[s] : *reinterpret_cast<const int4*>(buf + (size_t)(wrow + s * 128 + lane * 4) * 4);
          key[s * 4 + 0] = a.x; key[s * 4 + 1] = a.y; key[s * 4 + 2] = a.z; key[s * 4 + 3] = a.w;
        }
        if (kReg && tile + vgrid < ntiles) load_keys(P.fk, n, (tile + vgrid) * SC_TILE, wrow, lane, nk);
        if (want_pay) probe16<kPM, true>(P, table, bm, pa, bm_padded, key, flags, payload);
        else probe16<kPM, false>(P, table, bm, pa, bm_padded, key, flags, payload);
      }
    }
    // group scan of the per-slot survivor counts
    uint32_t packed = 0;
#pragma unroll
    for (int s = 0; s < SC_SLOTS; s++) packed |= (uint32_t)__popc((flags >> (4 * s)) & 0xFu) << (8 * s);
    const uint32_t incl = warp_incl_scan(packed, lane);
    const uint32_t excl = incl - packed;
    const uint32_t wtot = __shfl_sync(FULL, incl, 31);
    uint32_t slot_off[SC_SLOTS];
    uint32_t acc = 0;
#pragma unroll
    for (int s = 0; s < SC_SLOTS; s++) {
      slot_off[s] = acc;
      acc += (wtot >> (8 * s)) & 0xFFu;
    }
    if (lane == 0) s_warp_tot[g][warp] = acc;
    group_sync(g);  // (A) warp totals visible; the group is done computing on tile k-1
    uint32_t tot = 0, warp_off = 0;
#pragma unroll
    for (int w = 0; w < SC_GW; w++) {
      const uint32_t x = s_warp_tot[g][w];
      warp_off += (w < warp) ? x : 0;
      tot += x;
    }
    uint32_t my_base = 0;
    if (t == 0) {
      if (!kReg && have) {  // ring: refill stage (k-1)%S, released by (A)
        const uint32_t tl = tile + (uint32_t)ahead * vgrid;
        if (tl < ntiles) {
          fence_proxy_async();
          const int st = stg == 0 ? S - 1 : stg - 1;  // (k + S - 1) % S
          issue_tile(P, n, ring + (size_t)st * P.stage_bytes, &s_full[g][st], tl);
        }
      }
      my_base = tot ? atomicAdd(P.d_out_count, tot) : 0;  // consumed only before (B)
    }
    // copy out tile k-1 (reserved last iteration): coalesced, survivors only
    if (k > 0) {
      const uint16_t* pl = s_list;
      const int32_t* pp = s_pay;
      const uint32_t prow0 = (tile - vgrid) * SC_TILE;
      const uint32_t lim = prev_base + prev_tot <= P.out_cap ? prev_tot
                         : (P.out_cap > prev_base ? P.out_cap - prev_base : 0);
      if (lim < prev_tot && t == 0 && P.d_overflow) atomicMax(P.d_overflow, 4u);
      constexpr int U = 4;  // survivors per thread per batch: independent loads in flight
      for (uint32_t i0 = t; i0 < lim; i0 += U * SC_GT) {
        uint32_t it[U];
        int32_t pv[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
          const uint32_t i = i0 + u * SC_GT;
          it[u] = i < lim ? pl[i] : 0u;
          pv[u] = (want_pay && i < lim) ? pp[i] : 0;
        }
        if (kDirect && want_pay) {
#pragma unroll
          for (int u = 0; u < U; u++)
            if (i0 + u * SC_GT < lim) pv[u] = pa[(uint32_t)pv[u]];
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
          const uint32_t i = i0 + u * SC_GT;
          if (i < lim) {
            P.out_tids[prev_base + i] = kTids ? s_tid[i] : (int32_t)(prow0 + it[u]);
            if (want_pay) P.out_payload[prev_base + i] = pv[u];
            if (kTids)
              for (int c = 0; c < P.n_carry; c++)
                P.carry_out[c][prev_base + i] = __ldg(P.carry_in[c] + prow0 + it[u]);
          }
        }
      }
    }
    if (t == 0) s_base[g] = my_base;
    group_sync(g);  // (B) s_base visible; the list is free
    // stage tile k's survivors (tile-local item offsets + payloads) in the list,
    // which (B) released; (A) of the next iteration publishes it to the copy-out
    if (flags) {
#pragma unroll
      for (int s = 0; s < SC_SLOTS; s++) {
        const uint32_t m = (flags >> (4 * s)) & 0xFu;
        const uint32_t sb = warp_off + slot_off[s] + ((excl >> (8 * s)) & 0xFFu);
#pragma unroll
        for (int v = 0; v < 4; v++) {
          if ((m >> v) & 1u) {
            const uint32_t pos = sb + __popc(m & ((1u << v) - 1u));
            s_list[pos] = (uint16_t)(wrow + s * 128 + lane * 4 + v);
            if (want_pay) s_pay[pos] = payload[s * 4 + v];
            if (kTids) s_tid[pos] = row[s * 4 + v];
          }
        }
      }
    }
    prev_base = s_base[g];
    prev_tot = tot;
    if (++stg == S) {
      stg = 0;
      ph ^= 1u;
    }
    if (!have) break;
  }
  // the last CTA to finish clamps the count to the output capacity
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(P.d_out_count + 1, 1u) == gridDim.x - 1) {
      const uint32_t c = atomicAdd(P.d_out_count, 0u);
      if (c > P.out_cap) *P.d_out_count = P.out_cap;
    }
  }
}

static int g_smem_optin = 0;

template <int G, bool kTids>
static void set_attrs_g(int v) {
  cudaFuncSetAttribute(scan_kernel<G, kTids, SM_SEL_GENERIC>, cudaFuncAttributeMaxDynamicSharedMemorySize, v - 2048);
  cudaFuncSetAttribute(scan_kernel<G, kTids, SM_SEL_RANGE>, cudaFuncAttributeMaxDynamicSharedMemorySize, v - 2048);
  cudaFuncSetAttribute(scan_kernel<G, kTids, SM_PROBE_DIRECT>, cudaFuncAttributeMaxDynamicSharedMemorySize, v - 2048);
  cudaFuncSetAttribute(scan_kernel<G, kTids, SM_PROBE_HASH>, cudaFuncAttributeMaxDynamicSharedMemorySize, v - 2048);
  if (!kTids) {
    cudaFuncSetAttribute(scan_kernel<G, false, SM_PROBE_DIRECT_R>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         v - 2048);
    cudaFuncSetAttribute(scan_kernel<G, false, SM_PROBE_HASH_R>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         v - 2048);
  }
}

bool scan_supported(const FilterArgs& a) {
  if (a.n_carry > 4) return false;
  if (!a.probe && a.n_preds > SC_MAXCOLS) return false;
  if (!a.probe && a.n_preds < 1 && !a.eq_a) return false;
  if (a.in_tids) return ((uintptr_t)a.in_tids & 15) == 0;  // TMA needs 16-byte aligned bases
  if (a.eq_a || a.fk_by_pos || a.n_carry) return false;    // vectors exist only for TID inputs
  if (a.probe) return ((uintptr_t)a.fk & 15) == 0;
  for (int i = 0; i < a.n_preds; i++)
    if ((uintptr_t)a.preds[i].col & 15) return false;
  return true;
}

template <int G, bool kTids>
static void launch_m(int mode, int64_t grid, size_t smem, cudaStream_t st, const ScanParams& p) {
  switch (mode) {
    case SM_SEL_GENERIC: scan_kernel<G, kTids, SM_SEL_GENERIC><<<(int)grid, SC_GT * G, smem, st>>>(p); break;
    case SM_SEL_RANGE: scan_kernel<G, kTids, SM_SEL_RANGE><<<(int)grid, SC_GT * G, smem, st>>>(p); break;
    case SM_PROBE_DIRECT: scan_kernel<G, kTids, SM_PROBE_DIRECT><<<(int)grid, SC_GT * G, smem, st>>>(p); break;
    case SM_PROBE_HASH: scan_kernel<G, kTids, SM_PROBE_HASH><<<(int)grid, SC_GT * G, smem, st>>>(p); break;
    case SM_PROBE_DIRECT_R:
      if (!kTids) scan_kernel<G, false, SM_PROBE_DIRECT_R><<<(int)grid, SC_GT * G, smem, st>>>(p);
      break;
    default:
      if (!kTids) scan_kernel<G, false, SM_PROBE_HASH_R><<<(int)grid, SC_GT * G, smem, st>>>(p);
      break;
  }
}

cudaError_t launch_scan(const FilterArgs& a, cudaStream_t st) {
  static const bool scan_ready = [] {  // thread-safe one-time opt-in
    int dev = 0;
    cudaGetDevice(&dev);
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    set_attrs_g<1, false>(v);
    set_attrs_g<2, false>(v);
    set_attrs_g<3, false>(v);
    set_attrs_g<4, false>(v);
    set_attrs_g<1, true>(v);
    set_attrs_g<2, true>(v);
    g_smem_optin = v;
    return true;
  }();
  (void)scan_ready;
  const bool tids = a.in_tids != nullptr;
  ScanParams p{};
  p.n = (uint32_t)a.n_cap;
  p.d_in_count = a.d_in_count;
  int off = 0;
  if (tids) {  // stream the TID list; columns are gathered
    p.n_cols = 1;
    p.cols[0] = a.in_tids;
    p.width[0] = 4;
    off = SC_TILE * 4;
  } else if (a.probe) {
    p.n_cols = 1;
    p.cols[0] = a.fk;
    p.width[0] = 4;
    off = SC_TILE * 4;
  } else {
    p.n_cols = a.n_preds;
    for (int i = 0; i < a.n_preds; i++) {
      p.cols[i] = a.preds[i].col;
      p.width[i] = a.preds[i].width;
      p.col_off[i] = off;
      off += SC_TILE * a.preds[i].width;
    }
  }
  p.n_preds = a.probe ? 0 : a.n_preds;
  bool all_range = true;
  for (int i = 0; i < p.n_preds; i++) {
    const ddq_dev_pred& d = a.preds[i];
    ScanPred& q = p.preds[i];
    q.col = d.col;
    q.width = d.width;
    q.kind = d.kind;
    q.lo = d.lo;
    q.hi = d.hi;
    q.n_in = d.n_in;
    for (int j = 0; j < 8; j++) q.in_vals[j] = d.in_vals[j];
    all_range = all_range && d.kind == DDQ_PRED_RANGE;
    q.empty64 = d.hi < d.lo;
    q.d64 = q.empty64 ? 0 : (uint64_t)d.hi - (uint64_t)d.lo;
    const int64_t lo32 = d.lo < INT32_MIN ? INT32_MIN : d.lo, hi32 = d.hi > INT32_MAX ? INT32_MAX : d.hi;
    q.empty32 = hi32 < lo32;
    q.lo32 = q.empty32 ? 0 : (int32_t)lo32;
    q.d32 = q.empty32 ? 0 : (uint32_t)(hi32 - lo32);
  }
  p.eq_a = a.eq_a;
  p.eq_b = a.eq_b;
  p.eq_cmp = a.eq_cmp;
  p.stage_bytes = off;
  p.probe = a.probe ? 1 : 0;
  p.fk = a.fk;
  p.fk_by_pos = a.fk_by_pos ? 1 : 0;
  const bool direct = a.probe && a.bitmap != nullptr;
  int mode = a.probe ? (direct ? SM_PROBE_DIRECT : SM_PROBE_HASH)
                           : (all_range && !a.eq_a ? SM_SEL_RANGE : SM_SEL_GENERIC);
  // smem-resident structure: hash table, or join-index bitmap (+1 zero word) and,
  // when it fits too, the payload array
  const size_t kSmemTable = 144 * 1024;
  const size_t bm_bytes = direct ? ((size_t)a.range + 31) / 32 * 4 + 4 : 0;
  const size_t table_bytes = a.probe ? (direct ? bm_bytes : (size_t)a.capacity * 8) : 0;
  const size_t budget = (size_t)g_smem_optin - 2048;
  const bool in_smem = a.probe && table_bytes <= kSmemTable;
  p.table_in_smem = (in_smem && !direct) ? 1 : 0;
  p.bitmap_in_smem = (in_smem && direct) ? 1 : 0;
  const size_t pa_off = (bm_bytes + 15) / 16 * 16;
  const bool pa_smem = in_smem && direct && a.out_payload && pa_off + (size_t)a.range * 4 <= kSmemTable;
  p.payarr_in_smem = pa_smem ? 1 : 0;
  p.payarr_off = (int32_t)pa_off;
  const size_t shared = in_smem ? ((pa_smem ? pa_off + (size_t)a.range * 4 : table_bytes) + 127) / 128 * 128 : 0;
  const size_t pay_bytes = a.probe && a.out_payload ? (size_t)SC_TILE * 4 : 0;
  const size_t list_bytes = (size_t)SC_TILE * 2 + pay_bytes + (tids ? (size_t)SC_TILE * 4 : 0);
  // as many groups (up to 4) and stages (up to 4, at least 2) as shared memory allows
  const int min_s = 2;
  // TID mode: 2 groups (opprofile SF20: G=1 2105 us, G=2 1753 us, G=3 1894 us of
  // at-TID ops -- the 85-register cap of G=3 serialises the gathers; so did a
  // software-pipelined one-tile-ahead gather at G=2: spills, 1915 us)
  int G = tids ? 2 : 4, S = 4;
  {
    static const char* env = getenv("DDQ_SCAN_SMALL");
    if (env && a.n_cap <= atoll(env)) {
      G = 1;
      S = 2;
    }
  }
  auto need = [&](int gg, int ss) { return shared + (size_t)gg * ((size_t)ss * p.stage_bytes + list_bytes); };
  while (G > 1 && need(G, min_s) > budget) G--;
  while (S > min_s && need(G, S) > budget) S--;
  if (need(G, S) > budget) return cudaErrorInvalidConfiguration;
  // dense probes stream the keys through registers (microbench, 120M keys: 73 KB
  // bitmap + payloads 389 -> 258 us, 122 KB bitmap 431 -> 201 us vs the TMA ring,
  // whose smem competes with the bitmap); DDQ_SCAN_REG=0 selects the ring
  // TID mode always streams the TID list through registers (no ring)
  bool reg = tids;
  if (a.probe && !tids) {
    static const char* env = getenv("DDQ_SCAN_REG");
    reg = env ? env[0] == '1' : true;
  }
  if (reg) {
    if (!tids) mode = direct ? SM_PROBE_DIRECT_R : SM_PROBE_HASH_R;
    p.n_cols = tids ? 1 : 0;  // cols[0]: the TID list (streamed by the kernel itself)
    p.stage_bytes = 0;
    S = 1;
    // register budget (ptxas: no spills); hash probes hold 16 slots more
    G = tids ? 2 : (a.out_payload ? 3 : 4) - (direct ? 0 : 1);
    while (G > 1 && shared + (size_t)G * list_bytes > budget) G--;
    if (shared + (size_t)G * list_bytes > budget) return cudaErrorInvalidConfiguration;
  }
  p.stages = S;
  p.list_off = S * p.stage_bytes;
  p.group_bytes = (int32_t)((p.list_off + list_bytes + 127) / 128 * 128);
  p.tid_off = (int32_t)(p.list_off + SC_TILE * 2 + pay_bytes);
  p.shared_off = G * p.group_bytes;
  if (direct) {
    p.direct = 1;
    p.bitmap = a.bitmap;
    p.payarr = a.payarr;
    p.key_min = a.key_min;
    p.range = a.range;
    p.bitmap_words = (a.range + 31) / 32;
  } else if (a.probe) {
    p.table = a.table;
    p.cap_mask = a.capacity - 1;
    int lg = 0;
    while ((1u << lg) < a.capacity) lg++;
    p.shift = 32 - lg;
  }
  if (a.probe) p.out_payload = a.out_payload;
  p.n_carry = a.n_carry;
  for (int c = 0; c < a.n_carry; c++) {
    p.carry_in[c] = a.carry_in[c];
    p.carry_out[c] = a.carry_out[c];
  }
  p.out_tids = a.out_tids;
  p.d_out_count = a.d_out_count;
  p.out_cap = (uint32_t)(a.out_cap > 0 ? a.out_cap : a.n_cap);
  p.d_overflow = a.d_overflow;
  cudaError_t e = init_fill(a.d_out_count, 8, 0, st);
  if (e != cudaSuccess) return e;
  const size_t smem = (size_t)p.shared_off + shared;
  const int64_t ntiles = (a.n_cap + SC_TILE - 1) / SC_TILE;  // upper bound (TID mode: capacity)
  int64_t grid = num_sms();
  const int64_t need_ctas = (ntiles + G - 1) / G;
  if (grid > need_ctas) grid = need_ctas < 1 ? 1 : need_ctas;
  if (tids) {
    if (G == 1) launch_m<1, true>(mode, grid, smem, st, p);
    else launch_m<2, true>(mode, grid, smem, st, p);
  } else {
    switch (G) {
      case 1: launch_m<1, false>(mode, grid, smem, st, p); break;
      case 2: launch_m<2, false>(mode, grid, smem, st, p); break;
      case 3: launch_m<3, false>(mode, grid, smem, st, p); break;
      default: launch_m<4, false>(mode, grid, smem, st, p); break;
    }
  }
  return cudaGetLastError();
}

}  // namespace ddq
