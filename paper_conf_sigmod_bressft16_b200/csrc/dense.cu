// dense.cu -- warp-autonomous filter kernels of the hot path: the dense hash /
// join-index probe (S8(a4), every row of a fact FK column) and every operator over
// a TID list (S8(a2) selection at TIDs, S8(a4) probe at TIDs, FILTER_EQ), each
// emitting a compacted TID list (+ the hit's payload, + carried aligned vectors).
// The dense probe is the first fact operator of every SSB plan (SURVEY.md 8(d):
// the most selective dimension's FK column is scanned fully); the TID-input
// operators are the later steps of the same column-at-a-time chains.
//
// B200 design; the predecessor scan_kernel (one CTA per SM split into
// 256-thread groups with named barriers) was instruction- and barrier-bound (ncu:
// 46 thread-instructions per row; barrier, wait stalls) at 42 % of HBM peak:
//   * one persistent CTA of 32 warps per SM; every warp walks its own 512-item
//     tiles (32 lanes x 16 items, 16-byte loads, the next tile's keys / TIDs
//     prefetched into registers) -- no CTA-wide barrier inside the loop;
//   * the dimension bitmap (or hash table) is staged once per SM in shared memory
//     and probed with LDS (the kernel is specialised so the compiler sees a shared
//     pointer, not a generic one);
//   * compaction: a lane's 16 hit bits -> popc -> warp inclusive scan -> the warp
//     claims a range of a CTA-wide counter with ONE shared-memory atomic; the
//     survivors go straight from registers into a shared-memory write-combining
//     ring of R blocks x BLK entries (TID, payload, input position);
//   * the warp whose entries complete a ring block flushes it: one global atomicAdd
//     reserves BLK output slots (measured: 1.45 G same-address atomics/s on B200,
//     so one per 2048 survivors, not one per tile), then coalesced copies; carried
//     vectors are gathered at the survivors' input positions during the flush.
//     Its latency is that warp's alone; the other warps keep filling the remaining
//     blocks.  A block's slot is reused only after its flush (per-slot generation
//     counter); the oldest unflushed block's writers never wait, so the ring cannot
//     deadlock;
//   * after the loop the CTA flushes its last, partial block with an exact-size
//     reservation: the output has no holes.
// Output order: unspecified (reading O14': a TID list is a multiset; every consumer
// is order-free); each input item is emitted at most once.
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "ops_internal.h"

namespace ddq {

namespace {

constexpr int WS_ITEMS = 16;            // items per lane per tile
constexpr int WS_TILE = 32 * WS_ITEMS;  // items per warp tile
constexpr int WS_RMAX = 16;             // ring blocks (runtime R = 4..16, as shared memory allows)
// entries per ring block (one global reservation): 2048, or 1024 when carried
// vectors add up to 4 more int32 fields per entry (ring <= 96 KB)
__host__ __device__ constexpr int ws_blk(bool carry) { return carry ? 1024 : 2048; }
constexpr int WS_MAXF = 6;  // ring fields: TID, payload, <= 4 carried vectors
// warps per CTA: dense probes 32 (64 registers: 16 keys in use + 16 prefetched);
// TID-input operators 16 (128 registers: TIDs, gathered keys / values, payloads)
__host__ __device__ constexpr int ws_nw(bool tids) { return tids ? 16 : 32; }

// operator variants (compile time: a tile costs only the instructions it needs)
enum WsKind : int {
  WK_BM_SMEM = 0,    // join-index probe, bitmap in smem
  WK_BM_GLOBAL = 1,  // join-index probe, bitmap in global (L2)
  WK_HT_SMEM = 2,    // hash probe, table in smem
  WK_HT_GLOBAL = 3,  // hash probe, table in global
  WK_SEL_RANGE = 4,  // conjunctive range predicates (TID input)
  WK_SEL_GENERIC = 5,  // range / IN predicates (TID input)
  WK_EQ = 6,           // FILTER_EQ of two positional vectors (TID input)
  WK_BM_COARSE = 7     // join-index probe: a coarse bitmap (1 bit per 2^cg keys) in smem
                       // filters, the exact bit is read from the global (L2) bitmap
};

struct WsPred {
  const void* col;
  int32_t width, kind;
  int64_t lo, hi;
  uint64_t d64;  // RANGE: lo <= v <= hi  <=>  (u64)(v - lo) <= d64
  int32_t empty, n_in;
  int64_t in_vals[8];
};

struct WsParams {
  uint32_t n;                  // dense: rows; TID input: capacity (count in d_in_count)
  const uint32_t* d_in_count;  // TID input
  const int32_t* in_tids;      // TID input
  const uint32_t* in_bits;     // row-bitmap input (n = rows): 16 words per 512-row tile
  uint32_t* out_bits;          // row-bitmap output (dense probe / select, no payload)
  int32_t n_preds;
  WsPred preds[4];
  const int32_t* eq_a;
  const int32_t* eq_b;
  int eq_cmp;  // FILTER_EQ comparison: 0 a == b, 1 a < b, 2 a != b (DDQ_CMP_*)
  const int32_t* fk;  // probe keys: column (by row) or positional vector (fk_by_pos)
  int32_t fk_by_pos;
  // join index (direct): membership bitmap over [key_min, key_min + range) + payloads
  const uint32_t* bitmap;
  const int32_t* payarr;
  int32_t key_min;
  uint32_t range;
  uint32_t bitmap_words;
  uint32_t cg;              // WK_BM_COARSE: log2 keys per coarse bit
  const uint32_t* coarse;   // WK_BM_COARSE: the index's coarse bitmap (global)
  // hash table (open addressing, 8-byte slots key<<32|payload)
  const uint64_t* table;
  uint32_t cap_mask;
  int32_t shift;
  int32_t tab_off;  // byte offset of the staged table in dynamic smem
  int32_t ring_logr;  // log2 of the number of ring blocks
  int32_t n_carry;
  const int32_t* carry_in[4];
  int32_t* carry_out[4];
  int32_t n_fields;             // ring fields: TID, [payload], carried vectors
  int32_t* field_out[WS_MAXF];  // their outputs
  int32_t* out_tids;
  int32_t* out_payload;
  uint32_t* d_out_count;  // [0] survivors, [1] CTA completion counter (zeroed before launch)
  uint32_t out_cap;
  uint32_t* d_overflow;
};

__device__ __forceinline__ uint32_t ld_volatile_smem(const uint32_t* p) {
  return *reinterpret_cast<const volatile uint32_t*>(p);
}

// Copy `cnt` ring entries starting at ring offset `r0` (no wrap) of every field
// (field f lives at ring + f * ring_n) to its output at [g, g + cnt), clamped to
// out_cap.  Called by a whole warp (tid = lane, nthr = 32) or by the whole CTA.
// kXlate: field 1 holds the hits' KEYS and is written as their join-index payloads
// (payarr[key - key_min]) -- the lookups are done here, for dense survivors with every
// lane active, instead of per item (mostly dead) in the probe loop.
template <bool kXlate>
__device__ __forceinline__ void copy_out(const WsParams& P, const int32_t* ring, uint32_t ring_n, uint32_t r0,
                                         uint32_t cnt, uint32_t g, uint32_t tid, uint32_t nthr) {
  uint32_t lim = cnt;
  if (g + cnt > P.out_cap) {
    lim = P.out_cap > g ? P.out_cap - g : 0u;
    if (tid == 0 && P.d_overflow) atomicMax(P.d_overflow, 4u);
  }
  const int32_t* pa = P.payarr;
  const uint32_t kmin = (uint32_t)P.key_min;
  if ((g & 3u) == 0 && lim == cnt && (cnt & 3u) == 0) {  // 16-byte copies
    for (int f = 0; f < P.n_fields; f++) {
      const int4* src = reinterpret_cast<const int4*>(ring + (size_t)f * ring_n + r0);
      int4* dst = reinterpret_cast<int4*>(P.field_out[f] + g);
      if (kXlate && f == 1) {
#pragma unroll 4
        for (uint32_t i = tid; i < cnt / 4; i += nthr) {
          int4 k = src[i];
          k.x = __ldg(pa + ((uint32_t)k.x - kmin));
          k.y = __ldg(pa + ((uint32_t)k.y - kmin));
          k.z = __ldg(pa + ((uint32_t)k.z - kmin));
          k.w = __ldg(pa + ((uint32_t)k.w - kmin));
          dst[i] = k;
        }
      } else {
        for (uint32_t i = tid; i < cnt / 4; i += nthr) dst[i] = src[i];
      }
    }
    return;
  }
  for (int f = 0; f < P.n_fields; f++) {
    const int32_t* src = ring + (size_t)f * ring_n + r0;
    int32_t* dst = P.field_out[f] + g;
    if (kXlate && f == 1) {
      for (uint32_t i = tid; i < lim; i += nthr) dst[i] = __ldg(pa + ((uint32_t)src[i] - kmin));
    } else {
      for (uint32_t i = tid; i < lim; i += nthr) dst[i] = src[i];
    }
  }
}

__device__ __forceinline__ bool pred_generic(const WsPred& p, int64_t v) {
  if (p.kind == DDQ_PRED_RANGE) return (uint64_t)(v - p.lo) <= p.d64 && !p.empty;
  if (p.kind == DDQ_PRED_BITSET) return bitset_hit(p.in_vals, p.lo, v);
  bool m = false;
#pragma unroll
  for (int j = 0; j < 8; j++) m |= (j < p.n_in) && (v == p.in_vals[j]);
  return m;
}

// The lane's 16 int32 values of the tile starting at t0: positions
// t0 + s*128 + lofs + v (16-byte aligned), 0 past n.
__device__ __forceinline__ void load16(const int32_t* a, uint32_t t0, uint32_t lofs, uint32_t n, int4 (&r)[4]) {
  const uint32_t base = t0 + lofs;
  if (t0 + WS_TILE <= n) {
#pragma unroll
    for (int s = 0; s < 4; s++) r[s] = ld_stream_i4(a + base + s * 128);
  } else {
#pragma unroll
    for (int s = 0; s < 4; s++) {
      const uint32_t i = base + s * 128;
      r[s].x = i < n ? a[i] : 0;
      r[s].y = i + 1 < n ? a[i + 1] : 0;
      r[s].z = i + 2 < n ? a[i + 2] : 0;
      r[s].w = i + 3 < n ? a[i + 3] : 0;
    }
  }
}
__device__ __forceinline__ void unpack16(const int4 (&r)[4], int32_t (&v)[WS_ITEMS]) {
#pragma unroll
  for (int s = 0; s < 4; s++) {
    v[s * 4 + 0] = r[s].x; v[s * 4 + 1] = r[s].y; v[s * 4 + 2] = r[s].z; v[s * 4 + 3] = r[s].w;
  }
}

// kIn: 0 = every row of the table (keys streamed), 1 = a TID list, 2 = every row
// masked by a row bitmap (a dense probe of a dense intermediate: the key column is
// streamed like kIn 0 -- at >= 1/8 of the rows a gather would touch nearly every
// sector anyway -- and rows outside the bitmap are dead items).  Row bitmap: in the
// kernel's own item order, one 16-bit word per lane and tile (64 B per 512 rows):
// bit 4s+v of word tile*32+l = row tile*512 + s*128 + 4l + v.  kOutBits: the
// survivors are written as such a bitmap -- each lane stores its hit flags (no
// ring, no TIDs); a consumer prefetches one 16-bit word per tile.
template <int kKind, int kIn, bool kPay, bool kCarry, bool kOutBits>
__global__ void __launch_bounds__(ws_nw(kIn == 1) * 32, 1) ws_kernel(const __grid_constant__ WsParams P) {
  constexpr bool kTids = kIn == 1;  // sv[] holds TIDs (gathers at them)
  extern __shared__ __align__(16) uint8_t smem[];
  __shared__ uint32_t s_cnt, s_base;
  __shared__ uint32_t s_filled[WS_RMAX], s_gen[WS_RMAX];
  constexpr uint32_t BLK = ws_blk(kCarry);
  const uint32_t RL = P.ring_logr, RM = (1u << RL) - 1u, RING = BLK << RL;  // R = RM + 1 blocks
  int32_t* ring = reinterpret_cast<int32_t*>(smem);  // fields [tid | payload | carried...] x RING
  constexpr bool kProbe = kKind <= WK_HT_GLOBAL || kKind == WK_BM_COARSE;
  constexpr bool kHash = kKind == WK_HT_SMEM || kKind == WK_HT_GLOBAL;
  // bitmap-masked join-index probe with payloads: most items are dead rows, so the
  // payload lookups wait for the flush (copy_out<true>), where the survivors are dense
  constexpr bool kXlate = kPay && kIn == 2 && !kHash;
  uint32_t* s_bm = reinterpret_cast<uint32_t*>(smem + P.tab_off);
  uint64_t* s_ht = reinterpret_cast<uint64_t*>(smem + P.tab_off);

  if (threadIdx.x == 0) {
    s_cnt = 0;
#pragma unroll
    for (int r = 0; r < WS_RMAX; r++) s_filled[r] = 0, s_gen[r] = 0;
  }
  __shared__ __align__(8) uint64_t s_bar;
  if (kKind == WK_BM_SMEM) {  // + one zero word past the end: the range test is a clamp
    stage_bulk(s_bm, P.bitmap, (P.bitmap_words * 4 + 15) & ~15u, &s_bar);
    if (threadIdx.x == 0) s_bm[P.bitmap_words] = 0u;
  }
  if (kKind == WK_HT_SMEM) stage_bulk(s_ht, P.table, (P.cap_mask + 1) * 8, &s_bar);
  if (kKind == WK_BM_COARSE)  // the index's precomputed coarse bitmap
    stage_bulk(s_bm, P.coarse, (uint32_t)((((P.range >> P.cg) + 1 + 31) / 32 * 4 + 15) & ~15u), &s_bar);
  __syncthreads();

  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t n = kIn == 1 ? ld_relaxed_u32(P.d_in_count) : P.n;
  const uint32_t ntiles = (n + WS_TILE - 1) / WS_TILE;
  constexpr uint32_t NW = ws_nw(kTids);
  const uint32_t W = gridDim.x * NW;
  uint32_t tile = blockIdx.x * NW + warp;
  const uint32_t lofs = lane * 4;  // item (s, v) of lane l sits at tile*512 + s*128 + l*4 + v
  const int32_t* stream = kIn == 1 ? P.in_tids : P.fk;  // the column streamed through registers
  int4 nk[4];          // next tile: 16 keys / TIDs of this lane
  uint32_t nflags = 0;  // kIn 2: next tile's row-bitmap word of this lane
  const uint16_t* in_bits16 = reinterpret_cast<const uint16_t*>(P.in_bits);
  auto fetch = [&](uint32_t t) {
    load16(stream, t * WS_TILE, lofs, n, nk);
    if (kIn == 2) nflags = __ldg(in_bits16 + (size_t)t * 32 + lane);
  };
  if (tile < ntiles) fetch(tile);
  uint32_t bits_cnt = 0;  // kOutBits: survivors of this lane
  // kDefer (a dense or bitmap-masked semi-join: survivors are positions only): a tile's hit flags
  // wait for the warp's next tile and both are compacted with ONE scan / claim /
  // ring accounting (the per-tile compaction was ~60 instructions and three
  // dependent shared-memory atomics for a handful of survivors)
  constexpr bool kDefer = kIn != 1 && !kPay && !kCarry && !kOutBits;
  uint32_t pend = 0, pend_base = 0;
  bool have_pend = false;  // warp-uniform

  for (; tile < ntiles; tile += W) {
    int32_t sv[WS_ITEMS];  // streamed values: keys (dense probe) or TIDs
    unpack16(nk, sv);
    uint32_t flags = kIn == 2 ? nflags : 0xFFFFu;
    const uint32_t base = tile * WS_TILE + lofs;  // position of the lane's item 0
    if (tile + W < ntiles) fetch(tile + W);
    if (kIn == 2) {
      // an empty 512-row tile (unless it is the warp's last and a held tile waits)
      if (__all_sync(FULL, flags == 0) && (!kDefer || !have_pend || tile + W < ntiles)) continue;
    } else if (tile * WS_TILE + WS_TILE > n) {
      flags = 0;
#pragma unroll
      for (int j = 0; j < WS_ITEMS; j++) flags |= (base + (j >> 2) * 128 + (j & 3) < n ? 1u : 0u) << j;
    }
    int32_t pay[WS_ITEMS];
    if (kProbe) {
      int32_t key[WS_ITEMS];
      if (!kTids) {
#pragma unroll
        for (int j = 0; j < WS_ITEMS; j++) key[j] = sv[j];
      } else if (kIn == 1 && P.fk_by_pos) {  // positional key vector: coalesced
        int4 kk[4];
        load16(P.fk, tile * WS_TILE, lofs, n, kk);
        unpack16(kk, key);
      } else {  // key column gathered at the TIDs
#pragma unroll
        for (int j = 0; j < WS_ITEMS; j++) key[j] = ((flags >> j) & 1u) ? ldg_gather(P.fk + (uint32_t)sv[j]) : 0;
      }
      if (!kHash) {
        uint32_t m = 0;
#pragma unroll
        for (int j = 0; j < WS_ITEMS; j++) {
          uint32_t hit;
          if (kKind == WK_BM_SMEM) {
            uint32_t oo = min((uint32_t)(key[j] - P.key_min), P.range);
            // a row outside the input bitmap reads the clamp word like every other
            // dead lane (one broadcast address: fewer bank conflicts, no branch)
            if (kIn == 2) oo = ((flags >> j) & 1u) ? oo : P.range;
            hit = (s_bm[oo >> 5] >> (oo & 31)) & 1u;
          } else if (kKind == WK_BM_COARSE) {  // coarse filter here, exact bit below
            const uint32_t oo = min((uint32_t)(key[j] - P.key_min), P.range);
            const uint32_t cb = oo >> P.cg;
            hit = (s_bm[cb >> 5] >> (cb & 31)) & (oo < P.range ? 1u : 0u);
          } else {  // bitmap in L2: a masked probe looks up its live rows only
            const uint32_t o = (uint32_t)(key[j] - P.key_min);
            const bool look = o < P.range && (kIn != 2 || ((flags >> j) & 1u));
            hit = look ? (__ldg(P.bitmap + (o >> 5)) >> (o & 31)) & 1u : 0u;
          }
          m |= hit << j;
        }
        if (kKind == WK_BM_COARSE) {  // the exact bits of the coarse hits, loads in flight together
          uint32_t fine[WS_ITEMS];
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) {
            const uint32_t o = (uint32_t)(key[j] - P.key_min);
            fine[j] = ((m >> j) & 1u) ? __ldg(P.bitmap + (o >> 5)) : 0u;
          }
          uint32_t m2 = 0;
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) {
            const uint32_t o = (uint32_t)(key[j] - P.key_min);
            m2 |= ((fine[j] >> (o & 31)) & 1u) << j;
          }
          m = m2;
        }
        flags &= m;
        if (kPay && !kXlate) {
          const uint32_t any = __reduce_or_sync(FULL, flags);
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) {
            pay[j] = 0;
            if ((any >> j) & 1u)
              if ((flags >> j) & 1u) pay[j] = __ldg(P.payarr + (uint32_t)(key[j] - P.key_min));
          }
        }
        if (kXlate) {  // the key goes into the ring, translated at the flush
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) pay[j] = key[j];
        }
      } else {
#pragma unroll
        for (int j = 0; j < WS_ITEMS; j++) {
          pay[j] = 0;
          if ((flags >> j) & 1u) {
            uint32_t h = ht_hash(key[j], P.shift);
            uint64_t s = kKind == WK_HT_SMEM ? s_ht[h] : __ldg(P.table + h);
            while (s != HT_EMPTY && ht_key(s) != key[j]) {
              h = (h + 1) & P.cap_mask;
              s = kKind == WK_HT_SMEM ? s_ht[h] : __ldg(P.table + h);
            }
            if (s == HT_EMPTY) flags &= ~(1u << j);
            pay[j] = ht_val(s);
          }
        }
      }
    } else if (kKind == WK_EQ && kIn == 1) {
      int4 a4[4], b4[4];
      load16(P.eq_a, tile * WS_TILE, lofs, n, a4);
      load16(P.eq_b, tile * WS_TILE, lofs, n, b4);
      int32_t a[WS_ITEMS], b[WS_ITEMS];
      unpack16(a4, a);
      unpack16(b4, b);
      uint32_t m = 0;
#pragma unroll
      for (int j = 0; j < WS_ITEMS; j++) m |= (vec_cmp(P.eq_cmp, a[j], b[j]) ? 1u : 0u) << j;
      flags &= m;
    } else if (kIn == 0) {  // dense selection (row bitmap output): the one int32 column streamed
      const WsPred& pr = P.preds[0];
      uint32_t m = 0;
      if (kKind == WK_SEL_RANGE) {
#pragma unroll
        for (int j = 0; j < WS_ITEMS; j++) m |= ((uint64_t)((int64_t)sv[j] - pr.lo) <= pr.d64 ? 1u : 0u) << j;
        if (pr.empty) m = 0;
      } else {
#pragma unroll
        for (int j = 0; j < WS_ITEMS; j++) m |= (pred_generic(pr, (int64_t)sv[j]) ? 1u : 0u) << j;
      }
      flags &= m;
    } else {  // selection at TIDs: later columns gathered for the remaining rows only
      for (int p = 0; p < P.n_preds; p++) {
        const WsPred& pr = P.preds[p];
        int64_t v[WS_ITEMS];
        const uint32_t any = __reduce_or_sync(FULL, flags);
        if (pr.width == 8) {
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) {
            v[j] = 0;
            if ((any >> j) & 1u)
              if ((flags >> j) & 1u) v[j] = ldg_gather(reinterpret_cast<const long long*>(pr.col) + (uint32_t)sv[j]);
          }
        } else {
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) {
            v[j] = 0;
            if ((any >> j) & 1u)
              if ((flags >> j) & 1u) v[j] = ldg_gather(reinterpret_cast<const int32_t*>(pr.col) + (uint32_t)sv[j]);
          }
        }
        uint32_t m = 0;
        if (kKind == WK_SEL_RANGE) {
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) m |= ((uint64_t)(v[j] - pr.lo) <= pr.d64 ? 1u : 0u) << j;
          if (pr.empty) m = 0;
        } else {
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) m |= (pred_generic(pr, v[j]) ? 1u : 0u) << j;
        }
        flags &= m;
      }
    }
    if (kOutBits) {  // ---- row bitmap output: the lane's hit flags, 64 B per warp tile
      bits_cnt += __popc(flags);
      reinterpret_cast<uint16_t*>(P.out_bits)[(size_t)tile * 32 + lane] = (uint16_t)flags;
      continue;
    }
    if (kDefer && !have_pend && tile + W < ntiles) {  // hold this tile, compact with the next
      pend = flags;
      pend_base = base;
      have_pend = true;
      continue;
    }
    // ---- compaction: warp scan of the lanes' hit counts, one smem claim --------
    const uint32_t c = __popc(flags) + (kDefer && have_pend ? __popc(pend) : 0u);
    const uint32_t incl = warp_incl_scan(c, (int)lane);
    const uint32_t tot = __shfl_sync(FULL, incl, 31);
    if (tot == 0) {
      have_pend = false;
      continue;
    }
    uint32_t pos0 = 0;
    if (lane == 0) {
      pos0 = atomicAdd(&s_cnt, tot);
      // wait until the ring blocks this range touches are free (their previous
      // occupants flushed): block b lives in slot b % R, generation b / R
      const uint32_t b0 = pos0 / BLK, b1 = (pos0 + tot - 1) / BLK;
      while (ld_volatile_smem(&s_gen[b0 & RM]) != b0 >> RL) __nanosleep(64);
      if (b1 != b0)
        while (ld_volatile_smem(&s_gen[b1 & RM]) != b1 >> RL) __nanosleep(64);
    }
    pos0 = __shfl_sync(FULL, pos0, 0);
    __syncwarp();
    // predicated stores through a running ring pointer, no per-item branches (a
    // branchy version spent 43 % of the kernel's instructions here)
    const uint32_t r0 = (pos0 & (RING - 1)) + incl - c;  // this lane's first ring slot
    if ((kIn != 1 && !kPay && !kCarry) && (pos0 & (RING - 1)) + tot <= RING) {
      // positions only (a dense semi-join): visit the lane's set bits, not all 16
      // items -- most first probes keep <= 4 % of the rows, where 16 predicated
      // stores per lane and tile were mostly no-ops
      int32_t* wp = ring + r0;
      if (kDefer && have_pend)
        for (uint32_t f = pend; f; f &= f - 1) {
          const uint32_t j = __ffs(f) - 1;
          *wp++ = (int32_t)(pend_base + (j >> 2) * 128 + (j & 3));
        }
      for (uint32_t f = flags; f; f &= f - 1) {
        const uint32_t j = __ffs(f) - 1;
        *wp++ = (int32_t)(base + (j >> 2) * 128 + (j & 3));
      }
    } else if ((pos0 & (RING - 1)) + tot <= RING) {  // the claim does not wrap the ring
      int32_t* wp = ring + r0;
#pragma unroll
      for (int j = 0; j < WS_ITEMS; j++) {
        if (flags & (1u << j)) {
          const uint32_t pos = base + (j >> 2) * 128 + (j & 3);
          wp[0] = kTids ? sv[j] : (int32_t)pos;
          if (kPay) wp[RING] = pay[j];
          wp++;
        }
      }
      if (kCarry) {  // carried vectors: coalesced loads at the tile's positions
        for (int cc = 0; cc < P.n_carry; cc++) {
          int4 cv4[4];
          load16(P.carry_in[cc], tile * WS_TILE, lofs, n, cv4);
          int32_t cv[WS_ITEMS];
          unpack16(cv4, cv);
          int32_t* cp = ring + (size_t)((kPay ? 2 : 1) + cc) * RING + r0;
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) {
            if (flags & (1u << j)) {
              *cp = cv[j];
              cp++;
            }
          }
        }
      }
    } else {
      uint32_t p = r0;
      if (kDefer && have_pend)  // the held tile's positions first (ring wrap)
        for (uint32_t f = pend; f; f &= f - 1) {
          const uint32_t j = __ffs(f) - 1;
          ring[p & (RING - 1)] = (int32_t)(pend_base + (j >> 2) * 128 + (j & 3));
          p++;
        }
#pragma unroll
      for (int j = 0; j < WS_ITEMS; j++) {
        if ((flags >> j) & 1u) {
          const uint32_t r = p & (RING - 1);
          const uint32_t pos = base + (j >> 2) * 128 + (j & 3);
          ring[r] = kTids ? sv[j] : (int32_t)pos;
          if (kPay) ring[RING + r] = pay[j];
          p++;
        }
      }
      if (kCarry) {
        for (int cc = 0; cc < P.n_carry; cc++) {
          int4 cv4[4];
          load16(P.carry_in[cc], tile * WS_TILE, lofs, n, cv4);
          int32_t cv[WS_ITEMS];
          unpack16(cv4, cv);
          int32_t* cb = ring + (size_t)((kPay ? 2 : 1) + cc) * RING;
          uint32_t q = r0;
#pragma unroll
          for (int j = 0; j < WS_ITEMS; j++) {
            if ((flags >> j) & 1u) {
              cb[q & (RING - 1)] = cv[j];
              q++;
            }
          }
        }
      }
    }
    __threadfence_block();
    __syncwarp();
    have_pend = false;
    // account the written entries to their blocks; the warp completing a block flushes it
    uint32_t flush = 0;  // bit 0: block b0, bit 1: block b1
    if (lane == 0) {
      const uint32_t end = pos0 + tot;
      const uint32_t b0 = pos0 / BLK, b1 = (end - 1) / BLK;
      const uint32_t c0 = (b1 == b0 ? end : (b0 + 1) * BLK) - pos0;
      if (atomicAdd(&s_filled[b0 & RM], c0) + c0 == BLK) flush |= 1u;
      if (b1 != b0) {
        const uint32_t c1 = end - b1 * BLK;
        if (atomicAdd(&s_filled[b1 & RM], c1) + c1 == BLK) flush |= 2u;
      }
      __threadfence_block();
    }
    flush = __shfl_sync(FULL, flush, 0);
    // ring hand-off between warps is flag-synchronised, not barrier-synchronised:
    // writers fence (CTA) before their s_filled atomics, the flushing warp's lane 0
    // fences after its atomic, and this warp barrier orders that for all its lanes
    // before they read the block; the block is recycled through s_gen the same way.
    // (compute-sanitizer racecheck models only barriers and reports these hand-offs,
    // profiles/r2_sanitize_summary.txt)
    __syncwarp();
    while (flush) {
      const uint32_t b = (flush & 1u) ? pos0 / BLK : (pos0 + tot - 1) / BLK;
      flush &= flush - 1;
      const uint32_t slot = b & RM;
      uint32_t g = 0;
      if (lane == 0) g = atomicAdd(P.d_out_count, BLK);
      g = __shfl_sync(FULL, g, 0);
      copy_out<kXlate>(P, ring, RING, slot * BLK, BLK, g, lane, 32);
      __threadfence_block();
      __syncwarp();
      if (lane == 0) {
        s_filled[slot] = 0;
        __threadfence_block();
        atomicAdd(&s_gen[slot], 1u);
      }
    }
  }
  if (kOutBits) {  // survivor count: warp sum -> CTA -> one global atomic
    bits_cnt = __reduce_add_sync(FULL, bits_cnt);
    if (lane == 0 && bits_cnt) atomicAdd(&s_cnt, bits_cnt);
    __syncthreads();
    if (threadIdx.x == 0 && s_cnt) atomicAdd(P.d_out_count, s_cnt);
    return;
  }
  // the CTA's last, partial block: an exact reservation (no holes)
  __syncthreads();
  const uint32_t total = s_cnt;
  const uint32_t rem = total % BLK;
  if (rem) {
    if (threadIdx.x == 0) s_base = atomicAdd(P.d_out_count, rem);
    __syncthreads();
    copy_out<kXlate>(P, ring, RING, ((total / BLK) & RM) * BLK, rem, s_base, threadIdx.x, blockDim.x);
  }
  // the last CTA to finish clamps the count to the output capacity
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(P.d_out_count + 1, 1u) == gridDim.x - 1) {
      const uint32_t cnt = atomicAdd(P.d_out_count, 0u);
      if (cnt > P.out_cap) *P.d_out_count = P.out_cap;
    }
  }
}

int g_optin = 0;
constexpr size_t kWsCtl = 1024;  // static smem + reserve

template <int K, int In, bool Pa, bool C, bool Ob>
void ws_attr() {
  cudaFuncSetAttribute(ws_kernel<K, In, Pa, C, Ob>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       g_optin - (int)kWsCtl);
}
template <int K>
void ws_attr_kind() {
  constexpr bool kProbe = K <= WK_HT_GLOBAL || K == WK_BM_COARSE;
  if constexpr (kProbe) {  // dense inputs: probes only (payload, or a bitmap of the survivors)
    ws_attr<K, 0, false, false, false>();
    ws_attr<K, 0, true, false, false>();
    ws_attr<K, 0, false, false, true>();
  }
  if constexpr (K == WK_SEL_RANGE || K == WK_SEL_GENERIC)  // dense selection -> row bitmap
    ws_attr<K, 0, false, false, true>();
  ws_attr<K, 1, false, false, false>();
  ws_attr<K, 1, false, true, false>();
  if constexpr (kProbe) {
    ws_attr<K, 1, true, false, false>();
    ws_attr<K, 1, true, true, false>();
  }
  if constexpr (kProbe) {  // bitmap-masked dense probes (no carried vectors)
    ws_attr<K, 2, false, false, false>();
    ws_attr<K, 2, true, false, false>();
  }
}

template <int K>
void launch_k(int in, bool pay, bool carry, bool obits, int grid, size_t smem, cudaStream_t st,
              const WsParams& p) {
  constexpr bool kProbe = K <= WK_HT_GLOBAL || K == WK_BM_COARSE;
  if constexpr (kProbe) {
    if (in == 0) {
      const dim3 blk(ws_nw(false) * 32);
      if (obits) ws_kernel<K, 0, false, false, true><<<grid, blk, smem, st>>>(p);
      else if (pay) ws_kernel<K, 0, true, false, false><<<grid, blk, smem, st>>>(p);
      else ws_kernel<K, 0, false, false, false><<<grid, blk, smem, st>>>(p);
      return;
    }
  }
  if constexpr (kProbe) {
    if (in == 2) {
      const dim3 blk2(ws_nw(false) * 32);
      if (pay) ws_kernel<K, 2, true, false, false><<<grid, blk2, smem, st>>>(p);
      else ws_kernel<K, 2, false, false, false><<<grid, blk2, smem, st>>>(p);
      return;
    }
  }
  if constexpr (K == WK_SEL_RANGE || K == WK_SEL_GENERIC) {
    if (in == 0) {  // a dense selection writes a row bitmap (ws_supported)
      ws_kernel<K, 0, false, false, true><<<grid, dim3(ws_nw(false) * 32), smem, st>>>(p);
      return;
    }
  }
  const dim3 blk(ws_nw(true) * 32);
  if constexpr (kProbe) {
    if (pay) {
      if (carry) ws_kernel<K, 1, true, true, false><<<grid, blk, smem, st>>>(p);
      else ws_kernel<K, 1, true, false, false><<<grid, blk, smem, st>>>(p);
      return;
    }
  }
  if (carry) ws_kernel<K, 1, false, true, false><<<grid, blk, smem, st>>>(p);
  else ws_kernel<K, 1, false, false, false><<<grid, blk, smem, st>>>(p);
}

}  // namespace

bool ws_supported(const FilterArgs& a) {
  const bool tids = a.in_tids != nullptr;
  if (a.n_carry > 4 || a.n_cap > (int64_t)0x7FFFFFFF) return false;
  if (a.out_bits && (a.in_tids || a.in_bits || a.out_payload)) return false;
  if (a.in_bits) {  // row bitmap input: probes of a key column (streamed), no vectors
    if (!a.probe || a.fk_by_pos || a.eq_a || a.n_carry || ((uintptr_t)a.in_bits & 15) != 0) return false;
    if (((uintptr_t)a.fk & 15) != 0) return false;
  } else if (!tids) {  // dense: probes, or ONE int32 predicate column into a row bitmap (O27);
                       // other dense selections stream several columns: scan.cu
    if (!a.probe) {
      if (!a.out_bits || a.n_preds != 1 || a.preds[0].width != 4 || a.eq_a || a.n_carry) return false;
      if (((uintptr_t)a.preds[0].col & 15) != 0) return false;
    } else {
      if (a.fk_by_pos || a.eq_a || a.n_carry) return false;
      if (((uintptr_t)a.fk & 15) != 0) return false;
    }
  } else {
    if (((uintptr_t)a.in_tids & 15) != 0) return false;
    if (a.probe && a.fk_by_pos && ((uintptr_t)a.fk & 15) != 0) return false;
    if (a.eq_a && ((((uintptr_t)a.eq_a | (uintptr_t)a.eq_b) & 15) != 0)) return false;
    if (!a.probe && !a.eq_a && (a.n_preds < 1 || a.n_preds > 4)) return false;
    if (!a.probe && a.eq_a && a.n_preds) return false;
  }
  if (a.out_payload && ((uintptr_t)a.out_payload & 15) != 0) return false;
  for (int c = 0; c < a.n_carry; c++)  // carried vectors: 16-byte loads and copies
    if ((((uintptr_t)a.carry_in[c] | (uintptr_t)a.carry_out[c]) & 15) != 0) return false;
  return ((uintptr_t)a.out_tids & 15) == 0;
}

// Staging a table in every SM's shared memory costs ~tab x 148 bytes of L2 reads
// and one round trip per CTA; for small inputs the probes go to the L2-resident
// global copy instead (a few thousand late-materialisation lookups must not pay
// for a 75 KB bitmap per SM).
static bool stage_pays(int64_t n_cap, size_t tab) { return n_cap >= (int64_t)(tab * 4); }

// Whether launch_ws stages a probe's join-index bitmap (join index over `range`
// keys) or hash table (`capacity` slots) in shared memory for a bitmap-masked probe
// of n_rows rows (the WK_BM_SMEM / WK_HT_SMEM choice below).  ddq_prepare hands a
// row bitmap only to such consumers: with the table in L2 (customer at SF >= 60)
// the masked probe issues its L2 lookups at every row slot, live or dead
// (SF100 Q3.1: 1.26 ms against a TID list's fraction of that).
bool ws_masked_probe_smem(bool join_index, uint32_t range_or_capacity, int64_t n_rows, bool pay) {
  int dev = 0, v = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  const size_t budget = (size_t)v - kWsCtl;
  const size_t ring1 = (size_t)ws_blk(false) * 4 * (pay ? 2 : 1);
  const size_t tab = join_index ? ((size_t)((range_or_capacity + 31) / 32) * 4 + 15) / 16 * 16 + 16
                                : (size_t)range_or_capacity * 8;
  return 4 * ring1 + tab <= budget && stage_pays(n_rows, tab);
}

cudaError_t launch_ws(const FilterArgs& a, cudaStream_t st) {
  // one-time opt-in of every variant's dynamic shared memory; a function-local static
  // initialiser, so concurrent GPU workers wait for it (no launch before the attributes)
  static const bool ws_ready = [] {
    int dev = 0, v = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    g_optin = v;
    ws_attr_kind<WK_BM_SMEM>();
    ws_attr_kind<WK_BM_GLOBAL>();
    ws_attr_kind<WK_HT_SMEM>();
    ws_attr_kind<WK_HT_GLOBAL>();
    ws_attr_kind<WK_SEL_RANGE>();
    ws_attr_kind<WK_SEL_GENERIC>();
    ws_attr_kind<WK_EQ>();
    ws_attr_kind<WK_BM_COARSE>();
    return true;
  }();
  (void)ws_ready;
  const int in = a.in_bits ? 2 : (a.in_tids ? 1 : 0);
  WsParams p{};
  p.n = (uint32_t)a.n_cap;
  p.d_in_count = a.d_in_count;
  p.in_tids = a.in_tids;
  p.in_bits = a.in_bits;
  p.out_bits = a.out_bits;
  const bool obits = a.out_bits != nullptr;
  const bool pay = a.probe && a.out_payload != nullptr;
  const bool carry = in == 1 && a.n_carry > 0;
  const int n_fields = 1 + (pay ? 1 : 0) + (carry ? a.n_carry : 0);
  const size_t ring1 = (size_t)ws_blk(carry) * 4 * n_fields;  // one ring block, all fields
  const size_t budget = (size_t)g_optin - kWsCtl;
  int kind;
  size_t tab = 0;
  if (a.probe) {
    p.fk = a.fk;
    p.fk_by_pos = a.fk_by_pos ? 1 : 0;
    if (a.bitmap) {
      p.bitmap = a.bitmap;
      p.payarr = a.payarr;
      p.key_min = a.key_min;
      p.range = a.range;
      p.bitmap_words = (a.range + 31) / 32;
      tab = ((size_t)p.bitmap_words * 4 + 15) / 16 * 16 + 16;  // bulk-copy rounding + the zero word
      kind = (!a.no_smem && (obits ? 0 : 4 * ring1) + tab <= budget && stage_pays(a.n_cap, tab)) ? WK_BM_SMEM
                                                                                                 : WK_BM_GLOBAL;
      // a bitmap too large for one SM (customer at SF > 50, part at SF >= 128): the
      // index's coarse bitmap (1 bit per 2^cg keys) filters in shared memory; only
      // coarse hits read the exact bit from L2
      static const char* co_env = getenv("DDQ_BM_COARSE");  // "0": exact lookups in L2 instead
      // Probes of every row only: at a TID list (or row bitmap) the exact lookups
      // are L1-cached, and the coarse table's shared memory shrinks that L1 (SF80
      // Q3.1's customer probe at 24 M TIDs: 514 -> 720 us with it)
      if (kind == WK_BM_GLOBAL && a.coarse && in == 0 && !a.no_smem && !(co_env && co_env[0] == '0')) {
        const uint32_t cg = join_index_cg(a.range);
        const size_t ctab = ji_coarse_bytes_cg(a.range, cg);
        if ((obits ? 0 : 4 * ring1) + ctab <= budget && stage_pays(a.n_cap, ctab)) {
          kind = WK_BM_COARSE;
          p.cg = cg;
          p.coarse = a.coarse;
          tab = ctab;
        }
      }
    } else {
      p.table = a.table;
      p.cap_mask = a.capacity - 1;
      int lg = 0;
      while ((1u << lg) < a.capacity) lg++;
      p.shift = 32 - lg;
      tab = (size_t)a.capacity * 8;
      kind = (!a.no_smem && (obits ? 0 : 4 * ring1) + tab <= budget && stage_pays(a.n_cap, tab)) ? WK_HT_SMEM
                                                                                                 : WK_HT_GLOBAL;
    }
  } else if (a.eq_a) {
    kind = WK_EQ;
    p.eq_a = a.eq_a;
    p.eq_b = a.eq_b;
    p.eq_cmp = a.eq_cmp;
  } else {
    bool all_range = true;
    p.n_preds = a.n_preds;
    for (int i = 0; i < a.n_preds; i++) {
      const ddq_dev_pred& d = a.preds[i];
      WsPred& q = p.preds[i];
      q.col = d.col;
      q.width = d.width;
      q.kind = d.kind;
      q.lo = d.lo;
      q.hi = d.hi;
      q.empty = d.hi < d.lo;
      q.d64 = q.empty ? 0 : (uint64_t)d.hi - (uint64_t)d.lo;
      q.n_in = d.n_in;
      for (int j = 0; j < 8; j++) q.in_vals[j] = d.in_vals[j];
      all_range = all_range && d.kind == DDQ_PRED_RANGE;
    }
    kind = all_range ? WK_SEL_RANGE : WK_SEL_GENERIC;
    if (in == 0) p.fk = reinterpret_cast<const int32_t*>(a.preds[0].col);  // dense: the column streamed
  }
  // ring: 4 blocks.  More blocks would put more flushes in flight (ncu: a quarter
  // of a 100 %-pass late-fetch probe's instructions spin on a free slot), but
  // shared memory is carved out of the unified L1 where the payload-array lookups
  // live: 16 blocks made the date probe's d_year lookups miss (74 -> 141 us) and
  // 8 blocks slowed the late fetch itself (119 -> 195 us)
  const size_t tab_smem = (kind == WK_BM_SMEM || kind == WK_HT_SMEM || kind == WK_BM_COARSE) ? tab : 0;
  int logr = 2;
  // (Tried: 8-16 blocks for a dense semi-join probe with a dense known output --
  // ncu, SSB Q3.1 at 20 % survivors: 3.6 M spin loads on busy blocks next to 3.75 M
  // bitmap lookups.  Q3.1 / Q4.2's probes 147 / 151 -> 137 / 137 us alone, but the
  // 4-stream step 2.67 -> 3.03 ms: a 200 KB CTA leaves no room for the other
  // streams' kernels on its SM.)  DDQ_WS_RING_LOGR: A/B override.
  if (const char* e = getenv("DDQ_WS_RING_LOGR")) logr = std::max(2, std::min(4, atoi(e)));
  const size_t ring = obits ? 0 : ring1 << logr;
  p.ring_logr = logr;
  p.tab_off = (int32_t)ring;
  p.n_carry = carry ? a.n_carry : 0;
  for (int c = 0; c < p.n_carry; c++) {
    p.carry_in[c] = a.carry_in[c];
    p.carry_out[c] = a.carry_out[c];
  }
  p.out_tids = a.out_tids;
  p.out_payload = pay ? a.out_payload : nullptr;
  p.n_fields = n_fields;
  p.field_out[0] = a.out_tids;
  if (pay) p.field_out[1] = a.out_payload;
  for (int c = 0; c < p.n_carry; c++) p.field_out[(pay ? 2 : 1) + c] = a.carry_out[c];
  p.d_out_count = a.d_out_count;
  p.out_cap = (uint32_t)(a.out_cap > 0 ? a.out_cap : a.n_cap);
  p.d_overflow = a.d_overflow;
  cudaError_t e = init_fill(a.d_out_count, 8, 0, st);
  if (e != cudaSuccess) return e;
  const size_t smem = ring + tab_smem;
  const int64_t ntiles = (a.n_cap + WS_TILE - 1) / WS_TILE;  // TID input: an upper bound
  int64_t grid = num_sms();
  const int64_t need = (ntiles + ws_nw(in == 1) - 1) / ws_nw(in == 1);
  if (grid > need) grid = need < 1 ? 1 : need;
  switch (kind) {
    case WK_BM_SMEM: launch_k<WK_BM_SMEM>(in, pay, carry, obits, (int)grid, smem, st, p); break;
    case WK_BM_GLOBAL: launch_k<WK_BM_GLOBAL>(in, pay, carry, obits, (int)grid, smem, st, p); break;
    case WK_HT_SMEM: launch_k<WK_HT_SMEM>(in, pay, carry, obits, (int)grid, smem, st, p); break;
    case WK_HT_GLOBAL: launch_k<WK_HT_GLOBAL>(in, pay, carry, obits, (int)grid, smem, st, p); break;
    case WK_SEL_RANGE: launch_k<WK_SEL_RANGE>(in, false, carry, false, (int)grid, smem, st, p); break;
    case WK_SEL_GENERIC: launch_k<WK_SEL_GENERIC>(in, false, carry, false, (int)grid, smem, st, p); break;
    case WK_BM_COARSE: launch_k<WK_BM_COARSE>(in, pay, carry, obits, (int)grid, smem, st, p); break;
    default: launch_k<WK_EQ>(in, false, carry, false, (int)grid, smem, st, p); break;
  }
  return cudaGetLastError();
}

}  // namespace ddq
