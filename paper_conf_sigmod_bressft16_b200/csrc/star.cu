// star.cu -- n-ary semi-join over all rows of a fact table in ONE pass (DDQ_OP_STAR):
// a conjunction of predicates (S8(a2)) and dimension probes (S8(a4)), each on its
// own fact column, emitting the surviving TIDs and the probes' payloads.
//
// Why: ncu showed the column-at-a-time chain "dense probe -> probe
// at TIDs -> probe at TIDs" gathering the later FK columns at 64-128 B DRAM
// granularity, reading ~0.35-0.6 GB per 4-byte column regardless of the TID density,
// plus the TID lists in between.  Streaming every term column once with TMA costs
// exactly 4 B/row/column and removes the intermediate TID lists.  The operator is
// still an operator of the plan (children: the builds; data-driven placement needs
// all term columns cached), only n-ary.
//
// Structure = scan.cu's: one CTA per SM with G independent 256-thread groups, each a
// TMA ring (one bulk copy per column per tile) + named barrier + double-buffered
// survivor lists; per-tile output reservation by one atomicAdd, copied out one
// iteration later.  The stage of tile k-1 is refilled only after its copy-out (B),
// because payloads are looked up from the staged fk values at copy-out.  Membership
// structures (join-index bitmaps, small hash tables) of as many terms as fit are
// staged once per SM in shared memory; the rest are read through L2.
#include <cstdint>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "ops_internal.h"

namespace ddq {

constexpr int ST_GT = 256;
constexpr int ST_GW = ST_GT / 32;
constexpr int ST_MAXT = 4;
constexpr int ST_MAXG = 4;
constexpr int ST_MAXS = 4;

struct StarTerm {
  int32_t kind, width;
  const void* col;
  int32_t col_off;  // offset of the term's column inside a stage
  int32_t pred_kind, n_in;
  int64_t lo, hi;
  int64_t in_vals[8];
  // probe
  int32_t direct;
  const uint32_t* bitmap;
  const int32_t* payarr;
  int32_t key_min;
  uint32_t range;
  const uint64_t* table;
  uint32_t cap_mask;
  int32_t shift;
  int32_t smem_off;    // >= 0: membership structure staged at this shared-memory offset
  uint32_t smem_words; // 4-byte words staged
  int32_t* out_payload;
};

struct StarParams {
  uint32_t n;
  int32_t n_terms;
  StarTerm terms[ST_MAXT];
  int32_t tile;  // rows per tile (= 256 x ITEMS)
  int32_t stage_bytes, stages, group_bytes, list_off;
  int32_t* out_tids;
  uint32_t* d_out_count;
  uint32_t out_cap;
  uint32_t* d_overflow;
};

__device__ __forceinline__ uint32_t st_smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void st_mbar_init(uint64_t* bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(st_smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void st_mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
        : "=r"(done) : "r"(st_smem_u32(bar)), "r"(parity) : "memory");
  }
}
__device__ __forceinline__ void st_issue(const StarParams& P, uint8_t* buf, uint64_t* bar, uint32_t tile) {
  const uint64_t row0 = (uint64_t)tile * P.tile;
  const uint64_t rows = (uint64_t)P.n - row0 < (uint64_t)P.tile ? (uint64_t)P.n - row0 : (uint64_t)P.tile;
  uint32_t total = 0;
  for (int j = 0; j < P.n_terms; j++) total += (uint32_t)((rows * P.terms[j].width + 15) / 16 * 16);
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(st_smem_u32(bar)), "r"(total)
               : "memory");
  for (int j = 0; j < P.n_terms; j++) {
    const StarTerm& T = P.terms[j];
    const uint32_t bytes = (uint32_t)((rows * T.width + 15) / 16 * 16);
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(st_smem_u32(buf + T.col_off)), "l"(reinterpret_cast<const uint8_t*>(T.col) + row0 * T.width),
                 "r"(bytes), "r"(st_smem_u32(bar)) : "memory");
  }
}

__device__ __forceinline__ bool st_pred(const StarTerm& p, int64_t v) {
  if (p.pred_kind == DDQ_PRED_RANGE) return v >= p.lo && v <= p.hi;
  if (p.pred_kind == DDQ_PRED_BITSET) return bitset_hit(p.in_vals, p.lo, v);
  bool m = false;
#pragma unroll
  for (int j = 0; j < 8; j++) m |= (j < p.n_in) && (v == p.in_vals[j]);
  return m;
}

// hash lookup: payload or INT32_MIN sentinel-free "found" flag through *found
__device__ __forceinline__ int32_t st_hash_find(const StarTerm& T, const uint64_t* table, int32_t key, bool* found) {
  uint32_t h = ht_hash(key, T.shift);
  uint64_t s = table[h];
  while (s != HT_EMPTY && ht_key(s) != key) {
    h = (h + 1) & T.cap_mask;
    s = table[h];
  }
  *found = s != HT_EMPTY;
  return ht_val(s);
}

template <int G, int ST_ITEMS>
__global__ void __launch_bounds__(ST_GT* G, 1) star_kernel(const __grid_constant__ StarParams P) {
  constexpr int ST_TILE = ST_GT * ST_ITEMS;
  constexpr int ST_SLOTS = ST_ITEMS / 4;
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint32_t s_warp_tot[ST_MAXG][ST_GW];
  __shared__ uint32_t s_base[ST_MAXG];
  __shared__ __align__(8) uint64_t s_full[ST_MAXG][ST_MAXS];
  const int g = threadIdx.x / ST_GT, t = threadIdx.x % ST_GT;
  const int lane = t & 31, warp = t >> 5;
  const uint32_t ntiles = (P.n + ST_TILE - 1) / ST_TILE;
  const int S = P.stages;
  const uint32_t vb = blockIdx.x * G + g, vgrid = gridDim.x * G;
  uint8_t* ring = smem + (size_t)g * P.group_bytes;
  uint16_t* s_list = reinterpret_cast<uint16_t*>(ring + P.list_off);  // 2 x TILE

  if (t == 0) {
    for (int k = 0; k < S; k++) st_mbar_init(&s_full[g][k]);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    for (int k = 0; k < S - 1; k++) {
      const uint32_t tl = vb + (uint32_t)k * vgrid;
      if (tl < ntiles) st_issue(P, ring + (size_t)k * P.stage_bytes, &s_full[g][k], tl);
    }
  }
  // stage the membership structures that fit, once per SM
  for (int j = 0; j < P.n_terms; j++) {
    const StarTerm& T = P.terms[j];
    if (T.kind != DDQ_TERM_PROBE || T.smem_off < 0) continue;
    uint32_t* dst = reinterpret_cast<uint32_t*>(smem + T.smem_off);
    const uint32_t* src = T.direct ? T.bitmap : reinterpret_cast<const uint32_t*>(T.table);
    for (uint32_t i = threadIdx.x; i < T.smem_words; i += ST_GT * G) dst[i] = src[i];
  }
  __syncthreads();

  uint32_t prev_tot = 0, prev_base = 0;
  const uint32_t wrow = warp * (32 * ST_ITEMS);
  for (uint32_t k = 0;; k++) {
    const uint32_t tile = vb + k * vgrid;
    const bool have = tile < ntiles;
    const uint32_t row0 = tile * ST_TILE;
    uint32_t flags = 0;
    if (have) {
      st_mbar_wait(&s_full[g][k % S], (k / S) & 1u);
      const uint8_t* buf = ring + (size_t)(k % S) * P.stage_bytes;
      flags = (1u << ST_ITEMS) - 1u;
      if (row0 + ST_TILE > P.n) {
        flags = 0;
#pragma unroll
        for (int s = 0; s < ST_SLOTS; s++)
#pragma unroll
          for (int v = 0; v < 4; v++)
            flags |= (row0 + wrow + s * 128 + lane * 4 + v < P.n ? 1u : 0u) << (s * 4 + v);
      }
      for (int j = 0; j < P.n_terms; j++) {
        if (!__any_sync(FULL, flags != 0)) break;  // the whole warp is already rejected
        const StarTerm& T = P.terms[j];
        const uint8_t* cb = buf + T.col_off;
        if (T.kind == DDQ_TERM_PRED) {
#pragma unroll
          for (int s = 0; s < ST_SLOTS; s++) {
            const int it = wrow + s * 128 + lane * 4;
            int64_t v4[4];
            if (T.width == 8) {
              const longlong2 a = *reinterpret_cast<const longlong2*>(cb + (size_t)it * 8);
              const longlong2 b = *reinterpret_cast<const longlong2*>(cb + (size_t)it * 8 + 16);
              v4[0] = a.x; v4[1] = a.y; v4[2] = b.x; v4[3] = b.y;
            } else {
              const int4 a = *reinterpret_cast<const int4*>(cb + (size_t)it * 4);
              v4[0] = a.x; v4[1] = a.y; v4[2] = a.z; v4[3] = a.w;
            }
            uint32_t m = 0;
#pragma unroll
            for (int v = 0; v < 4; v++) m |= (st_pred(T, v4[v]) ? 1u : 0u) << v;
            flags &= ~((~m & 0xFu) << (s * 4));
          }
        } else if (T.direct) {
          const uint32_t* bm = T.smem_off >= 0 ? reinterpret_cast<const uint32_t*>(smem + T.smem_off) : T.bitmap;
          uint32_t m = 0;
#pragma unroll
          for (int s = 0; s < ST_SLOTS; s++) {
            const int4 a = *reinterpret_cast<const int4*>(cb + (size_t)(wrow + s * 128 + lane * 4) * 4);
            const int32_t kk[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
            for (int v = 0; v < 4; v++) {
              const uint32_t o = (uint32_t)(kk[v] - T.key_min);
              const bool live = ((flags >> (s * 4 + v)) & 1u) && o < T.range;
              const uint32_t w = live ? bm[o >> 5] : 0u;
              m |= ((w >> (o & 31)) & 1u) << (s * 4 + v);
            }
          }
          flags &= m;
        } else {
          const uint64_t* tb = T.smem_off >= 0 ? reinterpret_cast<const uint64_t*>(smem + T.smem_off) : T.table;
#pragma unroll
          for (int s = 0; s < ST_SLOTS; s++) {
            const int4 a = *reinterpret_cast<const int4*>(cb + (size_t)(wrow + s * 128 + lane * 4) * 4);
            const int32_t kk[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
            for (int v = 0; v < 4; v++) {
              if (!((flags >> (s * 4 + v)) & 1u)) continue;
              bool found;
              st_hash_find(T, tb, kk[v], &found);
              if (!found) flags &= ~(1u << (s * 4 + v));
            }
          }
        }
      }
    }
    // group scan of the per-slot survivor counts
    uint32_t packed = 0;
#pragma unroll
    for (int s = 0; s < ST_SLOTS; s++) packed |= (uint32_t)__popc((flags >> (4 * s)) & 0xFu) << (8 * s);
    const uint32_t incl = warp_incl_scan(packed, lane);
    const uint32_t excl = incl - packed;
    const uint32_t wtot = __shfl_sync(FULL, incl, 31);
    uint32_t slot_off[ST_SLOTS];
    uint32_t acc = 0;
#pragma unroll
    for (int s = 0; s < ST_SLOTS; s++) {
      slot_off[s] = acc;
      acc += (wtot >> (8 * s)) & 0xFFu;
    }
    if (lane == 0) s_warp_tot[g][warp] = acc;
    asm volatile("bar.sync %0, %1;" ::"r"(g + 1), "r"(ST_GT) : "memory");  // (A)
    uint32_t tot = 0, warp_off = 0;
#pragma unroll
    for (int w = 0; w < ST_GW; w++) {
      const uint32_t x = s_warp_tot[g][w];
      warp_off += (w < warp) ? x : 0;
      tot += x;
    }
    uint32_t my_base = 0;
    if (t == 0) my_base = tot ? atomicAdd(P.d_out_count, tot) : 0;  // consumed only before (B)
    uint16_t* lst = s_list + (k & 1) * ST_TILE;
#pragma unroll
    for (int s = 0; s < ST_SLOTS; s++) {
      const uint32_t m = (flags >> (4 * s)) & 0xFu;
      const uint32_t sb = warp_off + slot_off[s] + ((excl >> (8 * s)) & 0xFFu);
#pragma unroll
      for (int v = 0; v < 4; v++)
        if ((m >> v) & 1u) lst[sb + __popc(m & ((1u << v) - 1u))] = (uint16_t)(wrow + s * 128 + lane * 4 + v);
    }
    if (k > 0) {  // copy out tile k-1: TIDs + payloads from the (still staged) fk values
      const uint16_t* pl = s_list + ((k - 1) & 1) * ST_TILE;
      const uint8_t* pbuf = ring + (size_t)((k - 1) % S) * P.stage_bytes;
      const uint32_t prow0 = (tile - vgrid) * ST_TILE;
      const uint32_t lim = prev_base + prev_tot <= P.out_cap ? prev_tot
                         : (P.out_cap > prev_base ? P.out_cap - prev_base : 0);
      if (lim < prev_tot && t == 0 && P.d_overflow) atomicMax(P.d_overflow, 4u);
      for (uint32_t i = t; i < lim; i += ST_GT) {
        const uint32_t it = pl[i];
        P.out_tids[prev_base + i] = (int32_t)(prow0 + it);
        for (int j = 0; j < P.n_terms; j++) {
          const StarTerm& T = P.terms[j];
          if (T.kind != DDQ_TERM_PROBE || !T.out_payload) continue;
          const int32_t key = reinterpret_cast<const int32_t*>(pbuf + T.col_off)[it];
          int32_t pv;
          if (T.direct) {
            pv = __ldg(T.payarr + (uint32_t)(key - T.key_min));
          } else {
            const uint64_t* tb = T.smem_off >= 0 ? reinterpret_cast<const uint64_t*>(smem + T.smem_off) : T.table;
            bool found;
            pv = st_hash_find(T, tb, key, &found);
          }
          T.out_payload[prev_base + i] = pv;
        }
      }
    }
    if (t == 0) s_base[g] = my_base;
    asm volatile("bar.sync %0, %1;" ::"r"(g + 1), "r"(ST_GT) : "memory");  // (B)
    if (t == 0 && have) {  // refill stage (k-1)%S with tile k+S-1
      const uint32_t tl = tile + (uint32_t)(S - 1) * vgrid;
      if (tl < ntiles) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        const int st = (int)((k + S - 1) % S);
        st_issue(P, ring + (size_t)st * P.stage_bytes, &s_full[g][st], tl);
      }
    }
    prev_base = s_base[g];
    prev_tot = tot;
    if (!have) break;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(P.d_out_count + 1, 1u) == gridDim.x - 1) {
      const uint32_t c = atomicAdd(P.d_out_count, 0u);
      if (c > P.out_cap) *P.d_out_count = P.out_cap;
    }
  }
}

static int g_star_optin = 0;

template <int I>
static void star_attrs(int v) {
  cudaFuncSetAttribute(star_kernel<1, I>, cudaFuncAttributeMaxDynamicSharedMemorySize, v - 2048);
  cudaFuncSetAttribute(star_kernel<2, I>, cudaFuncAttributeMaxDynamicSharedMemorySize, v - 2048);
  cudaFuncSetAttribute(star_kernel<3, I>, cudaFuncAttributeMaxDynamicSharedMemorySize, v - 2048);
  cudaFuncSetAttribute(star_kernel<4, I>, cudaFuncAttributeMaxDynamicSharedMemorySize, v - 2048);
}

template <int I>
static void star_launch_g(int G, int64_t grid, size_t smem, cudaStream_t st, const StarParams& p) {
  switch (G) {
    case 1: star_kernel<1, I><<<(int)grid, ST_GT * 1, smem, st>>>(p); break;
    case 2: star_kernel<2, I><<<(int)grid, ST_GT * 2, smem, st>>>(p); break;
    case 3: star_kernel<3, I><<<(int)grid, ST_GT * 3, smem, st>>>(p); break;
    default: star_kernel<4, I><<<(int)grid, ST_GT * 4, smem, st>>>(p); break;
  }
}

cudaError_t launch_star(const ddq_dev_term* terms, int n_terms, int64_t n_rows, int32_t* out_tids,
                        uint32_t* d_out_count, int64_t out_cap, uint32_t* d_overflow, cudaStream_t st) {
  static const bool star_ready = [] {  // thread-safe one-time opt-in
    int dev = 0, v = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    star_attrs<4>(v);
    star_attrs<8>(v);
    g_star_optin = v;
    return true;
  }();
  (void)star_ready;
  StarParams p{};
  p.n = (uint32_t)n_rows;
  p.n_terms = n_terms;
  int row_bytes = 0;
  for (int j = 0; j < n_terms; j++) {
    const ddq_dev_term& d = terms[j];
    StarTerm& T = p.terms[j];
    T.kind = d.kind;
    T.width = d.width;
    T.col = d.col;
    T.col_off = row_bytes;  // scaled by the tile size below
    row_bytes += d.width;
    T.pred_kind = d.pred_kind;
    T.n_in = d.n_in;
    T.lo = d.lo;
    T.hi = d.hi;
    for (int i = 0; i < 8; i++) T.in_vals[i] = d.in_vals[i];
    T.smem_off = -1;
    if (d.kind == DDQ_TERM_PROBE) {
      T.out_payload = d.out_payload;
      if (d.index) {
        T.direct = 1;
        T.bitmap = join_index_bitmap(const_cast<void*>(d.index));
        T.payarr = join_index_payload(const_cast<void*>(d.index), d.range);
        T.key_min = d.key_min;
        T.range = d.range;
        T.smem_words = (d.range + 31) / 32;
      } else {
        T.table = d.table;
        T.cap_mask = d.capacity - 1;
        int lg = 0;
        while ((1u << lg) < d.capacity) lg++;
        T.shift = 32 - lg;
        T.smem_words = d.capacity * 2;
      }
    }
  }
  const size_t budget = (size_t)g_star_optin - 2048;
  auto group_need = [&](int items, int stages) {
    const size_t tile = (size_t)ST_GT * items;
    return (size_t)stages * tile * row_bytes + tile * 4;  // ring + 2 uint16 lists
  };
  // Membership structures into shared memory in term order (the first term is
  // evaluated on every row; later ones only on survivors and may stay in L2), while
  // two groups of 3 stages of 1024-row tiles remain possible.
  size_t shared = 0;
  for (int j = 0; j < n_terms; j++) {
    StarTerm& T = p.terms[j];
    if (T.kind != DDQ_TERM_PROBE) continue;
    const size_t b = ((size_t)T.smem_words * 4 + 127) / 128 * 128;
    const bool first = j == 0;
    if (b <= 160 * 1024 && (shared + b + 2 * group_need(4, 3) <= budget || (first && shared + b + group_need(4, 2) <= budget))) {
      T.smem_off = (int32_t)shared;  // rebased below
      shared += b;
    }
  }
  // tile size, groups and stages: prefer 2048-row tiles if >= 2 groups of 3 stages fit
  int items = 8, G = 4, S = 4;
  auto fits = [&](int it, int gg, int ss) { return shared + (size_t)gg * group_need(it, ss) <= budget; };
  while (G > 1 && !fits(8, G, 3)) G--;
  if (G < 2) {
    items = 4;
    G = 4;
    while (G > 1 && !fits(4, G, 3)) G--;
  }
  S = 4;
  while (S > 2 && !fits(items, G, S)) S--;
  if (!fits(items, G, S)) return cudaErrorInvalidConfiguration;
  p.tile = ST_GT * items;
  for (int j = 0; j < n_terms; j++) p.terms[j].col_off *= p.tile;
  p.stage_bytes = p.tile * row_bytes;
  p.stages = S;
  p.list_off = S * p.stage_bytes;
  p.group_bytes = (int32_t)((group_need(items, S) + 127) / 128 * 128);
  const int32_t shared_base = G * p.group_bytes;
  for (int j = 0; j < n_terms; j++)
    if (p.terms[j].smem_off >= 0) p.terms[j].smem_off += shared_base;
  p.out_tids = out_tids;
  p.d_out_count = d_out_count;
  p.out_cap = (uint32_t)(out_cap > 0 ? out_cap : n_rows);
  p.d_overflow = d_overflow;
  cudaError_t e = init_fill(d_out_count, 8, 0, st);
  if (e != cudaSuccess) return e;
  const size_t smem = (size_t)shared_base + shared;
  const int64_t ntiles = (n_rows + p.tile - 1) / p.tile;
  int64_t grid = num_sms();
  const int64_t need_ctas = (ntiles + G - 1) / G;
  if (grid > need_ctas) grid = need_ctas < 1 ? 1 : need_ctas;
  if (items == 8) star_launch_g<8>(G, grid, smem, st, p);
  else star_launch_g<4>(G, grid, smem, st, p);
  return cudaGetLastError();
}

}  // namespace ddq
