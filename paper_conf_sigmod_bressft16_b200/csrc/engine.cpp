// engine.cpp -- libddq database: column store, device column cache (Algorithm 1),
// heap-budget allocator, GPU operator runner, finalisation and prepared
// (CUDA-graph) plans.  Citations: P:n = PAPER.md line n.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <unordered_set>

#include "engine.h"
#include "ops_internal.h"

namespace ddq {

uint64_t now_ns() {
  return (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
             std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

int64_t pow2_at_least(int64_t x) {
  int64_t p = 1;
  while (p < x) p <<= 1;
  return p;
}

// ---------------------------------------------------------------- heap
// The rest of device memory after the cache is the heap for intermediates.
// Allocation never waits: it fails immediately so the operator can abort and be
// restarted elsewhere ("CoGaDB aborts operators immediately if an
// allocation fails").
static constexpr uint64_t kAlign = 256;

ddq_status Heap::init(uint64_t bytes, uint32_t fault_every) {
  cap_ = (bytes + kAlign - 1) / kAlign * kAlign;
  fault_every_ = fault_every;
  if (cap_ == 0) return DDQ_OK;
  cudaError_t e = cudaMalloc(&base_, cap_);
  if (e != cudaSuccess) return cuda_status(e, "heap cudaMalloc");
  free_[0] = cap_;
  return DDQ_OK;
}

Heap::~Heap() {
  if (base_) cudaFree(base_);
}

void* Heap::try_alloc(uint64_t bytes) {
  std::lock_guard<std::mutex> g(mu_);
  n_allocs_++;
  if (fault_every_ && n_allocs_ % fault_every_ == 0) return nullptr;  // fault injection
  uint64_t need = std::max<uint64_t>(kAlign, (bytes + kAlign - 1) / kAlign * kAlign);
  for (auto it = free_.begin(); it != free_.end(); ++it) {
    if (it->second < need) continue;
    uint64_t off = it->first, sz = it->second;
    free_.erase(it);
    if (sz > need) free_[off + need] = sz - need;
    alloc_[off] = need;
    used_ += need;
    peak_ = std::max(peak_, used_);
    return base_ + off;
  }
  return nullptr;
}

void Heap::free(void* p) {
  if (!p) return;
  std::lock_guard<std::mutex> g(mu_);
  uint64_t off = (uint64_t)((char*)p - base_);
  auto it = alloc_.find(off);
  if (it == alloc_.end()) return;
  uint64_t sz = it->second;
  alloc_.erase(it);
  used_ -= sz;
  auto nx = free_.lower_bound(off);
  if (nx != free_.end() && nx->first == off + sz) {
    sz += nx->second;
    nx = free_.erase(nx);
  }
  if (nx != free_.begin()) {
    auto pv = std::prev(nx);
    if (pv->first + pv->second == off) {
      pv->second += sz;
      return;
    }
  }
  free_[off] = sz;
}

const Column* col_of(ddq_db* db, int c) {
  if (c < 0 || c >= (int)db->cols.size()) return nullptr;
  return db->cols[(size_t)c].get();
}

void release_inter(ddq_db* db, Inter& x) {
  for (void* p : x.heap_blocks) db->heap.free(p);
  for (void* p : x.host_blocks) std::free(p);
  x.heap_blocks.clear();
  x.host_blocks.clear();
}

// A dimension key column whose values span a compact range gets a direct-mapped
// join index (bitmap + payload array) instead of a hash table: one probe per row,
// no collision chains.  Range <= 2^20 or <= 16 x the rows (primary keys 1..n).
bool use_join_index(const Column& kc, int64_t n_rows) {
  if (kc.vmax < kc.vmin) return false;
  const int64_t r = kc.vmax - kc.vmin + 1;
  return r <= (1ll << 28) && (r <= (1ll << 20) || r <= 16 * std::max<int64_t>(n_rows, 1));
}

// Input rows up to which an AGGREGATE evaluates its probe terms row by row (reading
// O37); about two waves of the warp-autonomous aggregation (148 SMs x 16 warps x
// 256-row tiles x 2 = 1.2 M rows on B200).  Longer inputs evaluate them term by term.
// The largest |value| one row can add to an aggregate of op, from the argument
// columns' load-time value ranges (include/ddq.h's expression set); -1 if unknown.
double max_row_abs(ddq_db* db, const ddq_op& op) {
  auto mx = [&](int c, long double off, long double sgn, long double* out) {
    const Column* col = col_of(db, c);
    if (!col || col->n <= 0 || col->vmax < col->vmin) return false;
    const long double a = fabsl(off + sgn * (long double)col->vmin), b = fabsl(off + sgn * (long double)col->vmax);
    *out = a > b ? a : b;
    return true;
  };
  long double best = 0;
  for (int a = 0; a < op.n_aggs; a++) {
    long double x = 1, y = 1, z = 1;
    switch (op.agg_kind[a]) {
      case DDQ_AGG_COUNT: break;
      case DDQ_AGG_SUM: if (!mx(op.agg_col[a][0], 0, 1, &x)) return -1; break;
      case DDQ_AGG_SUM_MUL:
        if (!mx(op.agg_col[a][0], 0, 1, &x) || !mx(op.agg_col[a][1], 0, 1, &y)) return -1;
        break;
      case DDQ_AGG_SUM_SUB:
        if (!mx(op.agg_col[a][0], 0, 1, &x) || !mx(op.agg_col[a][1], 0, 1, &y)) return -1;
        x += y;
        y = 1;
        break;
      case DDQ_AGG_SUM_MUL_100M:
        if (!mx(op.agg_col[a][0], 0, 1, &x) || !mx(op.agg_col[a][1], 100, -1, &y)) return -1;
        break;
      case DDQ_AGG_SUM_MUL_100M_100P:
        if (!mx(op.agg_col[a][0], 0, 1, &x) || !mx(op.agg_col[a][1], 100, -1, &y) ||
            !mx(op.agg_col[a][2], 100, 1, &z))
          return -1;
        break;
      default: return -1;
    }
    const long double v = x * y * z;
    if (v > best) best = v;
  }
  return (double)best;
}

int64_t fused_tail_max_rows() {
  if (const char* e = getenv("DDQ_FUSED_TAIL_MAX")) return (int64_t)strtoll(e, nullptr, 10);  // tests / A-B
  return (int64_t)num_sms() * 16 * 256 * 2;
}

// An int64 column whose load-time range fits int32 (exact narrowing) or an int32 column.
bool fits_int32(const Column& c) {
  return c.width == 4 || c.n == 0 || (c.vmin >= INT32_MIN && c.vmax <= INT32_MAX);
}

// ----------------------------------------------------------- GPU operator runner
struct Alloc {
  ddq_db* db;
  Inter* out;
  const std::vector<void*>* reuse = nullptr;  // replay: hand back these blocks in order
  size_t next = 0;
  bool failed = false;
  void* get(uint64_t bytes) {
    if (failed) return nullptr;
    if (reuse) {
      if (next >= reuse->size()) {
        failed = true;
        return nullptr;
      }
      void* p = (*reuse)[next++];
      out->heap_blocks.push_back(p);
      return p;
    }
    void* p = db->heap.try_alloc(bytes);
    if (!p) {
      failed = true;
      return nullptr;
    }
    out->heap_blocks.push_back(p);
    return p;
  }
};

static const void* dev_col(ddq_db* db, int c, bool count_access) {
  const Column* col = col_of(db, c);
  if (!col) return nullptr;
  if (count_access) {
    db->cols[(size_t)c]->access++;
    db->cols[(size_t)c]->last_access = ++db->clock;
  }
  return col->dev;
}

ddq_status run_gpu_op(GpuOpCtx& ctx, const ddq_op& op, Inter& out) {
  ddq_db* db = ctx.db;
  const std::vector<Inter>& I = *ctx.inters;
  cudaStream_t st = ctx.stream;
  const bool acc = ctx.count_column_access;
  Alloc A{db, &out};
  A.reuse = ctx.reuse;
  out = Inter();
  out.table = op.table;
  if (op.table < 0 || op.table >= (int)db->tables.size()) return set_error(DDQ_EINVAL, "op: bad table");
  const Table& T = db->tables[(size_t)op.table];
  const Inter* in = op.input >= 0 ? &I[(size_t)op.input] : nullptr;
  if (in && in->on_host) return set_error(DDQ_ESTATE, "GPU op with a host-resident input");
  if (in && in->bits && op.kind != DDQ_OP_SELECT && op.kind != DDQ_OP_HASH_PROBE)
    return set_error(DDQ_ESTATE, "op cannot read a row-bitmap input");
  const int32_t* in_tids = in ? in->tids : nullptr;
  const uint32_t* in_cnt = in ? in->d_count : nullptr;
  const int64_t in_cap = in ? in->cap : T.n_rows;
  const int64_t out_cap = ctx.forced_cap >= 0 ? std::min<int64_t>(ctx.forced_cap, in_cap) : in_cap;
  auto need_col = [&](int c) -> const void* {
    const void* p = dev_col(db, c, acc);
    return p;
  };
  switch (op.kind) {
    case DDQ_OP_SELECT:
    case DDQ_OP_FILTER_EQ:
    case DDQ_OP_HASH_PROBE: {
      const bool probe = op.kind == DDQ_OP_HASH_PROBE;
      ddq_dev_pred dp[DDQ_MAX_PREDS];
      std::memset(dp, 0, sizeof(dp));
      const int32_t* eq_a = nullptr;
      const int32_t* eq_b = nullptr;
      if (op.kind == DDQ_OP_FILTER_EQ) {
        if (!in) return set_error(DDQ_EINVAL, "filter_eq needs an input with aligned vectors");
        const int a = op.eq_vec[0] - 1, b = op.eq_vec[1] - 1;
        if (a < 0 || b < 0 || a >= (int)in->vecs.size() || b >= (int)in->vecs.size() ||
            in->vecs[(size_t)a].width != 4 || in->vecs[(size_t)b].width != 4)
          return set_error(DDQ_EINVAL, "filter_eq: bad vector indexes");
        eq_a = (const int32_t*)in->vecs[(size_t)a].ptr;
        eq_b = (const int32_t*)in->vecs[(size_t)b].ptr;
        if (op.eq_cmp < DDQ_CMP_EQ || op.eq_cmp > DDQ_CMP_NE) return set_error(DDQ_EINVAL, "filter_eq: bad eq_cmp");
      } else if (!probe) {
        if (op.n_preds < 0 || op.n_preds > DDQ_MAX_PREDS) return set_error(DDQ_EINVAL, "select: bad n_preds");
        for (int i = 0; i < op.n_preds; i++) {
          const ddq_pred& p = op.preds[i];
          const Column* c = col_of(db, p.column);
          if (!c || c->table != op.table) return set_error(DDQ_EINVAL, "select: predicate column not in table");
          dp[i].col = need_col(p.column);
          if (!dp[i].col) return set_error(DDQ_ESTATE, "select: column not cached on the GPU");
          dp[i].width = c->width;
          dp[i].kind = p.kind;
          dp[i].lo = p.lo;
          dp[i].hi = p.hi;
          dp[i].n_in = p.n_in;
          for (int j = 0; j < DDQ_MAX_IN; j++) dp[i].in_vals[j] = p.in_vals[j];
        }
      }
      const Inter* build = nullptr;
      const int32_t* fk = nullptr;
      if (probe) {
        if (op.build < 0 || op.build >= (int)I.size()) return set_error(DDQ_EINVAL, "probe: bad build index");
        build = &I[(size_t)op.build];
        if (!build->table_ptr && !build->jidx)
          return set_error(DDQ_ESTATE, "probe: build side is not a device hash table / join index");
        if (op.fk_vec > 0) {  // probe keys from an aligned vector of the input
          if (!in || op.fk_vec - 1 >= (int)in->vecs.size() || in->vecs[(size_t)op.fk_vec - 1].width != 4)
            return set_error(DDQ_EINVAL, "probe: bad fk vector");
          fk = (const int32_t*)in->vecs[(size_t)op.fk_vec - 1].ptr;
        } else {
          const Column* c = col_of(db, op.fk_col);
          if (!c || c->table != op.table || c->width != 4) return set_error(DDQ_EINVAL, "probe: bad fk column");
          fk = (const int32_t*)need_col(op.fk_col);
          if (!fk) return set_error(DDQ_ESTATE, "probe: fk column not cached on the GPU");
        }
      }
      // carried vectors (int32 only; int64 vectors are re-gathered by consumers)
      std::vector<const int32_t*> cin;
      std::vector<int32_t*> cout;
      if (in) {
        if (in->vecs.size() > DDQ_MAX_CARRY) return set_error(DDQ_EINVAL, "too many aligned vectors");
        for (const Vec& v : in->vecs) {
          if (v.width != 4) return set_error(DDQ_EINVAL, "only int32 vectors can be carried");
          cin.push_back((const int32_t*)v.ptr);
        }
      }
      // a row-bitmap output (O27): a dense semi-join probe, or a dense selection on one
      // int32 column (ws_kernel streams it; ddq_prepare decides, see bits_out)
      const bool obits = ctx.bits_out && !in && ((probe && !op.emit_payload) || (!probe && op.n_preds == 1));
      out.cap = obits ? T.n_rows : out_cap;
      if (obits) out.bits = (uint32_t*)A.get(row_bitmap_bytes(T.n_rows));
      else out.tids = (int32_t*)A.get((uint64_t)std::max<int64_t>(out_cap, 1) * 4);
      out.d_count = (uint32_t*)A.get(64);
      for (size_t c = 0; c < cin.size(); c++) {
        int32_t* p = (int32_t*)A.get((uint64_t)std::max<int64_t>(out_cap, 1) * 4);
        cout.push_back(p);
        out.vecs.push_back(Vec{p, 4, false});
      }
      int32_t* payload = nullptr;
      if (probe && op.emit_payload) {
        payload = (int32_t*)A.get((uint64_t)std::max<int64_t>(out_cap, 1) * 4);
        out.vecs.push_back(Vec{payload, 4, false});
      }
      size_t sb = filter_scratch_bytes(in_cap);
      void* scratch = A.get(sb);
      if (A.failed) return DDQ_ENOMEM_DEVICE;
      FilterArgs fa;
      fa.preds = dp;
      fa.n_preds = probe ? 0 : op.n_preds;
      fa.probe = probe;
      if (probe) {
        fa.table = build->table_ptr;
        fa.capacity = build->table_cap;
        if (build->jidx) {
          fa.bitmap = join_index_bitmap(build->jidx);
          fa.payarr = join_index_payload(build->jidx, build->jrange);
          fa.coarse = join_index_coarse(build->jidx, build->jrange);
          fa.key_min = build->jmin;
          fa.range = build->jrange;
        }
        fa.fk = fk;
        fa.fk_by_pos = op.fk_vec > 0;
        fa.out_payload = payload;
      }
      fa.eq_a = eq_a;
      fa.eq_b = eq_b;
      fa.eq_cmp = op.kind == DDQ_OP_FILTER_EQ ? op.eq_cmp : DDQ_CMP_EQ;
      fa.in_tids = in_tids;
      fa.d_in_count = in_cnt;
      fa.n_cap = in_cap;
      if (in && in->bits) {  // row bitmap input: every row of the table, masked
        fa.in_bits = in->bits;
        fa.in_tids = nullptr;
        fa.d_in_count = nullptr;
        fa.n_cap = T.n_rows;
      }
      if (obits) fa.out_bits = out.bits;
      fa.carry_in = cin.data();
      fa.carry_out = cout.data();
      fa.n_carry = (int)cin.size();
      fa.out_tids = out.tids;
      fa.d_out_count = out.d_count;
      fa.out_cap = out_cap;
      fa.d_overflow = ctx.forced_cap >= 0 && in && in->d_error ? in->d_error : nullptr;
      fa.scratch = scratch;
      // error cell propagates down the chain so a prepared plan can detect overflow
      // (its intermediates all live until ddq_prepared_free); in the chopping driver
      // an op's inputs are released as soon as their consumers are done, so every op
      // owns its cell there (a shared cell in a freed block was overwritten by a later
      // allocation: TPC-H Q2 on sparse keys)
      out.d_error = in && ctx.forced_cap >= 0 ? in->d_error : nullptr;
      if (!out.d_error) {
        out.d_error = (uint32_t*)A.get(64);
        if (A.failed) return DDQ_ENOMEM_DEVICE;
        init_fill(out.d_error, 4, 0, st);
      }
      fa.d_overflow = out.d_error;
      return cuda_status(launch_filter(fa, st), probe ? "probe" : "select");
    }
    case DDQ_OP_STAR: {
      if (in) return set_error(DDQ_EINVAL, "star: input must be all rows");
      if (op.n_terms < 1 || op.n_terms > 4) return set_error(DDQ_EINVAL, "star: 1..4 terms");
      ddq_dev_term terms[4];
      std::memset(terms, 0, sizeof(terms));
      out.cap = out_cap;
      out.tids = (int32_t*)A.get((uint64_t)std::max<int64_t>(out_cap, 1) * 4);
      out.d_count = (uint32_t*)A.get(64);
      for (int j = 0; j < op.n_terms; j++) {
        ddq_dev_term& d = terms[j];
        d.kind = op.term_kind[j];
        if (d.kind == DDQ_TERM_PRED) {
          const ddq_pred& p = op.preds[j];
          const Column* c = col_of(db, p.column);
          if (!c || c->table != op.table) return set_error(DDQ_EINVAL, "star: predicate column not in table");
          d.col = need_col(p.column);
          d.width = c->width;
          d.pred_kind = p.kind;
          d.lo = p.lo;
          d.hi = p.hi;
          d.n_in = p.n_in;
          for (int i = 0; i < DDQ_MAX_IN; i++) d.in_vals[i] = p.in_vals[i];
        } else if (d.kind == DDQ_TERM_PROBE) {
          const int b = op.term_build[j];
          if (b < 0 || b >= (int)I.size()) return set_error(DDQ_EINVAL, "star: bad build index");
          const Inter& B = I[(size_t)b];
          if (!B.table_ptr && !B.jidx) return set_error(DDQ_ESTATE, "star: build side is not on the device");
          const Column* c = col_of(db, op.term_fk[j]);
          if (!c || c->table != op.table || c->width != 4) return set_error(DDQ_EINVAL, "star: bad fk column");
          d.col = need_col(op.term_fk[j]);
          d.width = 4;
          if (B.jidx) {
            d.index = B.jidx;
            d.key_min = B.jmin;
            d.range = B.jrange;
          } else {
            d.table = B.table_ptr;
            d.capacity = B.table_cap;
          }
          if (op.term_emit[j]) {
            d.out_payload = (int32_t*)A.get((uint64_t)std::max<int64_t>(out_cap, 1) * 4);
            out.vecs.push_back(Vec{d.out_payload, 4, false});
          }
        } else {
          return set_error(DDQ_EINVAL, "star: bad term kind");
        }
        if (!d.col) return set_error(DDQ_ESTATE, "star: column not cached on the GPU");
      }
      out.d_error = (uint32_t*)A.get(64);
      if (A.failed) return DDQ_ENOMEM_DEVICE;
      init_fill(out.d_error, 4, 0, st);
      return cuda_status(launch_star(terms, op.n_terms, T.n_rows, out.tids, out.d_count, out_cap, out.d_error, st),
                         "star");
    }
    case DDQ_OP_HASH_BUILD: {
      const Column* kc = col_of(db, op.key_col);
      if (!kc || kc->table != op.table || kc->width != 4) return set_error(DDQ_EINVAL, "build: bad key column");
      const int32_t* keys = (const int32_t*)need_col(op.key_col);
      const int32_t* payload = nullptr;
      const long long* payload64 = nullptr;
      if (op.payload_col >= 0) {
        const Column* pc = col_of(db, op.payload_col);
        if (!pc || pc->table != op.table || !fits_int32(*pc)) return set_error(DDQ_EINVAL, "build: bad payload column");
        const void* pp = need_col(op.payload_col);
        if (!pp) return set_error(DDQ_ESTATE, "build: payload column not cached on the GPU");
        if (pc->width == 8) payload64 = (const long long*)pp;
        else payload = (const int32_t*)pp;
      }
      if (op.build_key_set < 0 || op.build_key_set > 2) return set_error(DDQ_EINVAL, "build: bad build_key_set");
      if (!keys) return set_error(DDQ_ESTATE, "build: key column not cached on the GPU");
      // fused selection (BUILD op with predicates): evaluated per input row in the
      // build kernel
      if (op.n_preds < 0 || op.n_preds > DDQ_MAX_PREDS) return set_error(DDQ_EINVAL, "build: bad n_preds");
      BuildPreds bp;
      bp.n = op.n_preds;
      bp.key_set = op.build_key_set;
      bp.payload64 = payload64;
      for (int i = 0; i < op.n_preds; i++) {
        const ddq_pred& p = op.preds[i];
        const Column* c = col_of(db, p.column);
        if (!c || c->table != op.table) return set_error(DDQ_EINVAL, "build: predicate column not in table");
        ddq_dev_pred& d = bp.p[i];
        std::memset(&d, 0, sizeof(d));
        d.col = need_col(p.column);
        if (!d.col) return set_error(DDQ_ESTATE, "build: predicate column not cached on the GPU");
        d.width = c->width;
        d.kind = p.kind;
        d.lo = p.lo;
        d.hi = p.hi;
        d.n_in = p.n_in;
        for (int j = 0; j < DDQ_MAX_IN; j++) d.in_vals[j] = p.in_vals[j];
      }
      if (use_join_index(*kc, T.n_rows)) {  // compact key range: direct-mapped join index
        out.jmin = (int32_t)kc->vmin;
        out.jrange = (uint32_t)(kc->vmax - kc->vmin + 1);
        out.jidx = A.get(join_index_bytes(out.jrange));
        out.d_error = (uint32_t*)A.get(64);
        out.cap = 0;
        if (A.failed) return DDQ_ENOMEM_DEVICE;
        init_fill(out.d_error, 4, 0, st);
        const bool recv = ctx.dist && dist_build_receives(db, op);  // built once, on rank 0 (S8(e))
        cudaError_t e = recv ? cudaSuccess : join_index_init(out.jidx, out.jrange, st);
        if (e == cudaSuccess && op.build_key_set == 2 && !recv)  // MIN build: payloads start at INT32_MAX
          e = init_fill(join_index_payload(out.jidx, out.jrange), (size_t)out.jrange * 4, 0x7FFFFFFF7FFFFFFFull, st);
        if (e == cudaSuccess && !recv)
          e = launch_join_index_build(keys, payload, in_tids, in_cnt, in_cap, out.jmin, out.jrange, out.jidx,
                                      out.d_error, st, &bp);
        if (e == cudaSuccess && ctx.dist)
          return dist_build_broadcast(db, op, out.jidx, join_index_bytes(out.jrange), st);
        return cuda_status(e, "join_index_build");
      }
      // sparse keys: open addressing; small tables (shared-memory resident) get load <= 0.25
      int64_t cap = pow2_at_least(std::max<int64_t>(16, 2 * out_cap));
      if (cap * 2 * 8 <= 64 * 1024) cap *= 2;
      if (cap > (1ll << 31)) return set_error(DDQ_EINVAL, "build: table too large");
      out.table_cap = (uint32_t)cap;
      out.table_ptr = (uint64_t*)A.get((uint64_t)cap * 8);
      out.d_error = (uint32_t*)A.get(64);
      out.cap = 0;
      if (A.failed) return DDQ_ENOMEM_DEVICE;
      init_fill(out.d_error, 4, 0, st);
      const bool recv = ctx.dist && dist_build_receives(db, op);  // built once, on rank 0 (S8(e))
      cudaError_t e = recv ? cudaSuccess : launch_hash_init(out.table_ptr, out.table_cap, st);
      if (e == cudaSuccess && !recv)
        e = launch_hash_build(keys, payload, in_tids, in_cnt, in_cap, out.table_ptr, out.table_cap, out.d_error, st,
                              &bp);
      if (e == cudaSuccess && ctx.dist)
        return dist_build_broadcast(db, op, out.table_ptr, (size_t)out.table_cap * 8, st);
      return cuda_status(e, "hash_build");
    }
    case DDQ_OP_GATHER: {
      const Column* c = col_of(db, op.gather_col);
      if (!c || c->table != op.table) return set_error(DDQ_EINVAL, "gather: bad column");
      if (!in) return set_error(DDQ_EINVAL, "gather needs an input TID list");
      const void* src = need_col(op.gather_col);
      if (!src) return set_error(DDQ_ESTATE, "gather: column not cached on the GPU");
      // pass-through of the input's TIDs and vectors (no copy), plus the new vector
      out.tids = in->tids;
      out.d_count = in->d_count;
      out.cap = in->cap;
      out.vecs = in->vecs;
      out.d_error = in->d_error;
      if (op.fetch_build > 0) {  // dimension attribute fetch through the build's index
        const int b = op.fetch_build - 1;
        if (b >= (int)I.size() || c->width != 4) return set_error(DDQ_EINVAL, "fetch: bad build / fk column");
        const Inter& B = I[(size_t)b];
        if (!B.table_ptr && !B.jidx) return set_error(DDQ_ESTATE, "fetch: build side is not on the device");
        if (!in->d_count) return set_error(DDQ_ESTATE, "fetch: input without a device count");
        int32_t* dst = (int32_t*)A.get((uint64_t)std::max<int64_t>(in->cap, 1) * 4);
        if (A.failed) return DDQ_ENOMEM_DEVICE;
        out.vecs.push_back(Vec{dst, 4, false});
        return cuda_status(launch_fetch(in->tids, in->d_count, in->cap, (const int32_t*)src,
                                        B.jidx ? join_index_bitmap(B.jidx) : nullptr,
                                        B.jidx ? join_index_payload(B.jidx, B.jrange) : nullptr, B.jmin, B.jrange,
                                        B.table_ptr, B.table_cap, dst, st),
                           "fetch");
      }
      if (op.gather_narrow && (c->width != 8 || !fits_int32(*c)))
        return set_error(DDQ_EINVAL, "gather: narrowing needs an int64 column whose values fit int32");
      const int w = op.gather_narrow ? 4 : c->width;
      void* dst = A.get((uint64_t)std::max<int64_t>(in->cap, 1) * w);
      if (A.failed) return DDQ_ENOMEM_DEVICE;
      out.vecs.push_back(Vec{dst, w, false});
      return cuda_status(launch_gather(src, op.gather_narrow ? -8 : c->width, in->tids, in->d_count, in->cap, dst, st),
                         "gather");
    }
    case DDQ_OP_AGGREGATE: {
      // no input: every row of op.table (a dense aggregation, e.g. TPC-H Q1 with
      // its selection fused, O26); keys must then be columns
      if (op.n_keys < 0 || op.n_keys > DDQ_MAX_KEYS || op.n_aggs < 1 || op.n_aggs > DDQ_MAX_AGGS)
        return set_error(DDQ_EINVAL, "aggregate: bad key/agg counts");
      const int32_t* kv[3] = {nullptr, nullptr, nullptr};
      const int32_t* kc[3] = {nullptr, nullptr, nullptr};
      // fused probe / fetch terms (reading O37): their emitted payloads follow the
      // input's vectors; a key naming one reads payload slot key_pay
      AggTerms terms;
      const int n_in_vecs = in ? (int)in->vecs.size() : 0;
      if (op.n_terms > 0) {
        if (!in) return set_error(DDQ_EINVAL, "aggregate: terms need an input TID list");
        terms.n = op.n_terms;
        int slot = 0;
        for (int j = 0; j < op.n_terms; j++) {
          const int b = op.term_build[j];
          if (b < 0 || b >= (int)I.size()) return set_error(DDQ_EINVAL, "aggregate: bad term build");
          const Inter& B = I[(size_t)b];
          if (!B.table_ptr && !B.jidx) return set_error(DDQ_ESTATE, "aggregate: term build is not on the device");
          const Column* c = col_of(db, op.term_fk[j]);
          if (!c || c->table != op.table || c->width != 4) return set_error(DDQ_EINVAL, "aggregate: bad term fk column");
          AggTerm& t = terms.t[j];
          t.kind = op.term_kind[j];
          t.fk = (const int32_t*)need_col(op.term_fk[j]);
          if (!t.fk) return set_error(DDQ_ESTATE, "aggregate: term fk column not cached on the GPU");
          const bool emits = op.term_kind[j] == DDQ_TERM_FETCH || op.term_emit[j];
          if (emits && slot >= 3) return set_error(DDQ_EINVAL, "aggregate: at most 3 emitting terms");
          t.emit = emits ? slot++ : -1;
          if (B.jidx) {
            t.bitmap = join_index_bitmap(B.jidx);
            t.payarr = join_index_payload(B.jidx, B.jrange);
            t.key_min = B.jmin;
            t.range = B.jrange;
          } else {
            t.table = B.table_ptr;
            t.capacity = B.table_cap;
          }
        }
      }
      for (int k = 0; k < op.n_keys; k++) {
        int src = op.key_src[k];
        if (src >= n_in_vecs && op.n_terms > 0) {  // an emitted payload of a term
          int e = src - n_in_vecs, slot = -1;
          for (int j = 0; j < op.n_terms; j++)
            if (terms.t[j].emit >= 0 && e-- == 0) slot = terms.t[j].emit;
          if (slot < 0) return set_error(DDQ_EINVAL, "aggregate: key names a term that emits nothing");
          terms.key_pay[k] = slot;
          kv[k] = nullptr;
          continue;
        }
        if (src >= 0) {
          if (!in || src >= (int)in->vecs.size() || in->vecs[(size_t)src].width != 4)
            return set_error(DDQ_EINVAL, "aggregate: bad key vector");
          kv[k] = (const int32_t*)in->vecs[(size_t)src].ptr;
        } else {
          const Column* c = col_of(db, -2 - src);
          if (!c || c->table != op.table || c->width != 4) return set_error(DDQ_EINVAL, "aggregate: bad key column");
          kc[k] = (const int32_t*)need_col(-2 - src);
          if (!kc[k]) return set_error(DDQ_ESTATE, "aggregate: key column not cached");
        }
      }
      ddq_dev_agg ag[DDQ_MAX_AGGS];
      std::memset(ag, 0, sizeof(ag));
      bool has_min = false;  // MIN: the generic global-table kernel (launch_groupby)
      for (int a = 0; a < op.n_aggs; a++) {
        ag[a].kind = op.agg_kind[a];
        if (op.agg_kind[a] < DDQ_AGG_COUNT || op.agg_kind[a] > DDQ_AGG_MIN)
          return set_error(DDQ_EINVAL, "aggregate: bad aggregate kind");
        has_min |= op.agg_kind[a] == DDQ_AGG_MIN;
        int need = op.agg_kind[a] == DDQ_AGG_COUNT ? 0 : (op.agg_kind[a] == DDQ_AGG_SUM || op.agg_kind[a] == DDQ_AGG_MIN) ? 1
                 : op.agg_kind[a] == DDQ_AGG_SUM_MUL_100M_100P ? 3 : 2;
        for (int j = 0; j < need; j++) {
          if (op.agg_col[a][j] <= -2) {  // MIN over an aligned vector: positional (negative width)
            const int v = -2 - op.agg_col[a][j];
            if (op.agg_kind[a] != DDQ_AGG_MIN || !in || op.n_preds > 0 || v >= (int)in->vecs.size())
              return set_error(DDQ_EINVAL, "aggregate: a vector operand needs MIN, an input and no fused predicates");
            ag[a].arg[j] = in->vecs[(size_t)v].ptr;
            ag[a].width[j] = -in->vecs[(size_t)v].width;
            continue;
          }
          const Column* c = col_of(db, op.agg_col[a][j]);
          if (!c || c->table != op.table) return set_error(DDQ_EINVAL, "aggregate: bad argument column");
          ag[a].arg[j] = need_col(op.agg_col[a][j]);
          ag[a].width[j] = c->width;
          if (!ag[a].arg[j]) return set_error(DDQ_ESTATE, "aggregate: argument column not cached");
        }
      }
      const int64_t in_cap = in ? in->cap : db->tables[(size_t)op.table].n_rows;
      int64_t groups = op.max_groups > 0 ? std::min<int64_t>(op.max_groups, std::max<int64_t>(in_cap, 1))
                                         : std::max<int64_t>(in_cap, 1);
      int64_t cap = pow2_at_least(std::max<int64_t>(64, 2 * groups));
      if (cap > (1ll << 31)) return set_error(DDQ_EINVAL, "aggregate: table too large");
      out.gb_cap = (uint32_t)cap;
      out.gb_table = A.get(groupby_table_bytes(out.gb_cap, op.n_aggs));
      out.gb_keys = (int64_t*)A.get((uint64_t)cap * 8);
      out.gb_accs = (int64_t*)A.get((uint64_t)cap * op.n_aggs * 16);
      out.gb_groups = (uint32_t*)A.get(64);
      out.d_error = in && ctx.forced_cap >= 0 ? in->d_error : nullptr;  // see the probe case
      if (!out.d_error) {
        out.d_error = (uint32_t*)A.get(64);
        if (!A.failed) init_fill(out.d_error, 4, 0, st);
      }
      if (A.failed) return DDQ_ENOMEM_DEVICE;
      // fused selection (reading O26): an AGGREGATE carrying predicates aggregates
      // only the input rows that pass them
      if (op.n_preds < 0 || op.n_preds > DDQ_MAX_PREDS) return set_error(DDQ_EINVAL, "aggregate: bad n_preds");
      BuildPreds bp;
      bp.n = op.n_preds;
      for (int i = 0; i < op.n_preds; i++) {
        const ddq_pred& p = op.preds[i];
        const Column* c = col_of(db, p.column);
        if (!c || c->table != op.table) return set_error(DDQ_EINVAL, "aggregate: predicate column not in table");
        ddq_dev_pred& d = bp.p[i];
        std::memset(&d, 0, sizeof(d));
        d.col = need_col(p.column);
        if (!d.col) return set_error(DDQ_ESTATE, "aggregate: predicate column not cached on the GPU");
        d.width = c->width;
        d.kind = p.kind;
        d.lo = p.lo;
        d.hi = p.hi;
        d.n_in = p.n_in;
        for (int j = 0; j < DDQ_MAX_IN; j++) d.in_vals[j] = p.in_vals[j];
      }
      if (op.n_terms > 0) {  // the fused tail (O37): the warp-autonomous aggregation only
        bool aligned = ((uintptr_t)in->tids & 15) == 0;
        for (int k = 0; k < op.n_keys; k++) aligned = aligned && (!kv[k] || ((uintptr_t)kv[k] & 15) == 0);
        if (has_min || op.n_aggs > 2 || out.gb_cap > 2048 || !aligned || !in->d_count)
          return set_error(DDQ_EINVAL, "aggregate: fused terms need <= 2 SUM/COUNT aggregates and <= 1024 groups");
        const int32_t* a_tids = in->tids;
        const uint32_t* a_count = in->d_count;
        const AggTerms* a_terms = &terms;
        if (in_cap > fused_tail_max_rows()) {
          // A long input: row-by-row terms would pay every term's gather latency for
          // every input tile while most rows are already dead.  The same operator
          // then evaluates its terms as the chain does -- one compacting probe (or
          // fetch) pass per term, survivors and payloads materialised -- and
          // aggregates the final rows (a physical algorithm choice).
          std::vector<const int32_t*> cv;
          for (const Vec& v : in->vecs) {
            if (v.width != 4) return set_error(DDQ_EINVAL, "aggregate: only int32 vectors can be carried");
            cv.push_back((const int32_t*)v.ptr);
          }
          const int64_t cap = in_cap;
          for (int j = 0; j < op.n_terms; j++) {
            const AggTerm& t = terms.t[j];
            if (t.kind == DDQ_TERM_FETCH) {
              int32_t* dst = (int32_t*)A.get((uint64_t)std::max<int64_t>(cap, 1) * 4);
              if (A.failed) return DDQ_ENOMEM_DEVICE;
              cudaError_t e0 = launch_fetch(a_tids, a_count, cap, t.fk, t.bitmap, t.payarr, t.key_min, t.range, t.table,
                                            t.capacity, dst, st);
              if (e0 != cudaSuccess) return cuda_status(e0, "aggregate: term fetch");
              cv.push_back(dst);
              continue;
            }
            if (cv.size() > DDQ_MAX_CARRY) return set_error(DDQ_EINVAL, "aggregate: too many aligned vectors");
            std::vector<int32_t*> co;
            int32_t* nt = (int32_t*)A.get((uint64_t)std::max<int64_t>(cap, 1) * 4);
            uint32_t* nc = (uint32_t*)A.get(64);
            for (size_t c = 0; c < cv.size(); c++) co.push_back((int32_t*)A.get((uint64_t)std::max<int64_t>(cap, 1) * 4));
            int32_t* pay = t.emit >= 0 ? (int32_t*)A.get((uint64_t)std::max<int64_t>(cap, 1) * 4) : nullptr;
            void* scr = A.get(filter_scratch_bytes(cap));
            if (A.failed) return DDQ_ENOMEM_DEVICE;
            FilterArgs fa;
            fa.probe = true;
            fa.table = t.table;
            fa.capacity = t.capacity;
            if (t.bitmap) {
              const Inter& B = I[(size_t)op.term_build[j]];
              fa.bitmap = t.bitmap;
              fa.payarr = t.payarr;
              fa.coarse = join_index_coarse(B.jidx, B.jrange);
              fa.key_min = t.key_min;
              fa.range = t.range;
            }
            fa.fk = t.fk;
            fa.out_payload = pay;
            fa.in_tids = a_tids;
            fa.d_in_count = a_count;
            fa.n_cap = cap;
            fa.carry_in = cv.data();
            fa.carry_out = co.data();
            fa.n_carry = (int)cv.size();
            fa.out_tids = nt;
            fa.d_out_count = nc;
            fa.out_cap = cap;
            fa.d_overflow = out.d_error;
            fa.scratch = scr;
            cudaError_t e0 = launch_filter(fa, st);
            if (e0 != cudaSuccess) return cuda_status(e0, "aggregate: term probe");
            a_tids = nt;
            a_count = nc;
            cv.assign(co.begin(), co.end());
            if (pay) cv.push_back(pay);
          }
          for (int k = 0; k < op.n_keys; k++) {  // keys: every vector is materialised now
            const int src = op.key_src[k];
            if (src >= 0) {
              if (src >= (int)cv.size()) return set_error(DDQ_EINVAL, "aggregate: bad key vector");
              kv[k] = cv[(size_t)src];
            }
          }
          a_terms = nullptr;
        }
        out.d_rows = (uint32_t*)A.get(64);
        if (A.failed) return DDQ_ENOMEM_DEVICE;
        init_fill(out.d_rows, 4, 0, st);
        cudaError_t e = launch_groupby_init(out.gb_table, out.gb_cap, op.n_aggs, st);
        if (e == cudaSuccess)
          e = launch_agg_ws(a_tids, a_count, in_cap, kv, kc, op.n_keys, op.key_bits, ag, op.n_aggs, out.gb_table,
                            out.gb_cap, out.d_error, st, &bp, out.d_rows, a_terms);
        if (e == cudaSuccess)
          e = launch_groupby_compact(out.gb_table, out.gb_cap, op.n_aggs, out.gb_keys, out.gb_accs, out.gb_groups, st);
        return cuda_status(e, "aggregate (fused terms)");
      }
      if (!in && !has_min && agg_dense_supported(in_cap, &bp, kc, op.n_keys, op.key_bits, ag, op.n_aggs)) {
        out.d_rows = (uint32_t*)A.get(64);
        if (A.failed) return DDQ_ENOMEM_DEVICE;
        init_fill(out.d_rows, 4, 0, st);
        cudaError_t e = launch_groupby_init(out.gb_table, out.gb_cap, op.n_aggs, st);
        if (e == cudaSuccess)
          e = launch_agg_dense(in_cap, kc, op.n_keys, op.key_bits, ag, op.n_aggs, out.gb_table, out.gb_cap,
                               out.d_error, st, &bp, out.d_rows, max_row_abs(db, op));
        if (e == cudaSuccess)
          e = launch_groupby_compact(out.gb_table, out.gb_cap, op.n_aggs, out.gb_keys, out.gb_accs, out.gb_groups, st);
        return cuda_status(e, "aggregate (dense)");
      }
      const int32_t* g_tids = in ? in->tids : nullptr;
      const uint32_t* g_count = in ? in->d_count : nullptr;
      if (!in && op.n_preds == 0) {  // other dense shapes: an all-rows TID list feeds the generic kernels
        int32_t* ft = (int32_t*)A.get((uint64_t)std::max<int64_t>(in_cap, 1) * 4);
        uint32_t* fc = (uint32_t*)A.get(64);
        if (A.failed) return DDQ_ENOMEM_DEVICE;
        cudaError_t e0 = launch_iota(ft, in_cap, fc, st);
        if (e0 != cudaSuccess) return cuda_status(e0, "aggregate: row list");
        g_tids = ft;
        g_count = fc;
      }
      if (op.n_preds > 0 && (has_min || !in || !agg_ws_supported(in->tids, kv, op.n_keys, op.n_aggs, out.gb_cap))) {
        // no fused kernel for this shape: a selection into a temporary TID list
        // (carrying the key vectors) feeds the aggregation
        int32_t* ft = (int32_t*)A.get((uint64_t)std::max<int64_t>(in_cap, 1) * 4);
        uint32_t* fc = (uint32_t*)A.get(64);
        void* fscr = A.get(filter_scratch_bytes(in_cap));
        const int32_t* cin[3] = {nullptr, nullptr, nullptr};
        int32_t* cout2[3] = {nullptr, nullptr, nullptr};
        int nc = 0;
        for (int k = 0; k < op.n_keys; k++)
          if (kv[k]) {
            cin[nc] = kv[k];
            cout2[nc] = (int32_t*)A.get((uint64_t)std::max<int64_t>(in_cap, 1) * 4);
            kv[k] = cout2[nc];
            nc++;
          }
        if (A.failed) return DDQ_ENOMEM_DEVICE;
        FilterArgs fa;
        fa.preds = bp.p;
        fa.n_preds = bp.n;
        fa.in_tids = in ? in->tids : nullptr;
        fa.d_in_count = in ? in->d_count : nullptr;
        fa.n_cap = in_cap;
        fa.carry_in = cin;
        fa.carry_out = cout2;
        fa.n_carry = nc;
        fa.out_tids = ft;
        fa.d_out_count = fc;
        fa.out_cap = in_cap;
        fa.d_overflow = out.d_error;
        fa.scratch = fscr;
        cudaError_t e0 = launch_filter(fa, st);
        if (e0 != cudaSuccess) return cuda_status(e0, "aggregate: fused selection");
        g_tids = ft;
        g_count = fc;
        bp.n = 0;
      }
      if (op.n_preds > 0 && bp.n > 0) {
        out.d_rows = (uint32_t*)A.get(64);
        if (A.failed) return DDQ_ENOMEM_DEVICE;
        init_fill(out.d_rows, 4, 0, st);
      }
      cudaError_t e = launch_groupby_init(out.gb_table, out.gb_cap, op.n_aggs, st);
      if (e == cudaSuccess) {
        if (bp.n > 0)
          e = launch_agg_ws(g_tids, g_count, in_cap, kv, kc, op.n_keys, op.key_bits, ag, op.n_aggs, out.gb_table,
                            out.gb_cap, out.d_error, st, &bp, out.d_rows);
        else
          e = launch_groupby(g_tids, g_count, in_cap, kv, kc, op.n_keys, op.key_bits, ag, op.n_aggs, out.gb_table,
                             out.gb_cap, out.d_error, st);
      }
      if (e == cudaSuccess)
        e = launch_groupby_compact(out.gb_table, out.gb_cap, op.n_aggs, out.gb_keys, out.gb_accs, out.gb_groups, st);
      return cuda_status(e, "aggregate");
    }
  }
  return set_error(DDQ_EINVAL, "unknown operator kind");
}

// ------------------------------------------------------------ finalisation
// S8(a7): decode the packed group key, ORDER BY (order-preserving codes, O4; the
// O8 tie-break = remaining keys ascending is encoded in the plan), LIMIT.
static inline __int128 acc128(const int64_t* accs, int64_t g, int n_aggs, int a) {
  unsigned __int128 lo = (uint64_t)accs[(g * n_aggs + a) * 2];
  __int128 hi = (__int128)accs[(g * n_aggs + a) * 2 + 1];
  return (__int128)((unsigned __int128)(hi << 64) | lo);
}

static ddq_status finalize_unique(const ddq_op& root, int64_t n_groups, const int64_t* keys, const int64_t* accs,
                                  ddq_result** out);

// Merge equal packed keys (partials of several shards, S8(e)) per aggregate kind:
// SUM / COUNT kinds by exact int128 addition, MIN by taking the smaller value (the
// merge of per-shard minima is the minimum); then finalise.
ddq_status finalize_result(const ddq_op& root, int64_t n_groups, const int64_t* keys, const int64_t* accs,
                           ddq_result** out, bool unique_keys) {
  const int na = root.n_aggs;
  bool dup = false;  // one device group table has unique keys; shards' partials may repeat them
  if (!unique_keys) {
    std::unordered_set<int64_t> seen;
    seen.reserve((size_t)n_groups * 2);
    for (int64_t i = 0; i < n_groups && !dup; i++) dup = !seen.insert(keys[i]).second;
  }
  if (!dup) return finalize_unique(root, n_groups, keys, accs, out);
  std::vector<int64_t> idx((size_t)n_groups);
  std::iota(idx.begin(), idx.end(), 0);
  std::sort(idx.begin(), idx.end(), [&](int64_t a, int64_t b) { return keys[a] < keys[b]; });
  std::vector<int64_t> mk, ma;
  for (size_t i = 0; i < idx.size(); i++) {
    const int64_t g = idx[i];
    if (i == 0 || keys[g] != mk.back()) {
      mk.push_back(keys[g]);
      for (int a = 0; a < na; a++) {
        ma.push_back(accs[(g * na + a) * 2]);
        ma.push_back(accs[(g * na + a) * 2 + 1]);
      }
    } else {
      const size_t m = mk.size() - 1;
      for (int a = 0; a < na; a++) {
        __int128 x = acc128(ma.data(), (int64_t)m, na, a), y = acc128(accs, g, na, a);
        if (root.agg_kind[a] == DDQ_AGG_MIN) x = std::min(x, y);
        else x = (__int128)((unsigned __int128)x + (unsigned __int128)y);
        ma[(m * na + a) * 2] = (int64_t)(uint64_t)(unsigned __int128)x;
        ma[(m * na + a) * 2 + 1] = (int64_t)(uint64_t)((unsigned __int128)x >> 64);
      }
    }
  }
  return finalize_unique(root, (int64_t)mk.size(), mk.data(), ma.data(), out);
}

static ddq_status finalize_unique(const ddq_op& root, int64_t n_groups, const int64_t* keys, const int64_t* accs,
                                  ddq_result** out) {
  const int nk = root.n_keys, na = root.n_aggs;
  if (root.n_avg < 0 || root.n_avg > 4) return set_error(DDQ_EINVAL, "finalize: n_avg must be 0..4");
  for (int k = 0; k < root.n_avg; k++)
    if (root.avg_sum[k] < 0 || root.avg_sum[k] >= na || root.avg_count < 0 || root.avg_count >= na ||
        root.agg_kind[root.avg_count] != DDQ_AGG_COUNT || root.avg_scale[k] < 0 || root.avg_scale[k] > 18)
      return set_error(DDQ_EINVAL, "finalize: bad AVG operands (sum aggregate, COUNT aggregate, scale 0..18)");
  // an aggregate without GROUP BY has exactly one row, also over an empty input
  // (reading O7: its SUMs / MINs are then SQL NULL, its COUNTs 0)
  std::vector<int64_t> zero_acc;
  bool empty_ungrouped = false;
  if (nk == 0 && n_groups == 0) {
    static const int64_t zero_key = 0;
    zero_acc.assign((size_t)std::max(na, 1) * 2, 0);
    keys = &zero_key;
    accs = zero_acc.data();
    n_groups = 1;
    empty_ungrouped = true;
  }
  std::vector<int64_t> idx((size_t)n_groups);
  std::iota(idx.begin(), idx.end(), 0);
  int shift[DDQ_MAX_KEYS], bits[DDQ_MAX_KEYS];
  for (int k = 0, sh = 0; k < DDQ_MAX_KEYS; k++) {
    bits[k] = root.key_bits[k] > 0 ? root.key_bits[k] : 21;
    shift[k] = sh;
    sh += bits[k];
  }
  auto keyk = [&](int64_t g, int k) { return (keys[g] >> shift[k]) & ((1ll << bits[k]) - 1); };
  auto before = [&](int64_t a, int64_t b) {
    for (int o = 0; o < root.n_order; o++) {
      int e = root.order_by[o];
      bool desc = e < 0;
      int v = desc ? -e : e;
      int c = 0;
      if (v >= 101) {
        __int128 x = acc128(accs, a, na, v - 101), y = acc128(accs, b, na, v - 101);
        c = x < y ? -1 : x > y ? 1 : 0;
      } else {
        int64_t x = keyk(a, v - 1), y = keyk(b, v - 1);
        c = x < y ? -1 : x > y ? 1 : 0;
      }
      if (desc) c = -c;
      if (c) return c < 0;
    }
    return keys[a] < keys[b];  // deterministic residual order
  };
  int64_t n = n_groups;
  if (root.limit > 0 && n > root.limit) n = root.limit;
  // LIMIT (O9): only the first n rows need their order (TPC-H Q3: 10 of ~3.6e5 groups)
  if (n < n_groups) std::partial_sort(idx.begin(), idx.begin() + n, idx.end(), before);
  else std::sort(idx.begin(), idx.end(), before);
  ddq_result* r = new ddq_result();
  std::memset(r, 0, sizeof(*r));
  int64_t* k = new int64_t[(size_t)std::max<int64_t>(1, n * nk)];
  int64_t* a = new int64_t[(size_t)std::max<int64_t>(1, n * na * 2)];
  uint8_t* nul = new uint8_t[(size_t)std::max<int64_t>(1, n * na)];
  double* av = root.n_avg > 0 ? new double[(size_t)std::max<int64_t>(1, n * root.n_avg)] : nullptr;
  for (int64_t i = 0; i < n; i++) {
    int64_t g = idx[(size_t)i];
    for (int j = 0; j < nk; j++) k[i * nk + j] = keyk(g, j);
    for (int j = 0; j < na; j++) {
      a[(i * na + j) * 2] = accs[(g * na + j) * 2];
      a[(i * na + j) * 2 + 1] = accs[(g * na + j) * 2 + 1];
      nul[i * na + j] = empty_ungrouped && root.agg_kind[j] != DDQ_AGG_COUNT ? 1 : 0;
    }
    // AVG = SUM / COUNT / 10^scale in double (reading O10): NULL (NaN) for no rows
    for (int j = 0; j < root.n_avg; j++) {
      const __int128 cnt = acc128(accs, g, na, root.avg_count);
      const __int128 sum = acc128(accs, g, na, root.avg_sum[j]);
      av[i * root.n_avg + j] = cnt == 0 ? std::nan("") : (double)sum / (double)cnt / std::pow(10.0, root.avg_scale[j]);
    }
  }
  r->n_rows = n;
  r->n_keys = nk;
  r->n_aggs = na;
  r->keys = k;
  r->aggs = a;
  r->agg_null = nul;
  r->n_avg = root.n_avg;
  r->avgs = av;
  *out = r;
  return DDQ_OK;
}

// Aligned vectors of op i's output, mirroring run_gpu_op / run_host_op: carried
// input vectors first (in order), then the vector the op appends -- a probe's
// emitted payload, a GATHER's column (or a fetch's payload); a STAR emits its
// probe terms' payloads in term order.
static int vec_count(const ddq_plan& plan, int i) {
  if (i < 0 || i >= plan.n_ops) return 0;
  const ddq_op& op = plan.ops[i];
  if (op.kind == DDQ_OP_STAR) {
    int e = 0;
    for (int j = 0; j < op.n_terms && j < 4; j++) e += op.term_kind[j] == DDQ_TERM_PROBE && op.term_emit[j];
    return e;
  }
  if (op.kind == DDQ_OP_HASH_BUILD || op.kind == DDQ_OP_AGGREGATE) return 0;
  const int base = op.input >= 0 && op.input < i ? vec_count(plan, op.input) : 0;
  if ((op.kind == DDQ_OP_HASH_PROBE && op.emit_payload) || op.kind == DDQ_OP_GATHER) return base + 1;
  return base;
}

// Column behind aligned vector v of op i's output (-1: a dimension row id or unknown).
static int vec_column(const ddq_plan& plan, int i, int v) {
  if (i < 0 || i >= plan.n_ops || v < 0) return -1;
  const ddq_op& op = plan.ops[i];
  auto payload_of = [&](int b) { return b >= 0 && b < i ? plan.ops[b].payload_col : -1; };
  if (op.kind == DDQ_OP_STAR) {
    for (int j = 0, e = 0; j < op.n_terms && j < 4; j++)
      if (op.term_kind[j] == DDQ_TERM_PROBE && op.term_emit[j] && e++ == v) return payload_of(op.term_build[j]);
    return -1;
  }
  const int base = op.input >= 0 && op.input < i ? vec_count(plan, op.input) : 0;
  if (v < base) return vec_column(plan, op.input, v);
  if (v == base && op.kind == DDQ_OP_HASH_PROBE && op.emit_payload) return payload_of(op.build);
  if (v == base && op.kind == DDQ_OP_GATHER) return op.fetch_build > 0 ? payload_of(op.fetch_build - 1) : op.gather_col;
  return -1;
}

void decode_result_keys(ddq_db* db, const ddq_plan& plan, ddq_result* r) {
  if (!db || !r || plan.n_ops < 1 || r->n_keys <= 0 || r->key_str) return;
  const ddq_op& root = plan.ops[plan.n_ops - 1];
  if (root.kind != DDQ_OP_AGGREGATE) return;
  const std::vector<std::string>* dict[DDQ_MAX_KEYS] = {nullptr, nullptr, nullptr};
  bool any = false;
  {
    std::lock_guard<std::mutex> g(db->mu);
    for (int k = 0; k < r->n_keys && k < DDQ_MAX_KEYS; k++) {
      const int src = root.key_src[k];
      const int nv = vec_count(plan, root.input);
      int c = src < -1 ? -2 - src : src >= 0 && src < nv ? vec_column(plan, root.input, src) : -1;
      if (src >= nv && root.n_terms > 0) {  // a fused term's emitted payload (O37)
        int e = src - nv;
        for (int j = 0; j < root.n_terms && j < 4; j++)
          if ((root.term_kind[j] == DDQ_TERM_FETCH || root.term_emit[j]) && e-- == 0) {
            const int b = root.term_build[j];
            c = b >= 0 && b < plan.n_ops ? plan.ops[b].payload_col : -1;
          }
      }
      if (c >= 0 && c < (int)db->cols.size() && !db->cols[(size_t)c]->dict.empty()) {
        dict[k] = &db->cols[(size_t)c]->dict;  // set once before queries, never reallocated
        any = true;
      }
    }
  }
  if (!any) return;
  const char** ks = new const char*[(size_t)std::max<int64_t>(1, r->n_rows * r->n_keys)];
  for (int64_t i = 0; i < r->n_rows; i++)
    for (int k = 0; k < r->n_keys; k++) {
      const int64_t code = r->keys[i * r->n_keys + k];
      const std::vector<std::string>* d = k < DDQ_MAX_KEYS ? dict[k] : nullptr;
      ks[i * r->n_keys + k] = d && code >= 0 && code < (int64_t)d->size() ? (*d)[(size_t)code].c_str() : nullptr;
    }
  r->key_str = ks;
}

}  // namespace ddq

using namespace ddq;

// ======================================================================= C ABI
extern "C" {

void ddq_config_default(ddq_config* c) {
  std::memset(c, 0, sizeof(*c));
  c->device = 0;
  c->rank = 0;
  c->world = 1;
  c->cache_bytes = 64ull << 30;
  c->heap_bytes = 32ull << 30;
  c->gpu_workers = 4;  // O17
  c->host_workers = 4;
  c->placement = DDQ_PLACE_DATA_DRIVEN;
  c->chopping = 1;
  c->cache_policy = 0;
  c->fault_alloc_every = 0;
  c->transfer_packing = 1;
}


ddq_status ddq_open(const ddq_config* cfg, ddq_db** out) {
  if (!cfg || !out) return set_error(DDQ_EINVAL, "ddq_open: null argument");
  ddq_db* db = new ddq_db();
  db->cfg = *cfg;
  if (db->cfg.gpu_workers < 1) db->cfg.gpu_workers = 1;
  if (db->cfg.host_workers < 1) db->cfg.host_workers = 1;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0) {
    delete db;
    return set_error(DDQ_ECUDA, "ddq_open: no CUDA device (the product path has no CPU fallback)");
  }
  if (cfg->device < 0 || cfg->device >= ndev) {
    delete db;
    return set_error(DDQ_EINVAL, "ddq_open: bad device ordinal");
  }
  db->device = cfg->device;
  cudaSetDevice(db->device);
  e = cudaStreamCreateWithFlags(&db->copy_stream, cudaStreamNonBlocking);
  if (e != cudaSuccess) {
    delete db;
    return cuda_status(e, "ddq_open stream");
  }
  {
    cudaMemPoolProps pp{};
    pp.allocType = cudaMemAllocationTypePinned;
    pp.location.type = cudaMemLocationTypeDevice;
    pp.location.id = db->device;
    e = cudaMemPoolCreate(&db->cache_pool, &pp);
    if (e != cudaSuccess) {
      cudaStreamDestroy(db->copy_stream);
      delete db;
      return cuda_status(e, "ddq_open cache pool");
    }
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(db->cache_pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  ddq_status s = db->heap.init(cfg->heap_bytes, cfg->fault_alloc_every);
  if (s != DDQ_OK) {
    delete db;
    return s;
  }
  ddq::driver_start(db);
  *out = db;
  return DDQ_OK;
}

void ddq_close(ddq_db* db) {
  if (!db) return;
  ddq::driver_stop(db);
  ddq::dist_free(db);
  cudaSetDevice(db->device);
  cudaDeviceSynchronize();
  for (auto& c : db->cols) {
    if (c->dev) cudaFreeAsync(c->dev, db->copy_stream);
    if (c->host) cudaFreeHost(c->host);
    if (c->host_packed) cudaFreeHost(c->host_packed);
    if (c->host_tdict) cudaFreeHost(c->host_tdict);
  }
  for (auto& kv : db->cache_free) cudaFreeAsync(kv.second, db->copy_stream);
  db->cache_free.clear();
  cudaStreamSynchronize(db->copy_stream);
  if (db->cache_pool) cudaMemPoolDestroy(db->cache_pool);
  if (db->copy_stream) cudaStreamDestroy(db->copy_stream);
  delete db;
}

ddq_status ddq_create_table(ddq_db* db, const char* name, int64_t n_rows, int64_t row_begin, ddq_table* out) {
  if (!db || !name || n_rows < 0 || n_rows > INT32_MAX || !out) return set_error(DDQ_EINVAL, "create_table");
  std::lock_guard<std::mutex> g(db->mu);
  for (auto& t : db->tables)
    if (t.name == name) return set_error(DDQ_EINVAL, "table exists");
  Table t;
  t.name = name;
  t.n_rows = n_rows;
  t.row_begin = row_begin;
  db->tables.push_back(t);
  *out = (ddq_table)(db->tables.size() - 1);
  return DDQ_OK;
}

ddq_status ddq_load_column(ddq_db* db, ddq_table t, const char* name, ddq_type type, const void* host_data,
                           int64_t n_rows, ddq_column* out) {
  if (!db || !name || !host_data || !out) return set_error(DDQ_EINVAL, "load_column: null argument");
  if (type != DDQ_I32 && type != DDQ_I64) return set_error(DDQ_EINVAL, "load_column: bad type");
  std::lock_guard<std::mutex> g(db->mu);
  if (t < 0 || t >= (int)db->tables.size()) return set_error(DDQ_ENOTFOUND, "load_column: bad table");
  if (n_rows != db->tables[(size_t)t].n_rows) return set_error(DDQ_EINVAL, "load_column: row count mismatch");
  auto c = std::make_unique<Column>();
  c->name = name;
  c->table = t;
  c->type = type;
  c->width = type == DDQ_I32 ? 4 : 8;
  c->n = n_rows;
  size_t bytes = (size_t)std::max<int64_t>(n_rows, 1) * c->width;
  cudaError_t e = cudaHostAlloc(&c->host, bytes, cudaHostAllocPortable);
  if (e != cudaSuccess) return set_error(DDQ_ENOMEM_HOST, "load_column: pinned alloc failed");
  std::memcpy(c->host, host_data, (size_t)n_rows * c->width);
  for (int64_t i = 0; i < n_rows; i++) {
    int64_t v = c->width == 4 ? ((const int32_t*)host_data)[i] : ((const int64_t*)host_data)[i];
    if (i == 0 || v < c->vmin) c->vmin = v;
    if (i == 0 || v > c->vmax) c->vmax = v;
  }
  // transfer encoding: value - vmin in the bit length of the range (1..32 bits, fewer
  // than the column's width), a little-endian bit stream (transfer.cu)
  if (db->cfg.transfer_packing && n_rows > 0) {
    const uint64_t range = (uint64_t)c->vmax - (uint64_t)c->vmin;
    int bits = 1;
    while (bits < 64 && (range >> bits) != 0) bits++;
    // dictionary transfer code (ranks of the distinct values) when its packed stream
    // plus the 8-byte dictionary is smaller: value ranges < 2^24 only (a presence
    // bitmap and a rank table over the range)
    std::vector<uint32_t> rank;
    std::vector<int64_t> dict;
    static const char* dict_env = getenv("DDQ_TRANSFER_DICT");  // "0": range code only (A/B)
    if (bits <= 32 && bits < 8 * c->width && range < (1u << 24) && !(dict_env && dict_env[0] == '0')) {
      const size_t pw = (size_t)(range >> 6) + 1;
      const int np = (int)std::max<int64_t>(1, std::min<int64_t>(std::thread::hardware_concurrency(),
                                                                  n_rows / (1 << 20)));
      std::vector<std::vector<uint64_t>> part((size_t)np, std::vector<uint64_t>(pw, 0));
      auto mark = [&](int t) {  // presence bitmap of rows [t*n/np, (t+1)*n/np)
        uint64_t* pr = part[(size_t)t].data();
        const int64_t b = n_rows * t / np, e = n_rows * (t + 1) / np;
        for (int64_t i = b; i < e; i++) {
          const int64_t v = c->width == 4 ? ((const int32_t*)host_data)[i] : ((const int64_t*)host_data)[i];
          const uint64_t o = (uint64_t)(v - c->vmin);
          pr[(size_t)(o >> 6)] |= 1ull << (o & 63);
        }
      };
      {
        std::vector<std::thread> th;
        for (int t = 1; t < np; t++) th.emplace_back(mark, t);
        mark(0);
        for (auto& x : th) x.join();
      }
      std::vector<uint64_t>& present = part[0];
      for (int t = 1; t < np; t++)
        for (size_t w = 0; w < pw; w++) present[w] |= part[(size_t)t][w];
      int64_t d = 0;
      for (uint64_t w : present) d += __builtin_popcountll(w);
      int dbits = 1;
      while (dbits < 32 && ((uint64_t)(d - 1) >> dbits) != 0) dbits++;
      if (packed_bytes(n_rows, dbits) + (size_t)d * 8 < packed_bytes(n_rows, bits)) {
        rank.assign((size_t)range + 1, 0);
        dict.reserve((size_t)d);
        for (size_t w = 0; w < present.size(); w++)
          for (uint64_t m = present[w]; m; m &= m - 1) {
            const uint64_t o = (uint64_t)w * 64 + (uint64_t)__builtin_ctzll(m);
            rank[(size_t)o] = (uint32_t)dict.size();
            dict.push_back(c->vmin + (int64_t)o);
          }
        bits = dbits;
      }
    }
    if (!dict.empty() && cudaHostAlloc((void**)&c->host_tdict, dict.size() * 8, cudaHostAllocPortable) != cudaSuccess)
      dict.clear(), rank.clear(), bits = 64;  // no pinned room for the dictionary: raw copy
    if (!dict.empty()) {
      std::memcpy(c->host_tdict, dict.data(), dict.size() * 8);
      c->tdict_n = (int64_t)dict.size();
    }
    if (bits <= 32 && bits < 8 * c->width &&
        cudaHostAlloc(&c->host_packed, packed_bytes(n_rows, bits), cudaHostAllocPortable) == cudaSuccess) {
      uint32_t* dst = (uint32_t*)c->host_packed;
      std::memset(dst, 0, packed_bytes(n_rows, bits));
      // 32 values fill exactly `bits` words, so chunks of 32k values pack in parallel
      const int64_t per = 32 * 65536;
      const int64_t chunks = (n_rows + per - 1) / per;
      const int nt = (int)std::max<int64_t>(1, std::min<int64_t>(chunks, std::thread::hardware_concurrency()));
      const int64_t vmin = c->vmin;
      const int width = c->width;
      const uint32_t* rk = rank.empty() ? nullptr : rank.data();
      auto pack = [&](int t) {
        for (int64_t ch = t; ch < chunks; ch += nt) {
          const int64_t b = ch * per, e = std::min<int64_t>(n_rows, b + per);
          uint64_t acc = 0;  // bits not yet flushed, low first
          int have = 0;
          size_t w = (size_t)(b / 32) * (size_t)bits;
          for (int64_t i = b; i < e; i++) {
            const int64_t v = width == 4 ? ((const int32_t*)host_data)[i] : ((const int64_t*)host_data)[i];
            const uint64_t x = (uint64_t)v - (uint64_t)vmin;
            acc |= (rk ? (uint64_t)rk[x] : x) << have;
            have += bits;
            if (have >= 32) {
              dst[w++] = (uint32_t)acc;
              acc >>= 32;
              have -= 32;
            }
          }
          if (have > 0) dst[w] = (uint32_t)acc;
        }
      };
      std::vector<std::thread> th;
      for (int t = 1; t < nt; t++) th.emplace_back(pack, t);
      pack(0);
      for (auto& x : th) x.join();
      c->tw = bits;
    } else if (c->host_tdict) {  // no packed copy after all: the raw column goes
      cudaFreeHost(c->host_tdict);
      c->host_tdict = nullptr;
      c->tdict_n = 0;
    }
  }
  db->cols.push_back(std::move(c));
  int id = (int)db->cols.size() - 1;
  db->tables[(size_t)t].cols.push_back(id);
  *out = id;
  return DDQ_OK;
}

ddq_status ddq_find_column(ddq_db* db, const char* table, const char* name, ddq_column* out) {
  if (!db || !table || !name || !out) return set_error(DDQ_EINVAL, "find_column");
  std::lock_guard<std::mutex> g(db->mu);
  for (size_t t = 0; t < db->tables.size(); t++) {
    if (db->tables[t].name != table) continue;
    for (int c : db->tables[t].cols)
      if (db->cols[(size_t)c]->name == name) {
        *out = c;
        return DDQ_OK;
      }
  }
  return set_error(DDQ_ENOTFOUND, std::string("column ") + table + "." + name);
}

ddq_status ddq_column_stats(ddq_db* db, ddq_column c, int64_t* n, int64_t* vmin, int64_t* vmax) {
  if (!db || !n || !vmin || !vmax) return set_error(DDQ_EINVAL, "column_stats: null argument");
  std::lock_guard<std::mutex> g(db->mu);
  if (c < 0 || c >= (int)db->cols.size()) return set_error(DDQ_ENOTFOUND, "column_stats: bad column");
  const Column& col = *db->cols[(size_t)c];
  *n = col.n;
  *vmin = col.n > 0 ? col.vmin : 1;
  *vmax = col.n > 0 ? col.vmax : 0;
  return DDQ_OK;
}

ddq_status ddq_set_dictionary(ddq_db* db, ddq_column c, const char* const* sorted_strings, int32_t n) {
  if (!db || n < 0 || (n > 0 && !sorted_strings)) return set_error(DDQ_EINVAL, "set_dictionary: null argument");
  std::vector<std::string> d;
  d.reserve((size_t)n);
  for (int32_t i = 0; i < n; i++) {
    if (!sorted_strings[i]) return set_error(DDQ_EINVAL, "set_dictionary: null string");
    d.emplace_back(sorted_strings[i]);
    if (i > 0 && !(d[(size_t)i - 1] < d[(size_t)i]))  // std::string compares bytewise (C locale)
      return set_error(DDQ_EINVAL, "set_dictionary: strings not strictly ascending (bytewise)");
  }
  std::lock_guard<std::mutex> g(db->mu);
  if (c < 0 || c >= (int)db->cols.size()) return set_error(DDQ_ENOTFOUND, "set_dictionary: bad column");
  Column& col = *db->cols[(size_t)c];
  if (col.width != 4) return set_error(DDQ_EINVAL, "set_dictionary: codes are int32");
  if (col.n > 0 && (col.vmin < 0 || col.vmax >= (int64_t)n))
    return set_error(DDQ_EINVAL, "set_dictionary: column holds codes outside the dictionary");
  col.dict = std::move(d);
  return DDQ_OK;
}

ddq_status ddq_dictionary_range(ddq_db* db, ddq_column c, const char* s, int32_t* lower, int32_t* upper) {
  if (!db || !s || !lower || !upper) return set_error(DDQ_EINVAL, "dictionary_range: null argument");
  std::lock_guard<std::mutex> g(db->mu);
  if (c < 0 || c >= (int)db->cols.size()) return set_error(DDQ_ENOTFOUND, "dictionary_range: bad column");
  const std::vector<std::string>& d = db->cols[(size_t)c]->dict;
  if (d.empty()) return set_error(DDQ_ENOTFOUND, "dictionary_range: column has no dictionary");
  *lower = (int32_t)(std::lower_bound(d.begin(), d.end(), std::string(s)) - d.begin());
  *upper = (int32_t)(std::upper_bound(d.begin(), d.end(), std::string(s)) - d.begin());
  return DDQ_OK;
}

// SQL LIKE: '%' matches any run of bytes, '_' exactly one byte (no escape character)
static bool like_match(const char* s, const char* p) {
  if (*p == 0) return *s == 0;
  if (*p == '%') {
    while (*p == '%') p++;
    if (*p == 0) return true;
    for (; *s; s++)
      if (like_match(s, p)) return true;
    return false;
  }
  if (*s == 0) return false;
  return (*p == '_' || *p == *s) && like_match(s + 1, p + 1);
}

ddq_status ddq_dictionary_like(ddq_db* db, ddq_column c, const char* pattern, ddq_pred* out) {
  if (!db || !pattern || !out) return set_error(DDQ_EINVAL, "dictionary_like: null argument");
  std::lock_guard<std::mutex> g(db->mu);
  if (c < 0 || c >= (int)db->cols.size()) return set_error(DDQ_ENOTFOUND, "dictionary_like: bad column");
  const std::vector<std::string>& d = db->cols[(size_t)c]->dict;
  if (d.empty()) return set_error(DDQ_ENOTFOUND, "dictionary_like: column has no dictionary");
  std::vector<int64_t> hits;
  for (size_t i = 0; i < d.size(); i++)
    if (like_match(d[i].c_str(), pattern)) hits.push_back((int64_t)i);
  std::memset(out, 0, sizeof(*out));
  out->column = c;
  if (hits.empty()) {  // matches nothing: an empty range
    out->kind = DDQ_PRED_RANGE;
    out->lo = 1;
    out->hi = 0;
    return DDQ_OK;
  }
  if (hits.size() <= DDQ_MAX_IN) {
    out->kind = DDQ_PRED_IN;
    out->n_in = (int32_t)hits.size();
    for (size_t i = 0; i < hits.size(); i++) out->in_vals[i] = hits[i];
    return DDQ_OK;
  }
  if (hits.back() - hits.front() >= 512) return set_error(DDQ_EINVAL, "dictionary_like: matches span > 512 codes");
  out->kind = DDQ_PRED_BITSET;
  out->lo = hits.front();
  out->hi = hits.back();
  for (int64_t h : hits) out->in_vals[(h - out->lo) >> 6] |= (int64_t)(1ull << ((h - out->lo) & 63));
  return DDQ_OK;
}

}  // extern "C"

namespace ddq {
// Cache blocks: an exact-size free list in front of the stream-ordered pool.  The
// pool alone let cold steps stretch from 52 ms to 150-600 ms (tools/e2e_steps.py):
// blocks freed and re-requested in a different order each step.
static void* cache_block(ddq_db* db, size_t bytes) {
  auto it = db->cache_free.find(bytes);
  if (it != db->cache_free.end()) {
    void* p = it->second;
    db->cache_free.erase(it);
    return p;
  }
  void* p = nullptr;
  if (cudaMallocFromPoolAsync(&p, bytes, db->cache_pool, db->copy_stream) != cudaSuccess) {
    cudaGetLastError();
    // drop the free list back into the pool and retry once
    for (auto& kv : db->cache_free) cudaFreeAsync(kv.second, db->copy_stream);
    db->cache_free.clear();
    if (cudaMallocFromPoolAsync(&p, bytes, db->cache_pool, db->copy_stream) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
  }
  return p;
}
static void cache_unblock(ddq_db* db, void* p, size_t bytes) { db->cache_free.emplace(bytes, p); }

// H2D copy of one column into the cache.  The caller holds db->mu through `lk`;
// it is released for the copy itself, so operators of other queries keep
// launching while PCIe is busy (a concurrent request for the same column waits
// on cache_cv).  The bytes are reserved against the budget before unlocking.
ddq_status cache_column_locked(ddq_db* db, int c, bool on_demand, std::unique_lock<std::mutex>& lk) {
  Column& col = *db->cols[(size_t)c];
  while (col.loading) db->cache_cv.wait(lk);
  if (col.dev) {
    col.evict_pending = false;
    return DDQ_OK;
  }
  uint64_t bytes = (uint64_t)std::max<int64_t>(col.n, 1) * col.width;
  if (db->cache_used + bytes > db->cfg.cache_bytes)
    return set_error(DDQ_ENOMEM_DEVICE, "cache budget exceeded for " + col.name);
  cudaSetDevice(db->device);
  void* p = nullptr;
  // padded: TMA reads whole 16-byte chunks
  const size_t dbytes = (bytes + 255) / 256 * 256;
  p = cache_block(db, dbytes);
  if (!p) return set_error(DDQ_ENOMEM_DEVICE, "cache: device memory exhausted for " + col.name);
  cudaError_t e = cudaSuccess;
  cudaEvent_t done = nullptr;
  e = cudaEventCreateWithFlags(&done, cudaEventDisableTiming);
  if (e != cudaSuccess) {
    cache_unblock(db, p, dbytes);
    return cuda_status(e, "cache event");
  }
  db->cache_used += bytes;
  col.loading = true;
  // packed transfer: stage the packed bytes in a pool block, widen into the column
  void* stage = nullptr;
  const size_t sbytes = col.tw ? packed_bytes(col.n, col.tw) : 0;  // the stream, 16-byte multiple
  const size_t dict_bytes = (size_t)col.tdict_n * 8;
  const size_t pbytes = sbytes + dict_bytes;  // the dictionary travels behind the stream
  if (col.tw) stage = cache_block(db, pbytes);  // null: no room, send the raw column
  lk.unlock();
  uint64_t t0 = now_ns();
  uint64_t moved = 0;
  if (stage) {
    e = cudaMemcpyAsync(stage, col.host_packed, sbytes, cudaMemcpyHostToDevice, db->copy_stream);
    void* ddict = dict_bytes ? (void*)((char*)stage + sbytes) : nullptr;
    if (e == cudaSuccess && ddict)
      e = cudaMemcpyAsync(ddict, col.host_tdict, dict_bytes, cudaMemcpyHostToDevice, db->copy_stream);
    if (e == cudaSuccess) e = launch_unpack(stage, col.tw, col.vmin, p, col.width, col.n, db->copy_stream, ddict);
    moved = pbytes;
  } else {
    e = cudaMemcpyAsync(p, col.host, (size_t)col.n * col.width, cudaMemcpyHostToDevice, db->copy_stream);
    moved = (uint64_t)col.n * col.width;
  }
  if (e == cudaSuccess) e = cudaEventRecord(done, db->copy_stream);
  if (e == cudaSuccess) e = cudaEventSynchronize(done);
  const uint64_t dt = now_ns() - t0;
  cudaEventDestroy(done);
  lk.lock();
  col.loading = false;
  db->cache_cv.notify_all();
  if (stage) cache_unblock(db, stage, pbytes);  // later users are ordered after the unpack on copy_stream
  if (e != cudaSuccess) {
    cache_unblock(db, p, dbytes);
    db->cache_used -= bytes;
    return cuda_status(e, "cache H2D");
  }
  db->stats.h2d_ns += dt;
  db->stats.h2d_bytes += moved;
  col.dev = p;
  col.on_demand = on_demand;
  col.evict_pending = false;
  return DDQ_OK;
}

// Evict (deferred while running operators hold references).  Prepared
// plans launched asynchronously may still read the column: wait for the device
// (cudaFree's implicit synchronisation), then return the block to the pool.
// Drop cache references (one per entry of cols); a column whose eviction was
// deferred is evicted when its last reference goes.
void release_column_refs(ddq_db* db, const std::vector<int>& cols) {
  std::lock_guard<std::mutex> g(db->mu);
  for (int c : cols) {
    Column& col = *db->cols[(size_t)c];
    if (--col.refs == 0 && col.evict_pending) evict_column_locked(db, c);
  }
}

void evict_column_locked(ddq_db* db, int c) {
  Column& col = *db->cols[(size_t)c];
  if (!col.dev) return;
  if (col.refs > 0) {
    col.evict_pending = true;
    return;
  }
  cudaSetDevice(db->device);
  cudaDeviceSynchronize();
  cache_unblock(db, col.dev, ((size_t)std::max<int64_t>(col.n, 1) * col.width + 255) / 256 * 256);
  col.dev = nullptr;
  col.evict_pending = false;
  db->cache_used -= (uint64_t)std::max<int64_t>(col.n, 1) * col.width;
}
}  // namespace ddq

extern "C" {

ddq_status ddq_cache_column(ddq_db* db, ddq_column c) {
  if (!db || c < 0 || c >= (int)db->cols.size()) return set_error(DDQ_ENOTFOUND, "cache_column");
  std::unique_lock<std::mutex> g(db->mu);
  return cache_column_locked(db, c, false, g);
}

ddq_status ddq_evict_column(ddq_db* db, ddq_column c) {
  if (!db || c < 0 || c >= (int)db->cols.size()) return set_error(DDQ_ENOTFOUND, "evict_column");
  std::lock_guard<std::mutex> g(db->mu);
  evict_column_locked(db, c);
  return DDQ_OK;
}

int32_t ddq_column_is_cached(ddq_db* db, ddq_column c) {
  if (!db || c < 0 || c >= (int)db->cols.size()) return 0;
  std::lock_guard<std::mutex> g(db->mu);
  return db->cols[(size_t)c]->dev && !db->cols[(size_t)c]->evict_pending ? 1 : 0;
}

const void* ddq_column_device_ptr(ddq_db* db, ddq_column c) {
  if (!db || c < 0 || c >= (int)db->cols.size()) return nullptr;
  std::lock_guard<std::mutex> g(db->mu);
  return db->cols[(size_t)c]->dev;
}

uint64_t ddq_column_access_count(ddq_db* db, ddq_column c) {
  if (!db || c < 0 || c >= (int)db->cols.size()) return 0;
  return db->cols[(size_t)c]->access.load();
}

ddq_status ddq_reset_access_counts(ddq_db* db) {
  if (!db) return set_error(DDQ_EINVAL, "reset_access_counts");
  for (auto& c : db->cols) c->access = 0;
  return DDQ_OK;
}

// Algorithm 1 (Sec. 3.2).  LFU by access count (cache_policy 0) or
// LRU by last access (policy 1, App. E).  Reading O16: i runs over all
// of K, ties by column id, and the loop stops at the first column that does not fit.
ddq_status ddq_update_placement(ddq_db* db) {
  if (!db) return set_error(DDQ_EINVAL, "update_placement");
  std::unique_lock<std::mutex> lk(db->mu);
  std::vector<int> K(db->cols.size());
  std::iota(K.begin(), K.end(), 0);
  std::stable_sort(K.begin(), K.end(), [&](int a, int b) {
    uint64_t x = db->cfg.cache_policy == 1 ? db->cols[(size_t)a]->last_access.load() : db->cols[(size_t)a]->access.load();
    uint64_t y = db->cfg.cache_policy == 1 ? db->cols[(size_t)b]->last_access.load() : db->cols[(size_t)b]->access.load();
    return x > y;
  });
  uint64_t used = 0;
  std::vector<bool> keep(db->cols.size(), false);
  for (size_t i = 0; i < K.size(); i++) {
    const Column& c = *db->cols[(size_t)K[i]];
    uint64_t sz = (uint64_t)std::max<int64_t>(c.n, 1) * c.width;
    if (used + sz > db->cfg.cache_bytes) break;
    keep[(size_t)K[i]] = true;
    used += sz;
  }
  for (size_t c = 0; c < db->cols.size(); c++)  // evict(C_old \ C_new)
    if (!keep[c] && db->cols[c]->dev) evict_column_locked(db, (int)c);
  for (size_t c = 0; c < db->cols.size(); c++)  // a kept column no longer pending eviction
    if (keep[c] && db->cols[c]->dev) db->cols[c]->evict_pending = false;
  for (size_t c = 0; c < db->cols.size(); c++)  // cache(C_new \ C_old)
    if (keep[c] && !db->cols[c]->dev) {
      ddq_status s = cache_column_locked(db, (int)c, false, lk);
      if (s != DDQ_OK && s != DDQ_ENOMEM_DEVICE) return s;  // deferred evictions may still hold memory
    }
  return DDQ_OK;
}

ddq_status ddq_get_stats(ddq_db* db, ddq_stats* o) {
  if (!db || !o) return set_error(DDQ_EINVAL, "get_stats");
  std::memset(o, 0, sizeof(*o));
  o->h2d_bytes = db->stats.h2d_bytes;
  o->d2h_bytes = db->stats.d2h_bytes;
  o->h2d_ns = db->stats.h2d_ns;
  o->d2h_ns = db->stats.d2h_ns;
  o->gpu_ops = db->stats.gpu_ops;
  o->host_ops = db->stats.host_ops;
  o->aborts = db->stats.aborts;
  o->wasted_ns = db->stats.wasted_ns;
  o->heap_peak_bytes = db->heap.peak();
  o->heap_used_bytes = db->heap.used();
  o->cache_used_bytes = db->cache_used;
  o->cache_hits = db->stats.cache_hits;
  o->cache_misses = db->stats.cache_misses;
  o->queries_done = db->stats.queries_done;
  return DDQ_OK;
}

ddq_status ddq_reset_stats(ddq_db* db) {
  if (!db) return set_error(DDQ_EINVAL, "reset_stats");
  db->stats.h2d_bytes = 0;
  db->stats.d2h_bytes = 0;
  db->stats.h2d_ns = 0;
  db->stats.d2h_ns = 0;
  db->stats.gpu_ops = 0;
  db->stats.host_ops = 0;
  db->stats.aborts = 0;
  db->stats.wasted_ns = 0;
  db->stats.cache_hits = 0;
  db->stats.cache_misses = 0;
  db->stats.queries_done = 0;
  db->heap.reset_peak();
  return DDQ_OK;
}

void* ddq_heap_try_alloc(ddq_db* db, uint64_t bytes) { return db ? db->heap.try_alloc(bytes) : nullptr; }
void ddq_heap_free(ddq_db* db, void* p) {
  if (db) db->heap.free(p);
}

void ddq_result_free(ddq_result* r) {
  if (!r) return;
  delete[] r->keys;
  delete[] r->aggs;
  delete[] r->tids;
  delete[] r->agg_null;
  delete[] r->avgs;
  delete[] r->key_str;
  delete[] r->op_place;
  delete[] r->op_ms;
  delete r;
}

}  // extern "C"

// ============================================================ prepared plans
struct ddq_prepared {
  ddq_db* db = nullptr;
  // cache references on every column the plan reads: an eviction (explicit,
  // Algorithm 1 or the GPU-only LRU) is deferred until ddq_prepared_free, so the
  // graph never reads a freed or reused column block
  std::vector<int> held;
  ddq_plan plan{};
  std::vector<ddq::Inter> inters;
  std::vector<int64_t> forced;  // per-op output capacity (exact count + slack)
  std::vector<char> bits_out;   // per op: survivors as a row bitmap (see GpuOpCtx)
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t exec = nullptr;
  bool use_graph = false;
  int kernels = 0;
  cudaStream_t cap_stream = nullptr;
  // graph capture with parallel branches: side streams + one event per op
  std::vector<cudaStream_t> side;
  std::vector<cudaEvent_t> ev;
  std::vector<ddq::FillRec> fills;  // buffer initialisations, hoisted to the graph root
};

namespace ddq {

static ddq_status validate_plan(ddq_db* db, const ddq_plan* plan) {
  if (!plan || plan->n_ops < 1 || plan->n_ops > DDQ_MAX_OPS) return set_error(DDQ_EINVAL, "plan: bad op count");
  for (int i = 0; i < plan->n_ops; i++) {
    const ddq_op& op = plan->ops[i];
    if (op.kind < DDQ_OP_SELECT || op.kind > DDQ_OP_STAR) return set_error(DDQ_EINVAL, "plan: bad op kind");
    if (op.kind == DDQ_OP_STAR) {
      if (op.input >= 0) return set_error(DDQ_EINVAL, "plan: a STAR op scans all rows");
      if (op.n_terms < 1 || op.n_terms > 4) return set_error(DDQ_EINVAL, "plan: STAR needs 1..4 terms");
      for (int j = 0; j < op.n_terms; j++)
        if (op.term_kind[j] == DDQ_TERM_PROBE &&
            (op.term_build[j] < 0 || op.term_build[j] >= i || plan->ops[op.term_build[j]].kind != DDQ_OP_HASH_BUILD))
          return set_error(DDQ_EINVAL, "plan: STAR probe must reference an earlier HASH_BUILD");
    }
    if (op.kind == DDQ_OP_AGGREGATE && op.n_terms != 0) {  // fused probe / fetch terms (O37)
      if (op.input < 0) return set_error(DDQ_EINVAL, "plan: aggregate terms need an input TID list");
      if (op.n_terms < 0 || op.n_terms > 4) return set_error(DDQ_EINVAL, "plan: aggregate needs 0..4 terms");
      for (int j = 0; j < op.n_terms; j++)
        if ((op.term_kind[j] != DDQ_TERM_PROBE && op.term_kind[j] != DDQ_TERM_FETCH) || op.term_build[j] < 0 ||
            op.term_build[j] >= i || plan->ops[op.term_build[j]].kind != DDQ_OP_HASH_BUILD)
          return set_error(DDQ_EINVAL, "plan: an aggregate term probes / fetches an earlier HASH_BUILD");
    }
    if (op.kind == DDQ_OP_FILTER_EQ && op.input < 0) return set_error(DDQ_EINVAL, "plan: filter_eq needs an input");
    if (op.fetch_build != 0 && (op.kind != DDQ_OP_GATHER || op.fetch_build - 1 < 0 || op.fetch_build - 1 >= i ||
                                plan->ops[op.fetch_build - 1].kind != DDQ_OP_HASH_BUILD))
      return set_error(DDQ_EINVAL, "plan: a fetch must be a GATHER referencing an earlier HASH_BUILD");
    if (op.kind == DDQ_OP_HASH_PROBE && op.fk_vec > 0 && op.input < 0)
      return set_error(DDQ_EINVAL, "plan: a vector-keyed probe needs an input");
    if (op.kind == DDQ_OP_AGGREGATE && op.input < 0)
      for (int k = 0; k < op.n_keys && k < DDQ_MAX_KEYS; k++)
        if (op.key_src[k] >= 0) return set_error(DDQ_EINVAL, "plan: an aggregate over all rows keys on columns only");
    if (op.kind == DDQ_OP_AGGREGATE) {
      int bits = 0;
      for (int k = 0; k < op.n_keys && k < DDQ_MAX_KEYS; k++) bits += op.key_bits[k] > 0 ? op.key_bits[k] : 21;
      if (bits > 63) return set_error(DDQ_EINVAL, "plan: packed group key wider than 63 bits");
    }
    if (op.n_preds < 0 || op.n_preds > DDQ_MAX_PREDS) return set_error(DDQ_EINVAL, "plan: bad n_preds");
    for (int k = 0; k < op.n_preds; k++) {
      const ddq_pred& pr = op.preds[k];
      if (pr.kind != DDQ_PRED_RANGE && pr.kind != DDQ_PRED_IN && pr.kind != DDQ_PRED_BITSET)
        return set_error(DDQ_EINVAL, "plan: bad predicate kind");
      if (pr.kind == DDQ_PRED_IN && (pr.n_in < 0 || pr.n_in > DDQ_MAX_IN))
        return set_error(DDQ_EINVAL, "plan: IN list must hold 0..8 values");
    }
    if (op.kind == DDQ_OP_AGGREGATE && (op.n_avg < 0 || op.n_avg > 4)) return set_error(DDQ_EINVAL, "plan: n_avg 0..4");
    if (op.kind == DDQ_OP_HASH_BUILD && (op.build_key_set < 0 || op.build_key_set > 2))
      return set_error(DDQ_EINVAL, "plan: build_key_set must be 0, 1 or 2");
    if (op.input >= i || op.input < -1) return set_error(DDQ_EINVAL, "plan: input must precede the op");
    if (op.kind == DDQ_OP_HASH_PROBE && (op.build < 0 || op.build >= i ||
                                         plan->ops[op.build].kind != DDQ_OP_HASH_BUILD))
      return set_error(DDQ_EINVAL, "plan: probe must reference an earlier HASH_BUILD");
    if (op.input >= 0 && plan->ops[op.input].kind == DDQ_OP_HASH_BUILD)
      return set_error(DDQ_EINVAL, "plan: a hash table is not a TID input");
    if (op.input >= 0 && plan->ops[op.input].kind == DDQ_OP_AGGREGATE)
      return set_error(DDQ_EINVAL, "plan: an aggregate is not a TID input");
    if (op.input >= 0 && plan->ops[op.input].table != op.table)
      return set_error(DDQ_EINVAL, "plan: input TIDs belong to another table");
    if (op.table < 0 || op.table >= (int)db->tables.size()) return set_error(DDQ_EINVAL, "plan: bad table");
  }
  const ddq_op& root = plan->ops[plan->n_ops - 1];
  if (root.kind == DDQ_OP_HASH_BUILD) return set_error(DDQ_EINVAL, "plan: root cannot be a HASH_BUILD");
  return DDQ_OK;
}
ddq_status validate_plan_public(ddq_db* db, const ddq_plan* plan) { return validate_plan(db, plan); }

// kernels an operator launches in a prepared graph (its buffer initialisations are
// hoisted into the graph's one multi-range fill kernel, counted separately)
static int kernels_of(const ddq_op& op) {
  switch (op.kind) {
    case DDQ_OP_SELECT:
    case DDQ_OP_HASH_PROBE: return 1;
    case DDQ_OP_HASH_BUILD: return 1;
    case DDQ_OP_GATHER: return 1;
    case DDQ_OP_AGGREGATE: return 2;
    case DDQ_OP_FILTER_EQ: return 1;
    case DDQ_OP_STAR: return 1;
  }
  return 0;
}

static void free_inters(ddq_db* db, std::vector<Inter>& v) {
  for (auto& x : v) release_inter(db, x);
  v.clear();
}

// Re-issue the launches of a prepared plan on its existing buffers.
static ddq_status replay_op(ddq_prepared* P, int i, cudaStream_t st) {
  std::vector<void*> blocks = P->inters[(size_t)i].heap_blocks;
  GpuOpCtx ctx{P->db, st, &P->inters};
  ctx.forced_cap = P->forced[(size_t)i];
  ctx.count_column_access = false;
  ctx.reuse = &blocks;
  ctx.bits_out = P->bits_out[(size_t)i] != 0;
  ctx.dist = true;
  return run_gpu_op(ctx, P->plan.ops[i], P->inters[(size_t)i]);
}
static ddq_status replay(ddq_prepared* P, cudaStream_t st) {
  for (int i = 0; i < P->plan.n_ops; i++)
    if (ddq_status s = replay_op(P, i, st)) return s;
  return DDQ_OK;
}

// The plan DAG's edges: an op depends on its TID input, its build side and the
// builds its STAR terms probe (every other buffer it reads -- carried vectors,
// error cells -- comes down its input chain).
static std::vector<int> op_deps(const ddq_op& op, int i) {
  std::vector<int> d;
  auto add = [&](int x) {
    if (x >= 0 && x < i && std::find(d.begin(), d.end(), x) == d.end()) d.push_back(x);
  };
  add(op.input);
  if (op.kind == DDQ_OP_HASH_PROBE) add(op.build);
  if (op.kind == DDQ_OP_GATHER && op.fetch_build > 0) add(op.fetch_build - 1);
  if (op.kind == DDQ_OP_STAR || op.kind == DDQ_OP_AGGREGATE)
    for (int j = 0; j < op.n_terms && j < 4; j++)
      if (op.term_kind[j] == DDQ_TERM_PROBE || op.term_kind[j] == DDQ_TERM_FETCH) add(op.term_build[j]);
  return d;
}

// Capture the plan as a graph whose branches follow the DAG: independent
// operators (the dimension builds of a star query, and the fact chain's first
// probe against the builds it does not read) run concurrently, so the small,
// latency-bound build kernels leave the critical path.  An op continues the
// stream of its first dependency when it is that stream's last op, else forks a
// side stream; other dependencies are event waits.  All branches join `st`.
static ddq_status replay_branches(ddq_prepared* P, cudaStream_t st) {
  const int n = P->plan.n_ops;
  if ((int)P->ev.size() < n + 1) {
    for (int i = (int)P->ev.size(); i < n + 1; i++) {
      cudaEvent_t e;
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
        return set_error(DDQ_ECUDA, "prepare: event");
      P->ev.push_back(e);
    }
  }
  std::vector<cudaStream_t> streams;  // capture lanes; lane 0 = st
  std::vector<int> tail;              // last op on each lane
  std::vector<int> lane_of((size_t)n, -1);
  streams.push_back(st);
  tail.push_back(-1);
  cudaEvent_t start = P->ev[(size_t)n];
  if (cudaEventRecord(start, st) != cudaSuccess) return set_error(DDQ_ECUDA, "prepare: fork");
  size_t next_side = 0;
  for (int i = 0; i < n; i++) {
    const std::vector<int> d = op_deps(P->plan.ops[i], i);
    int lane = -1;
    if (!d.empty() && tail[(size_t)lane_of[(size_t)d[0]]] == d[0]) lane = lane_of[(size_t)d[0]];
    if (lane < 0 && d.empty() && tail[0] == -1) lane = 0;  // the first root op stays on st
    if (lane < 0) {
      if (next_side == P->side.size()) {
        cudaStream_t s2;
        if (cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking) != cudaSuccess)
          return set_error(DDQ_ECUDA, "prepare: side stream");
        P->side.push_back(s2);
      }
      streams.push_back(P->side[next_side++]);
      tail.push_back(-1);
      lane = (int)streams.size() - 1;
      if (d.empty() && cudaStreamWaitEvent(streams[(size_t)lane], start, 0) != cudaSuccess)
        return set_error(DDQ_ECUDA, "prepare: fork");
    }
    for (int x : d)
      if (lane_of[(size_t)x] != lane && cudaStreamWaitEvent(streams[(size_t)lane], P->ev[(size_t)x], 0) != cudaSuccess)
        return set_error(DDQ_ECUDA, "prepare: edge");
    if (ddq_status s = replay_op(P, i, streams[(size_t)lane])) return s;
    if (cudaEventRecord(P->ev[(size_t)i], streams[(size_t)lane]) != cudaSuccess)
      return set_error(DDQ_ECUDA, "prepare: event record");
    lane_of[(size_t)i] = lane;
    tail[(size_t)lane] = i;
  }
  for (size_t l = 1; l < streams.size(); l++)
    if (tail[l] >= 0 && cudaStreamWaitEvent(st, P->ev[(size_t)tail[l]], 0) != cudaSuccess)
      return set_error(DDQ_ECUDA, "prepare: join");
  return DDQ_OK;
}

void count_accesses(ddq_db* db, const ddq_op& op) {
  auto touch = [&](int c) {
    if (c < 0 || c >= (int)db->cols.size()) return;
    db->cols[(size_t)c]->access++;
    db->cols[(size_t)c]->last_access = ++db->clock;
  };
  switch (op.kind) {
    case DDQ_OP_SELECT:
      for (int i = 0; i < op.n_preds; i++) touch(op.preds[i].column);
      break;
    case DDQ_OP_HASH_BUILD:
      touch(op.key_col);
      touch(op.payload_col);
      for (int i = 0; i < op.n_preds; i++) touch(op.preds[i].column);
      break;
    case DDQ_OP_HASH_PROBE: touch(op.fk_col); break;
    case DDQ_OP_GATHER: touch(op.gather_col); break;
    case DDQ_OP_STAR:
      for (int j = 0; j < op.n_terms; j++) touch(op.term_kind[j] == DDQ_TERM_PRED ? op.preds[j].column : op.term_fk[j]);
      break;
    case DDQ_OP_AGGREGATE:
      for (int i = 0; i < op.n_preds; i++) touch(op.preds[i].column);  // fused selection
      for (int j = 0; j < op.n_terms && j < 4; j++) touch(op.term_fk[j]);  // fused probe terms
      for (int k = 0; k < op.n_keys; k++)
        if (op.key_src[k] < -1) touch(-2 - op.key_src[k]);
      for (int a = 0; a < op.n_aggs; a++) {
        int need = op.agg_kind[a] == DDQ_AGG_COUNT ? 0 : (op.agg_kind[a] == DDQ_AGG_SUM || op.agg_kind[a] == DDQ_AGG_MIN) ? 1
                 : op.agg_kind[a] == DDQ_AGG_SUM_MUL_100M_100P ? 3 : 2;
        for (int j = 0; j < need; j++) touch(op.agg_col[a][j]);
      }
      break;
  }
}

}  // namespace ddq

extern "C" {

// Data-driven placement for the hot path: every input column must be
// cached on this GPU; run once with worst-case capacities to learn the exact
// intermediate cardinalities (run-time placement knows them), then
// allocate exactly and capture the operator sequence into one CUDA graph.
ddq_status ddq_prepare(ddq_db* db, const ddq_plan* plan, int32_t use_graph, ddq_prepared** out) {
  if (!db || !out) return set_error(DDQ_EINVAL, "prepare: null argument");
  if (ddq_status s = validate_plan(db, plan)) return s;
  cudaSetDevice(db->device);
  auto P = std::make_unique<ddq_prepared>();
  P->db = db;
  P->plan = *plan;
  P->use_graph = use_graph != 0;
  {  // data-driven placement: every input column resident; pin them
    std::vector<int> cols;
    for (int i = 0; i < plan->n_ops; i++)
      for (int c : op_columns(plan->ops[i])) cols.push_back(c);
    std::lock_guard<std::mutex> g(db->mu);
    for (int c : cols) {
      const Column* col = col_of(db, c);
      if (!col || !col->dev || col->evict_pending)
        return set_error(DDQ_ESTATE, "prepare: an input column is not cached on the GPU (data-driven placement)");
    }
    for (int c : cols) db->cols[(size_t)c]->refs++;
    P->held = std::move(cols);
  }
  cudaStream_t st;
  if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess) {
    release_column_refs(db, P->held);
    return set_error(DDQ_ECUDA, "prepare: stream");
  }
  P->cap_stream = st;
  auto fail = [&](ddq_status s) {
    free_inters(db, P->inters);
    cudaStreamDestroy(st);
    P->cap_stream = nullptr;
    release_column_refs(db, P->held);
    return s;
  };
  // 1. calibration run (worst-case capacities) -> exact counts
  std::vector<int64_t> counts((size_t)plan->n_ops, -1);
  // per build op: its join index's key range (>= 0) or hash table capacity (-2 - cap)
  std::vector<int64_t> build_tab((size_t)plan->n_ops, -1);
  {
    std::vector<Inter> cal((size_t)plan->n_ops);
    GpuOpCtx ctx{db, st, &cal};
    ctx.count_column_access = false;
    uint32_t err = 0;
    for (int i = 0; i < plan->n_ops; i++) {
      ddq_status s = run_gpu_op(ctx, plan->ops[i], cal[(size_t)i]);
      if (s != DDQ_OK) {
        free_inters(db, cal);
        return fail(s == DDQ_ENOMEM_DEVICE ? set_error(s, "prepare: device heap exhausted (calibration)") : s);
      }
      if (plan->ops[i].kind == DDQ_OP_HASH_BUILD)
        build_tab[(size_t)i] = cal[(size_t)i].jidx ? (int64_t)cal[(size_t)i].jrange
                                                   : -2 - (int64_t)cal[(size_t)i].table_cap;
      if (cal[(size_t)i].d_count && plan->ops[i].kind != DDQ_OP_GATHER) {
        uint32_t c = 0;
        cudaMemcpyAsync(&c, cal[(size_t)i].d_count, 4, cudaMemcpyDeviceToHost, st);
        cudaError_t e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) {
          free_inters(db, cal);
          return fail(cuda_status(e, "prepare: calibration"));
        }
        counts[(size_t)i] = c;
      }
    }
    for (auto& x : cal)
      if (x.d_error) {
        uint32_t e2 = 0;
        cudaMemcpy(&e2, x.d_error, 4, cudaMemcpyDeviceToHost);
        err = std::max(err, e2);
      }
    free_inters(db, cal);
    if (err == 1 || err == 3) return fail(set_error(DDQ_EINVAL, "prepare: duplicate or invalid build key"));
    if (err) return fail(set_error(DDQ_EOVERFLOW, "prepare: hash table overflow"));
  }
  // 2. exact capacities, allocate, eager run
  P->forced.assign((size_t)plan->n_ops, -1);
  for (int i = 0; i < plan->n_ops; i++) {
    const ddq_op& op = plan->ops[i];
    if (op.kind == DDQ_OP_HASH_BUILD && op.input >= 0) P->forced[(size_t)i] = counts[(size_t)op.input];
    if (op.kind == DDQ_OP_SELECT || op.kind == DDQ_OP_HASH_PROBE || op.kind == DDQ_OP_STAR ||
        op.kind == DDQ_OP_FILTER_EQ)
      P->forced[(size_t)i] = counts[(size_t)i] + counts[(size_t)i] / 64 + 256;
  }
  // a dense semi-join probe (no payload) keeping >= 1/8 of the rows, whose consumers
  // are all probes of a key column, hands them a row bitmap (N/8 bytes) instead of a
  // TID list; they stream their key column masked by it (a gather at that density
  // touches nearly every sector anyway).  Sparser outputs stay TID lists: a bitmap
  // consumer pays for every row.
  P->bits_out.assign((size_t)plan->n_ops, 0);
  {
    static const char* env = getenv("DDQ_ROW_BITMAPS");  // "0": TID lists only
    const bool allow = !env || env[0] != '0';
    for (int i = 0; i < plan->n_ops && allow; i++) {
      const ddq_op& op = plan->ops[i];
      const bool sel1 = op.kind == DDQ_OP_SELECT && op.input < 0 && op.n_preds == 1 && [&] {
        const Column* c = col_of(db, op.preds[0].column);
        return c && c->width == 4;
      }();  // a dense selection on one int32 column (TPC-H Q3's l_shipdate)
      if (!sel1 && (op.kind != DDQ_OP_HASH_PROBE || op.input >= 0 || op.emit_payload || op.fk_vec > 0)) continue;
      int consumers = 0;
      bool ok = true;
      for (int j = i + 1; j < plan->n_ops; j++) {
        const ddq_op& c = plan->ops[j];
        if (c.input != i) continue;
        consumers++;
        // consumers that emit payloads too: over the bitmap they do the probe work for
        // every row (opprofile SF20: Q3.1's s_nation probe 109 -> 160 us), but the
        // producer no longer compacts 24 M TIDs through its ring (152 -> 84 us), and the
        // 4-stream step drops 2.67 -> 2.60 ms (Q3.1, Q4.2)
        ok = ok && c.kind == DDQ_OP_HASH_PROBE && c.fk_vec <= 0;
        // ... (round 2, final session) wherever its table lives: a masked probe of a
        // join index in L2 looks up its live rows only (dense.cu), so the producer
        // writes its bitmap at the kOutBits rate instead of compacting >= 1/8 of the
        // rows into a TID list.  DDQ_MASKED_GLOBAL=0: only consumers whose table the
        // masked probe stages in shared memory (the earlier rule; SF80-SF160 dims and
        // SF100: customer's join index no longer fits one SM)
        static const char* mg_env = getenv("DDQ_MASKED_GLOBAL");
        const bool masked_global = !(mg_env && mg_env[0] == '0');
        if (ok && !masked_global && c.build >= 0 && c.build < plan->n_ops) {
          const int64_t bt = build_tab[(size_t)c.build];
          const int64_t rows_c = db->tables[(size_t)c.table].n_rows;
          ok = bt >= 0 ? ws_masked_probe_smem(true, (uint32_t)bt, rows_c, c.emit_payload != 0)
                       : (bt <= -2 && ws_masked_probe_smem(false, (uint32_t)(-2 - bt), rows_c, c.emit_payload != 0));
        }
      }
      const int64_t rows = db->tables[(size_t)op.table].n_rows;
      const bool dense_enough = counts[(size_t)i] >= 0 && counts[(size_t)i] * 8 >= rows;
      P->bits_out[(size_t)i] = (ok && consumers > 0 && dense_enough) ? 1 : 0;
    }
  }
  P->inters.resize((size_t)plan->n_ops);
  fill_hoist().rec = &P->fills;  // record every buffer initialisation of the eager run
  for (int i = 0; i < plan->n_ops; i++) {
    GpuOpCtx ctx{db, st, &P->inters};
    ctx.forced_cap = P->forced[(size_t)i];
    ctx.count_column_access = false;
    ctx.bits_out = P->bits_out[(size_t)i] != 0;
    ctx.dist = true;
    ddq_status s = run_gpu_op(ctx, plan->ops[i], P->inters[(size_t)i]);
    if (s != DDQ_OK) {
      fill_hoist().rec = nullptr;
      return fail(s == DDQ_ENOMEM_DEVICE ? set_error(s, "prepare: device heap exhausted") : s);
    }
    P->kernels += kernels_of(plan->ops[i]);
  }
  fill_hoist().rec = nullptr;
  cudaError_t e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return fail(cuda_status(e, "prepare: eager run"));
  // 3. capture the same launches on the same buffers into one CUDA graph
  if (P->use_graph) {
    e = cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
    if (e != cudaSuccess) return fail(cuda_status(e, "prepare: begin capture"));
    static const char* env = getenv("DDQ_GRAPH_BRANCHES");  // "0": one serial chain
    // multi-GPU build broadcasts: one collective order on every rank -> serial capture
    const bool branches = (!env || env[0] != '0') && !dist_serial_capture(db);
    // all buffer initialisations as ONE fill kernel at the graph root; the
    // operators' own fills are skipped while capturing
    ddq_status s = DDQ_OK;
    if (branches) {
      if (launch_multi_fill(P->fills, st) != cudaSuccess) s = set_error(DDQ_ECUDA, "prepare: fill");
      fill_hoist().skip = true;
    }
    if (s == DDQ_OK) s = branches ? replay_branches(P.get(), st) : replay(P.get(), st);
    fill_hoist().skip = false;
    if (branches) P->kernels += (int)((P->fills.size() + 47) / 48);
    cudaGraph_t g = nullptr;
    e = cudaStreamEndCapture(st, &g);
    if (s != DDQ_OK || e != cudaSuccess) {
      if (g) cudaGraphDestroy(g);
      return fail(s != DDQ_OK ? s : cuda_status(e, "prepare: end capture"));
    }
    P->graph = g;
    e = cudaGraphInstantiate(&P->exec, g, 0);
    if (e != cudaSuccess) return fail(cuda_status(e, "prepare: instantiate"));
  }
  *out = P.release();
  return DDQ_OK;
}

ddq_status ddq_prepared_launch(ddq_prepared* p, void* stream) {
  if (!p) return set_error(DDQ_EINVAL, "prepared_launch: null");
  cudaStream_t st = (cudaStream_t)stream;
  // column access counts (LFU statistics)
  for (int i = 0; i < p->plan.n_ops; i++) count_accesses(p->db, p->plan.ops[i]);
  p->db->stats.gpu_ops += (uint64_t)p->plan.n_ops;
  if (p->use_graph) return cuda_status(cudaGraphLaunch(p->exec, st), "prepared_launch");
  return replay(p, st);
}

int32_t ddq_prepared_kernel_count(ddq_prepared* p) { return p ? p->kernels : 0; }

static double sector_bytes(double N, double m, int w) {
  if (N <= 0 || m <= 0) return 0;
  double rho = std::min(1.0, m / N);
  return N * w * (1.0 - std::pow(1.0 - rho, 32.0 / w));
}

int32_t ddq_prepared_profile(ddq_prepared* p, void* stream, int32_t max_ops, float* op_ms, double* op_bytes,
                             int32_t* op_class) {
  if (!p) return set_error(DDQ_EINVAL, "prepared_profile: null");
  cudaStream_t st = (cudaStream_t)stream;
  const int n = p->plan.n_ops;
  std::vector<cudaEvent_t> ev((size_t)n + 1);
  for (auto& e : ev) cudaEventCreate(&e);
  // the operators are enqueued behind a device-side delay (longer than their host
  // set-up and launches take), so each event pair brackets device time only
  launch_delay((uint64_t)(500 + 100 * n) * 1000, st);
  cudaEventRecord(ev[0], st);
  for (int i = 0; i < n; i++) {
    std::vector<void*> blocks = p->inters[(size_t)i].heap_blocks;
    GpuOpCtx ctx{p->db, st, &p->inters};
    ctx.forced_cap = p->forced[(size_t)i];
    ctx.count_column_access = false;
    ctx.reuse = &blocks;
    ctx.bits_out = p->bits_out[(size_t)i] != 0;
    ctx.dist = true;
    ddq_status s = run_gpu_op(ctx, p->plan.ops[i], p->inters[(size_t)i]);
    if (s != DDQ_OK) {
      for (auto& e : ev) cudaEventDestroy(e);
      return s;
    }
    cudaEventRecord(ev[(size_t)i + 1], st);
  }
  cudaError_t e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) {
    for (auto& x : ev) cudaEventDestroy(x);
    return cuda_status(e, "prepared_profile");
  }
  std::vector<int64_t> cnt((size_t)n, -1);
  for (int i = 0; i < n; i++)
    if (p->inters[(size_t)i].d_count) {
      uint32_t c = 0;
      cudaMemcpy(&c, p->inters[(size_t)i].d_count, 4, cudaMemcpyDeviceToHost);
      cnt[(size_t)i] = c;
    }
  auto width = [&](int c) { const Column* col = col_of(p->db, c); return col ? col->width : 4; };
  for (int i = 0; i < n && i < max_ops; i++) {
    const ddq_op& op = p->plan.ops[i];
    const Inter& o = p->inters[(size_t)i];
    const double N = (double)p->db->tables[(size_t)op.table].n_rows;
    const double m = op.input >= 0 ? (double)cnt[(size_t)op.input] : N;
    const double out = cnt[(size_t)i] >= 0 ? (double)cnt[(size_t)i] : 0;
    const int nvec_in = op.input >= 0 ? (int)p->inters[(size_t)op.input].vecs.size() : 0;
    double bytes = 0;
    int cls = 0;
    float ms = 0;
    cudaEventElapsedTime(&ms, ev[(size_t)i], ev[(size_t)i + 1]);
    switch (op.kind) {
      case DDQ_OP_SELECT:
      case DDQ_OP_HASH_PROBE: {
        std::vector<int> cols;
        if (op.kind == DDQ_OP_SELECT)
          for (int k = 0; k < op.n_preds; k++) cols.push_back(op.preds[k].column);
        else
          cols.push_back(op.fk_col);
        const int emit = op.kind == DDQ_OP_HASH_PROBE && op.emit_payload ? 1 : 0;
        const bool in_bits = op.input >= 0 && p->inters[(size_t)op.input].bits;
        if (op.input < 0) {
          cls = 0;
          for (int c : cols) bytes += N * width(c);
        } else {
          // a row-bitmap input streams the whole key column (class 5), a TID list gathers
          cls = in_bits ? 5 : 1;
          bytes += in_bits ? N / 8 : m * 4;  // the input: a row bitmap or a TID list
          // a conjunction reads its first column at every input TID and the
          // others only at rows still alive (counted at the final survivors: a
          // lower bound, intermediate counts are not kept)
          for (size_t k = 0; k < cols.size(); k++) bytes += sector_bytes(N, k == 0 ? m : out, width(cols[k]));
          bytes += out * 4 * nvec_in;  // carried vectors read at survivors
        }
        bytes += o.bits ? N / 8 : out * 4 * (1 + nvec_in + emit);  // row bitmap or TIDs + vectors
      } break;
      case DDQ_OP_STAR: {
        cls = 0;
        int emit = 0;
        for (int j = 0; j < op.n_terms; j++) {
          bytes += N * (op.term_kind[j] == DDQ_TERM_PRED ? width(op.preds[j].column) : 4);
          emit += op.term_kind[j] == DDQ_TERM_PROBE && op.term_emit[j] ? 1 : 0;
        }
        bytes += out * 4 * (1 + emit);
      } break;
      case DDQ_OP_FILTER_EQ:
        cls = 1;
        bytes = m * 4 + m * 8 + out * 4 * (1 + 2 * nvec_in);
        break;
      case DDQ_OP_HASH_BUILD:
        cls = 2;
        bytes = m * 4 * (op.payload_col >= 0 ? 2 : 1) + (double)o.table_cap * 8 * 2;
        for (int k = 0; k < op.n_preds; k++) bytes += m * width(op.preds[k].column);  // fused selection
        break;
      case DDQ_OP_GATHER:
        cls = op.fetch_build > 0 ? 1 : 3;  // a fetch is an at-TIDs lookup like a probe
        bytes = m * 4 + sector_bytes(N, m, width(op.gather_col)) + m * (op.fetch_build > 0 ? 4 : width(op.gather_col));
        break;
      case DDQ_OP_AGGREGATE: {
        cls = 4;
        bytes = op.input >= 0 ? m * 4 : 0;  // the input TID list (none over all rows)
        // fused selection: first predicate column at every input TID, the rest
        // and everything below at the rows that passed (d_rows)
        double mr = m;
        if ((op.n_preds > 0 || op.n_terms > 0) && o.d_rows) {
          uint32_t r = 0;
          cudaMemcpy(&r, o.d_rows, 4, cudaMemcpyDeviceToHost);
          mr = r;
          for (int k = 0; k < op.n_preds; k++) bytes += sector_bytes(N, k == 0 ? m : mr, width(op.preds[k].column));
          // fused probe / fetch terms (O37): the first term's fk at every input row that
          // passed the predicates, later ones at least at the final rows (a lower bound)
          for (int j = 0; j < op.n_terms && j < 4; j++)
            bytes += sector_bytes(N, j == 0 && op.n_preds == 0 ? m : mr, 4);
        }
        for (int k = 0; k < op.n_keys; k++) bytes += op.key_src[k] >= 0 ? m * 4 : sector_bytes(N, mr, 4);
        std::vector<int> seen;
        for (int a = 0; a < op.n_aggs; a++)
          for (int j = 0; j < 3; j++) {
            int c = op.agg_col[a][j];
            if (c < 0 || std::find(seen.begin(), seen.end(), c) != seen.end()) continue;
            int need = op.agg_kind[a] == DDQ_AGG_COUNT ? 0 : (op.agg_kind[a] == DDQ_AGG_SUM || op.agg_kind[a] == DDQ_AGG_MIN) ? 1
                     : op.agg_kind[a] == DDQ_AGG_SUM_MUL_100M_100P ? 3 : 2;
            if (j >= need) continue;
            seen.push_back(c);
            bytes += sector_bytes(N, mr, width(c));
          }
      } break;
    }
    if (op_ms) op_ms[i] = ms;
    if (op_bytes) op_bytes[i] = bytes;
    if (op_class) op_class[i] = cls;
  }
  for (auto& x : ev) cudaEventDestroy(x);
  return n;
}

int64_t ddq_prepared_group_capacity(ddq_prepared* p) {
  if (!p) return 0;
  const Inter& r = p->inters.back();
  return r.gb_cap ? (int64_t)r.gb_cap : r.cap;
}

static ddq_status check_errors(ddq_prepared* p, cudaStream_t st) {
  uint32_t err = 0;
  for (auto& x : p->inters)
    if (x.d_error) {
      uint32_t e2 = 0;
      cudaMemcpyAsync(&e2, x.d_error, 4, cudaMemcpyDeviceToHost, st);
      cudaError_t e = cudaStreamSynchronize(st);
      if (e != cudaSuccess) return cuda_status(e, "prepared: error cell");
      err = std::max(err, e2);
    }
  if (err == 1 || err == 3) return set_error(DDQ_EINVAL, "duplicate or invalid build key");
  if (err == 4) return set_error(DDQ_EOVERFLOW, "intermediate exceeded its prepared capacity (data changed?)");
  if (err) return set_error(DDQ_EOVERFLOW, "hash table overflow");
  return DDQ_OK;
}

ddq_status ddq_prepared_partials(ddq_prepared* p, void* stream, int64_t* h_n_groups, int64_t* h_keys,
                                 int64_t* h_accs, int64_t cap) {
  if (!p || !h_n_groups) return set_error(DDQ_EINVAL, "prepared_partials: null");
  cudaStream_t st = (cudaStream_t)stream;
  const Inter& r = p->inters.back();
  if (!r.gb_table) return set_error(DDQ_ESTATE, "prepared_partials: root is not an aggregate");
  if (ddq_status s = check_errors(p, st)) return s;
  uint32_t g = 0;
  uint64_t t0 = now_ns();
  cudaMemcpyAsync(&g, r.gb_groups, 4, cudaMemcpyDeviceToHost, st);
  cudaError_t e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_status(e, "prepared_partials");
  if ((int64_t)g > cap) return set_error(DDQ_EINVAL, "prepared_partials: buffer too small");
  const int na = p->plan.ops[p->plan.n_ops - 1].n_aggs;
  if (g) {
    cudaMemcpyAsync(h_keys, r.gb_keys, (size_t)g * 8, cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(h_accs, r.gb_accs, (size_t)g * na * 16, cudaMemcpyDeviceToHost, st);
    e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_status(e, "prepared_partials copy");
  }
  p->db->stats.d2h_bytes += 4 + (uint64_t)g * (8 + 16 * na);
  p->db->stats.d2h_ns += now_ns() - t0;
  *h_n_groups = g;
  return DDQ_OK;
}

ddq_status ddq_prepared_partials_device(ddq_prepared* p, int64_t** keys, int64_t** accs, uint32_t** count,
                                        int64_t* cap);
}  // extern "C"
namespace ddq {
const ddq_plan& prepared_plan(const ddq_prepared* p) { return p->plan; }
ddq_status prepared_partials_device(ddq_prepared* p, int64_t** keys, int64_t** accs, uint32_t** count, int64_t* cap) {
  return ddq_prepared_partials_device(p, keys, accs, count, cap);
}
}  // namespace ddq
extern "C" {
ddq_status ddq_prepared_partials_device(ddq_prepared* p, int64_t** keys, int64_t** accs, uint32_t** count,
                                        int64_t* cap) {
  if (!p || !keys || !accs || !count || !cap) return set_error(DDQ_EINVAL, "prepared_partials_device: null");
  const Inter& r = p->inters.back();
  if (!r.gb_table) return set_error(DDQ_ESTATE, "prepared_partials_device: root is not an aggregate");
  *keys = r.gb_keys;
  *accs = r.gb_accs;
  *count = r.gb_groups;
  *cap = r.gb_cap;
  return DDQ_OK;
}

ddq_status ddq_finalize_partials(const ddq_op* root, int64_t n, const int64_t* keys, const int64_t* accs,
                                 ddq_result** out) {
  if (!root || !out || n < 0 || (n > 0 && (!keys || !accs))) return set_error(DDQ_EINVAL, "finalize_partials");
  if (root->kind != DDQ_OP_AGGREGATE || root->n_aggs < 1 || root->n_aggs > DDQ_MAX_AGGS ||
      root->n_keys < 0 || root->n_keys > DDQ_MAX_KEYS)
    return set_error(DDQ_EINVAL, "finalize_partials: root must be an AGGREGATE");
  return finalize_result(*root, n, keys, accs, out);
}

ddq_status ddq_prepared_finalize(ddq_prepared* p, int64_t n_groups, const int64_t* h_keys, const int64_t* h_accs,
                                 ddq_result** out) {
  if (!p || !out) return set_error(DDQ_EINVAL, "prepared_finalize: null");
  ddq_status s = finalize_result(p->plan.ops[p->plan.n_ops - 1], n_groups, h_keys, h_accs, out);
  if (s == DDQ_OK) decode_result_keys(p->db, p->plan, *out);
  return s;
}

ddq_status ddq_prepared_fetch(ddq_prepared* p, void* stream, ddq_result** out) {
  if (!p || !out) return set_error(DDQ_EINVAL, "prepared_fetch: null");
  cudaStream_t st = (cudaStream_t)stream;
  const ddq_op& root = p->plan.ops[p->plan.n_ops - 1];
  const Inter& r = p->inters.back();
  if (root.kind != DDQ_OP_AGGREGATE) {  // select-* root: return the TID list
    if (ddq_status s = check_errors(p, st)) return s;
    uint32_t n = 0;
    cudaMemcpyAsync(&n, r.d_count, 4, cudaMemcpyDeviceToHost, st);
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_status(e, "prepared_fetch");
    ddq_result* res = new ddq_result();
    std::memset(res, 0, sizeof(*res));
    int32_t* t = new int32_t[std::max<uint32_t>(n, 1)];
    if (n) cudaMemcpyAsync(t, r.tids, (size_t)n * 4, cudaMemcpyDeviceToHost, st);
    e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) {
      delete[] t;
      delete res;
      return cuda_status(e, "prepared_fetch tids");
    }
    // a select-* result is a set of rows; present it in row order (S8(a7))
    std::sort(t, t + n);
    const int64_t base = p->db->tables[(size_t)root.table].row_begin;
    for (uint32_t i = 0; i < n; i++) t[i] = (int32_t)(t[i] + base);
    res->n_tids = n;
    res->tids = t;
    res->gpu_ops = p->plan.n_ops;
    *out = res;
    return DDQ_OK;
  }
  const int na = root.n_aggs;
  std::vector<int64_t> keys(r.gb_cap), accs((size_t)r.gb_cap * na * 2);
  int64_t g = 0;
  if (ddq_status s = ddq_prepared_partials(p, stream, &g, keys.data(), accs.data(), r.gb_cap)) return s;
  ddq_status s = finalize_result(root, g, keys.data(), accs.data(), out, true);
  if (s == DDQ_OK) {
    (*out)->gpu_ops = p->plan.n_ops;
    decode_result_keys(p->db, p->plan, *out);
  }
  return s;
}

void ddq_prepared_free(ddq_prepared* p) {
  if (!p) return;
  if (p->cap_stream) cudaStreamSynchronize(p->cap_stream);
  if (p->exec) cudaGraphExecDestroy(p->exec);
  if (p->graph) cudaGraphDestroy(p->graph);
  free_inters(p->db, p->inters);
  release_column_refs(p->db, p->held);
  if (p->cap_stream) cudaStreamDestroy(p->cap_stream);
  for (cudaStream_t s2 : p->side) cudaStreamDestroy(s2);
  for (cudaEvent_t e : p->ev) cudaEventDestroy(e);
  delete p;
}

}  // extern "C"
