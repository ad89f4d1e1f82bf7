// driver.cpp -- the paper's execution policy around the operators:
//   * query chopping (Sec. 5.1-5.2): the leaf operators of every
//     submitted query enter a global operator stream; each processor has a ready
//     queue served by a bounded pool of worker threads that PULL operators; a
//     finished operator notifies its parent, which enqueues itself once all its
//     children are done (Fig. 11);
//   * run-time data-driven placement (Sec. 3.1, Sec. 3.3
//     Sec. 5.4): an operator goes to the GPU iff all its input columns are cached
//     there and all its child intermediates live there; otherwise to the host;
//   * abort and restart (Sec. 2.5.1, Sec. 4.1): a GPU operator
//     whose heap allocation fails aborts at once (no wait-and-admit), its
//     begin->abort time is counted as wasted time, and it is restarted on
//     the host; its successors follow the data to the host;
//   * the comparison arms of Sec. 6.2: GPU-only with operator-driven data
//     placement (inputs copied on demand, LRU), compile-time placement (chopping=0:
//     placement fixed at submit, no concurrency bound), and CPU-only.
// The host executor (run_host_op) is the CPU fallback handler that exists for
// every operator.  It is product code and shares nothing with oracle/.
#include <algorithm>
#include <array>
#include <cstring>
#include <numeric>
#include <unordered_map>

#include "engine.h"
#include "ops_internal.h"

namespace ddq {

ddq_status cache_column_locked(ddq_db* db, int c, bool on_demand, std::unique_lock<std::mutex>& lk);
void evict_column_locked(ddq_db* db, int c);
ddq_status validate_plan_public(ddq_db* db, const ddq_plan* plan);

enum Place { P_NONE = 0, P_GPU = 1, P_HOST = 2 };

struct QueryState {
  int64_t id = 0;
  ddq_plan plan{};
  std::vector<Inter> inters;
  std::vector<int> pending;                 // unfinished children per op
  std::vector<std::vector<int>> parents;
  std::vector<int> place;                   // compile-time placement (chopping=0)
  std::vector<int> consumers_left;          // for freeing intermediates early
  int ops_left = 0;
  int inflight = 0;          // operators of this query a worker is running right now
  bool failed = false;       // an operator failed: remaining ops are dropped
  bool released = false;     // intermediates of a failed query freed (once, at inflight == 0)
  bool done = false;
  ddq_status status = DDQ_OK;
  std::string error;
  ddq_result* result = nullptr;
  uint64_t t_submit = 0, t_done = 0;
  int gpu_ops = 0, host_ops = 0, aborts = 0;
  std::vector<uint8_t> trace;               // per op: DDQ_RAN_GPU / _HOST / _ABORTED
  std::vector<float> op_ms;                 // per op: wall time from pull to completion
  std::vector<uint64_t> op_t0;
  std::mutex mu;
  std::condition_variable cv;
};

// ------------------------------------------------------------ column helpers
std::vector<int> op_columns(const ddq_op& op) {
  std::vector<int> c;
  switch (op.kind) {
    case DDQ_OP_SELECT:
      for (int i = 0; i < op.n_preds; i++) c.push_back(op.preds[i].column);
      break;
    case DDQ_OP_HASH_BUILD:
      c.push_back(op.key_col);
      if (op.payload_col >= 0) c.push_back(op.payload_col);
      for (int i = 0; i < op.n_preds; i++) c.push_back(op.preds[i].column);  // fused selection
      break;
    case DDQ_OP_HASH_PROBE:
      if (op.fk_vec <= 0) c.push_back(op.fk_col);
      break;
    case DDQ_OP_FILTER_EQ: break;
    case DDQ_OP_STAR:
      for (int j = 0; j < op.n_terms && j < 4; j++)
        c.push_back(op.term_kind[j] == DDQ_TERM_PRED ? op.preds[j].column : op.term_fk[j]);
      break;
    case DDQ_OP_GATHER: c.push_back(op.gather_col); break;
    case DDQ_OP_AGGREGATE:
      for (int i = 0; i < op.n_preds; i++) c.push_back(op.preds[i].column);  // fused selection
      for (int j = 0; j < op.n_terms && j < 4; j++) c.push_back(op.term_fk[j]);  // fused probe terms (O37)
      for (int k = 0; k < op.n_keys; k++)
        if (op.key_src[k] < -1) c.push_back(-2 - op.key_src[k]);
      for (int a = 0; a < op.n_aggs; a++) {
        int need = op.agg_kind[a] == DDQ_AGG_COUNT ? 0 : (op.agg_kind[a] == DDQ_AGG_SUM || op.agg_kind[a] == DDQ_AGG_MIN) ? 1
                 : op.agg_kind[a] == DDQ_AGG_SUM_MUL_100M_100P ? 3 : 2;
        for (int j = 0; j < need; j++)
          if (op.agg_col[a][j] >= 0) c.push_back(op.agg_col[a][j]);  // <= -2: an aligned vector
      }
      break;
  }
  return c;
}

static std::vector<int> op_children(const ddq_op& op) {
  std::vector<int> ch;
  if (op.input >= 0) ch.push_back(op.input);
  if (op.kind == DDQ_OP_HASH_PROBE && op.build >= 0 && op.build != op.input) ch.push_back(op.build);
  if (op.kind == DDQ_OP_GATHER && op.fetch_build > 0 && op.fetch_build - 1 != op.input)
    ch.push_back(op.fetch_build - 1);
  if (op.kind == DDQ_OP_STAR || op.kind == DDQ_OP_AGGREGATE)
    for (int j = 0; j < op.n_terms && j < 4; j++)
      if ((op.term_kind[j] == DDQ_TERM_PROBE || op.term_kind[j] == DDQ_TERM_FETCH) &&
          std::find(ch.begin(), ch.end(), op.term_build[j]) == ch.end())
        ch.push_back(op.term_build[j]);
  return ch;
}

// ------------------------------------------------------------ transfers
static void* host_alloc(Inter& x, size_t bytes) {
  void* p = std::malloc(std::max<size_t>(bytes, 8));
  if (p) x.host_blocks.push_back(p);
  return p;
}

// Move an intermediate to host memory (D2H; counted as GPU->CPU transfer).
ddq_status inter_to_host(ddq_db* db, Inter& x, cudaStream_t st) {
  if (x.on_host) return DDQ_OK;
  Inter h;
  h.on_host = true;
  h.table = x.table;
  uint64_t t0 = now_ns();
  uint64_t bytes = 0;
  if (x.table_ptr) {
    auto t = std::make_shared<std::vector<uint64_t>>(x.table_cap);
    cudaMemcpyAsync(t->data(), x.table_ptr, (size_t)x.table_cap * 8, cudaMemcpyDeviceToHost, st);
    h.host_table = t;
    h.table_cap = x.table_cap;
    bytes += (uint64_t)x.table_cap * 8;
  }
  if (x.jidx) {
    const size_t words = ((size_t)x.jrange + 31) / 32;
    auto bm = std::make_shared<std::vector<uint32_t>>(words);
    auto pa = std::make_shared<std::vector<int32_t>>(x.jrange);
    cudaMemcpyAsync(bm->data(), x.jidx, words * 4, cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(pa->data(), join_index_payload(x.jidx, x.jrange), (size_t)x.jrange * 4,
                    cudaMemcpyDeviceToHost, st);
    h.h_bitmap = bm;
    h.h_payarr = pa;
    h.jmin = x.jmin;
    h.jrange = x.jrange;
    bytes += words * 4 + (uint64_t)x.jrange * 4;
  }
  if (x.gb_table) {
    // aggregate outputs are consumed by finalisation only
    return set_error(DDQ_ESTATE, "aggregate output cannot move");
  }
  if (x.tids || x.d_count) {
    uint32_t n = 0;
    cudaMemcpyAsync(&n, x.d_count, 4, cudaMemcpyDeviceToHost, st);
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_status(e, "inter_to_host count");
    h.count = n;
    h.cap = n;
    h.tids = (int32_t*)host_alloc(h, (size_t)n * 4);
    if (!h.tids) return set_error(DDQ_ENOMEM_HOST, "inter_to_host");
    if (n) cudaMemcpyAsync(h.tids, x.tids, (size_t)n * 4, cudaMemcpyDeviceToHost, st);
    bytes += (uint64_t)n * 4;
    for (const Vec& v : x.vecs) {
      void* p = host_alloc(h, (size_t)n * v.width);
      if (!p) return set_error(DDQ_ENOMEM_HOST, "inter_to_host");
      if (n) cudaMemcpyAsync(p, v.ptr, (size_t)n * v.width, cudaMemcpyDeviceToHost, st);
      h.vecs.push_back(Vec{p, v.width, true});
      bytes += (uint64_t)n * v.width;
    }
  }
  cudaError_t e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_status(e, "inter_to_host");
  db->stats.d2h_bytes += bytes;
  db->stats.d2h_ns += now_ns() - t0;
  release_inter(db, x);
  x = std::move(h);
  return DDQ_OK;
}

// Move a host intermediate to the device heap (H2D; CPU->GPU transfer).
// Returns DDQ_ENOMEM_DEVICE if the heap cannot hold it (-> abort).
static ddq_status inter_to_device(ddq_db* db, Inter& x, cudaStream_t st) {
  if (!x.on_host) return DDQ_OK;
  Inter d;
  d.table = x.table;
  uint64_t t0 = now_ns(), bytes = 0;
  auto get = [&](uint64_t b) -> void* {
    void* p = db->heap.try_alloc(b);
    if (p) d.heap_blocks.push_back(p);
    return p;
  };
  if (x.h_bitmap) {
    d.jmin = x.jmin;
    d.jrange = x.jrange;
    d.jidx = get(join_index_bytes(x.jrange));
    d.d_error = (uint32_t*)get(64);
    if (!d.jidx || !d.d_error) {
      release_inter(db, d);
      return DDQ_ENOMEM_DEVICE;
    }
    cudaMemsetAsync(d.d_error, 0, 4, st);
    cudaMemcpyAsync(d.jidx, x.h_bitmap->data(), x.h_bitmap->size() * 4, cudaMemcpyHostToDevice, st);
    cudaMemcpyAsync(join_index_payload(d.jidx, d.jrange), x.h_payarr->data(), (size_t)x.jrange * 4,
                    cudaMemcpyHostToDevice, st);
    bytes += x.h_bitmap->size() * 4 + (uint64_t)x.jrange * 4;
    if (join_index_cg(x.jrange)) {  // derived from the membership bits (a host-built index)
      std::vector<uint32_t> co(join_index_coarse_bytes(x.jrange) / 4);
      join_index_coarse_host(x.h_bitmap->data(), x.jrange, co.data());
      cudaMemcpyAsync(join_index_coarse(d.jidx, d.jrange), co.data(), co.size() * 4, cudaMemcpyHostToDevice, st);
      cudaStreamSynchronize(st);  // `co` is a stack buffer
      bytes += co.size() * 4;
    }
  } else if (x.host_table) {
    d.table_cap = x.table_cap;
    d.table_ptr = (uint64_t*)get((uint64_t)x.table_cap * 8);
    d.d_error = (uint32_t*)get(64);
    if (!d.table_ptr || !d.d_error) {
      release_inter(db, d);
      return DDQ_ENOMEM_DEVICE;
    }
    cudaMemsetAsync(d.d_error, 0, 4, st);
    cudaMemcpyAsync(d.table_ptr, x.host_table->data(), (size_t)x.table_cap * 8, cudaMemcpyHostToDevice, st);
    bytes += (uint64_t)x.table_cap * 8;
  } else {
    int64_t n = x.count;
    d.cap = n;
    d.count = n;
    d.tids = (int32_t*)get((uint64_t)std::max<int64_t>(n, 1) * 4);
    d.d_count = (uint32_t*)get(64);
    d.d_error = (uint32_t*)get(64);
    for (const Vec& v : x.vecs) d.vecs.push_back(Vec{get((uint64_t)std::max<int64_t>(n, 1) * v.width), v.width, false});
    bool ok = d.tids && d.d_count && d.d_error;
    for (auto& v : d.vecs) ok = ok && v.ptr;
    if (!ok) {
      release_inter(db, d);
      return DDQ_ENOMEM_DEVICE;
    }
    uint32_t n32 = (uint32_t)n;
    cudaMemcpyAsync(d.d_count, &n32, 4, cudaMemcpyHostToDevice, st);
    cudaMemsetAsync(d.d_error, 0, 4, st);
    if (n) cudaMemcpyAsync(d.tids, x.tids, (size_t)n * 4, cudaMemcpyHostToDevice, st);
    for (size_t i = 0; i < x.vecs.size(); i++)
      if (n) cudaMemcpyAsync(d.vecs[i].ptr, x.vecs[i].ptr, (size_t)n * x.vecs[i].width, cudaMemcpyHostToDevice, st);
    bytes += (uint64_t)n * 4;
    for (auto& v : x.vecs) bytes += (uint64_t)n * v.width;
  }
  cudaError_t e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) {
    release_inter(db, d);
    return cuda_status(e, "inter_to_device");
  }
  db->stats.h2d_bytes += bytes;
  db->stats.h2d_ns += now_ns() - t0;
  release_inter(db, x);
  x = std::move(d);
  return DDQ_OK;
}

// ------------------------------------------------------------ host executor
static inline uint32_t host_hash32(int32_t k, int shift) { return ((uint32_t)k * 0x9E3779B1u) >> shift; }
static constexpr uint64_t kHostEmpty = 0x8000000000000000ull;

template <class F>
static void parallel_chunks(int64_t n, int threads, F f) {  // f(chunk, begin, end)
  if (threads <= 1 || n < (1 << 16)) {
    f(0, 0, n);
    return;
  }
  std::vector<std::thread> th;
  int64_t step = (n + threads - 1) / threads;
  for (int t = 0; t < threads; t++) {
    int64_t b = t * step, e = std::min<int64_t>(n, b + step);
    if (b >= e) break;
    th.emplace_back([=] { f(t, b, e); });
  }
  for (auto& x : th) x.join();
}

static int host_threads(ddq_db* db) {
  int hw = (int)std::thread::hardware_concurrency();
  int t = hw / std::max(1, db->cfg.host_workers);
  return std::max(1, t);
}

// one predicate of the plan IR on a host value (RANGE, IN, BITSET; include/ddq.h)
static inline bool host_pred(const ddq_pred& pr, int64_t v) {
  if (pr.kind == DDQ_PRED_RANGE) return v >= pr.lo && v <= pr.hi;
  if (pr.kind == DDQ_PRED_BITSET) {
    const uint64_t o = (uint64_t)(v - pr.lo);
    return o < 512 && (((uint64_t)pr.in_vals[o >> 6] >> (o & 63)) & 1);
  }
  bool m = false;
  for (int j = 0; j < pr.n_in && j < DDQ_MAX_IN; j++) m |= v == pr.in_vals[j];
  return m;
}

// Look key k up in a host-resident build (hash table or join index copy).
static bool host_lookup(const Inter& B, int32_t k, int32_t* v) {
  if (B.h_bitmap) {
    const uint32_t o = (uint32_t)(k - B.jmin);
    if (o < B.jrange && (((*B.h_bitmap)[o >> 5] >> (o & 31)) & 1u)) {
      *v = (*B.h_payarr)[o];
      return true;
    }
    return false;
  }
  int lg = 0;
  while ((1u << lg) < B.table_cap) lg++;
  uint32_t h = ((uint32_t)k * 0x9E3779B1u) >> (32 - lg);
  while (true) {
    const uint64_t sl = (*B.host_table)[h];
    if (sl == 0x8000000000000000ull) return false;
    if ((int32_t)(sl >> 32) == k) {
      *v = (int32_t)(uint32_t)sl;
      return true;
    }
    h = (h + 1) & (B.table_cap - 1);
  }
}

static inline int64_t hcol(const Column* c, int64_t r) {
  return c->width == 8 ? ((const int64_t*)c->host)[r] : (int64_t)((const int32_t*)c->host)[r];
}

ddq_status run_host_op(ddq_db* db, const ddq_op& op, const std::vector<Inter>& I, Inter& out) {
  out = Inter();
  out.on_host = true;
  out.table = op.table;
  const Table& T = db->tables[(size_t)op.table];
  const Inter* in = op.input >= 0 ? &I[(size_t)op.input] : nullptr;
  if (in && !in->on_host) return set_error(DDQ_ESTATE, "host op with a device-resident input");
  const int64_t n = in ? in->count : T.n_rows;
  auto row_of = [&](int64_t i) -> int32_t { return in ? in->tids[i] : (int32_t)i; };
  const int threads = host_threads(db);
  for (int c : op_columns(op)) {
    db->cols[(size_t)c]->access++;
    db->cols[(size_t)c]->last_access = ++db->clock;
  }
  switch (op.kind) {
    case DDQ_OP_STAR: {  // conjunction of predicates / probes over all rows
      struct HT {
        const Column* col;
        const Inter* b;
        int lg;
      };
      std::vector<HT> ts;
      int n_emit = 0;
      for (int j = 0; j < op.n_terms; j++) {
        HT h{nullptr, nullptr, 0};
        if (op.term_kind[j] == DDQ_TERM_PRED) {
          h.col = col_of(db, op.preds[j].column);
        } else {
          h.col = col_of(db, op.term_fk[j]);
          h.b = &I[(size_t)op.term_build[j]];
          if (!h.b->host_table && !h.b->h_bitmap) return set_error(DDQ_ESTATE, "host star needs host tables");
          while (h.b->host_table && (1u << h.lg) < h.b->table_cap) h.lg++;
          n_emit += op.term_emit[j] ? 1 : 0;
        }
        ts.push_back(h);
      }
      int nchunks = (threads <= 1 || n < (1 << 16)) ? 1 : threads;
      std::vector<std::vector<int32_t>> sel((size_t)nchunks);
      std::vector<std::vector<int32_t>> pay((size_t)nchunks);  // n_emit values per survivor
      parallel_chunks(n, nchunks, [&](int t, int64_t b, int64_t e) {
        int32_t pv[4];
        for (int64_t r = b; r < e; r++) {
          bool ok = true;
          int ne = 0;
          for (int j = 0; j < op.n_terms && ok; j++) {
            const int64_t v = hcol(ts[(size_t)j].col, r);
            if (op.term_kind[j] == DDQ_TERM_PRED) {
              const ddq_pred& pr = op.preds[j];
              ok = host_pred(pr, v);
              continue;
            }
            const Inter& B = *ts[(size_t)j].b;
            int32_t p = 0;
            if (B.h_bitmap) {
              const uint32_t o = (uint32_t)((int32_t)v - B.jmin);
              ok = o < B.jrange && (((*B.h_bitmap)[o >> 5] >> (o & 31)) & 1u);
              if (ok) p = (*B.h_payarr)[o];
            } else {
              uint32_t h = host_hash32((int32_t)v, 32 - ts[(size_t)j].lg);
              ok = false;
              while (true) {
                const uint64_t s = (*B.host_table)[h];
                if (s == kHostEmpty) break;
                if ((int32_t)(s >> 32) == (int32_t)v) {
                  ok = true;
                  p = (int32_t)(uint32_t)s;
                  break;
                }
                h = (h + 1) & (B.table_cap - 1);
              }
            }
            if (ok && op.term_emit[j]) pv[ne++] = p;
          }
          if (!ok) continue;
          sel[(size_t)t].push_back((int32_t)r);
          for (int x = 0; x < ne; x++) pay[(size_t)t].push_back(pv[x]);
        }
      });
      int64_t total = 0;
      for (auto& s : sel) total += (int64_t)s.size();
      out.count = out.cap = total;
      out.tids = (int32_t*)host_alloc(out, (size_t)total * 4);
      std::vector<int32_t*> pv;
      for (int x = 0; x < n_emit; x++) {
        pv.push_back((int32_t*)host_alloc(out, (size_t)total * 4));
        out.vecs.push_back(Vec{pv.back(), 4, true});
      }
      int64_t o = 0;
      for (int t = 0; t < nchunks; t++)
        for (size_t i = 0; i < sel[(size_t)t].size(); i++, o++) {
          out.tids[o] = sel[(size_t)t][i];
          for (int x = 0; x < n_emit; x++) pv[(size_t)x][o] = pay[(size_t)t][i * n_emit + x];
        }
      return DDQ_OK;
    }
    case DDQ_OP_SELECT:
    case DDQ_OP_FILTER_EQ:
    case DDQ_OP_HASH_PROBE: {
      const bool probe = op.kind == DDQ_OP_HASH_PROBE;
      const Inter* build = probe ? &I[(size_t)op.build] : nullptr;
      if (probe && !build->host_table && !build->h_bitmap) return set_error(DDQ_ESTATE, "host probe needs a host table");
      const bool direct = probe && build->h_bitmap != nullptr;
      std::vector<const Column*> pc;
      for (int i = 0; i < op.n_preds && op.kind == DDQ_OP_SELECT; i++) pc.push_back(col_of(db, op.preds[i].column));
      const int32_t* eqa = nullptr;
      const int32_t* eqb = nullptr;
      if (op.kind == DDQ_OP_FILTER_EQ) {
        const int a = op.eq_vec[0] - 1, b = op.eq_vec[1] - 1;
        if (!in || a < 0 || b < 0 || a >= (int)in->vecs.size() || b >= (int)in->vecs.size())
          return set_error(DDQ_EINVAL, "filter_eq: bad vector indexes");
        eqa = (const int32_t*)in->vecs[(size_t)a].ptr;
        eqb = (const int32_t*)in->vecs[(size_t)b].ptr;
        if (op.eq_cmp < DDQ_CMP_EQ || op.eq_cmp > DDQ_CMP_NE) return set_error(DDQ_EINVAL, "filter_eq: bad eq_cmp");
      }
      const Column* fk = (probe && op.fk_vec <= 0) ? col_of(db, op.fk_col) : nullptr;
      const int32_t* fkv = (probe && op.fk_vec > 0) ? (const int32_t*)in->vecs[(size_t)op.fk_vec - 1].ptr : nullptr;
      int lg = 0;
      if (probe && !direct)
        while ((1u << lg) < build->table_cap) lg++;
      const uint64_t* tab = (probe && !direct) ? build->host_table->data() : nullptr;
      const uint32_t mask = (probe && !direct) ? build->table_cap - 1 : 0;
      int nchunks = (threads <= 1 || n < (1 << 16)) ? 1 : threads;
      std::vector<std::vector<int64_t>> sel((size_t)nchunks);     // positions i
      std::vector<std::vector<int32_t>> pay((size_t)nchunks);
      parallel_chunks(n, nchunks, [&](int t, int64_t b, int64_t e) {
        auto& S = sel[(size_t)t];
        auto& Pv = pay[(size_t)t];
        for (int64_t i = b; i < e; i++) {
          int32_t r = row_of(i);
          bool ok = true;
          if (eqa) {
            const bool keep = op.eq_cmp == DDQ_CMP_LT ? eqa[i] < eqb[i]
                            : op.eq_cmp == DDQ_CMP_NE ? eqa[i] != eqb[i] : eqa[i] == eqb[i];
            if (keep) S.push_back(i);
          } else if (!probe) {
            for (int p = 0; p < op.n_preds && ok; p++) {
              int64_t v = hcol(pc[(size_t)p], r);
              const ddq_pred& pr = op.preds[p];
              ok = host_pred(pr, v);
            }
            if (ok) S.push_back(i);
          } else {
            int32_t k = fkv ? fkv[i] : ((const int32_t*)fk->host)[r];
            if (direct) {
              const uint32_t o = (uint32_t)(k - build->jmin);
              ok = o < build->jrange && (((*build->h_bitmap)[o >> 5] >> (o & 31)) & 1u);
              if (ok) {
                Pv.push_back((*build->h_payarr)[o]);
                S.push_back(i);
              }
              continue;
            }
            uint32_t h = host_hash32(k, 32 - lg);
            while (true) {
              uint64_t s = tab[h];
              if (s == kHostEmpty) { ok = false; break; }
              if ((int32_t)(s >> 32) == k) { Pv.push_back((int32_t)(uint32_t)s); break; }
              h = (h + 1) & mask;
            }
            if (ok) S.push_back(i);
          }
        }
      });
      int64_t total = 0;
      for (auto& s : sel) total += (int64_t)s.size();
      out.count = out.cap = total;
      out.tids = (int32_t*)host_alloc(out, (size_t)total * 4);
      size_t nv = in ? in->vecs.size() : 0;
      for (size_t v = 0; v < nv; v++) out.vecs.push_back(Vec{host_alloc(out, (size_t)total * in->vecs[v].width), in->vecs[v].width, true});
      int32_t* payout = nullptr;
      if (probe && op.emit_payload) {
        payout = (int32_t*)host_alloc(out, (size_t)total * 4);
        out.vecs.push_back(Vec{payout, 4, true});
      }
      int64_t o = 0;
      for (int t = 0; t < nchunks; t++) {
        for (size_t j = 0; j < sel[(size_t)t].size(); j++, o++) {
          int64_t i = sel[(size_t)t][j];
          out.tids[o] = row_of(i);
          for (size_t v = 0; v < nv; v++) {
            if (in->vecs[v].width == 4) ((int32_t*)out.vecs[v].ptr)[o] = ((const int32_t*)in->vecs[v].ptr)[i];
            else ((int64_t*)out.vecs[v].ptr)[o] = ((const int64_t*)in->vecs[v].ptr)[i];
          }
          if (payout) payout[o] = pay[(size_t)t][j];
        }
      }
      return DDQ_OK;
    }
    case DDQ_OP_HASH_BUILD: {
      const Column* kc = col_of(db, op.key_col);
      const Column* pc = op.payload_col >= 0 ? col_of(db, op.payload_col) : nullptr;
      if (pc && !fits_int32(*pc)) return set_error(DDQ_EINVAL, "build: payload values do not fit int32");
      int64_t cap = pow2_at_least(std::max<int64_t>(16, 2 * n));
      int lg = 0;
      while ((1ll << lg) < cap) lg++;
      auto t = std::make_shared<std::vector<uint64_t>>((size_t)cap, kHostEmpty);
      std::vector<const Column*> bpc;  // fused selection (BUILD op with predicates)
      for (int p = 0; p < op.n_preds; p++) bpc.push_back(col_of(db, op.preds[p].column));
      for (int64_t i = 0; i < n; i++) {
        int32_t r = row_of(i);
        bool ok = true;
        for (int p = 0; p < op.n_preds && ok; p++) {
          const int64_t v = hcol(bpc[(size_t)p], r);
          const ddq_pred& pr = op.preds[p];
          ok = host_pred(pr, v);
        }
        if (!ok) continue;
        int32_t k = ((const int32_t*)kc->host)[r];
        int32_t v = pc ? (int32_t)hcol(pc, r) : r;  // an int64 payload fits int32 (checked below)
        uint32_t h = host_hash32(k, 32 - lg);
        bool dup = false;
        while ((*t)[h] != kHostEmpty) {
          if ((int32_t)((*t)[h] >> 32) == k) {
            if (!op.build_key_set) return set_error(DDQ_EINVAL, "duplicate build key");
            dup = true;  // key set (semi-join): the first row stays
            if (op.build_key_set == 2 && v < (int32_t)(uint32_t)(*t)[h])  // MIN build: keep the smallest
              (*t)[h] = ((uint64_t)(uint32_t)k << 32) | (uint32_t)v;
            break;
          }
          h = (h + 1) & (uint32_t)(cap - 1);
        }
        if (!dup) (*t)[h] = ((uint64_t)(uint32_t)k << 32) | (uint32_t)v;
      }
      out.host_table = t;
      out.table_cap = (uint32_t)cap;
      return DDQ_OK;
    }
    case DDQ_OP_GATHER: {
      const Column* c = col_of(db, op.gather_col);
      out.count = out.cap = n;
      out.tids = (int32_t*)host_alloc(out, (size_t)n * 4);
      std::memcpy(out.tids, in->tids, (size_t)n * 4);
      for (const Vec& v : in->vecs) {
        void* p = host_alloc(out, (size_t)n * v.width);
        std::memcpy(p, v.ptr, (size_t)n * v.width);
        out.vecs.push_back(Vec{p, v.width, true});
      }
      if (op.fetch_build > 0) {  // dimension attribute fetch (INT32_MIN for a missing key)
        const Inter* B = &I[(size_t)op.fetch_build - 1];
        if (!B->host_table && !B->h_bitmap) return set_error(DDQ_ESTATE, "host fetch needs a host table");
        int32_t* dst = (int32_t*)host_alloc(out, (size_t)n * 4);
        int lg = 0;
        while (B->host_table && (1u << lg) < B->table_cap) lg++;
        for (int64_t i = 0; i < n; i++) {
          const int32_t k = ((const int32_t*)c->host)[in->tids[i]];
          int32_t v = INT32_MIN;
          if (B->h_bitmap) {
            const uint32_t o = (uint32_t)(k - B->jmin);
            if (o < B->jrange && (((*B->h_bitmap)[o >> 5] >> (o & 31)) & 1u)) v = (*B->h_payarr)[o];
          } else {
            uint32_t h = host_hash32(k, 32 - lg);
            while (true) {
              const uint64_t sl = (*B->host_table)[h];
              if (sl == kHostEmpty) break;
              if ((int32_t)(sl >> 32) == k) {
                v = (int32_t)(uint32_t)sl;
                break;
              }
              h = (h + 1) & (B->table_cap - 1);
            }
          }
          dst[i] = v;
        }
        out.vecs.push_back(Vec{dst, 4, true});
        return DDQ_OK;
      }
      if (op.gather_narrow && (c->width != 8 || !fits_int32(*c)))
        return set_error(DDQ_EINVAL, "gather: narrowing needs an int64 column whose values fit int32");
      const int w = op.gather_narrow ? 4 : c->width;
      void* dst = host_alloc(out, (size_t)n * w);
      for (int64_t i = 0; i < n; i++) {
        if (w == 8) ((int64_t*)dst)[i] = ((const int64_t*)c->host)[in->tids[i]];
        else ((int32_t*)dst)[i] = (int32_t)hcol(c, in->tids[i]);
      }
      out.vecs.push_back(Vec{dst, w, true});
      return DDQ_OK;
    }
    case DDQ_OP_AGGREGATE: {
      const int na = op.n_aggs;
      std::vector<const Column*> kc(3, nullptr);
      for (int k = 0; k < op.n_keys; k++)
        if (op.key_src[k] < -1) kc[(size_t)k] = col_of(db, -2 - op.key_src[k]);
      std::vector<std::array<const Column*, 3>> ac((size_t)na);
      for (int a = 0; a < na; a++)
        for (int j = 0; j < 3; j++) ac[(size_t)a][(size_t)j] = op.agg_col[a][j] >= 0 ? col_of(db, op.agg_col[a][j]) : nullptr;
      int kshift[DDQ_MAX_KEYS];
      for (int k = 0, sh = 0; k < DDQ_MAX_KEYS; k++) {
        kshift[k] = sh;
        sh += op.key_bits[k] > 0 ? op.key_bits[k] : 21;
      }
      // fused probe / fetch terms (reading O37): builds on the host, emitted payloads
      // numbered after the input's vectors
      std::vector<const Inter*> tb;
      std::vector<const Column*> tfk;
      for (int j = 0; j < op.n_terms && j < 4; j++) {
        tb.push_back(&I[(size_t)op.term_build[j]]);
        tfk.push_back(col_of(db, op.term_fk[j]));
        if (!tb.back()->host_table && !tb.back()->h_bitmap) return set_error(DDQ_ESTATE, "host aggregate: term build not on the host");
      }
      const int n_in_vecs = in ? (int)in->vecs.size() : 0;
      std::vector<const Column*> apc;  // fused selection (AGGREGATE op with predicates)
      for (int p = 0; p < op.n_preds; p++) apc.push_back(col_of(db, op.preds[p].column));
      // every core of the op's share aggregates a row range into its own table
      // (A2: an operator uses all cores); the tables merge exactly below
      std::vector<std::unordered_map<int64_t, std::vector<__int128>>> part((size_t)std::max(threads, 1));
      parallel_chunks(n, threads, [&](int chunk, int64_t b, int64_t e) {
      auto& g = part[(size_t)chunk];
      for (int64_t i = b; i < e; i++) {
        int32_t r = row_of(i);
        bool ok = true;
        for (int p = 0; p < op.n_preds && ok; p++) {
          const int64_t v = hcol(apc[(size_t)p], r);
          const ddq_pred& pr = op.preds[p];
          ok = host_pred(pr, v);
        }
        if (!ok) continue;
        int32_t tpay[4];
        int ne = 0;
        for (size_t j = 0; j < tb.size() && ok; j++) {
          int32_t v = INT32_MIN;
          const bool hit = host_lookup(*tb[j], ((const int32_t*)tfk[j]->host)[r], &v);
          if (op.term_kind[j] == DDQ_TERM_PROBE && !hit) ok = false;
          if (op.term_kind[j] == DDQ_TERM_FETCH || op.term_emit[j]) tpay[ne++] = v;
        }
        if (!ok) continue;
        int64_t key = 0;
        for (int k = 0; k < op.n_keys; k++) {
          const int src = op.key_src[k];
          int32_t c = src >= n_in_vecs && !tb.empty() ? tpay[src - n_in_vecs]
                      : src >= 0 ? ((const int32_t*)in->vecs[(size_t)src].ptr)[i]
                                 : ((const int32_t*)kc[(size_t)k]->host)[r];
          key |= (int64_t)(uint32_t)c << kshift[k];
        }
        auto& acc = g[key];
        const bool fresh = acc.empty();
        if (fresh) acc.assign((size_t)na, 0);
        for (int a = 0; a < na; a++) {
          int kind = op.agg_kind[a];
          if (kind == DDQ_AGG_MIN) {  // operand: a column, or an aligned vector (agg_col <= -2)
            const int vs = -2 - op.agg_col[a][0];
            const __int128 x = op.agg_col[a][0] <= -2
                                   ? (in->vecs[(size_t)vs].width == 8 ? ((const int64_t*)in->vecs[(size_t)vs].ptr)[i]
                                                                      : ((const int32_t*)in->vecs[(size_t)vs].ptr)[i])
                                   : (__int128)hcol(ac[(size_t)a][0], r);
            if (fresh || x < acc[(size_t)a]) acc[(size_t)a] = x;
            continue;
          }
          __int128 v = 1;
          if (kind != DDQ_AGG_COUNT) {
            __int128 x = hcol(ac[(size_t)a][0], r);
            if (kind == DDQ_AGG_SUM) v = x;
            else {
              __int128 y = hcol(ac[(size_t)a][1], r);
              if (kind == DDQ_AGG_SUM_MUL) v = x * y;
              else if (kind == DDQ_AGG_SUM_SUB) v = x - y;
              else if (kind == DDQ_AGG_SUM_MUL_100M) v = x * (100 - y);
              else v = x * (100 - y) * (100 + hcol(ac[(size_t)a][2], r));
            }
          }
          acc[(size_t)a] += v;
        }
      }
      });
      std::unordered_map<int64_t, std::vector<__int128>>& g = part[0];
      for (size_t t = 1; t < part.size(); t++)
        for (auto& kv : part[t]) {
          auto it = g.find(kv.first);
          if (it == g.end()) {
            g.emplace(kv.first, std::move(kv.second));
            continue;
          }
          for (int a = 0; a < na; a++)
            it->second[(size_t)a] = op.agg_kind[a] == DDQ_AGG_MIN ? std::min(it->second[(size_t)a], kv.second[(size_t)a])
                                                                 : it->second[(size_t)a] + kv.second[(size_t)a];
        }
      auto keys = std::make_shared<std::vector<int64_t>>();
      auto accs = std::make_shared<std::vector<int64_t>>();
      for (auto& kv : g) {
        keys->push_back(kv.first);
        for (int a = 0; a < na; a++) {
          unsigned __int128 u = (unsigned __int128)kv.second[(size_t)a];
          accs->push_back((int64_t)(uint64_t)u);
          accs->push_back((int64_t)(uint64_t)(u >> 64));
        }
      }
      out.h_keys = keys;
      out.h_accs = accs;
      out.h_groups = (int64_t)keys->size();
      return DDQ_OK;
    }
  }
  return set_error(DDQ_EINVAL, "unknown operator");
}

// ------------------------------------------------------------ scheduling
static bool columns_cached(ddq_db* db, const ddq_op& op) {
  std::lock_guard<std::mutex> g(db->mu);
  for (int c : op_columns(op)) {
    const Column* col = col_of(db, c);
    if (!col || !col->dev || col->evict_pending) return false;
  }
  return true;
}

static bool children_on_gpu(QueryState& q, int i) {
  for (int c : op_children(q.plan.ops[i]))
    if (q.inters[(size_t)c].on_host) return false;
  return true;
}

// Operator-driven data placement for the GPU-only arm: make the
// op's columns resident, evicting least-recently-used unreferenced columns.
static ddq_status ensure_cached_lru(ddq_db* db, const ddq_op& op) {
  std::unique_lock<std::mutex> g(db->mu);
  for (int c : op_columns(op)) {
    Column& col = *db->cols[(size_t)c];
    while (col.loading) db->cache_cv.wait(g);  // another worker is copying it
    if (col.dev && !col.evict_pending) {
      db->stats.cache_hits++;
      continue;
    }
    db->stats.cache_misses++;
    uint64_t need = (uint64_t)std::max<int64_t>(col.n, 1) * col.width;
    while (db->cache_used + need > db->cfg.cache_bytes) {
      int victim = -1;
      uint64_t best = UINT64_MAX;
      std::vector<int> mine = op_columns(op);
      for (size_t k = 0; k < db->cols.size(); k++) {
        const Column& o = *db->cols[k];
        if (!o.dev || o.refs > 0 || std::find(mine.begin(), mine.end(), (int)k) != mine.end()) continue;
        if (o.last_access < best) {
          best = o.last_access;
          victim = (int)k;
        }
      }
      if (victim < 0) return DDQ_ENOMEM_DEVICE;
      evict_column_locked(db, victim);
    }
    ddq_status s = cache_column_locked(db, c, true, g);
    if (s != DDQ_OK) return s;
  }
  return DDQ_OK;
}

static void hold_columns(ddq_db* db, const ddq_op& op, int delta) {
  std::lock_guard<std::mutex> g(db->mu);
  for (int c : op_columns(op)) {
    Column& col = *db->cols[(size_t)c];
    col.refs += delta;
    if (delta < 0 && col.refs == 0 && col.evict_pending) evict_column_locked(db, c);
  }
}

// Pin the op's columns iff all are resident (check and pin under one lock, so an
// eviction cannot slip between them).
static bool hold_if_cached(ddq_db* db, const ddq_op& op) {
  std::lock_guard<std::mutex> g(db->mu);
  const std::vector<int> cols = op_columns(op);
  for (int c : cols) {
    const Column* col = col_of(db, c);
    if (!col || !col->dev || col->evict_pending) return false;
  }
  for (int c : cols) db->cols[(size_t)c]->refs++;
  return true;
}

static void enqueue(ddq_db* db, std::shared_ptr<QueryState> q, int i);

// The leaf operators of a query enter the global operator stream.  Collect
// them first: once one is enqueued, workers may finish it and make parents ready.
static void start_query(ddq_db* db, std::shared_ptr<QueryState> q) {
  std::vector<int> leaves;
  for (int i = 0; i < q->plan.n_ops; i++)
    if (q->pending[(size_t)i] == 0) leaves.push_back(i);
  for (int i : leaves) enqueue(db, q, i);
}

// A query finished or failed: its admission slot goes to the oldest waiting query.
static void release_admission(ddq_db* db) {
  std::shared_ptr<QueryState> next;
  {
    std::lock_guard<std::mutex> g(db->qmu);
    db->running_queries--;
    if (!db->admit_queue.empty() && (db->cfg.max_queries <= 0 || db->running_queries < db->cfg.max_queries)) {
      next = db->admit_queue.front();
      db->admit_queue.pop_front();
      db->running_queries++;
    }
  }
  if (next) start_query(db, next);
}

static void finish_query(ddq_db* db, QueryState& q) {
  const ddq_op& root = q.plan.ops[q.plan.n_ops - 1];
  Inter& r = q.inters.back();
  ddq_result* res = nullptr;
  ddq_status s = DDQ_OK;
  if (root.kind == DDQ_OP_AGGREGATE) {
    if (r.on_host) {
      s = finalize_result(root, r.h_groups, r.h_keys->data(), r.h_accs->data(), &res, true);
    } else {
      cudaStream_t st;
      cudaSetDevice(db->device);
      cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
      uint32_t g = 0;
      uint64_t t0 = now_ns();
      cudaMemcpyAsync(&g, r.gb_groups, 4, cudaMemcpyDeviceToHost, st);
      cudaStreamSynchronize(st);
      std::vector<int64_t> keys(g), accs((size_t)g * root.n_aggs * 2);
      if (g) {
        cudaMemcpyAsync(keys.data(), r.gb_keys, (size_t)g * 8, cudaMemcpyDeviceToHost, st);
        cudaMemcpyAsync(accs.data(), r.gb_accs, (size_t)g * root.n_aggs * 16, cudaMemcpyDeviceToHost, st);
      }
      cudaError_t e = cudaStreamSynchronize(st);
      cudaStreamDestroy(st);
      db->stats.d2h_bytes += 4 + (uint64_t)g * (8 + 16 * root.n_aggs);
      db->stats.d2h_ns += now_ns() - t0;
      s = e == cudaSuccess ? finalize_result(root, g, keys.data(), accs.data(), &res, true) : cuda_status(e, "fetch");
    }
  } else {
    cudaStream_t st;
    cudaSetDevice(db->device);
    cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
    s = inter_to_host(db, r, st);
    cudaStreamDestroy(st);
    if (s == DDQ_OK) {
      res = new ddq_result();
      std::memset(res, 0, sizeof(*res));
      int32_t* t = new int32_t[(size_t)std::max<int64_t>(r.count, 1)];
      const int64_t base = db->tables[(size_t)root.table].row_begin;
      for (int64_t i = 0; i < r.count; i++) t[i] = (int32_t)(r.tids[i] + base);
      std::sort(t, t + r.count);  // a select-* result is a set of rows: row order (S8(a7))
      res->n_tids = r.count;
      res->tids = t;
    }
  }
  if (s == DDQ_OK && res) decode_result_keys(db, q.plan, res);
  for (auto& x : q.inters) release_inter(db, x);
  std::lock_guard<std::mutex> g(q.mu);
  q.status = s;
  if (s != DDQ_OK) q.error = ddq_last_error();
  if (res) {
    res->gpu_ops = q.gpu_ops;
    res->host_ops = q.host_ops;
    res->aborts = q.aborts;
    uint8_t* tr = new uint8_t[std::max<size_t>(q.trace.size(), 1)];
    std::copy(q.trace.begin(), q.trace.end(), tr);
    res->n_ops = (int32_t)q.trace.size();
    res->op_place = tr;
    float* om = new float[std::max<size_t>(q.op_ms.size(), 1)];
    std::copy(q.op_ms.begin(), q.op_ms.end(), om);
    res->op_ms = om;
  }
  q.t_done = now_ns();
  if (res) res->exec_ms = (double)(q.t_done - q.t_submit) / 1e6;
  q.result = res;
  q.done = true;
  db->stats.queries_done++;
  q.cv.notify_all();
}

static void finish_query_and_admit(ddq_db* db, QueryState& q) {
  finish_query(db, q);
  release_admission(db);
}

// A failed operator fails its query: waiters are woken at once, but the query's
// intermediates are released only when no operator of it is still running (the
// caller is itself in flight; worker_loop releases when the count drains).
static void fail_query(ddq_db* db, QueryState& q, ddq_status s) {
  std::string msg = ddq_last_error();
  {
    std::lock_guard<std::mutex> g(q.mu);
    if (q.done) return;
    q.status = s;
    q.error = msg;
    q.failed = true;
    q.done = true;
    q.cv.notify_all();
  }
  release_admission(db);
}

// Called when op i of q finished: notify parents, free consumed inputs.
static void op_finished(ddq_db* db, std::shared_ptr<QueryState> q, int i) {
  std::vector<int> ready;
  bool last = false;
  {
    std::lock_guard<std::mutex> g(q->mu);
    for (int p : q->parents[(size_t)i])
      if (--q->pending[(size_t)p] == 0) ready.push_back(p);
    // intermediates whose consumers are all done can be released
    // (a GATHER output aliases its input's TIDs: such inputs live until the query ends)
    for (int c : op_children(q->plan.ops[i]))
      if (--q->consumers_left[(size_t)c] == 0 && q->plan.ops[i].kind != DDQ_OP_GATHER)
        release_inter(db, q->inters[(size_t)c]);
    last = --q->ops_left == 0;
  }
  for (int p : ready) enqueue(db, q, p);
  if (last) finish_query_and_admit(db, *q);
}

static int decide_place(ddq_db* db, QueryState& q, int i) {
  const ddq_op& op = q.plan.ops[i];
  if (!db->cfg.chopping && q.place[(size_t)i] != P_NONE) return q.place[(size_t)i];  // compile time
  switch (db->cfg.placement) {
    case DDQ_PLACE_CPU_ONLY: return P_HOST;
    case DDQ_PLACE_GPU_ONLY: return P_GPU;
    default:  // data-driven, run time
      return (columns_cached(db, op) && children_on_gpu(q, i)) ? P_GPU : P_HOST;
  }
}

static void enqueue(ddq_db* db, std::shared_ptr<QueryState> q, int i) {
  int where = decide_place(db, *q, i);
  std::lock_guard<std::mutex> g(db->qmu);
  if (where == P_GPU) db->gpu_ready.emplace_back(q, i);
  else db->host_ready.emplace_back(q, i);
  db->qcv.notify_all();
}

static void run_on_host(ddq_db* db, std::shared_ptr<QueryState> q, int i, cudaStream_t st) {
  const ddq_op& op = q->plan.ops[i];
  for (int c : op_children(op)) {  // data follows the operator to the host
    ddq_status s = inter_to_host(db, q->inters[(size_t)c], st);
    if (s != DDQ_OK) {
      fail_query(db, *q, s);
      return;
    }
  }
  Inter out;
  ddq_status s = run_host_op(db, op, q->inters, out);
  if (s != DDQ_OK) {
    release_inter(db, out);
    fail_query(db, *q, s);
    return;
  }
  q->inters[(size_t)i] = std::move(out);
  q->op_ms[(size_t)i] = (float)((now_ns() - q->op_t0[(size_t)i]) / 1e6);
  q->host_ops++;
  if (q->trace[(size_t)i] != DDQ_RAN_ABORTED) q->trace[(size_t)i] = DDQ_RAN_HOST;
  db->stats.host_ops++;
  op_finished(db, q, i);
}

static void run_on_gpu(ddq_db* db, std::shared_ptr<QueryState> q, int i, cudaStream_t st) {
  const ddq_op& op = q->plan.ops[i];
  const uint64_t t0 = now_ns();
  ddq_status s = DDQ_OK;
  if (db->cfg.placement == DDQ_PLACE_GPU_ONLY || !db->cfg.chopping) s = ensure_cached_lru(db, op);
  bool abort = s == DDQ_ENOMEM_DEVICE || (i < 32 && ((db->cfg.fault_op_mask >> i) & 1u));
  if (s != DDQ_OK && !abort) {
    fail_query(db, *q, s);
    return;
  }
  if (!abort) {
    for (int c : op_children(op)) {  // compile-time arm: copy host data back (Fig. 8)
      s = inter_to_device(db, q->inters[(size_t)c], st);
      if (s == DDQ_ENOMEM_DEVICE) {
        abort = true;
        break;
      }
      if (s != DDQ_OK) {
        fail_query(db, *q, s);
        return;
      }
    }
  }
  if (!abort && !hold_if_cached(db, op)) abort = true;  // evicted meanwhile: follow the data
  Inter out;
  if (!abort) {
    GpuOpCtx ctx{db, st, &q->inters};
    s = run_gpu_op(ctx, op, out);
    if (s == DDQ_OK) {
      cudaError_t e = cudaStreamSynchronize(st);
      if (e != cudaSuccess) s = cuda_status(e, "gpu op");
    }
    hold_columns(db, op, -1);
    if (s == DDQ_OK && out.d_count && op.kind != DDQ_OP_GATHER) {
      uint32_t c = 0;
      cudaMemcpy(&c, out.d_count, 4, cudaMemcpyDeviceToHost);
      out.count = c;
      out.cap = c;  // exact cardinality is known at run time: consumers allocate exactly
    }
    if (s == DDQ_OK && (out.table_ptr || out.jidx) && out.d_error) {
      uint32_t e2 = 0;
      cudaMemcpy(&e2, out.d_error, 4, cudaMemcpyDeviceToHost);
      if (e2) s = set_error(e2 == 2 ? DDQ_EOVERFLOW : DDQ_EINVAL, "hash build failed (duplicate key or overflow)");
    }
    static const bool dbg = getenv("DDQ_DEBUG_ERRORS") != nullptr;
    if (dbg && s == DDQ_OK && out.d_error) {
      uint32_t e2 = 0;
      cudaMemcpy(&e2, out.d_error, 4, cudaMemcpyDeviceToHost);
      fprintf(stderr, "ddq: query %lld op %d kind %d error cell %u count %lld\n", (long long)q->id, i, op.kind, e2,
              (long long)out.count);
    }
    if (s == DDQ_OK && op.kind == DDQ_OP_AGGREGATE && out.d_error) {  // group table overflow (max_groups)
      uint32_t e2 = 0;
      cudaMemcpy(&e2, out.d_error, 4, cudaMemcpyDeviceToHost);
      if (e2) s = set_error(DDQ_EOVERFLOW, "aggregate: more groups than the plan's max_groups allows");
    }
    if (s == DDQ_ENOMEM_DEVICE) {
      abort = true;
      release_inter(db, out);
    } else if (s != DDQ_OK) {
      release_inter(db, out);
      fail_query(db, *q, s);
      return;
    }
  }
  if (abort) {  // abort immediately, restart on the host
    q->trace[(size_t)i] = DDQ_RAN_ABORTED;
    q->aborts++;
    db->stats.aborts++;
    db->stats.wasted_ns += now_ns() - t0;
    run_on_host(db, q, i, st);
    return;
  }
  if (op.kind == DDQ_OP_GATHER) out.count = q->inters[(size_t)op.input].count;
  q->inters[(size_t)i] = std::move(out);
  q->op_ms[(size_t)i] = (float)((now_ns() - q->op_t0[(size_t)i]) / 1e6);
  q->trace[(size_t)i] = DDQ_RAN_GPU;
  q->gpu_ops++;
  db->stats.gpu_ops++;
  op_finished(db, q, i);
}

// Streamed cold path (N1): copy the queued columns in order on the copy stream
// while the operators of earlier-arriving data compute.  A column that no longer
// fits the cache budget is skipped (the operator copies it on demand, LRU).
static void prefetch_loop(ddq_db* db) {
  cudaSetDevice(db->device);
  while (true) {
    int c = -1;
    {
      std::unique_lock<std::mutex> g(db->qmu);
      db->qcv.wait(g, [&] { return db->stopping || !db->prefetch_queue.empty(); });
      if (db->stopping) break;
      c = db->prefetch_queue.front();
      db->prefetch_queue.pop_front();
    }
    std::unique_lock<std::mutex> lk(db->mu);
    if (c < 0 || c >= (int)db->cols.size()) continue;
    Column& col = *db->cols[(size_t)c];
    if (col.dev || col.loading) continue;
    const uint64_t bytes = (uint64_t)std::max<int64_t>(col.n, 1) * col.width;
    if (db->cache_used + bytes > db->cfg.cache_bytes) continue;
    (void)cache_column_locked(db, c, true, lk);  // failures: the operator fetches on demand
  }
}

// The paper's background data-placement job: Algorithm 1 every
// placement_period_ms; running queries keep going (evictions are deferred while
// referenced).
static void placement_loop(ddq_db* db) {
  cudaSetDevice(db->device);
  std::unique_lock<std::mutex> g(db->qmu);
  while (!db->stopping) {
    db->qcv.wait_for(g, std::chrono::milliseconds(db->cfg.placement_period_ms), [&] { return db->stopping; });
    if (db->stopping) break;
    g.unlock();
    (void)ddq_update_placement(db);
    g.lock();
  }
}

// every input column of op resident on the GPU (the cached-first pull order)
static bool op_resident(ddq_db* db, const ddq_op& op) {
  std::lock_guard<std::mutex> g(db->mu);
  for (int c : op_columns(op)) {
    const Column* col = col_of(db, c);
    if (!col || !col->dev || col->loading) return false;
  }
  return true;
}

static void worker_loop(ddq_db* db, bool gpu) {
  cudaSetDevice(db->device);
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  while (true) {
    std::shared_ptr<QueryState> q;
    int i = -1;
    {
      std::unique_lock<std::mutex> g(db->qmu);
      auto& Q = gpu ? db->gpu_ready : db->host_ready;
      db->qcv.wait(g, [&] { return db->stopping || !Q.empty(); });
      if (db->stopping) break;
      // pull the ready operator of the OLDEST query (FIFO among its ops): a query
      // already in flight finishes before the leaves of newer ones start, so the
      // heap holds the intermediates of about gpu_workers queries, not of every
      // submitted one (measured M5: FIFO pulls let 32 users' first intermediates
      // pile up and abort, profiles/r2_config5_sf20.jsonl)
      auto pick = Q.begin();
      for (auto it = Q.begin(); it != Q.end(); ++it)
        if (it->first->id < pick->first->id) pick = it;
      if (gpu && db->cfg.prefetch && !op_resident(db, pick->first->plan.ops[pick->second]))
        for (auto it = Q.begin(); it != Q.end(); ++it)  // cached-first: an op whose data is here
          if (op_resident(db, it->first->plan.ops[it->second]) &&
              (!op_resident(db, pick->first->plan.ops[pick->second]) || it->first->id < pick->first->id))
            pick = it;
      q = pick->first;
      i = pick->second;
      Q.erase(pick);
    }
    {
      std::lock_guard<std::mutex> g(q->mu);
      if (q->done) continue;  // failed query: drop remaining ops
      q->inflight++;
    }
    q->op_t0[(size_t)i] = now_ns();  // op_ms: pull -> completion (recorded before op_finished)
    if (gpu) run_on_gpu(db, q, i, st);
    else run_on_host(db, q, i, st);
    std::lock_guard<std::mutex> g(q->mu);
    if (--q->inflight == 0 && q->failed && !q->released) {  // last running op of a failed query
      q->released = true;
      for (auto& x : q->inters) release_inter(db, x);
    }
  }
  cudaStreamDestroy(st);
}

void driver_start(ddq_db* db) {
  // chopping: a bounded pool pulls GPU operators; without chopping
  // every operator gets its own thread (unbounded inter-operator parallelism).
  int g = db->cfg.chopping ? db->cfg.gpu_workers : 64;
  int h = db->cfg.chopping ? db->cfg.host_workers : std::max(db->cfg.host_workers, 16);
  for (int i = 0; i < g; i++) db->workers.emplace_back(worker_loop, db, true);
  for (int i = 0; i < h; i++) db->workers.emplace_back(worker_loop, db, false);
  if (db->cfg.prefetch && db->cfg.placement != DDQ_PLACE_CPU_ONLY) db->prefetcher = std::thread(prefetch_loop, db);
  if (db->cfg.placement_period_ms > 0) db->placer = std::thread(placement_loop, db);
}

void driver_stop(ddq_db* db) {
  {
    std::lock_guard<std::mutex> g(db->qmu);
    db->stopping = true;
    db->qcv.notify_all();
  }
  for (auto& t : db->workers) t.join();
  db->workers.clear();
  if (db->prefetcher.joinable()) db->prefetcher.join();
  if (db->placer.joinable()) db->placer.join();
  for (auto& kv : db->queries) {
    for (auto& x : kv.second->inters) release_inter(db, x);
    if (kv.second->result) ddq_result_free(kv.second->result);
  }
  db->queries.clear();
}

}  // namespace ddq

using namespace ddq;

extern "C" {

ddq_status ddq_submit(ddq_db* db, const ddq_plan* plan, ddq_query* out) {
  if (!db || !out) return set_error(DDQ_EINVAL, "submit: null argument");
  if (ddq_status s = validate_plan_public(db, plan)) return s;
  auto q = std::make_shared<QueryState>();
  q->plan = *plan;  // plans are copied at submit (S8(b))
  const int n = plan->n_ops;
  q->inters.resize((size_t)n);
  q->pending.assign((size_t)n, 0);
  q->parents.assign((size_t)n, {});
  q->consumers_left.assign((size_t)n, 0);
  q->place.assign((size_t)n, P_NONE);
  q->trace.assign((size_t)n, 0);
  q->op_ms.assign((size_t)n, 0.f);
  q->op_t0.assign((size_t)n, 0);
  q->ops_left = n;
  q->t_submit = now_ns();
  for (int i = 0; i < n; i++)
    for (int c : op_children(plan->ops[i])) {
      q->pending[(size_t)i]++;
      q->parents[(size_t)c].push_back(i);
      q->consumers_left[(size_t)c]++;
    }
  if (!db->cfg.chopping) {  // compile-time placement from the cache state at submit
    for (int i = 0; i < n; i++) {
      if (db->cfg.placement == DDQ_PLACE_CPU_ONLY) q->place[(size_t)i] = P_HOST;
      else if (db->cfg.placement == DDQ_PLACE_GPU_ONLY) q->place[(size_t)i] = P_GPU;
      else {
        bool ok = columns_cached(db, plan->ops[i]);
        for (int c : op_children(plan->ops[i])) ok = ok && q->place[(size_t)c] == P_GPU;
        q->place[(size_t)i] = ok ? P_GPU : P_HOST;
      }
    }
  }
  bool admitted = true;
  {
    std::lock_guard<std::mutex> g(db->qmu);
    q->id = db->next_query++;
    db->queries[q->id] = q;
    // admission control (max_queries): beyond the limit the query waits its turn
    if (db->cfg.max_queries > 0 && db->running_queries >= db->cfg.max_queries) {
      db->admit_queue.push_back(q);
      admitted = false;
    } else {
      db->running_queries++;
    }
  }
  *out = q->id;
  if (db->cfg.prefetch && db->cfg.placement != DDQ_PLACE_CPU_ONLY) {  // N1: stream the plan's columns in
    std::vector<int> cols;
    for (int i = 0; i < n; i++)
      for (int c : op_columns(plan->ops[i]))
        if (std::find(cols.begin(), cols.end(), c) == cols.end()) cols.push_back(c);
    std::lock_guard<std::mutex> g(db->qmu);
    for (int c : cols) db->prefetch_queue.push_back(c);
    db->qcv.notify_all();
  }
  if (admitted) start_query(db, q);
  return DDQ_OK;
}

ddq_status ddq_wait(ddq_db* db, ddq_query id, int64_t timeout_ns) {
  if (!db) return set_error(DDQ_EINVAL, "wait: null");
  std::shared_ptr<QueryState> q;
  {
    std::lock_guard<std::mutex> g(db->qmu);
    auto it = db->queries.find(id);
    if (it == db->queries.end()) return set_error(DDQ_ENOTFOUND, "wait: unknown query");
    q = it->second;
  }
  std::unique_lock<std::mutex> g(q->mu);
  if (timeout_ns < 0) q->cv.wait(g, [&] { return q->done; });
  else if (!q->cv.wait_for(g, std::chrono::nanoseconds(timeout_ns), [&] { return q->done; }))
    return set_error(DDQ_ETIMEOUT, "wait: timeout");
  if (q->status != DDQ_OK) return set_error(q->status, q->error);
  return DDQ_OK;
}

ddq_status ddq_fetch(ddq_db* db, ddq_query id, ddq_result** out) {
  if (!db || !out) return set_error(DDQ_EINVAL, "fetch: null");
  std::shared_ptr<QueryState> q;
  {
    std::lock_guard<std::mutex> g(db->qmu);
    auto it = db->queries.find(id);
    if (it == db->queries.end()) return set_error(DDQ_ENOTFOUND, "fetch: unknown query");
    q = it->second;
  }
  std::unique_lock<std::mutex> g(q->mu);
  q->cv.wait(g, [&] { return q->done; });
  const ddq_status s = q->status;
  const std::string err = q->error;
  *out = s == DDQ_OK ? q->result : nullptr;
  q->result = nullptr;
  g.unlock();
  {  // a fetched query -- failed or not -- leaves the table (its intermediates are
     // released by the workers: at the root for a result, at the last in-flight op
     // of a failed query)
    std::lock_guard<std::mutex> g2(db->qmu);
    db->queries.erase(id);
  }
  if (s != DDQ_OK) return set_error(s, err);
  return DDQ_OK;
}

}  // extern "C"
