// cluster.cpp -- multi-GPU data-driven placement (Sec. 6.3:
// "Our Data-Driven strategy can support multiple co-processors").  One database per
// GPU, each with its own column cache and heap, all holding the same tables in
// pinned host memory.  Data placement stays Algorithm 1 per GPU, over the
// access counts of the queries THAT GPU ran; query placement is data-driven: a
// submitted plan goes to the GPU whose cache holds the most of its input bytes (all of
// them if any GPU has them), ties to the GPU with the fewest queries in flight, and
// inside that GPU's driver every operator is still placed by Sec. 3.1-5.4 (GPU iff its
// inputs are resident there, else the host).  Over a workload the GPUs' caches
// specialise on the queries routed to them, so each column is copied to the GPU its
// queries run on -- the data-driven principle across co-processors.
// Rows are not partitioned here (S8(e)'s row sharding is dist.cpp); this is
// placement of whole queries over per-GPU caches.
#include <algorithm>
#include <atomic>
#include <mutex>
#include <vector>

#include "engine.h"

struct ddq_cluster {
  std::vector<ddq_db*> dbs;
  std::vector<std::atomic<int64_t>*> inflight;  // queries submitted and not fetched, per member
  std::mutex mu;
  uint64_t rr = 0;  // round-robin origin for full ties (an empty cluster spreads queries)
};

namespace ddq {

// Bytes of the plan's input columns resident on db (cache, not pending eviction).
static uint64_t resident_bytes(ddq_db* db, const ddq_plan& plan, uint64_t* total) {
  std::vector<int> cols;
  for (int i = 0; i < plan.n_ops; i++)
    for (int c : op_columns(plan.ops[i]))
      if (std::find(cols.begin(), cols.end(), c) == cols.end()) cols.push_back(c);
  uint64_t r = 0, t = 0;
  std::lock_guard<std::mutex> g(db->mu);
  for (int c : cols) {
    const Column* col = col_of(db, c);
    if (!col) continue;
    const uint64_t b = (uint64_t)std::max<int64_t>(col->n, 1) * col->width;
    t += b;
    if (col->dev && !col->evict_pending) r += b;
  }
  if (total) *total = t;
  return r;
}

}  // namespace ddq

using namespace ddq;

extern "C" {

ddq_status ddq_cluster_open(const ddq_config* cfg, const int32_t* devices, int32_t n, ddq_cluster** out) {
  if (!cfg || !devices || n < 1 || !out) return set_error(DDQ_EINVAL, "cluster_open");
  auto* c = new ddq_cluster();
  for (int32_t i = 0; i < n; i++) {
    ddq_config ci = *cfg;
    ci.device = devices[i];
    ddq_db* db = nullptr;
    ddq_status s = ddq_open(&ci, &db);
    if (s != DDQ_OK) {
      for (ddq_db* d : c->dbs) ddq_close(d);
      for (auto* a : c->inflight) delete a;
      delete c;
      return s;
    }
    c->dbs.push_back(db);
    c->inflight.push_back(new std::atomic<int64_t>(0));
  }
  *out = c;
  return DDQ_OK;
}

void ddq_cluster_close(ddq_cluster* c) {
  if (!c) return;
  for (ddq_db* d : c->dbs) ddq_close(d);
  for (auto* a : c->inflight) delete a;
  delete c;
}

int32_t ddq_cluster_size(ddq_cluster* c) { return c ? (int32_t)c->dbs.size() : 0; }

ddq_db* ddq_cluster_db(ddq_cluster* c, int32_t i) {
  return c && i >= 0 && i < (int32_t)c->dbs.size() ? c->dbs[(size_t)i] : nullptr;
}

ddq_status ddq_cluster_submit(ddq_cluster* c, const ddq_plan* plan, int32_t* member, ddq_query* out) {
  if (!c || !plan || !member || !out) return set_error(DDQ_EINVAL, "cluster_submit");
  int best = 0;
  {
    std::lock_guard<std::mutex> g(c->mu);
    uint64_t best_r = 0;
    int64_t best_q = INT64_MAX;
    const size_t m = c->dbs.size();
    for (size_t k = 0; k < m; k++) {
      const size_t i = (c->rr + k) % m;  // full ties: round robin
      uint64_t total = 0;
      const uint64_t r = resident_bytes(c->dbs[i], *plan, &total);
      const int64_t q = c->inflight[i]->load();
      if (k == 0 || r > best_r || (r == best_r && q < best_q)) {
        best = (int)i;
        best_r = r;
        best_q = q;
      }
    }
    c->rr++;
    c->inflight[(size_t)best]->fetch_add(1);
  }
  ddq_status s = ddq_submit(c->dbs[(size_t)best], plan, out);
  if (s != DDQ_OK) {
    c->inflight[(size_t)best]->fetch_sub(1);
    return s;
  }
  *member = best;
  return DDQ_OK;
}

ddq_status ddq_cluster_fetch(ddq_cluster* c, int32_t member, ddq_query q, ddq_result** out) {
  if (!c || member < 0 || member >= (int32_t)c->dbs.size()) return set_error(DDQ_EINVAL, "cluster_fetch");
  ddq_status s = ddq_fetch(c->dbs[(size_t)member], q, out);
  c->inflight[(size_t)member]->fetch_sub(1);
  return s;
}

ddq_status ddq_cluster_update_placement(ddq_cluster* c) {
  if (!c) return set_error(DDQ_EINVAL, "cluster_update_placement");
  for (ddq_db* d : c->dbs)
    if (ddq_status s = ddq_update_placement(d)) return s;
  return DDQ_OK;
}

}  // extern "C"
