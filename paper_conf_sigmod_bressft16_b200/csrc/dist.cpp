// dist.cpp -- multi-GPU execution inside libddq (S8(e); Sec. 6.3: "Our
// Data-Driven strategy can support multiple co-processors by performing horizontal
// partitioning").  One process per GPU.  The fact table is range-sharded by row
// (each rank loads its rows; ddq_table_set_partitioned), dimension tables are
// replicated.  Two collectives:
//   * build once (ddq_dist_init_nccl with build_once = 1): a prepared plan's build over
//     a replicated table runs on rank 0 only and its index (join-index bitmap +
//     payload array + coarse bitmap, or the hash table) is broadcast to every rank
//     with ncclBroadcast on the plan's stream -- captured into the plan's CUDA graph
//     (serial capture: one NCCL stream order on every rank);
//   * partial aggregates: ddq_dist_exchange packs the compacted group table of each
//     prepared plan ([count, keys[cap], accs[cap * n_aggs * 2]] int64 words) into one
//     device buffer and all-gathers it (ncclAllGather over NVLink / NVSwitch, or a
//     host all-gather callback -- the gloo transport of the CPU tests);
//     ddq_dist_result merges the ranks' partials exactly (SUM / COUNT by int128
//     addition, MIN by minimum) and finalises (S8(a7)).
// NCCL is loaded at run time (dlopen "libnccl.so.2": the copy PyTorch already loaded,
// else the system one) so libddq has no link-time NCCL dependency.
#include <dlfcn.h>

#include <algorithm>
#include <cstring>
#include <vector>

#include <nccl.h>

#include "engine.h"
#include "ops_internal.h"

struct ddq_prepared;

namespace ddq {

// the prepared plans' internals this module reads (engine.cpp)
const ddq_plan& prepared_plan(const ddq_prepared* p);
ddq_status prepared_partials_device(ddq_prepared* p, int64_t** keys, int64_t** accs, uint32_t** count, int64_t* cap);

namespace {

struct Nccl {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  bool ok = false;
};

Nccl& nccl() {
  static Nccl n = [] {
    Nccl x;
    x.h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!x.h) return x;
    x.GetUniqueId = (decltype(x.GetUniqueId))dlsym(x.h, "ncclGetUniqueId");
    x.CommInitRank = (decltype(x.CommInitRank))dlsym(x.h, "ncclCommInitRank");
    x.CommDestroy = (decltype(x.CommDestroy))dlsym(x.h, "ncclCommDestroy");
    x.AllGather = (decltype(x.AllGather))dlsym(x.h, "ncclAllGather");
    x.Broadcast = (decltype(x.Broadcast))dlsym(x.h, "ncclBroadcast");
    x.GetErrorString = (decltype(x.GetErrorString))dlsym(x.h, "ncclGetErrorString");
    x.ok = x.GetUniqueId && x.CommInitRank && x.CommDestroy && x.AllGather && x.Broadcast && x.GetErrorString;
    return x;
  }();
  return n;
}

ddq_status nccl_status(ncclResult_t r, const char* where) {
  if (r == ncclSuccess) return DDQ_OK;
  return set_error(DDQ_ENCCL, std::string(where) + ": " + nccl().GetErrorString(r));
}

}  // namespace

struct DistState {
  int rank = 0, world = 1;
  ncclComm_t comm = nullptr;
  bool build_once = false;
  ddq_allgather_fn host_fn = nullptr;
  void* host_user = nullptr;
  // the last exchange
  std::vector<ddq_prepared*> plans;
  std::vector<int64_t> off;   // word offset of each plan in the packed buffer
  int64_t words = 0;          // packed words per rank
  int64_t* d_send = nullptr;  // device packed buffer (this rank)
  int64_t* d_recv = nullptr;  // device gathered buffer (NCCL path)
  size_t dcap = 0;
  std::vector<int64_t> h_send, h_recv;
  cudaStream_t stream = nullptr;
  bool host_ready = false;
};

static DistState* dist_of(ddq_db* db) { return db ? (DistState*)db->dist : nullptr; }

// words of one plan's packed partials: [count, keys[cap], accs[cap * na * 2]]
static int64_t packed_words(int64_t cap, int na) { return 1 + cap + cap * na * 2; }

void dist_free(ddq_db* db) {
  DistState* d = dist_of(db);
  if (!d) return;
  cudaSetDevice(db->device);
  if (d->stream) cudaStreamSynchronize(d->stream);
  if (d->comm) nccl().CommDestroy(d->comm);
  if (d->d_send) cudaFree(d->d_send);
  if (d->d_recv) cudaFree(d->d_recv);
  delete d;
  db->dist = nullptr;
}

// Build once (called by run_gpu_op for a HASH_BUILD in a prepared plan): true if this
// rank must not build this table's index itself (it receives rank 0's copy).
bool dist_build_receives(ddq_db* db, const ddq_op& op) {
  DistState* d = dist_of(db);
  if (!d || !d->comm || !d->build_once || d->world < 2) return false;
  if (op.table < 0 || op.table >= (int)db->tables.size() || db->tables[(size_t)op.table].partitioned) return false;
  return d->rank != 0;
}

// ... and the broadcast of its index bytes from rank 0, on the op's stream.
ddq_status dist_build_broadcast(ddq_db* db, const ddq_op& op, void* buf, size_t bytes, cudaStream_t st) {
  DistState* d = dist_of(db);  // (also at world 1: an in-place self-broadcast, so the path is testable)
  if (!d || !d->comm || !d->build_once || !buf || !bytes) return DDQ_OK;
  if (op.table < 0 || op.table >= (int)db->tables.size() || db->tables[(size_t)op.table].partitioned) return DDQ_OK;
  return nccl_status(nccl().Broadcast(buf, buf, bytes, ncclUint8, 0, d->comm, st), "build broadcast");
}

bool dist_serial_capture(ddq_db* db) {
  DistState* d = dist_of(db);
  return d && d->comm && d->build_once;
}

}  // namespace ddq

using namespace ddq;

extern "C" {

ddq_status ddq_dist_nccl_unique_id(void* out128) {
  if (!out128) return set_error(DDQ_EINVAL, "dist_nccl_unique_id: null");
  if (!nccl().ok) return set_error(DDQ_ENCCL, "libnccl.so.2 not loadable");
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  ncclUniqueId id;
  if (ddq_status s = nccl_status(nccl().GetUniqueId(&id), "ncclGetUniqueId")) return s;
  std::memcpy(out128, &id, 128);
  return DDQ_OK;
}

ddq_status ddq_dist_init_nccl(ddq_db* db, const void* id128, int32_t rank, int32_t world, int32_t build_once) {
  if (!db || !id128 || world < 1 || rank < 0 || rank >= world) return set_error(DDQ_EINVAL, "dist_init_nccl");
  if (db->dist) return set_error(DDQ_ESTATE, "dist_init_nccl: already initialised");
  if (!nccl().ok) return set_error(DDQ_ENCCL, "libnccl.so.2 not loadable");
  cudaSetDevice(db->device);
  auto* d = new DistState();
  d->rank = rank;
  d->world = world;
  d->build_once = build_once != 0;
  ncclUniqueId id;
  std::memcpy(&id, id128, 128);
  ddq_status s = nccl_status(nccl().CommInitRank(&d->comm, world, id, rank), "ncclCommInitRank");
  if (s != DDQ_OK) {
    delete d;
    return s;
  }
  db->dist = d;
  db->cfg.rank = rank;
  db->cfg.world = world;
  return DDQ_OK;
}

ddq_status ddq_dist_init_host(ddq_db* db, int32_t rank, int32_t world, ddq_allgather_fn fn, void* user) {
  if (!db || !fn || world < 1 || rank < 0 || rank >= world) return set_error(DDQ_EINVAL, "dist_init_host");
  if (db->dist) return set_error(DDQ_ESTATE, "dist_init_host: already initialised");
  auto* d = new DistState();
  d->rank = rank;
  d->world = world;
  d->host_fn = fn;
  d->host_user = user;
  db->dist = d;
  db->cfg.rank = rank;
  db->cfg.world = world;
  return DDQ_OK;
}

ddq_status ddq_table_set_partitioned(ddq_db* db, ddq_table t, int32_t partitioned) {
  if (!db) return set_error(DDQ_EINVAL, "table_set_partitioned");
  std::lock_guard<std::mutex> g(db->mu);
  if (t < 0 || t >= (int)db->tables.size()) return set_error(DDQ_ENOTFOUND, "table_set_partitioned: bad table");
  db->tables[(size_t)t].partitioned = partitioned != 0;
  return DDQ_OK;
}

ddq_status ddq_dist_exchange(ddq_db* db, ddq_prepared* const* plans, int32_t n, void* stream) {
  DistState* d = dist_of(db);
  if (!d) return set_error(DDQ_ESTATE, "dist_exchange: ddq_dist_init_* first");
  if (!plans || n < 1) return set_error(DDQ_EINVAL, "dist_exchange: no plans");
  cudaSetDevice(db->device);
  cudaStream_t st = (cudaStream_t)stream;
  d->plans.assign(plans, plans + n);
  d->off.assign((size_t)n, 0);
  int64_t words = 0;
  std::vector<int64_t*> k((size_t)n), a((size_t)n);
  std::vector<uint32_t*> c((size_t)n);
  std::vector<int64_t> cap((size_t)n);
  for (int i = 0; i < n; i++) {
    if (ddq_status s = prepared_partials_device(plans[i], &k[(size_t)i], &a[(size_t)i], &c[(size_t)i], &cap[(size_t)i]))
      return s;
    d->off[(size_t)i] = words;
    words += packed_words(cap[(size_t)i], prepared_plan(plans[i]).ops[prepared_plan(plans[i]).n_ops - 1].n_aggs);
  }
  d->words = words;
  const size_t bytes = (size_t)words * 8;
  if (d->dcap < bytes) {
    if (d->d_send) cudaFree(d->d_send);
    if (d->d_recv) cudaFree(d->d_recv);
    d->d_send = d->d_recv = nullptr;
    if (cudaMalloc(&d->d_send, bytes) != cudaSuccess ||
        (d->comm && cudaMalloc(&d->d_recv, bytes * (size_t)d->world) != cudaSuccess))
      return set_error(DDQ_ENOMEM_DEVICE, "dist_exchange: buffers");
    d->dcap = bytes;
  }
  // pack on the stream: the count cell (uint32) widened into word 0, keys, accs
  for (int i = 0; i < n; i++) {
    int64_t* w = d->d_send + d->off[(size_t)i];
    const int na = prepared_plan(plans[i]).ops[prepared_plan(plans[i]).n_ops - 1].n_aggs;
    cudaError_t e = cudaMemsetAsync(w, 0, 8, st);
    if (e == cudaSuccess) e = cudaMemcpyAsync(w, c[(size_t)i], 4, cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(w + 1, k[(size_t)i], (size_t)cap[(size_t)i] * 8, cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(w + 1 + cap[(size_t)i], a[(size_t)i], (size_t)cap[(size_t)i] * na * 16,
                          cudaMemcpyDeviceToDevice, st);
    if (e != cudaSuccess) return cuda_status(e, "dist_exchange: pack");
  }
  d->stream = st;
  d->host_ready = false;
  if (d->comm)  // all ranks' packed buffers, rank-major, on the device (NVLink / NVSwitch)
    return nccl_status(nccl().AllGather(d->d_send, d->d_recv, (size_t)words, ncclInt64, d->comm, st),
                       "ncclAllGather");
  // host transport (gloo tests): D2H, the caller's all-gather, kept on the host
  d->h_send.resize((size_t)words);
  d->h_recv.resize((size_t)words * d->world);
  cudaError_t e = cudaMemcpyAsync(d->h_send.data(), d->d_send, bytes, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_status(e, "dist_exchange: D2H");
  if (d->host_fn(d->h_send.data(), d->h_recv.data(), bytes, d->host_user) != 0)
    return set_error(DDQ_ENCCL, "dist_exchange: host all-gather failed");
  d->host_ready = true;
  return DDQ_OK;
}

ddq_status ddq_dist_result(ddq_db* db, int32_t i, ddq_result** out) {
  DistState* d = dist_of(db);
  if (!d || d->plans.empty()) return set_error(DDQ_ESTATE, "dist_result: no exchange");
  if (!out || i < 0 || i >= (int)d->plans.size()) return set_error(DDQ_EINVAL, "dist_result: bad plan index");
  if (!d->host_ready) {  // NCCL path: the gathered buffer to the host once per exchange
    cudaSetDevice(db->device);
    d->h_recv.resize((size_t)d->words * d->world);
    cudaError_t e = cudaMemcpyAsync(d->h_recv.data(), d->d_recv, (size_t)d->words * d->world * 8,
                                    cudaMemcpyDeviceToHost, d->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(d->stream);
    if (e != cudaSuccess) return cuda_status(e, "dist_result: D2H");
    d->host_ready = true;
  }
  const ddq_plan& plan = prepared_plan(d->plans[(size_t)i]);
  const ddq_op& root = plan.ops[plan.n_ops - 1];
  const int na = root.n_aggs;
  int64_t* kp = nullptr;
  int64_t* ap = nullptr;
  uint32_t* cp = nullptr;
  int64_t cap = 0;
  if (ddq_status s = prepared_partials_device(d->plans[(size_t)i], &kp, &ap, &cp, &cap)) return s;
  std::vector<int64_t> keys, accs;
  for (int r = 0; r < d->world; r++) {
    const int64_t* w = d->h_recv.data() + (size_t)r * d->words + d->off[(size_t)i];
    const int64_t g = w[0];
    if (g < 0 || g > cap) return set_error(DDQ_EINVAL, "dist_result: corrupt partials");
    keys.insert(keys.end(), w + 1, w + 1 + g);
    for (int64_t x = 0; x < g; x++)  // group-major accs of group x
      accs.insert(accs.end(), w + 1 + cap + x * na * 2, w + 1 + cap + (x + 1) * na * 2);
  }
  ddq_status s = finalize_result(root, (int64_t)keys.size(), keys.data(), accs.data(), out);
  if (s == DDQ_OK) decode_result_keys(db, plan, *out);
  return s;
}

}  // extern "C"
