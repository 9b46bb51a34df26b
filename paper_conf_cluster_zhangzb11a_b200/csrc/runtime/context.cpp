// Error state, device setup and NCCL plumbing of the runtime.
#include <cstdarg>
#include <cstdio>
#include <chrono>
#include <cstdlib>
#include <map>
#include <mutex>
#include <thread>

#include "internal.h"

namespace gpa {

namespace {
thread_local std::string t_last_error = "no error";
}

void set_last_error(gpa_status st, const std::string& msg) {
  (void)st;
  t_last_error = msg;
}

const char* last_error_cstr() { return t_last_error.c_str(); }



void fail(gpa_status st, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  throw Error{st, std::string(buf)};
}

DeviceInfo use_device(int requested) {
  static std::mutex mu;
  static bool pool_done[64] = {false};
  static int sms[64] = {0};
  int dev = requested;
  if (dev < 0) GPA_CUDA(cudaGetDevice(&dev));
  int n_dev = 0;
  GPA_CUDA(cudaGetDeviceCount(&n_dev));
  GPA_REQUIRE(dev >= 0 && dev < n_dev && dev < 64, GPA_ERR_INVALID, "invalid CUDA device %d (have %d)", dev, n_dev);
  GPA_CUDA(cudaSetDevice(dev));
  std::lock_guard<std::mutex> lk(mu);
  if (!pool_done[dev]) {
    int major = 0, minor = 0;
    GPA_CUDA(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev));
    GPA_CUDA(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev));
    GPA_REQUIRE(major == 10 && minor == 0, GPA_ERR_CUDA,
                "device %d is sm_%d%d; this library is built for sm_100a (B200) only", dev, major, minor);
    cudaMemPool_t pool;
    GPA_CUDA(cudaDeviceGetDefaultMemPool(&pool, dev));
    uint64_t thr = UINT64_MAX;
    GPA_CUDA(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
    GPA_CUDA(cudaDeviceGetAttribute(&sms[dev], cudaDevAttrMultiProcessorCount, dev));
    pool_done[dev] = true;
  }
  return DeviceInfo{dev, sms[dev]};
}

#define GPA_NCCL(call)                                                                                    \
  do {                                                                                                    \
    ncclResult_t r_ = (call);                                                                             \
    if (r_ != ncclSuccess) ::gpa::fail(GPA_ERR_NCCL, "%s failed: %s", #call, ncclGetErrorString(r_));     \
  } while (0)

void dist_check(const gpa_dist* d) {
  if (!d) return;
  GPA_REQUIRE(!d->failed, GPA_ERR_STATE, "communicator unusable after a failed collective");
}

namespace {

thread_local const gpa_dist* t_scope = nullptr;

[[noreturn]] void dist_abort(const gpa_dist* d, const char* why) {
  auto* m = const_cast<gpa_dist*>(d);
  m->failed = true;
  if (m->comm) {
    ncclCommAbort(m->comm);   // unblocks this rank's pending NCCL kernels
    m->comm = nullptr;
  }
  fail(GPA_ERR_NCCL, "collective failed on rank %d of %d: %s", d->rank, d->world, why);
}

void log_collective(const gpa_dist* d, size_t n, uint32_t dtype, uint32_t op) {
  const_cast<gpa_dist*>(d)->log.push_back(((uint64_t)op << 60) | ((uint64_t)dtype << 56) | (uint64_t)n);
}

void collective(const gpa_dist* d, void* buf, size_t n, uint32_t dtype, uint32_t op, cudaStream_t s) {
  if (!d || n == 0) return;  // a 1-rank communicator still runs the collective (exercises NCCL)
  dist_check(d);
  log_collective(d, n, dtype, op);
  const size_t bytes = n * (dtype == GPA_DT_U64 ? 8 : 4);
  if (d->host_fn) {
    auto* m = const_cast<gpa_dist*>(d);
    if (m->stage_bytes < bytes) {
      if (m->stage) cudaFreeHost(m->stage);
      m->stage = nullptr;
      m->stage_bytes = 0;
      GPA_CUDA(cudaHostAlloc(&m->stage, bytes, cudaHostAllocDefault));
      m->stage_bytes = bytes;
    }
    GPA_CUDA(cudaMemcpyAsync(m->stage, buf, bytes, cudaMemcpyDeviceToHost, s));
    GPA_CUDA(cudaStreamSynchronize(s));
    const int rc = d->host_fn(d->host_ctx, m->stage, (uint64_t)n, dtype, op);
    if (rc != 0) {
      m->failed = true;
      fail(GPA_ERR_NCCL, "host all-reduce callback returned %d on rank %d", rc, d->rank);
    }
    GPA_CUDA(cudaMemcpyAsync(buf, m->stage, bytes, cudaMemcpyHostToDevice, s));
    GPA_CUDA(cudaStreamSynchronize(s));   // the staging buffer is reused by the next collective
    return;
  }
  const ncclDataType_t t = dtype == GPA_DT_U64 ? ncclUint64 : ncclUint32;
  ncclResult_t r = ncclAllReduce(buf, buf, n, t, op == GPA_OP_MAX ? ncclMax : ncclSum, d->comm, s);
  if (r != ncclSuccess) dist_abort(d, ncclGetErrorString(r));
}
}  // namespace

DistScope::DistScope(const gpa_dist* d) : prev(t_scope) { t_scope = d; }
DistScope::~DistScope() { t_scope = prev; }

}  // namespace gpa

namespace gpa {
namespace {
std::mutex g_bundle_mu;
std::vector<StreamBundle*>& free_bundles() {
  static auto* v = new std::vector<StreamBundle*>();   // never destroyed (used until process exit)
  return *v;
}
}  // namespace

StreamBundle* acquire_bundle(int device) {
  {
    std::lock_guard<std::mutex> lk(g_bundle_mu);
    auto& v = free_bundles();
    for (size_t i = 0; i < v.size(); ++i)
      if (v[i]->device == device) {
        StreamBundle* b = v[i];
        v.erase(v.begin() + (long)i);
        return b;
      }
  }
  auto* b = new StreamBundle();
  b->device = device;
  GPA_CUDA(cudaStreamCreateWithFlags(&b->s, cudaStreamNonBlocking));
  for (auto& e : b->ev) GPA_CUDA(cudaEventCreate(&e));
  return b;
}

void release_bundle(StreamBundle* b) {
  if (!b) return;
  std::lock_guard<std::mutex> lk(g_bundle_mu);
  free_bundles().push_back(b);
}
}  // namespace gpa

void gpa::stream_wait(cudaStream_t s) {
  const gpa_dist* d = t_scope;
  if (!d || !d->comm) {
    GPA_CUDA(cudaStreamSynchronize(s));
    return;
  }
  // poll: stream done? asynchronous NCCL error? timeout?
  const double t0 = wall_ms();
  for (uint32_t it = 0;; ++it) {
    const cudaError_t q = cudaStreamQuery(s);
    if (q == cudaSuccess) return;
    if (q != cudaErrorNotReady) GPA_CUDA(q);
    ncclResult_t ar = ncclSuccess;
    if (ncclCommGetAsyncError(d->comm, &ar) == ncclSuccess && ar != ncclSuccess && ar != ncclInProgress)
      dist_abort(d, ncclGetErrorString(ar));
    if (d->timeout_s > 0 && (it & 255) == 0 && wall_ms() - t0 > d->timeout_s * 1e3)
      dist_abort(d, "timed out waiting for the stream (a peer rank failed or left the collective sequence)");
    if (it > 64) std::this_thread::sleep_for(std::chrono::microseconds(20));
  }
}

namespace gpa {

void allreduce_sum_u32(const gpa_dist* d, uint32_t* buf, size_t n, cudaStream_t s) {
  collective(d, buf, n, GPA_DT_U32, GPA_OP_SUM, s);
}
void allreduce_sum_u64(const gpa_dist* d, uint64_t* buf, size_t n, cudaStream_t s) {
  collective(d, buf, n, GPA_DT_U64, GPA_OP_SUM, s);
}
void allreduce_max_u32(const gpa_dist* d, uint32_t* buf, size_t n, cudaStream_t s) {
  collective(d, buf, n, GPA_DT_U32, GPA_OP_MAX, s);
}

void dist_agree_max(const gpa_dist* d, uint32_t* vals, size_t n) {
  if (!d || n == 0) return;
  dist_check(d);
  use_device(d->device);
  struct Ws {   // per thread: a small device buffer and a stream per device
    std::map<int, std::pair<cudaStream_t, uint32_t*>> m;
    ~Ws() {
      for (auto& kv : m) {
        cudaFree(kv.second.second);
        cudaStreamDestroy(kv.second.first);
      }
    }
  };
  thread_local Ws ws;
  auto it = ws.m.find(d->device);
  if (it == ws.m.end()) {
    cudaStream_t st = nullptr;
    uint32_t* p = nullptr;
    GPA_CUDA(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    GPA_CUDA(cudaMalloc(reinterpret_cast<void**>(&p), 64 * sizeof(uint32_t)));
    it = ws.m.emplace(d->device, std::make_pair(st, p)).first;
  }
  GPA_REQUIRE(n <= 64, GPA_ERR_INVALID, "dist_agree_max: too many values");
  cudaStream_t st = it->second.first;
  uint32_t* p = it->second.second;
  GPA_CUDA(cudaMemcpyAsync(p, vals, n * 4, cudaMemcpyHostToDevice, st));
  allreduce_max_u32(d, p, n, st);
  GPA_CUDA(cudaMemcpyAsync(vals, p, n * 4, cudaMemcpyDeviceToHost, st));
  DistScope scope(d);
  stream_wait(st);
}

}  // namespace gpa

// ---------------------------------------------------------------- C ABI: dist

extern "C" gpa_status gpa_dist_unique_id(uint8_t id_out[128]) {
  return gpa::guard([&] {
    GPA_REQUIRE(id_out, GPA_ERR_INVALID, "id_out is NULL");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    ncclUniqueId id;
    GPA_NCCL(ncclGetUniqueId(&id));
    memcpy(id_out, &id, 128);
  });
}

extern "C" gpa_status gpa_dist_create(int rank, int world, int device, const uint8_t id[128], gpa_dist** out) {
  return gpa::guard([&] {
    GPA_REQUIRE(out && id, GPA_ERR_INVALID, "NULL argument");
    GPA_REQUIRE(world >= 1 && rank >= 0 && rank < world, GPA_ERR_INVALID, "bad rank %d / world %d", rank, world);
    gpa::DeviceInfo di = gpa::use_device(device);
    auto* d = new gpa_dist();
    d->rank = rank;
    d->world = world;
    d->device = di.device;
    ncclUniqueId uid;
    memcpy(&uid, id, 128);
    ncclResult_t r = ncclCommInitRank(&d->comm, world, uid, rank);
    if (r != ncclSuccess) {
      delete d;
      gpa::fail(GPA_ERR_NCCL, "ncclCommInitRank failed: %s", ncclGetErrorString(r));
    }
    *out = d;
  });
}

extern "C" gpa_status gpa_dist_create_host(int rank, int world, int device, gpa_host_allreduce_fn fn, void* ctx,
                                           gpa_dist** out) {
  return gpa::guard([&] {
    GPA_REQUIRE(out && fn, GPA_ERR_INVALID, "NULL argument");
    GPA_REQUIRE(world >= 1 && rank >= 0 && rank < world, GPA_ERR_INVALID, "bad rank %d / world %d", rank, world);
    gpa::DeviceInfo di = gpa::use_device(device);
    auto* d = new gpa_dist();
    d->rank = rank;
    d->world = world;
    d->device = di.device;
    d->host_fn = fn;
    d->host_ctx = ctx;
    *out = d;
  });
}

extern "C" gpa_status gpa_dist_destroy(gpa_dist* dist) {
  return gpa::guard([&] {
    if (!dist) return;
    if (dist->comm) ncclCommDestroy(dist->comm);
    if (dist->stage) cudaFreeHost(dist->stage);
    delete dist;
  });
}

extern "C" gpa_status gpa_dist_log(const gpa_dist* dist, uint64_t* entries, uint64_t cap, uint64_t* n_total) {
  return gpa::guard([&] {
    GPA_REQUIRE(dist, GPA_ERR_INVALID, "dist is NULL");
    GPA_REQUIRE(entries || cap == 0, GPA_ERR_INVALID, "entries is NULL");
    const uint64_t n = dist->log.size();
    if (n_total) *n_total = n;
    for (uint64_t i = 0; i < n && i < cap; ++i) entries[i] = dist->log[i];
  });
}

extern "C" gpa_status gpa_dist_set_timeout(gpa_dist* dist, double seconds) {
  return gpa::guard([&] {
    GPA_REQUIRE(dist, GPA_ERR_INVALID, "dist is NULL");
    dist->timeout_s = seconds;
  });
}

extern "C" gpa_status gpa_dist_info(const gpa_dist* dist, int* rank, int* world) {
  return gpa::guard([&] {
    GPA_REQUIRE(dist, GPA_ERR_INVALID, "dist is NULL");
    if (rank) *rank = dist->rank;
    if (world) *world = dist->world;
  });
}
