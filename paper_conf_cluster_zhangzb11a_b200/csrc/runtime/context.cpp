// Error state, device setup and NCCL plumbing of the runtime.
#include <cstdarg>
#include <cstdio>
#include <chrono>
#include <cstdlib>
#include <mutex>

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
void collective(const gpa_dist* d, void* buf, size_t n, ncclDataType_t t, ncclRedOp_t op, cudaStream_t s) {
  if (!d || n == 0) return;  // a 1-rank communicator still runs the collective (exercises NCCL)
  dist_check(d);
  ncclResult_t r = ncclAllReduce(buf, buf, n, t, op, d->comm, s);
  if (r != ncclSuccess) {
    const_cast<gpa_dist*>(d)->failed = true;
    fail(GPA_ERR_NCCL, "ncclAllReduce failed: %s", ncclGetErrorString(r));
  }
}
}  // namespace

void allreduce_sum_u32(const gpa_dist* d, uint32_t* buf, size_t n, cudaStream_t s) {
  collective(d, buf, n, ncclUint32, ncclSum, s);
}
void allreduce_sum_u64(const gpa_dist* d, uint64_t* buf, size_t n, cudaStream_t s) {
  collective(d, buf, n, ncclUint64, ncclSum, s);
}
void allreduce_max_u32(const gpa_dist* d, uint32_t* buf, size_t n, cudaStream_t s) {
  collective(d, buf, n, ncclUint32, ncclMax, s);
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

extern "C" gpa_status gpa_dist_destroy(gpa_dist* dist) {
  return gpa::guard([&] {
    if (!dist) return;
    if (dist->comm) ncclCommDestroy(dist->comm);
    delete dist;
  });
}

extern "C" gpa_status gpa_dist_info(const gpa_dist* dist, int* rank, int* world) {
  return gpa::guard([&] {
    GPA_REQUIRE(dist, GPA_ERR_INVALID, "dist is NULL");
    if (rank) *rank = dist->rank;
    if (world) *world = dist->world;
  });
}
