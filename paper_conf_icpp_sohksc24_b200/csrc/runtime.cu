// Host runtime of libcstf: error plumbing, device info, buffers, launch
// counter, NCCL (loaded at run time) and the row partitioner.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstring>
#include <mutex>
#include <numeric>

#include "internal.h"

namespace cstf {

static thread_local std::string g_err;
static std::atomic<int64_t> g_launches{0};

void set_error(const std::string& msg) { g_err = msg; }
cstf_status fail(cstf_status s, const std::string& msg) {
  g_err = std::string(cstf_status_string(s)) + ": " + msg;
  return s;
}
cstf_status cuda_fail(cudaError_t e, const char* what) {
  cstf_status s = (e == cudaErrorMemoryAllocation) ? CSTF_ERR_OUT_OF_MEMORY : CSTF_ERR_CUDA;
  g_err = std::string(cudaGetErrorName(e)) + " (" + cudaGetErrorString(e) + ") in " + what;
  return s;
}
void count_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

const DeviceInfo& device_info() {
  static thread_local DeviceInfo info[64];
  int dev = 0;
  cudaGetDevice(&dev);
  DeviceInfo& d = info[dev & 63];
  if (d.device != dev) {
    d.device = dev;
    cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev);
    int l2 = 0;
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    d.l2 = (size_t)l2;
    cudaDeviceGetAttribute(&d.max_smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  }
  return d;
}

void DevBuf::release() {
  if (p) cudaFree(p);
  p = nullptr;
  bytes = 0;
}
cstf_status DevBuf::alloc(size_t n) {
  release();
  if (n == 0) return CSTF_OK;
  cudaError_t e = cudaMalloc(&p, n);
  if (e != cudaSuccess) {
    p = nullptr;
    cudaGetLastError();
    return cuda_fail(e, "cudaMalloc");
  }
  bytes = n;
  return CSTF_OK;
}
cstf_status DevBuf::ensure(size_t n) {
  if (n <= bytes) return CSTF_OK;
  return alloc(n);
}

// ------------------------------------------------------------------ NCCL (dlopen)
namespace {
struct NcclApi {
  bool tried = false, ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};
NcclApi g_nccl;
std::mutex g_nccl_mu;

cstf_status nccl_load() {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  if (g_nccl.tried) return g_nccl.ok ? CSTF_OK : fail(CSTF_ERR_NCCL, "libnccl.so.2 not loadable");
  g_nccl.tried = true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) return fail(CSTF_ERR_NCCL, std::string("dlopen libnccl.so.2: ") + dlerror());
#define LOAD(name) g_nccl.name = reinterpret_cast<decltype(g_nccl.name)>(dlsym(h, "nccl" #name))
  LOAD(GetUniqueId); LOAD(CommInitRank); LOAD(CommDestroy); LOAD(AllReduce); LOAD(AllGather);
  LOAD(GetErrorString);
#undef LOAD
  g_nccl.ok = g_nccl.GetUniqueId && g_nccl.CommInitRank && g_nccl.CommDestroy && g_nccl.AllReduce &&
              g_nccl.AllGather;
  return g_nccl.ok ? CSTF_OK : fail(CSTF_ERR_NCCL, "libnccl.so.2 lacks required symbols");
}
cstf_status nccl_check(ncclResult_t r, const char* what) {
  if (r == ncclSuccess) return CSTF_OK;
  std::string m = what;
  if (g_nccl.GetErrorString) m += std::string(": ") + g_nccl.GetErrorString(r);
  return fail(CSTF_ERR_NCCL, m);
}
}  // namespace

int comm_nranks(const cstf_comm* c) { return c ? c->c.nranks : 1; }
int comm_rank(const cstf_comm* c) { return c ? c->c.rank : 0; }

cstf_status comm_allreduce_f64(const cstf_comm* c, double* d_buf, size_t count, cudaStream_t st) {
  if (!c || count == 0 || (c->c.nranks <= 1 && !c->c.nccl)) return CSTF_OK;
  if (c->c.host_allreduce) {
    std::vector<double> h(count);
    CSTF_CUDA(cudaMemcpyAsync(h.data(), d_buf, count * 8, cudaMemcpyDeviceToHost, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    if (c->c.host_allreduce(h.data(), (int64_t)count, c->c.user) != 0)
      return fail(CSTF_ERR_NCCL, "host all-reduce callback failed");
    CSTF_CUDA(cudaMemcpyAsync(d_buf, h.data(), count * 8, cudaMemcpyHostToDevice, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    return CSTF_OK;
  }
  return nccl_check(g_nccl.AllReduce(d_buf, d_buf, count, ncclFloat64, ncclSum,
                                     (ncclComm_t)c->c.nccl, st), "ncclAllReduce");
}
cstf_status comm_allgather_f64(const cstf_comm* c, const double* d_send, double* d_recv,
                               size_t count_per_rank, cudaStream_t st) {
  if (!c || (c->c.nranks <= 1 && !c->c.nccl)) {
    if (d_send != d_recv && count_per_rank)
      CSTF_CUDA(cudaMemcpyAsync(d_recv, d_send, count_per_rank * 8, cudaMemcpyDeviceToDevice, st));
    return CSTF_OK;
  }
  if (c->c.host_allgather) {
    const size_t P = (size_t)c->c.nranks;
    std::vector<double> hs(count_per_rank), hr(count_per_rank * P);
    CSTF_CUDA(cudaMemcpyAsync(hs.data(), d_send, count_per_rank * 8, cudaMemcpyDeviceToHost, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    if (c->c.host_allgather(hs.data(), hr.data(), (int64_t)count_per_rank, c->c.user) != 0)
      return fail(CSTF_ERR_NCCL, "host all-gather callback failed");
    CSTF_CUDA(cudaMemcpyAsync(d_recv, hr.data(), hr.size() * 8, cudaMemcpyHostToDevice, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    return CSTF_OK;
  }
  return nccl_check(g_nccl.AllGather(d_send, d_recv, count_per_rank, ncclFloat64,
                                     (ncclComm_t)c->c.nccl, st), "ncclAllGather");
}

}  // namespace cstf

using namespace cstf;

extern "C" {

const char* cstf_status_string(cstf_status s) {
  switch (s) {
    case CSTF_OK: return "CSTF_OK";
    case CSTF_ERR_INVALID_ARG: return "CSTF_ERR_INVALID_ARG";
    case CSTF_ERR_UNSUPPORTED: return "CSTF_ERR_UNSUPPORTED";
    case CSTF_ERR_OUT_OF_MEMORY: return "CSTF_ERR_OUT_OF_MEMORY";
    case CSTF_ERR_CUDA: return "CSTF_ERR_CUDA";
    case CSTF_ERR_NCCL: return "CSTF_ERR_NCCL";
    case CSTF_ERR_NOT_SPD: return "CSTF_ERR_NOT_SPD";
    case CSTF_ERR_NUMERIC: return "CSTF_ERR_NUMERIC";
  }
  return "CSTF_ERR_UNKNOWN";
}

const char* cstf_last_error_message(void) { return g_err.c_str(); }
int cstf_version(void) { return CSTF_VERSION_MAJOR * 100 + CSTF_VERSION_MINOR; }
int64_t cstf_kernel_launch_count(void) { return g_launches.load(); }

cstf_status cstf_get_unique_id(unsigned char id[128]) {
  if (!id) return fail(CSTF_ERR_INVALID_ARG, "id is NULL");
  CSTF_TRY(nccl_load());
  ncclUniqueId u;
  CSTF_TRY(nccl_check(g_nccl.GetUniqueId(&u), "ncclGetUniqueId"));
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  memcpy(id, &u, 128);
  return CSTF_OK;
}

cstf_status cstf_comm_create(int nranks, int rank, const unsigned char id[128], cstf_comm** out) {
  if (!out || !id || nranks < 1 || rank < 0 || rank >= nranks)
    return fail(CSTF_ERR_INVALID_ARG, "cstf_comm_create arguments");
  *out = nullptr;
  cstf_comm* c = new cstf_comm();
  c->c.nranks = nranks;
  c->c.rank = rank;
  {   // also for one rank: the same NCCL calls run (a 1-rank job exercises the transport)
    cstf_status s = nccl_load();
    if (s != CSTF_OK) { delete c; return s; }
    ncclUniqueId u;
    memcpy(&u, id, 128);
    ncclComm_t nc = nullptr;
    s = nccl_check(g_nccl.CommInitRank(&nc, nranks, u, rank), "ncclCommInitRank");
    if (s != CSTF_OK) { delete c; return s; }
    c->c.nccl = nc;
  }
  *out = c;
  return CSTF_OK;
}

cstf_status cstf_comm_create_host(int nranks, int rank, cstf_host_allreduce_fn allreduce,
                                  cstf_host_allgather_fn allgather, void* user, cstf_comm** out) {
  if (!out || nranks < 1 || rank < 0 || rank >= nranks || !allreduce || !allgather)
    return fail(CSTF_ERR_INVALID_ARG, "cstf_comm_create_host arguments");
  cstf_comm* c = new cstf_comm();
  c->c.nranks = nranks;
  c->c.rank = rank;
  c->c.host_allreduce = allreduce;
  c->c.host_allgather = allgather;
  c->c.user = user;
  *out = c;
  return CSTF_OK;
}

}  // extern "C"

// ------------------------------------------------------------------ loopback group
// cstf_comm_loopback: nparts communicators of ONE process (one thread per part,
// sharing a GPU).  Collectives meet at a host barrier; the all-reduce sums the
// parts' host copies in rank order (identical bits on every part), the all-gather
// concatenates them.  A part that does not arrive within kLoopTimeout makes the
// collective fail (CSTF_ERR_NCCL) instead of hanging.
namespace {
constexpr auto kLoopTimeout = std::chrono::seconds(120);
struct LoopGroup {
  int n = 0;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  bool broken = false;
  std::vector<const double*> src;
  std::atomic<int> refs{0};
  bool barrier() {
    std::unique_lock<std::mutex> lk(mu);
    if (broken) return false;
    const uint64_t g = gen;
    if (++arrived == n) {
      arrived = 0;
      gen++;
      cv.notify_all();
      return true;
    }
    if (!cv.wait_for(lk, kLoopTimeout, [&] { return gen != g || broken; }) || broken) {
      broken = true;
      cv.notify_all();
      return false;
    }
    return true;
  }
};
struct LoopMember {
  LoopGroup* g;
  int rank;
};
int loop_allreduce(double* buf, int64_t count, void* user) {
  LoopMember* m = static_cast<LoopMember*>(user);
  LoopGroup* g = m->g;
  std::vector<double> mine(buf, buf + count);
  g->src[(size_t)m->rank] = mine.data();
  if (!g->barrier()) return 1;
  for (int64_t i = 0; i < count; i++) {
    double s = 0.0;
    for (int r = 0; r < g->n; r++) s += g->src[(size_t)r][i];
    buf[i] = s;
  }
  return g->barrier() ? 0 : 1;       // nobody releases `mine` while others still read it
}
int loop_allgather(const double* send, double* recv, int64_t count, void* user) {
  LoopMember* m = static_cast<LoopMember*>(user);
  LoopGroup* g = m->g;
  g->src[(size_t)m->rank] = send;
  if (!g->barrier()) return 1;
  for (int r = 0; r < g->n; r++) memcpy(recv + (size_t)r * count, g->src[(size_t)r], (size_t)count * 8);
  return g->barrier() ? 0 : 1;
}
}  // namespace

extern "C" {

cstf_status cstf_comm_loopback(int nparts, cstf_comm** out) {
  if (!out || nparts < 1 || nparts > 64) return fail(CSTF_ERR_INVALID_ARG, "cstf_comm_loopback arguments");
  LoopGroup* g = new LoopGroup();
  g->n = nparts;
  g->src.assign((size_t)nparts, nullptr);
  g->refs = nparts;
  for (int r = 0; r < nparts; r++) {
    cstf_comm* c = new cstf_comm();
    c->c.nranks = nparts;
    c->c.rank = r;
    c->c.host_allreduce = loop_allreduce;
    c->c.host_allgather = loop_allgather;
    LoopMember* m = new LoopMember{g, r};
    c->c.user = m;
    c->c.loop = m;
    out[r] = c;
  }
  return CSTF_OK;
}

cstf_status cstf_comm_info(const cstf_comm* comm, int* nranks, int* rank) {
  if (!comm) return fail(CSTF_ERR_INVALID_ARG, "comm is NULL");
  if (nranks) *nranks = comm->c.nranks;
  if (rank) *rank = comm->c.rank;
  return CSTF_OK;
}

void cstf_comm_destroy(cstf_comm* comm) {
  if (!comm) return;
  if (comm->c.nccl && g_nccl.CommDestroy) g_nccl.CommDestroy((ncclComm_t)comm->c.nccl);
  if (comm->c.loop) {
    LoopMember* m = static_cast<LoopMember*>(comm->c.loop);
    if (--m->g->refs == 0) delete m->g;
    delete m;
  }
  delete comm;
}

cstf_status cstf_partition_rows(int64_t I, const int64_t* counts, int nranks, int32_t* owner,
                                int64_t* local) {
  if (I < 0 || nranks < 1 || (I > 0 && (!counts || !owner || !local)))
    return fail(CSTF_ERR_INVALID_ARG, "cstf_partition_rows arguments");
  std::vector<int64_t> order((size_t)I);
  std::iota(order.begin(), order.end(), 0);
  std::stable_sort(order.begin(), order.end(),
                   [&](int64_t a, int64_t b) { return counts[a] > counts[b]; });
  std::vector<int64_t> next((size_t)nranks, 0);
  for (int64_t t = 0; t < I; t++) {
    int64_t round = t / nranks, pos = t % nranks;
    int r = (round % 2 == 0) ? (int)pos : (int)(nranks - 1 - pos);   // snake order
    int64_t row = order[(size_t)t];
    owner[row] = r;
    local[row] = next[(size_t)r]++;
  }
  return CSTF_OK;
}

}  // extern "C"
