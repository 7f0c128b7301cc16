// Communicators for the value-range row-sharded fit (dt_fit_sharded).
//
// Two backends behind one interface, both stream-ordered from the caller's view:
//   * NCCL (one process per GPU; NVLink / NVSwitch): ncclAllGather / ncclAllReduce on the
//     fit's stream.  libnccl.so.2 is dlopen'ed on first use (the one torch already loaded
//     when present), so libdt.so itself has no hard NCCL dependency.
//   * local: `world` ranks as host threads of ONE process (same or different devices),
//     exchanging through device-to-device copies behind a host barrier.  Used to run and
//     verify the sharded path on a single GPU.
#include <dlfcn.h>
#include <nccl.h>
#include <string.h>

#include <condition_variable>
#include <memory>
#include <mutex>
#include <vector>

#include "dt_internal.cuh"

namespace dtl {

namespace {

// ---- NCCL entry points (dlopen)
struct NcclApi {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  bool ok = false;
};
NcclApi g_nccl;
std::mutex g_nccl_mu;

bool load_nccl() {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  if (g_nccl.ok) return true;
  const char* names[] = {"libnccl.so.2", "libnccl.so"};
  for (const char* nm : names) {
    g_nccl.h = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
    if (g_nccl.h) break;
  }
  if (!g_nccl.h) return false;
#define LOAD(field, sym) g_nccl.field = (decltype(g_nccl.field))dlsym(g_nccl.h, sym)
  LOAD(GetUniqueId, "ncclGetUniqueId");
  LOAD(CommInitRank, "ncclCommInitRank");
  LOAD(CommDestroy, "ncclCommDestroy");
  LOAD(AllGather, "ncclAllGather");
  LOAD(AllReduce, "ncclAllReduce");
  LOAD(GetErrorString, "ncclGetErrorString");
  LOAD(Send, "ncclSend");
  LOAD(Recv, "ncclRecv");
  LOAD(GroupStart, "ncclGroupStart");
  LOAD(GroupEnd, "ncclGroupEnd");
#undef LOAD
  g_nccl.ok = g_nccl.GetUniqueId && g_nccl.CommInitRank && g_nccl.CommDestroy && g_nccl.AllGather &&
              g_nccl.AllReduce && g_nccl.GetErrorString && g_nccl.Send && g_nccl.Recv && g_nccl.GroupStart &&
              g_nccl.GroupEnd;
  return g_nccl.ok;
}

dt_status nccl_fail(ncclResult_t r, const char* what) {
  return fail(DT_ERR_NCCL, std::string("NCCL error in ") + what + ": " +
                               (g_nccl.GetErrorString ? g_nccl.GetErrorString(r) : "?"));
}

// ---- in-process group
struct LocalGroup {
  int world;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  long long gen = 0;
  std::vector<const void*> send;
  std::vector<int> device;
  std::vector<const size_t*> sdispl;  // all-to-all: each rank's byte displacements per destination
  explicit LocalGroup(int w) : world(w), send((size_t)w, nullptr), device((size_t)w, 0), sdispl((size_t)w, nullptr) {}
  void barrier() {
    std::unique_lock<std::mutex> lk(mu);
    const long long g = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != g; });
    }
  }
};

__global__ void sum_u64_kernel(const unsigned long long* const* __restrict__ src, int nsrc,
                               unsigned long long* __restrict__ dst, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    unsigned long long m = 0;
    for (int r = 0; r < nsrc; ++r) m += src[r][i];
    dst[i] = m;
  }
}

__global__ void or_u32_kernel(const uint32_t* const* __restrict__ src, int nsrc, uint32_t* __restrict__ dst,
                              int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint32_t m = 0;
    for (int r = 0; r < nsrc; ++r) m |= src[r][i];
    dst[i] = m;
  }
}

}  // namespace

struct CommImpl {
  int rank = 0, world = 1;
  int backend = 0;  // 0 = NCCL, 1 = local
  int device = -1;  // NCCL: the device the communicator is bound to
  ncclComm_t nccl = nullptr;
  std::shared_ptr<LocalGroup> group;
  uint32_t** dev_ptrs = nullptr;  // local backend: device array of peer pointers
};

}  // namespace dtl

struct dt_comm {
  dtl::CommImpl impl;
};

namespace dtl {

int comm_rank(const dt_comm* c) { return c->impl.rank; }
int comm_world(const dt_comm* c) { return c->impl.world; }

// recv[r * bytes .. (r+1) * bytes) = rank r's send buffer; stream-ordered for NCCL, blocking
// (stream synchronised) for the local backend.
dt_status comm_allgather(dt_comm* c, const void* send, void* recv, size_t bytes, cudaStream_t s) {
  CommImpl& m = c->impl;
  if (m.backend == 0) {  // NCCL, any world size (a 1-rank communicator runs the real collective)
    ncclResult_t r = g_nccl.AllGather(send, recv, bytes, ncclUint8, m.nccl, s);
    if (r != ncclSuccess) return nccl_fail(r, "ncclAllGather");
    return DT_OK;
  }
  if (m.world == 1) {
    if (send != recv) DT_CK(cudaMemcpyAsync(recv, send, bytes, cudaMemcpyDeviceToDevice, s));
    return DT_OK;
  }
  LocalGroup& g = *m.group;
  DT_CK(cudaStreamSynchronize(s));
  g.send[(size_t)m.rank] = send;
  g.barrier();
  for (int r = 0; r < m.world; ++r)
    DT_CK(cudaMemcpyAsync((char*)recv + (size_t)r * bytes, g.send[(size_t)r], bytes, cudaMemcpyDefault, s));
  DT_CK(cudaStreamSynchronize(s));
  g.barrier();
  return DT_OK;
}

// buf[i] = OR over ranks of buf[i], in place, for bitmaps whose set bits are disjoint
// across ranks (each row's go-left bit is set by exactly one rank): NCCL sums the words,
// which equals the OR when no two ranks set the same bit.
dt_status comm_allreduce_or_u32(dt_comm* c, uint32_t* buf, int64_t n, cudaStream_t s) {
  CommImpl& m = c->impl;
  if (m.backend == 0) {
    ncclResult_t r = g_nccl.AllReduce(buf, buf, (size_t)n, ncclUint32, ncclSum, m.nccl, s);
    if (r != ncclSuccess) return nccl_fail(r, "ncclAllReduce");
    return DT_OK;
  }
  if (m.world == 1) return DT_OK;
  LocalGroup& g = *m.group;
  // every rank computes the OR of all ranks' (unchanged) inputs into a private copy
  uint32_t* tmp = nullptr;
  DT_CK(cudaMallocAsync((void**)&tmp, sizeof(uint32_t) * (size_t)n, s));
  DT_CK(cudaStreamSynchronize(s));
  g.send[(size_t)m.rank] = buf;
  g.barrier();
  std::vector<uint32_t*> ptrs((size_t)m.world);
  for (int r = 0; r < m.world; ++r) ptrs[(size_t)r] = (uint32_t*)g.send[(size_t)r];
  DT_CK(cudaMemcpyAsync(m.dev_ptrs, ptrs.data(), sizeof(uint32_t*) * ptrs.size(), cudaMemcpyHostToDevice, s));
  or_u32_kernel<<<num_sms() * 4, 256, 0, s>>>(m.dev_ptrs, m.world, tmp, n);
  DT_CK(cudaGetLastError());
  DT_CK(cudaStreamSynchronize(s));
  g.barrier();  // everybody has read every input
  DT_CK(cudaMemcpyAsync(buf, tmp, sizeof(uint32_t) * (size_t)n, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaFreeAsync(tmp, s));
  DT_CK(cudaStreamSynchronize(s));
  return DT_OK;
}

// buf[i] = sum over ranks of buf[i] (u64), in place.
dt_status comm_allreduce_sum_u64(dt_comm* c, unsigned long long* buf, int64_t n, cudaStream_t s) {
  CommImpl& m = c->impl;
  if (m.backend == 0) {
    ncclResult_t r = g_nccl.AllReduce(buf, buf, (size_t)n, ncclUint64, ncclSum, m.nccl, s);
    if (r != ncclSuccess) return nccl_fail(r, "ncclAllReduce");
    return DT_OK;
  }
  if (m.world == 1) return DT_OK;
  LocalGroup& g = *m.group;
  unsigned long long* tmp = nullptr;
  DT_CK(cudaMallocAsync((void**)&tmp, sizeof(unsigned long long) * (size_t)n, s));
  DT_CK(cudaStreamSynchronize(s));
  g.send[(size_t)m.rank] = buf;
  g.barrier();
  std::vector<unsigned long long*> ptrs((size_t)m.world);
  for (int r = 0; r < m.world; ++r) ptrs[(size_t)r] = (unsigned long long*)g.send[(size_t)r];
  DT_CK(cudaMemcpyAsync(m.dev_ptrs, ptrs.data(), sizeof(void*) * ptrs.size(), cudaMemcpyHostToDevice, s));
  sum_u64_kernel<<<num_sms() * 2, 256, 0, s>>>(reinterpret_cast<unsigned long long**>(m.dev_ptrs), m.world, tmp, n);
  DT_CK(cudaGetLastError());
  DT_CK(cudaStreamSynchronize(s));
  g.barrier();  // everybody has read every input
  DT_CK(cudaMemcpyAsync(buf, tmp, sizeof(unsigned long long) * (size_t)n, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaFreeAsync(tmp, s));
  DT_CK(cudaStreamSynchronize(s));
  return DT_OK;
}

// All-to-all of byte ranges: this rank sends send[sdispl[q], sdispl[q] + scount[q]) to rank
// q and receives rank q's range for it at recv + rdispl[q] (rcount[q] bytes).  Host arrays.
dt_status comm_alltoallv(dt_comm* c, const void* send, const size_t* scount, const size_t* sdispl, void* recv,
                         const size_t* rcount, const size_t* rdispl, cudaStream_t s) {
  CommImpl& m = c->impl;
  if (m.backend == 0) {
    ncclResult_t r = g_nccl.GroupStart();
    for (int q = 0; q < m.world && r == ncclSuccess; ++q) {
      if (scount[q]) r = g_nccl.Send((const char*)send + sdispl[q], scount[q], ncclUint8, q, m.nccl, s);
      if (r == ncclSuccess && rcount[q]) r = g_nccl.Recv((char*)recv + rdispl[q], rcount[q], ncclUint8, q, m.nccl, s);
    }
    ncclResult_t r2 = g_nccl.GroupEnd();
    if (r != ncclSuccess) return nccl_fail(r, "ncclSend/ncclRecv");
    if (r2 != ncclSuccess) return nccl_fail(r2, "ncclGroupEnd");
    return DT_OK;
  }
  LocalGroup& g = *m.group;
  DT_CK(cudaStreamSynchronize(s));
  g.send[(size_t)m.rank] = send;
  g.sdispl[(size_t)m.rank] = sdispl;
  g.barrier();
  for (int q = 0; q < m.world; ++q)
    if (rcount[q])
      DT_CK(cudaMemcpyAsync((char*)recv + rdispl[q], (const char*)g.send[(size_t)q] + g.sdispl[(size_t)q][m.rank],
                            rcount[q], cudaMemcpyDefault, s));
  DT_CK(cudaStreamSynchronize(s));
  g.barrier();
  return DT_OK;
}

}  // namespace dtl

using namespace dtl;

extern "C" {

dt_status dt_comm_unique_id(void* id_out) {
  if (!id_out) return fail(DT_ERR_INVALID_ARG, "dt_comm_unique_id: NULL");
  if (!load_nccl()) return fail(DT_ERR_NCCL, "dt_comm_unique_id: libnccl.so.2 not loadable");
  ncclUniqueId id;
  ncclResult_t r = g_nccl.GetUniqueId(&id);
  if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
  memcpy(id_out, &id, sizeof(id));
  return DT_OK;
}

int32_t dt_comm_unique_id_bytes(void) { return (int32_t)sizeof(ncclUniqueId); }

dt_status dt_comm_init(const void* id, int32_t rank, int32_t world, int32_t device, dt_comm** out) {
  if (!out) return fail(DT_ERR_INVALID_ARG, "dt_comm_init: out is NULL");
  *out = nullptr;
  if (!id || world < 1 || rank < 0 || rank >= world)
    return fail(DT_ERR_INVALID_ARG, "dt_comm_init: need id, 0 <= rank < world");
  int ndev = 0;
  DT_CK(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev) return fail(DT_ERR_INVALID_ARG, "dt_comm_init: bad device");
  // the communicator is bound to `device`: made current for this thread (NCCL binds the
  // communicator to the current device at init)
  DT_CK(cudaSetDevice(device));
  std::unique_ptr<dt_comm> c(new dt_comm());
  c->impl.rank = rank;
  c->impl.world = world;
  c->impl.backend = 0;
  c->impl.device = device;
  if (!load_nccl()) return fail(DT_ERR_NCCL, "dt_comm_init: libnccl.so.2 not loadable");
  ncclUniqueId uid;
  memcpy(&uid, id, sizeof(uid));
  ncclResult_t r = g_nccl.CommInitRank(&c->impl.nccl, world, uid, rank);
  if (r != ncclSuccess) return nccl_fail(r, "ncclCommInitRank");
  *out = c.release();
  return DT_OK;
}

dt_status dt_comm_init_local(int32_t world, dt_comm** comms_out) {
  if (!comms_out || world < 1 || world > 64) return fail(DT_ERR_INVALID_ARG, "dt_comm_init_local: bad args");
  auto g = std::make_shared<LocalGroup>(world);
  for (int r = 0; r < world; ++r) {
    dt_comm* c = new dt_comm();
    c->impl.rank = r;
    c->impl.world = world;
    c->impl.backend = 1;
    c->impl.group = g;
    cudaError_t e = cudaMalloc((void**)&c->impl.dev_ptrs, sizeof(void*) * (size_t)world);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc", __FILE__, __LINE__);
    comms_out[r] = c;
  }
  return DT_OK;
}

void dt_comm_free(dt_comm* c) {
  if (!c) return;
  if (c->impl.nccl && g_nccl.CommDestroy) g_nccl.CommDestroy(c->impl.nccl);
  if (c->impl.dev_ptrs) cudaFree(c->impl.dev_ptrs);
  delete c;
}

int32_t dt_comm_rank(const dt_comm* c) { return c ? c->impl.rank : -1; }
int32_t dt_comm_world(const dt_comm* c) { return c ? c->impl.world : 0; }

}  // extern "C"
