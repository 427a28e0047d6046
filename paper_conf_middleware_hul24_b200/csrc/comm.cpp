// Tensor-parallel collectives for the Llama-2-70B path (include/menos.h menos_tp_cfg).
//
// Two transports behind one interface, chosen at menos_server_create:
//   * NCCL, driven from C++ (no Python on the per-layer path): the caller broadcasts a 128-byte ncclUniqueId
//     (menos_tp_unique_id on rank 0) and every rank passes it in menos_tp_cfg.nccl_id; the library builds the
//     communicator with ncclCommInitRank and issues ncclAllGather / ncclReduceScatter / ncclAllReduce on the stream
//     of the call.  libnccl.so.2 is dlopen'ed: inside a PyTorch process that resolves to the NCCL torch already
//     loaded (same soname), so there is one NCCL in the process.
//   * a caller callback (menos_tp_cfg.collective), e.g. torch.distributed over gloo for the single-GPU tests.
#include <dlfcn.h>
#include <cstring>
#include <mutex>

#include <cuda_runtime.h>

#include "menos.h"
#include "comm.h"

namespace menos {
void set_last_error(const char* fmt, ...);

namespace {
// the subset of nccl.h the library uses (ABI-stable since NCCL 2.0)
typedef struct ncclComm* ncclComm_t;
typedef struct { char internal[128]; } ncclUniqueId;
typedef int ncclResult_t;
enum { nccl_sum = 0 };
enum { nccl_float32 = 7, nccl_bfloat16 = 9 };

struct NcclApi {
  bool tried = false, ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*ReduceScatter)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};
NcclApi g_nccl;
std::mutex g_nccl_mu;

bool load_nccl() {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  if (g_nccl.tried) return g_nccl.ok;
  g_nccl.tried = true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
  if (!h) return false;
  auto sym = [&](const char* n) { return dlsym(h, n); };
  g_nccl.GetUniqueId = (decltype(g_nccl.GetUniqueId))sym("ncclGetUniqueId");
  g_nccl.CommInitRank = (decltype(g_nccl.CommInitRank))sym("ncclCommInitRank");
  g_nccl.CommDestroy = (decltype(g_nccl.CommDestroy))sym("ncclCommDestroy");
  g_nccl.AllReduce = (decltype(g_nccl.AllReduce))sym("ncclAllReduce");
  g_nccl.AllGather = (decltype(g_nccl.AllGather))sym("ncclAllGather");
  g_nccl.ReduceScatter = (decltype(g_nccl.ReduceScatter))sym("ncclReduceScatter");
  g_nccl.GetErrorString = (decltype(g_nccl.GetErrorString))sym("ncclGetErrorString");
  g_nccl.ok = g_nccl.GetUniqueId && g_nccl.CommInitRank && g_nccl.CommDestroy && g_nccl.AllReduce &&
              g_nccl.AllGather && g_nccl.ReduceScatter && g_nccl.GetErrorString;
  return g_nccl.ok;
}

int nccl_dtype(int dt) { return dt == MENOS_DT_BF16 ? nccl_bfloat16 : nccl_float32; }
}  // namespace

int Comm::init(const menos_tp_cfg& tp, int device) {
  rank = tp.rank; world = tp.world;
  fn = tp.collective; user = tp.user;
  if (tp.nccl_id == nullptr) {
    if (world > 1 && !fn) { set_last_error("tensor parallelism needs menos_tp_cfg.collective or .nccl_id"); return MENOS_EINVAL; }
    return MENOS_OK;
  }
  if (!load_nccl()) { set_last_error("libnccl.so.2 not loadable (dlopen: %s)", dlerror()); return MENOS_ENCCL; }
  ncclUniqueId id;
  memcpy(&id, tp.nccl_id, sizeof id);
  cudaSetDevice(device);
  ncclComm_t c = nullptr;
  const ncclResult_t r = g_nccl.CommInitRank(&c, world, id, rank);
  if (r != 0) { set_last_error("ncclCommInitRank(rank %d of %d): %s", rank, world, g_nccl.GetErrorString(r)); return MENOS_ENCCL; }
  nccl = c;
  return MENOS_OK;
}

void Comm::destroy() {
  if (nccl && g_nccl.ok) g_nccl.CommDestroy((ncclComm_t)nccl);
  nccl = nullptr;
}

int Comm::run(int op, const void* send, void* recv, size_t count, int dtype, cudaStream_t st) {
  if (world <= 1 && !nccl) {   // a single rank: the collective is the identity
    if (op == MENOS_COLL_ALLREDUCE || send == recv || count == 0) return MENOS_OK;
    const size_t el = dtype == MENOS_DT_BF16 ? 2 : 4;
    return cudaMemcpyAsync(recv, send, count * el, cudaMemcpyDeviceToDevice, st) == cudaSuccess ? MENOS_OK : MENOS_ECUDA;
  }
  ++calls;
  bytes += (double)count * (dtype == MENOS_DT_BF16 ? 2 : 4) * (op == MENOS_COLL_ALLREDUCE ? 1 : world);
  if (nccl) {
    ncclResult_t r = 0;
    const int dt = nccl_dtype(dtype);
    if (op == MENOS_COLL_ALLREDUCE) r = g_nccl.AllReduce(send, recv, count, dt, nccl_sum, (ncclComm_t)nccl, st);
    else if (op == MENOS_COLL_ALLGATHER) r = g_nccl.AllGather(send, recv, count, dt, (ncclComm_t)nccl, st);
    else r = g_nccl.ReduceScatter(send, recv, count, dt, nccl_sum, (ncclComm_t)nccl, st);
    if (r != 0) { set_last_error("NCCL collective %d failed on rank %d: %s", op, rank, g_nccl.GetErrorString(r)); return MENOS_ENCCL; }
    return MENOS_OK;
  }
  const int rc = fn(op, send, recv, count, dtype, (void*)st, user);
  if (rc) { set_last_error("tensor-parallel collective %d failed (%d) on rank %d", op, rc, rank); return MENOS_ENCCL; }
  return MENOS_OK;
}

}  // namespace menos

extern "C" MENOS_API int menos_tp_unique_id(void* out) {
  if (!out) { menos::set_last_error("null output"); return MENOS_EINVAL; }
  if (!menos::load_nccl()) { menos::set_last_error("libnccl.so.2 not loadable"); return MENOS_ENCCL; }
  menos::ncclUniqueId id;
  const menos::ncclResult_t r = menos::g_nccl.GetUniqueId(&id);
  if (r != 0) { menos::set_last_error("ncclGetUniqueId: %s", menos::g_nccl.GetErrorString(r)); return MENOS_ENCCL; }
  memcpy(out, &id, sizeof id);
  return MENOS_OK;
}
