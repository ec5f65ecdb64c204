// comm.cpp -- NCCL shim for attribute-sharded multi-GPU training.
//
// Per level the only exchanges are (1) an allgather of every shard's per-node best split record
// and (2) a sum-allreduce of the byte map "instance goes to the non-default child", whose
// non-zero entries are written by exactly one shard (the owner of the winning attribute), so the
// sum equals the OR.  NCCL is loaded with dlopen so that single-GPU use never needs it.
#include <dlfcn.h>
#include <nccl.h>

#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "internal.h"

namespace gbdt {
namespace {

struct NcclApi {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi& api() {
  static NcclApi a;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* names[] = {"libnccl.so.2", "libnccl.so"};
    for (const char* nm : names) {
      a.h = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
      if (a.h) break;
    }
    if (!a.h) return;
    a.GetUniqueId = (decltype(a.GetUniqueId))dlsym(a.h, "ncclGetUniqueId");
    a.CommInitRank = (decltype(a.CommInitRank))dlsym(a.h, "ncclCommInitRank");
    a.CommDestroy = (decltype(a.CommDestroy))dlsym(a.h, "ncclCommDestroy");
    a.AllGather = (decltype(a.AllGather))dlsym(a.h, "ncclAllGather");
    a.AllReduce = (decltype(a.AllReduce))dlsym(a.h, "ncclAllReduce");
    a.GetErrorString = (decltype(a.GetErrorString))dlsym(a.h, "ncclGetErrorString");
  });
  if (!a.h || !a.GetUniqueId || !a.CommInitRank || !a.AllGather || !a.AllReduce)
    fail(GBDT_E_NCCL, std::string("NCCL not loadable: ") + (dlerror() ? dlerror() : "libnccl.so.2 missing"));
  return a;
}

void check(ncclResult_t r, const char* what) {
  if (r != ncclSuccess)
    fail(GBDT_E_NCCL, std::string(what) + ": " + (api().GetErrorString ? api().GetErrorString(r) : "nccl error"));
}

}  // namespace

void Comm::allgather(const void* send, void* recv, size_t bytes, cudaStream_t st) {
  if (!nccl) {  // host-staged callback
    std::vector<unsigned char> hs(bytes), hr(bytes * (size_t)world);
    GBDT_CUDA(cudaMemcpyAsync(hs.data(), send, bytes, cudaMemcpyDeviceToHost, st));
    GBDT_CUDA(cudaStreamSynchronize(st));
    if (cb_allgather(hs.data(), hr.data(), bytes, cb_user) != 0) fail(GBDT_E_NCCL, "allgather callback failed");
    GBDT_CUDA(cudaMemcpyAsync(recv, hr.data(), hr.size(), cudaMemcpyHostToDevice, st));
    GBDT_CUDA(cudaStreamSynchronize(st));
    return;
  }
  count_launch();
  check(api().AllGather(send, recv, bytes, ncclUint8, (ncclComm_t)nccl, st), "ncclAllGather");
}

void Comm::allreduce_sum_u8(void* buf, size_t n, cudaStream_t st) {
  if (!nccl) {
    std::vector<unsigned char> hb(n);
    GBDT_CUDA(cudaMemcpyAsync(hb.data(), buf, n, cudaMemcpyDeviceToHost, st));
    GBDT_CUDA(cudaStreamSynchronize(st));
    if (cb_allreduce(hb.data(), n, cb_user) != 0) fail(GBDT_E_NCCL, "allreduce callback failed");
    GBDT_CUDA(cudaMemcpyAsync(buf, hb.data(), n, cudaMemcpyHostToDevice, st));
    GBDT_CUDA(cudaStreamSynchronize(st));
    return;
  }
  count_launch();
  check(api().AllReduce(buf, buf, n, ncclUint8, ncclSum, (ncclComm_t)nccl, st), "ncclAllReduce");
}

void comm_unique_id(uint8_t id[128]) {
  ncclUniqueId u;
  check(api().GetUniqueId(&u), "ncclGetUniqueId");
  static_assert(sizeof(u) == 128, "ncclUniqueId is 128 bytes");
  std::memcpy(id, &u, 128);
}

Comm* comm_init(int rank, int world, const uint8_t id[128], int device) {
  ncclUniqueId u;
  std::memcpy(&u, id, 128);
  if (device >= 0) GBDT_CUDA(cudaSetDevice(device));
  int dev = 0;
  GBDT_CUDA(cudaGetDevice(&dev));
  ncclComm_t c;
  check(api().CommInitRank(&c, world, u, rank), "ncclCommInitRank");
  Comm* cm = new Comm();
  cm->rank = rank;
  cm->world = world;
  cm->device = dev;
  cm->nccl = c;
  return cm;
}

void comm_free(Comm* c) {
  if (!c) return;
  if (c->nccl && api().CommDestroy) api().CommDestroy((ncclComm_t)c->nccl);
  delete c;
}

}  // namespace gbdt
