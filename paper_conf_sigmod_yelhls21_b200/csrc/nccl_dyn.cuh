// nccl_dyn.cuh -- NCCL resolved at run time (the exchange itself: comm.cuh).
//
// NCCL is resolved with dlopen("libnccl.so.2") on first use so that libglp.so
// loads (and its single-GPU path runs) without NCCL; inside a PyTorch process
// the already-loaded torch NCCL is reused.
#pragma once
#include <dlfcn.h>
#include <nccl.h>

#include <string>

#include "glp_internal.cuh"

namespace glp {

struct NcclApi {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*ReduceScatter)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

inline NcclApi& nccl_api() {
  static NcclApi api;
  if (!api.h) {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) throw Err{GLP_ERR_NCCL, std::string("dlopen(libnccl.so.2) failed: ") + dlerror()};
#define GLP_SYM(f, name) api.f = (decltype(api.f))dlsym(h, name)
    GLP_SYM(GetUniqueId, "ncclGetUniqueId");
    GLP_SYM(CommInitRank, "ncclCommInitRank");
    GLP_SYM(CommDestroy, "ncclCommDestroy");
    GLP_SYM(AllGather, "ncclAllGather");
    GLP_SYM(AllReduce, "ncclAllReduce");
    GLP_SYM(ReduceScatter, "ncclReduceScatter");
    GLP_SYM(Broadcast, "ncclBroadcast");
    GLP_SYM(GroupStart, "ncclGroupStart");
    GLP_SYM(GroupEnd, "ncclGroupEnd");
    GLP_SYM(GetErrorString, "ncclGetErrorString");
#undef GLP_SYM
    if (!api.GetUniqueId || !api.CommInitRank || !api.AllGather || !api.AllReduce || !api.ReduceScatter ||
        !api.Broadcast || !api.GroupStart || !api.GroupEnd || !api.CommDestroy)
      throw Err{GLP_ERR_NCCL, "libnccl.so.2 lacks required symbols"};
    api.h = h;
  }
  return api;
}

#define NCK(x)                                                                                    \
  do {                                                                                            \
    ncclResult_t r_ = (x);                                                                        \
    if (r_ != ncclSuccess)                                                                        \
      throw Err{GLP_ERR_NCCL, std::string(#x) + ": " +                                            \
                                  (nccl_api().GetErrorString ? nccl_api().GetErrorString(r_) : "?")}; \
  } while (0)

inline void nccl_unique_id(uint8_t out[128]) {
  ncclUniqueId id;
  NCK(nccl_api().GetUniqueId(&id));
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  memcpy(out, &id, 128);
}

}  // namespace glp
