// nccl_dyn.cuh -- the multi-GPU exchange of the 1-D vertex-range partition.
//
// NCCL is resolved with dlopen("libnccl.so.2") on first use so that libglp.so
// loads (and its single-GPU path runs) without NCCL; inside a PyTorch process
// the already-loaded torch NCCL is reused.  Per iteration:
//   * ncclAllGather of the owned slice of L_t into the replicated label array
//     (in place; grouped ncclBroadcast when the slices are unequal);
//   * ncclAllReduce(sum) of the per-bin counters -> every rank takes the same
//     stop / frontier decision;
//   * sparse iterations: ncclReduceScatter(max) (or AllReduce when slices are
//     unequal) of the global frontier marks written by each rank's push.
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

inline void nccl_init(glp_graph* g, const void* uid) {
  NcclApi& A = nccl_api();
  ncclUniqueId id;
  memcpy(&id, uid, sizeof(id));
  ncclComm_t comm;
  NCK(A.CommInitRank(&comm, g->nranks, id, g->rank));
  g->nccl = comm;
  // exchange row bounds and arc counts of every rank
  int64_t* d = nullptr;
  if (cudaMalloc(&d, sizeof(int64_t) * 3 * g->nranks) != cudaSuccess) throw Err{GLP_ERR_OUT_OF_MEMORY, "cudaMalloc"};
  int64_t mine[3] = {g->vb, g->ve, g->nnz};
  cudaMemcpy(d + 3 * g->rank, mine, sizeof(mine), cudaMemcpyHostToDevice);
  NCK(A.AllGather(d + 3 * g->rank, d, 3, ncclInt64, comm, g->stream));
  std::vector<int64_t> all(3 * g->nranks);
  cudaMemcpyAsync(all.data(), d, sizeof(int64_t) * 3 * g->nranks, cudaMemcpyDeviceToHost, g->stream);
  cudaStreamSynchronize(g->stream);
  cudaFree(d);
  g->bounds.assign(g->nranks + 1, 0);
  g->nnz_global = 0;
  g->equal_slices = true;
  const int64_t per = g->npad / g->nranks;
  for (int r = 0; r < g->nranks; ++r) {
    g->bounds[r] = all[3 * r];
    g->bounds[r + 1] = all[3 * r + 1];
    g->nnz_global += all[3 * r + 2];
    if (all[3 * r] != per * r || (r + 1 < g->nranks && all[3 * r + 1] != per * (r + 1))) g->equal_slices = false;
    if (r > 0 && all[3 * r] != all[3 * (r - 1) + 1])
      throw Err{GLP_ERR_INVALID_ARGUMENT, "rank row ranges are not contiguous"};
  }
  if (g->bounds[0] != 0 || g->bounds[g->nranks] != g->n)
    throw Err{GLP_ERR_INVALID_ARGUMENT, "rank row ranges do not cover [0, n_global)"};
}

inline void nccl_destroy(glp_graph* g) {
  if (g->nccl) {
    nccl_api().CommDestroy((ncclComm_t)g->nccl);
    g->nccl = nullptr;
  }
}

// Replicate L_t: every rank contributes its owned rows.
inline void nccl_exchange(glp_graph* g, int32_t* W) {
  NcclApi& A = nccl_api();
  ncclComm_t c = (ncclComm_t)g->nccl;
  if (g->equal_slices) {
    const size_t per = (size_t)(g->npad / g->nranks);
    NCK(A.AllGather(W + per * g->rank, W, per, ncclInt32, c, g->stream));
  } else {
    NCK(A.GroupStart());
    for (int r = 0; r < g->nranks; ++r) {
      const size_t cnt = (size_t)(g->bounds[r + 1] - g->bounds[r]);
      if (cnt) NCK(A.Broadcast(W + g->bounds[r], W + g->bounds[r], cnt, ncclInt32, r, c, g->stream));
    }
    NCK(A.GroupEnd());
  }
}

inline void nccl_sum_counters(glp_graph* g, void* d_cnt, size_t n_u64) {
  NCK(nccl_api().AllReduce(d_cnt, d_cnt, n_u64, ncclUint64, ncclSum, (ncclComm_t)g->nccl, g->stream));
}

// Merge the global frontier marks (n bytes, global ids) of all ranks.
inline void nccl_merge_flags(glp_graph* g, uint8_t* flag) {
  NcclApi& A = nccl_api();
  ncclComm_t c = (ncclComm_t)g->nccl;
  if (g->equal_slices) {
    const size_t per = (size_t)(g->npad / g->nranks);
    NCK(A.ReduceScatter(flag, flag + per * g->rank, per, ncclUint8, ncclMax, c, g->stream));
  } else {
    NCK(A.AllReduce(flag, flag, (size_t)g->npad, ncclUint8, ncclMax, c, g->stream));
  }
}

}  // namespace glp
