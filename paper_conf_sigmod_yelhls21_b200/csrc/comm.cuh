// comm.cuh -- the label exchange of the 1-D vertex-range partition (§8 a10).
//
// Synchronous LP [P:48, P:68] makes every vertex's update independent given
// L_{t-1}, so P ranks each compute their owned rows [b_r, b_{r+1}) and then
// replicate the result ("handled by one or multiple GPUs" [P:103]; 2 GPUs ->
// 1.8x [P:355]).  Every exchange the iteration needs goes through `Comm`:
//
//   allgather(buf, eb)        rank r's slice [b_r, b_{r+1}) of an n-element
//                             array (element size eb) to every rank, in place
//                             (labels L_t; LLP: (label, V) pairs; pos/orig)
//   allreduce_u64(p, k)       sum of k counters (changed, d2, arcs, ...) so
//                             every rank takes the same stop/frontier decision
//   allreduce_i32(s, r, k)    r = sum over ranks of s (LLP sharded histogram)
//   merge_flags(flag)         owned slice of the frontier marks = max over the
//                             ranks' marks (each rank's push marks global ids)
//   exchange_changes(W, ...)  §8(f)1 sparse exchange: instead of the label
//                             slices, every rank's (id, label) pairs of the
//                             vertices it changed at t-1 and at t (W holds
//                             L_{t-2} outside the owned rows; applying both
//                             lists in order yields L_t) -- volume 8 B per
//                             change instead of 4 B per vertex
//
// Two implementations:
//   NcclComm   one process per GPU: ncclAllGather (grouped ncclBroadcast when
//              the slices are unequal), ncclAllReduce, ncclReduceScatter.
//   LocalComm  P ranks in ONE process (glp_local_group), e.g. P graphs on one
//              device: each rank publishes a device pointer and an event, the
//              others wait for the event and pull the data straight from the
//              peer's buffer (cudaMemcpyAsync for slices, small kernels for the
//              reductions) -- the peer-memory shape of an NVLink exchange.  It
//              runs the library's real partitioned code path (layout, pos/orig
//              exchange, counters, frontier merge, sharded LLP histogram) on
//              one GPU, which is how that path is parity-tested here.
#pragma once
#include <cuda_runtime.h>

#include <chrono>
#include <condition_variable>
#include <mutex>
#include <string>
#include <vector>

#include "glp_internal.cuh"
#include "nccl_dyn.cuh"

namespace glp {

inline void cuda_ok(cudaError_t e, const char* what) {
  if (e != cudaSuccess) {
    if (e == cudaErrorMemoryAllocation) throw Err{GLP_ERR_OUT_OF_MEMORY, std::string(what) + ": out of memory"};
    throw Err{GLP_ERR_CUDA, std::string(what) + ": " + cudaGetErrorName(e) + " " + cudaGetErrorString(e)};
  }
}

struct Comm {
  virtual ~Comm() = default;
  virtual const char* name() const = 0;
  // every rank's (v_begin, v_end, nnz_local) -> g->bounds, nnz_global, equal_slices
  virtual void setup(glp_graph* g) = 0;
  virtual void allgather(glp_graph* g, void* buf, size_t eb) = 0;
  virtual void allreduce_u64(glp_graph* g, unsigned long long* p, size_t k) = 0;
  virtual void allreduce_i32(glp_graph* g, const int32_t* send, int32_t* recv, size_t k) = 0;
  virtual void merge_flags(glp_graph* g, uint8_t* flag) = 0;
  // sparse replacement of allgather(L_t) (§8(f)1): W holds L_{t-2} outside
  // this rank's rows; applying every other rank's changes of t-1 (lists[0],
  // counts[0]) and then of t (lists[1], counts[1]) turns it into L_t.
  // Lists and counts are device memory.
  virtual void exchange_changes(glp_graph* g, int32_t* W, const int2* const lists[2],
                                const unsigned* const counts[2]) = 0;
  // a rank failed: release the others (local group) instead of letting them wait
  virtual void abort(const std::string&) {}
};

// Shared by both: row bounds from every rank's (vb, ve, nnz).
inline void set_bounds(glp_graph* g, const std::vector<int64_t>& all) {
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

constexpr int kMaxLocalRanks = 16;

// ---- sparse exchange (§8(f)1): only (vertex, label) pairs of changed vertices
// This rank's owned vertices changed at t (so.x == t): (global internal id,
// new label), compacted with one atomic per warp.
__global__ void k_collect_changes(const int2* __restrict__ so, const int32_t* __restrict__ W, int64_t nl, int64_t vb,
                                  int32_t t, int2* __restrict__ out, unsigned* __restrict__ n_out) {
  const int lane = threadIdx.x & 31;
  for (int64_t base = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) & ~31ll; base < nl;
       base += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = base + lane;
    const bool ch = v < nl && so[v].x == t;
    const unsigned m = __ballot_sync(0xffffffffu, ch);
    unsigned at = 0;
    if (lane == 0 && m) at = atomicAdd(n_out, (unsigned)__popc(m));
    at = __shfl_sync(0xffffffffu, at, 0);
    if (ch) out[at + __popc(m & ((1u << lane) - 1u))] = make_int2((int)(vb + v), W[vb + v]);
  }
}
// W[q] = label for every pair of the given lists (other ranks' changes)
struct ChgLists {
  const int2* p[kMaxLocalRanks];
  const unsigned* n[kMaxLocalRanks];
  int nranks, skip;  // skip = this rank (its own changes are already in W)
};
__global__ void k_apply_changes(ChgLists L, int32_t* __restrict__ W) {
  for (int r = 0; r < L.nranks; ++r) {
    if (r == L.skip) continue;
    const unsigned cnt = *L.n[r];
    for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += gridDim.x * blockDim.x) {
      const int2 x = L.p[r][i];
      W[x.x] = x.y;
    }
  }
}
__global__ void k_apply_pairs(const int2* __restrict__ p, int64_t cnt, int32_t* __restrict__ W) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x)
    W[p[i].x] = p[i].y;
}


// ------------------------------------------------------------------ NCCL
struct NcclComm : Comm {
  ncclComm_t c = nullptr;
  NcclComm(glp_graph* g, const void* uid) {
    NcclApi& A = nccl_api();
    ncclUniqueId id;
    memcpy(&id, uid, sizeof(id));
    NCK(A.CommInitRank(&c, g->nranks, id, g->rank));
  }
  ~NcclComm() override {
    if (c) nccl_api().CommDestroy(c);
  }
  const char* name() const override { return "nccl"; }
  void setup(glp_graph* g) override {
    int64_t* d = nullptr;
    cuda_ok(cudaMalloc(&d, sizeof(int64_t) * 3 * g->nranks), "cudaMalloc");
    int64_t mine[3] = {g->vb, g->ve, g->nnz};
    std::vector<int64_t> all(3 * g->nranks);
    try {
      cuda_ok(cudaMemcpy(d + 3 * g->rank, mine, sizeof(mine), cudaMemcpyHostToDevice), "cudaMemcpy");
      NCK(nccl_api().AllGather(d + 3 * g->rank, d, 3, ncclInt64, c, g->stream));
      cuda_ok(cudaMemcpyAsync(all.data(), d, sizeof(int64_t) * 3 * g->nranks, cudaMemcpyDeviceToHost, g->stream),
              "cudaMemcpyAsync");
      cuda_ok(cudaStreamSynchronize(g->stream), "cudaStreamSynchronize");
    } catch (...) {
      cudaFree(d);
      throw;
    }
    cudaFree(d);
    set_bounds(g, all);
  }
  void allgather(glp_graph* g, void* buf, size_t eb) override {
    NcclApi& A = nccl_api();
    char* b = (char*)buf;
    if (g->equal_slices) {
      const size_t per = (size_t)(g->npad / g->nranks) * eb;
      NCK(A.AllGather(b + per * g->rank, b, per, ncclInt8, c, g->stream));
    } else {
      NCK(A.GroupStart());
      for (int r = 0; r < g->nranks; ++r) {
        const size_t cnt = (size_t)(g->bounds[r + 1] - g->bounds[r]) * eb;
        if (cnt) NCK(A.Broadcast(b + g->bounds[r] * eb, b + g->bounds[r] * eb, cnt, ncclInt8, r, c, g->stream));
      }
      NCK(A.GroupEnd());
    }
  }
  void allreduce_u64(glp_graph* g, unsigned long long* p, size_t k) override {
    NCK(nccl_api().AllReduce(p, p, k, ncclUint64, ncclSum, c, g->stream));
  }
  void allreduce_i32(glp_graph* g, const int32_t* send, int32_t* recv, size_t k) override {
    NCK(nccl_api().AllReduce(send, recv, k, ncclInt32, ncclSum, c, g->stream));
  }
  // counts all-gathered (one host sync), then each rank's lists broadcast
  // into one receive buffer per list (grouped), then applied in order
  void exchange_changes(glp_graph* g, int32_t* W, const int2* const lists[2], const unsigned* const counts[2]) override {
    NcclApi& A = nccl_api();
    const int P = g->nranks;
    unsigned* d = nullptr;
    cuda_ok(cudaMallocAsync((void**)&d, sizeof(unsigned) * 2 * P, g->stream), "cudaMallocAsync");
    cuda_ok(cudaMemcpyAsync(d + 2 * g->rank, counts[0], sizeof(unsigned), cudaMemcpyDeviceToDevice, g->stream), "copy");
    cuda_ok(cudaMemcpyAsync(d + 2 * g->rank + 1, counts[1], sizeof(unsigned), cudaMemcpyDeviceToDevice, g->stream),
            "copy");
    NCK(A.AllGather(d + 2 * g->rank, d, 2, ncclUint32, c, g->stream));
    std::vector<unsigned> all(2 * P);
    cuda_ok(cudaMemcpyAsync(all.data(), d, sizeof(unsigned) * 2 * P, cudaMemcpyDeviceToHost, g->stream), "copy");
    cuda_ok(cudaStreamSynchronize(g->stream), "sync");
    cudaFreeAsync(d, g->stream);
    for (int j = 0; j < 2; ++j) {
      int64_t tot = 0;
      for (int r = 0; r < P; ++r) tot += all[2 * r + j];
      if (tot == 0) continue;
      int2* recv = nullptr;
      cuda_ok(cudaMallocAsync((void**)&recv, sizeof(int2) * tot, g->stream), "cudaMallocAsync");
      NCK(A.GroupStart());
      int64_t at = 0;
      for (int r = 0; r < P; ++r) {
        const unsigned k = all[2 * r + j];
        if (k) NCK(A.Broadcast(r == g->rank ? (const void*)lists[j] : (const void*)(recv + at), recv + at,
                               (size_t)k * 2, ncclInt32, r, c, g->stream));
        at += k;
      }
      NCK(A.GroupEnd());
      k_apply_pairs<<<g->sms * 2, 256, 0, g->stream>>>(recv, tot, W);  // own pairs rewrite own values: harmless
      cuda_ok(cudaGetLastError(), "k_apply_pairs");
      cudaFreeAsync(recv, g->stream);
    }
  }
  void merge_flags(glp_graph* g, uint8_t* flag) override {
    NcclApi& A = nccl_api();
    if (g->equal_slices) {
      const size_t per = (size_t)(g->npad / g->nranks);
      NCK(A.ReduceScatter(flag, flag + per * g->rank, per, ncclUint8, ncclMax, c, g->stream));
    } else {
      NCK(A.AllReduce(flag, flag, (size_t)g->npad, ncclUint8, ncclMax, c, g->stream));
    }
  }
};

// ------------------------------------------------------------------ local group
struct Peers {
  const void* p[kMaxLocalRanks];
  int nranks;
};

// sum of the ranks' arrays (out of place: the sources are the peers' send buffers)
__global__ void k_sum_u64(Peers src, unsigned long long* __restrict__ dst, int64_t k) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < k; i += (int64_t)gridDim.x * blockDim.x) {
    unsigned long long s = 0;
    for (int r = 0; r < src.nranks; ++r) s += ((const unsigned long long*)src.p[r])[i];
    dst[i] = s;
  }
}
__global__ void k_sum_i32(Peers src, int32_t* __restrict__ dst, int64_t k) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < k; i += (int64_t)gridDim.x * blockDim.x) {
    int32_t s = 0;
    for (int r = 0; r < src.nranks; ++r) s += ((const int32_t*)src.p[r])[i];
    dst[i] = s;
  }
}
// owned slice [b, e) of this rank's marks = max over the ranks' marks (in place:
// every rank writes only its own slice, and reads the others' marks there)
__global__ void k_max_flags(Peers src, uint8_t* __restrict__ dst, int64_t b, int64_t e) {
  for (int64_t i = b + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < e; i += (int64_t)gridDim.x * blockDim.x) {
    uint8_t m = 0;
    for (int r = 0; r < src.nranks; ++r) m = max(m, ((const uint8_t*)src.p[r])[i]);
    dst[i] = m;
  }
}

}  // namespace glp

// The in-process group: a host barrier plus a table of published pointers and
// events, one slot per rank.
struct glp_local_group {
  int nranks = 0;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  bool broken = false;
  std::string why;
  std::vector<const void*> ptr;
  std::vector<cudaEvent_t> ready, done;
  std::vector<int64_t> host;  // 3 per rank (setup)
  std::vector<int> joined;

  explicit glp_local_group(int p) : nranks(p), ptr(p, nullptr), ready(p, nullptr), done(p, nullptr), host(3 * p, 0),
                                    joined(p, 0) {}

  // generation barrier; throws if the group was aborted or a rank never came
  void barrier() {
    std::unique_lock<std::mutex> lk(mu);
    if (broken) throw glp::Err{GLP_ERR_STATE, "local group aborted: " + why};
    const uint64_t my = gen;
    if (++arrived == nranks) {
      arrived = 0;
      ++gen;
      cv.notify_all();
      return;
    }
    const bool ok = cv.wait_for(lk, std::chrono::seconds(600), [&] { return gen != my || broken; });
    if (!ok) {
      broken = true;
      why = "barrier timeout (a rank never reached the exchange)";
      cv.notify_all();
    }
    if (gen == my) throw glp::Err{GLP_ERR_STATE, "local group aborted: " + why};
  }
  void abort(const std::string& m) {
    std::lock_guard<std::mutex> lk(mu);
    if (!broken) {
      broken = true;
      why = m;
    }
    cv.notify_all();
  }
};

namespace glp {

struct LocalComm : Comm {
  glp_local_group* grp;
  int rank;
  cudaEvent_t ready = nullptr, done = nullptr;
  unsigned long long* stage = nullptr;  // allreduce_u64 send copy
  size_t stage_k = 0;
  struct Desc {
    const int2* p[2];
    const unsigned* n[2];
  };
  Desc host_desc;  // this rank's change lists (device pointers), read by the peers' host threads

  LocalComm(glp_graph* g, glp_local_group* grp_) : grp(grp_), rank(g->rank) {
    if (grp->nranks != g->nranks) throw Err{GLP_ERR_INVALID_ARGUMENT, "local group size != nranks"};
    if (g->nranks > kMaxLocalRanks) throw Err{GLP_ERR_INVALID_ARGUMENT, "local group: at most 16 ranks"};
    {
      std::lock_guard<std::mutex> lk(grp->mu);
      if (grp->joined[rank]) throw Err{GLP_ERR_INVALID_ARGUMENT, "local group: rank already joined"};
      grp->joined[rank] = 1;
    }
    cuda_ok(cudaEventCreateWithFlags(&ready, cudaEventDisableTiming), "cudaEventCreate");
    cuda_ok(cudaEventCreateWithFlags(&done, cudaEventDisableTiming), "cudaEventCreate");
    grp->ready[rank] = ready;
    grp->done[rank] = done;
  }
  ~LocalComm() override {
    if (stage) cudaFree(stage);
    if (ready) cudaEventDestroy(ready);
    if (done) cudaEventDestroy(done);
    std::lock_guard<std::mutex> lk(grp->mu);
    grp->joined[rank] = 0;
  }
  const char* name() const override { return "local"; }
  void abort(const std::string& m) override { grp->abort(m); }

  // publish `mine` (ready on this rank's stream), run `work` on this rank's
  // stream after every peer's data is ready, then wait until every peer has
  // finished reading before this rank's buffers may change again
  template <class F>
  void collective(glp_graph* g, const void* mine, F work) {
    cuda_ok(cudaEventRecord(ready, g->stream), "cudaEventRecord");
    grp->ptr[rank] = mine;
    grp->barrier();
    Peers pe;
    memset(&pe, 0, sizeof(pe));
    pe.nranks = grp->nranks;
    for (int r = 0; r < grp->nranks; ++r) {
      pe.p[r] = grp->ptr[r];
      if (r != rank) cuda_ok(cudaStreamWaitEvent(g->stream, grp->ready[r], 0), "cudaStreamWaitEvent");
    }
    work(pe);
    cuda_ok(cudaGetLastError(), "local exchange");
    cuda_ok(cudaEventRecord(done, g->stream), "cudaEventRecord");
    grp->barrier();
    for (int r = 0; r < grp->nranks; ++r)
      if (r != rank) cuda_ok(cudaStreamWaitEvent(g->stream, grp->done[r], 0), "cudaStreamWaitEvent");
  }

  void setup(glp_graph* g) override {
    grp->host[3 * rank] = g->vb;
    grp->host[3 * rank + 1] = g->ve;
    grp->host[3 * rank + 2] = g->nnz;
    grp->barrier();
    std::vector<int64_t> all(grp->host.begin(), grp->host.end());
    grp->barrier();  // every rank has read the table
    set_bounds(g, all);
  }
  void allgather(glp_graph* g, void* buf, size_t eb) override {
    collective(g, buf, [&](const Peers& pe) {
      for (int r = 0; r < g->nranks; ++r) {
        const int64_t b = g->bounds[r], e = g->bounds[r + 1];
        if (r == rank || e <= b) continue;
        cuda_ok(cudaMemcpyAsync((char*)buf + b * eb, (const char*)pe.p[r] + b * eb, (size_t)(e - b) * eb,
                                cudaMemcpyDeviceToDevice, g->stream),
                "cudaMemcpyAsync (peer slice)");
      }
    });
  }
  void allreduce_u64(glp_graph* g, unsigned long long* p, size_t k) override {
    if (stage_k < k) {
      if (stage) cudaFree(stage);
      stage = nullptr;
      cuda_ok(cudaMalloc(&stage, k * sizeof(unsigned long long)), "cudaMalloc");
      stage_k = k;
    }
    cuda_ok(cudaMemcpyAsync(stage, p, k * sizeof(unsigned long long), cudaMemcpyDeviceToDevice, g->stream),
            "cudaMemcpyAsync");
    collective(g, stage, [&](const Peers& pe) { k_sum_u64<<<1, 256, 0, g->stream>>>(pe, p, (int64_t)k); });
  }
  void allreduce_i32(glp_graph* g, const int32_t* send, int32_t* recv, size_t k) override {
    collective(g, send, [&](const Peers& pe) {
      k_sum_i32<<<g->sms * 4, 256, 0, g->stream>>>(pe, recv, (int64_t)k);
    });
  }
  // peers' lists read in place: publish a device descriptor of this rank's
  // two lists, then apply every other rank's t-1 lists, then their t lists
  void exchange_changes(glp_graph* g, int32_t* W, const int2* const lists[2], const unsigned* const counts[2]) override {
    Desc h;
    h.p[0] = lists[0]; h.p[1] = lists[1]; h.n[0] = counts[0]; h.n[1] = counts[1];
    host_desc = h;  // peers read the host copy (pointers are process-wide)
    collective(g, &host_desc, [&](const Peers& pe) {
      for (int j = 0; j < 2; ++j) {
        ChgLists L;
        memset(&L, 0, sizeof(L));
        L.nranks = g->nranks;
        L.skip = rank;
        for (int r = 0; r < g->nranks; ++r) {
          const Desc* dr = (const Desc*)pe.p[r];
          L.p[r] = dr->p[j];
          L.n[r] = dr->n[j];
        }
        k_apply_changes<<<g->sms * 2, 256, 0, g->stream>>>(L, W);
      }
    });
  }
  void merge_flags(glp_graph* g, uint8_t* flag) override {
    collective(g, flag, [&](const Peers& pe) {
      k_max_flags<<<g->sms * 4, 256, 0, g->stream>>>(pe, flag, g->vb, g->ve);
    });
  }
};

}  // namespace glp
