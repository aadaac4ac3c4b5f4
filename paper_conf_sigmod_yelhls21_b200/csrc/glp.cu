// glp.cu -- host runtime and C ABI of libglp.so (see include/glp.h).
//
// Per LP iteration t, all on the graph's stream:
//   1. reset per-bin counters                                  (memset 256 B)
//   2. MFL kernels huge, high, mid, low        R = L_{t-1} -> W = L_t
//   3. [P > 1] all-gather of the owned label slice, counters all-reduce
//      (comm.cuh: NCCL across processes, or an in-process local group)
//   4. read the counters (changed, d2, sum of changed degrees) -> stop rule R8
//   5. frontier decision: dense when sum_{changed} deg > nnz / dense_divisor,
//      else k_push marks N(v) + v for changed v (exact for CLASSIC/SEEDED, R9)
//   6. LLP: rebuild the label histogram V from L_t               [P:119]
//   7. swap R/W
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <array>
#include <chrono>
#include <mutex>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <string>
#include <vector>

#include "aux_kernels.cuh"
#include "comm.cuh"
#include "glp_internal.cuh"
#include "layout.cuh"
#include "mfl_kernels.cuh"
#include "mfl_weighted.cuh"

using namespace glp;

namespace {

thread_local std::string g_last_error = "";

// GLP_TRACE_CREATE=1: host timestamps of the create phases on stderr
struct CreateTrace {
  bool on = false;
  std::chrono::steady_clock::time_point t0;
  CreateTrace() {
    const char* e = getenv("GLP_TRACE_CREATE");
    on = e && e[0] == '1';
    t0 = std::chrono::steady_clock::now();
  }
  void mark(const char* what) const {
    if (on)
      fprintf(stderr, "[glp create] %-28s %8.2f ms\n", what,
              std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
  }
};
thread_local CreateTrace* g_trace = nullptr;
void trace(const char* what) {
  if (g_trace) g_trace->mark(what);
}

[[noreturn]] void fail(glp_status st, const std::string& m) { throw Err{st, m}; }

#define CK(x)                                                                              \
  do {                                                                                     \
    cudaError_t e_ = (x);                                                                  \
    if (e_ != cudaSuccess) {                                                               \
      if (e_ == cudaErrorMemoryAllocation)                                                 \
        fail(GLP_ERR_OUT_OF_MEMORY, std::string(#x) + ": " + cudaGetErrorString(e_));      \
      fail(GLP_ERR_CUDA, std::string(#x) + ": " + cudaGetErrorName(e_) + " " + cudaGetErrorString(e_)); \
    }                                                                                      \
  } while (0)

// Device memory comes from a PRIVATE stream-ordered memory pool per device
// (cudaMemPoolCreate; not the device's default pool, which torch's
// cudaMallocAsync backend may share), which keeps up to kPoolKeep bytes (env
// GLP_POOL_KEEP_GB) of freed memory mapped between graphs: create/destroy of
// a multi-GB graph then costs no driver map/unmap (plain cudaMalloc/cudaFree
// made end-to-end create times vary from 0.1 to 2 s on the B200 box).  When an
// allocation fails, the pool's unused reserve is returned to the driver
// (cudaMemPoolTrimTo) and the allocation is retried once.
constexpr uint64_t kPoolKeep = 16ull << 30;
cudaMemPool_t device_pool(int dev) {
  static std::mutex mu;
  static std::vector<cudaMemPool_t> pools;
  std::lock_guard<std::mutex> lock(mu);
  if ((int)pools.size() <= dev) pools.resize(dev + 1, nullptr);
  if (!pools[dev]) {
    cudaMemPoolProps props;
    memset(&props, 0, sizeof(props));
    props.allocType = cudaMemAllocationTypePinned;
    props.handleTypes = cudaMemHandleTypeNone;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t pool = nullptr;
    if (cudaMemPoolCreate(&pool, &props) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    uint64_t keep = kPoolKeep;
    if (const char* e = getenv("GLP_POOL_KEEP_GB")) keep = (uint64_t)(atof(e) * (double)(1ull << 30));
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
    pools[dev] = pool;
  }
  return pools[dev];
}
cudaError_t pool_malloc(void** p, size_t bytes, cudaStream_t s) {
  int dev = 0;
  cudaGetDevice(&dev);
  cudaMemPool_t pool = device_pool(dev);
  if (!pool) return cudaMallocAsync(p, bytes, s);
  cudaError_t e = cudaMallocFromPoolAsync(p, bytes, pool, s);
  if (e == cudaErrorMemoryAllocation) {
    cudaGetLastError();
    cudaStreamSynchronize(s);  // frees queued on this stream complete first
    cudaMemPoolTrimTo(pool, 0);
    e = cudaMallocFromPoolAsync(p, bytes, pool, s);
  }
  return e;
}
void pool_free(void* p, cudaStream_t s) {
  if (p) cudaFreeAsync(p, s);
}
// thrust temporaries from the same pool
struct PoolAlloc {
  typedef char value_type;
  cudaStream_t s;
  char* allocate(std::ptrdiff_t n) {
    void* p = nullptr;
    if (pool_malloc(&p, std::max<std::ptrdiff_t>(n, 16), s) != cudaSuccess) {
      cudaGetLastError();
      throw std::bad_alloc();
    }
    return (char*)p;
  }
  void deallocate(char* p, size_t) { pool_free(p, s); }
};

template <class T>
T* dalloc(glp_graph* g, size_t count) {
  void* p = nullptr;
  size_t bytes = std::max<size_t>(count * sizeof(T), 16);
  cudaError_t e = pool_malloc(&p, bytes, g->stream);
  if (e != cudaSuccess) {
    cudaGetLastError();
    fail(GLP_ERR_OUT_OF_MEMORY, "cudaMalloc(" + std::to_string(bytes) + " B) failed: " + cudaGetErrorString(e));
  }
  g->allocs.push_back(p);
  return (T*)p;
}

template <class T>
T* upload(glp_graph* g, const std::vector<T>& h) {
  T* d = dalloc<T>(g, h.size());
  if (!h.empty()) CK(cudaMemcpyAsync(d, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice, g->stream));
  return d;
}

int grid_for(int sms, const void* fn, int block, size_t smem) {
  int per_sm = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, block, smem));
  return std::max(1, per_sm) * sms;
}

glp_params default_params() {
  glp_params p;
  memset(&p, 0, sizeof(p));
  p.struct_size = sizeof(glp_params);
  p.gamma = 0.0;
  p.frontier = -1;
  p.stop_on_2cycle = 1;
  p.validate = 1;
  p.profile = 0;
  p.dense_divisor = 4;
  p.sparse_exchange = -1;
  return p;
}

glp_params get_params(const glp_params* p) {
  if (!p) return default_params();
  if (p->struct_size != sizeof(glp_params))
    fail(GLP_ERR_INVALID_ARGUMENT, "glp_params.struct_size mismatch (got " + std::to_string(p->struct_size) +
                                       ", expected " + std::to_string(sizeof(glp_params)) + ")");
  glp_params q = *p;
  if (q.dense_divisor <= 0) q.dense_divisor = 4;
  return q;
}

template <class F>
glp_status guard(F f) {
  try {
    f();
    return GLP_OK;
  } catch (const Err& e) {
    g_last_error = e.msg;
    return e.st;
  } catch (const std::bad_alloc&) {
    g_last_error = "host allocation failed";
    return GLP_ERR_OUT_OF_MEMORY;
  } catch (...) {
    g_last_error = "unknown internal error";
    return GLP_ERR_CUDA;
  }
}

void free_graph(glp_graph* g) {
  if (!g) return;
  if (g->device >= 0) cudaSetDevice(g->device);
  if (g->stream) cudaStreamSynchronize(g->stream);
  for (void* p : g->allocs) pool_free(p, g->stream);
  if (g->stream) cudaStreamSynchronize(g->stream);
  g->allocs.clear();
  if (g->h_cnt) cudaFreeHost(g->h_cnt);
  if (g->h_stop) cudaFreeHost((void*)g->h_stop);
  if (g->col2_host) cudaFreeHost(g->col2_host);
  if (g->registered) cudaHostUnregister(g->registered);
  if (g->ev_a) cudaEventDestroy(g->ev_a);
  if (g->ev_b) cudaEventDestroy(g->ev_b);
  for (auto& e : g->ev_pool) cudaEventDestroy(e);
  for (auto& e : g->xev) if (e) cudaEventDestroy(e);
  for (auto& e : g->arc_chunk_ev) cudaEventDestroy(e);
  delete g->comm;
  g->comm = nullptr;
  if (g->own_stream && g->stream) cudaStreamDestroy(g->stream);
  delete g;
}

// Side streams of the concurrent class kernels: one set per device for the
// process lifetime (stream creation/destruction per graph made graph create
// and destroy times erratic).  Graphs on different threads may share them:
// every graph forks and joins through its own events, so sharing only orders
// their side-stream kernels, never breaks a dependency.
void side_streams(int dev, cudaStream_t (&xs)[4]) {
  static std::mutex mu;
  static std::vector<std::array<cudaStream_t, 4>> pool;
  std::lock_guard<std::mutex> lock(mu);
  if ((int)pool.size() <= dev) pool.resize(dev + 1, std::array<cudaStream_t, 4>{nullptr, nullptr, nullptr, nullptr});
  for (int i = 0; i < 4; ++i) {
    if (!pool[dev][i]) CK(cudaStreamCreateWithFlags(&pool[dev][i], cudaStreamNonBlocking));
    xs[i] = pool[dev][i];
  }
}

// ---------------------------------------------------------------- layout
#define GLP_M_KERNEL(VAR) mfl_block<VAR, kMBlock, kMSlots, false, kMUnroll, CLS_M>
#define GLP_L_KERNEL(VAR) mfl_block<VAR, kLBlock, kLSlots, true, kLUnroll, CLS_L>

// Degree bins, low-degree warp chunks and the bin-major arc copy col2
// (DESIGN.md §Layout), built on the device (layout.cuh).  off_d/col_d: the
// caller's CSR on the device (borrowed or staged).
void build_layout(glp_graph* g, const int64_t* off_d, const int32_t* col_d) {
  cudaStream_t s = g->stream;
  PoolAlloc palloc{s};
  auto pol = thrust::cuda::par(palloc).on(s);
  const int64_t nl = g->nl;
  std::vector<void*> tmp;
  auto talloc = [&](size_t bytes) {
    void* p = nullptr;
    if (pool_malloc(&p, std::max<size_t>(bytes, 16), s) != cudaSuccess) {
      cudaGetLastError();
      for (void* q : tmp) pool_free(q, s);
      fail(GLP_ERR_OUT_OF_MEMORY, "layout scratch allocation failed");
    }
    tmp.push_back(p);
    return p;
  };
  struct Free {
    std::vector<void*>& v;
    cudaStream_t s;
    ~Free() {
      for (void* p : v) pool_free(p, s);
    }
  } fr{tmp, s};
  int32_t* deg = (int32_t*)talloc(nl * sizeof(int32_t));
  LayoutStats* dst = (LayoutStats*)talloc(sizeof(LayoutStats));
  CK(cudaMemsetAsync(dst, 0, sizeof(LayoutStats), s));
  const int gb = g->sms * 8;
  if (nl) k_degree_stats<<<gb, 256, 0, s>>>(off_d, nl, deg, dst);
  CK(cudaGetLastError());
  LayoutStats st;
  CK(cudaMemcpyAsync(&st, dst, sizeof(st), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  trace("degree stats");
  for (int b = 0; b < NBINS; ++b) {
    g->bin_verts[b] = (int64_t)st.verts[b];
    g->bin_arcs[b] = (int64_t)st.arcs[b];
  }
  g->max_deg = (int64_t)st.max_deg;
  if (g->max_deg >= ((int64_t)1 << 30)) fail(GLP_ERR_INVALID_GRAPH, "row degree >= 2^30 is not supported");
  const int64_t n_low = g->bin_verts[BIN_LOW];
  const int64_t n_rows = nl - g->bin_verts[BIN_ISO] - n_low;
  g->ioff = dalloc<int64_t>(g, nl);
  g->ideg = dalloc<int32_t>(g, nl);
  CK(cudaMemsetAsync(g->ioff, 0, std::max<int64_t>(nl, 1) * sizeof(int64_t), s));
  CK(cudaMemsetAsync(g->ideg, 0, std::max<int64_t>(nl, 1) * sizeof(int32_t), s));
  unsigned long long* keys = (unsigned long long*)talloc(std::max(n_low, n_rows) * sizeof(unsigned long long));
  // orig_local[p] = local original id of internal vertex p: rows, low rows,
  // isolated vertices (layout.cuh, internal vertex order)
  int32_t* orig_local = (int32_t*)talloc(std::max<int64_t>(nl, 1) * sizeof(int32_t));
  // ---- low rows: sorted by (deg, id), packed floor(32/deg) per chunk
  int32_t* low_list = orig_local + n_rows;
  LowGroups grp;
  memset(&grp, 0, sizeof(grp));
  int64_t vb = 0, cb = 0, ab = 0;
  for (int d = 1; d <= 33; ++d) {
    grp.vbase[d] = vb;
    grp.cbase[d] = cb;
    grp.abase[d] = ab;
    if (d <= 32) {
      const int64_t cnt = (int64_t)st.low_hist[d];
      vb += cnt;
      cb += (cnt + (32 / d) - 1) / (32 / d);
      ab += cnt * d;
    }
  }
  g->n_low = (int32_t)n_low;
  g->low_base = n_rows;
  g->n_chunks = (int32_t)cb;
  g->chunks = dalloc<LowChunk>(g, cb);
  g->cflag = dalloc<uint8_t>(g, std::max<int64_t>(cb, 1));
  const int64_t low_arcs = ab;
  if (n_low) {
    thrust::copy_if(pol, thrust::counting_iterator<int32_t>(0), thrust::counting_iterator<int32_t>((int32_t)nl),
                    thrust::device_pointer_cast(low_list), IsLow{deg});
    k_make_keys<<<gb, 256, 0, s>>>(low_list, n_low, deg, 0, keys);
    thrust::sort(pol, thrust::device_pointer_cast(keys), thrust::device_pointer_cast(keys) + n_low);
    k_keys_to_ids<<<gb, 256, 0, s>>>(keys, n_low, low_list);
    k_low_chunks<<<gb, 256, 0, s>>>(grp, cb, n_low, g->chunks);
    k_low_place<<<gb, 256, 0, s>>>(grp, low_list, n_low, deg, n_rows, g->ioff, g->ideg);
    CK(cudaGetLastError());
  }
  // ---- other rows: (deg desc, id), 16-B aligned, padded to a multiple of 4
  int32_t* rows = orig_local;
  int64_t* pstart = (int64_t*)talloc((n_rows + 1) * sizeof(int64_t));
  const int64_t rows_base = (low_arcs + 3) & ~(int64_t)3;
  g->n_rows = (int32_t)n_rows;
  g->rows = dalloc<BinItem>(g, n_rows);
  std::vector<BinItem> row_i(n_rows);
  int64_t padded_total = 0;
  if (n_rows) {
    thrust::copy_if(pol, thrust::counting_iterator<int32_t>(0), thrust::counting_iterator<int32_t>((int32_t)nl),
                    thrust::device_pointer_cast(rows), IsRow{deg});
    k_make_keys<<<gb, 256, 0, s>>>(rows, n_rows, deg, 1, keys);
    thrust::sort(pol, thrust::device_pointer_cast(keys), thrust::device_pointer_cast(keys) + n_rows);
    k_keys_to_ids<<<gb, 256, 0, s>>>(keys, n_rows, rows);
    k_padded_deg<<<gb, 256, 0, s>>>(rows, n_rows, deg, pstart);
    CK(cudaGetLastError());
    thrust::exclusive_scan(pol, thrust::device_pointer_cast(pstart), thrust::device_pointer_cast(pstart) + n_rows + 1,
                           thrust::device_pointer_cast(pstart));
    k_row_place<<<gb, 256, 0, s>>>(rows, n_rows, deg, pstart, rows_base, g->rows, g->ioff, g->ideg);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(row_i.data(), g->rows, n_rows * sizeof(BinItem), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&padded_total, pstart + n_rows, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    trace("row order + placement");
  }
  g->nnz2 = rows_base + padded_total;
  if (g->nnz2 >= ((int64_t)1 << 48)) fail(GLP_ERR_INVALID_ARGUMENT, "graph too large");
  g->n_gt256 = g->n_gt2048 = g->n_ge8k = g->n_gt512 = 0;
  int64_t arcs_le64 = 0, arcs_rows = 0;
  for (const BinItem& it : row_i) {
    arcs_le64 += it.d <= 64 ? it.d : 0;
    arcs_rows += it.d;
    g->n_gt256 += it.d > 256;
    g->n_gt2048 += it.d > 2048;
    g->n_ge8k += it.d >= 8192;
    g->n_gt512 += it.d > kWtWarpMax;
  }
  const char* wse = getenv("GLP_W_SHORT");  // A/B: 0 / 1 forces the W variant
  g->w_short = wse ? wse[0] == '1' : 2 * arcs_le64 > arcs_rows;
  for (int k = 0; k < 3; ++k) g->pred[k] = dalloc<unsigned>(g, std::max<int64_t>(n_rows, 1));
  g->redo_m = dalloc<int32_t>(g, std::max<int64_t>(n_rows, 1));
  g->redo_l = dalloc<int32_t>(g, std::max<int64_t>(n_rows, 1));
  g->d_sched = dalloc<Sched>(g, 1);
  // giant rows: the prefix with deg > kGiantMin, split into segments
  g->n_giant = 0;
  for (const BinItem& it : row_i) g->n_giant += it.d > kGiantMin;
  if (g->n_giant > 0) {
    if (g->max_deg >= ((int64_t)1 << kGCountBits))
      fail(GLP_ERR_UNSUPPORTED, "a row has >= 2^25 arcs (giant-row table count field)");
    std::vector<GiantSeg> segs;
    std::vector<int32_t> first;
    std::vector<int64_t> toff;
    int64_t slots = 0;
    for (int32_t r = 0; r < g->n_giant; ++r) {
      first.push_back((int32_t)segs.size());
      toff.push_back(slots);
      for (int32_t b = 0; b < row_i[r].d; b += kGiantSeg) segs.push_back(GiantSeg{r, b});
      int64_t tsz = 1;
      while (tsz < 2 * (int64_t)row_i[r].d) tsz <<= 1;
      slots += tsz;
    }
    first.push_back((int32_t)segs.size());
    toff.push_back(slots);
    g->n_gsegs = (int32_t)segs.size();
    g->gsegs = upload(g, segs);
    g->gseg_first = upload(g, first);
    g->gtab_off = upload(g, toff);
    g->gtab_slots = slots;
    g->gtab = dalloc<unsigned long long>(g, slots);
    CK(cudaMemsetAsync(g->gtab, 0, slots * sizeof(unsigned long long), s));
    g->gepoch = 0;
    g->gcand_key = dalloc<unsigned long long>(g, segs.size());
    g->gcand_lab = dalloc<unsigned>(g, segs.size());
    g->gdistinct = dalloc<unsigned>(g, g->n_giant);
    CK(cudaMemsetAsync(g->gdistinct, 0, g->n_giant * sizeof(unsigned), s));
  }
  // ---- internal vertex order: isolated vertices last, then pos/orig of the
  // owned slice; with several ranks the slices are all-gathered (every rank
  // renames the global column ids of its arcs)
  const int64_t n_iso = nl - n_rows - n_low;
  if (n_iso)
    thrust::copy_if(pol, thrust::counting_iterator<int32_t>(0), thrust::counting_iterator<int32_t>((int32_t)nl),
                    thrust::device_pointer_cast(orig_local + n_rows + n_low), IsIso{deg});
  g->pos = dalloc<int32_t>(g, std::max<int64_t>(g->npad, 1));
  g->orig = dalloc<int32_t>(g, std::max<int64_t>(g->npad, 1));
  if (nl) k_perm<<<gb, 256, 0, s>>>(orig_local, nl, g->vb, g->pos, g->orig);
  if (g->npad > g->n) k_iota2<<<1, 256, 0, s>>>(g->pos, g->orig, g->n, g->npad);
  CK(cudaGetLastError());
  if (g->comm) {
    g->comm->allgather(g, g->pos, sizeof(int32_t));
    g->comm->allgather(g, g->orig, sizeof(int32_t));
  }
  // ---- the arcs themselves (copied and checked on the side stream, in
  // chunks of rows: each chunk is relayouted as soon as its copy landed)
  if (g->host_arcs) {
    // hybrid mode [P:103]: the bin-major arc array lives in pinned, mapped
    // host memory; the MFL kernels stream it over the host link (labels,
    // counters and tables stay in HBM)
    void* hp = nullptr;
    const size_t bytes = std::max<int64_t>(g->nnz2, 1) * sizeof(int32_t);
    if (cudaHostAlloc(&hp, bytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
      cudaGetLastError();
      fail(GLP_ERR_OUT_OF_MEMORY, "pinned host allocation of the arc array failed");
    }
    g->col2_host = hp;
    memset(hp, 0xff, bytes);  // padding = -1
    void* dp = nullptr;
    CK(cudaHostGetDevicePointer(&dp, hp, 0));
    g->col2 = (int32_t*)dp;
  } else {
    g->col2 = dalloc<int32_t>(g, g->nnz2);
    CK(cudaMemsetAsync(g->col2, 0xff, std::max<int64_t>(g->nnz2, 1) * sizeof(int32_t), s));  // padding = -1
  }
  if (nl > 0 && g->nnz > 0) {
    // rows past kRelayBig arcs: listed by k_relayout, copied by the grid
    int32_t* rbig = nullptr;
    unsigned* rnbig = nullptr;
    if (g->max_deg > kRelayBig) {
      const int64_t big_cap = g->nnz / kRelayBig + 1;
      rbig = dalloc<int32_t>(g, big_cap + 1);
      rnbig = (unsigned*)(rbig + big_cap);
      g->relay_big = rbig;
      g->relay_nbig = rnbig;
      CK(cudaMemsetAsync(rnbig, 0, sizeof(unsigned), s));
    }
    for (size_t c = 0; c + 1 < g->arc_chunks.size(); ++c) {
      if (c < g->arc_chunk_ev.size()) CK(cudaStreamWaitEvent(s, g->arc_chunk_ev[c], 0));
      else CK(cudaStreamWaitEvent(s, g->xev[1], 0));
      k_relayout<<<gb, 256, 0, s>>>(off_d, col_d, g->ioff, g->pos, g->arc_chunks[c], g->arc_chunks[c + 1], g->vb,
                                    g->n, g->col2, rbig, rnbig);
      CK(cudaGetLastError());
    }
    if (rbig) {
      k_relayout_big<<<gb, 256, 0, s>>>(off_d, col_d, g->ioff, g->pos, g->vb, g->n, g->col2, rbig, rnbig);
      CK(cudaGetLastError());
    }
  }
  CK(cudaStreamWaitEvent(s, g->xev[1], 0));
  {
    int bad = 0;
    CK(cudaMemcpyAsync(&bad, g->col_bad, sizeof(int), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    trace("arcs copied + checked + relayout");
    if (bad & 8) fail(GLP_ERR_INVALID_GRAPH, "col_idx entry outside [0, n_global)");
  }
}

void create_impl(const glp_csr* csr, const glp_dist* dist, const glp_params* prm, glp_graph** out) {
  CreateTrace tr;
  g_trace = &tr;
  struct Reset {
    ~Reset() { g_trace = nullptr; }
  } reset_trace;
  if (!out) fail(GLP_ERR_INVALID_ARGUMENT, "out is NULL");
  *out = nullptr;
  if (!csr) fail(GLP_ERR_INVALID_ARGUMENT, "csr is NULL");
  glp_params p = get_params(prm);
  const int64_t n = csr->n_global;
  if (n < 0 || n >= (int64_t)INT32_MAX) fail(GLP_ERR_INVALID_ARGUMENT, "n_global out of range [0, 2^31-1)");
  if (csr->v_begin < 0 || csr->v_end < csr->v_begin || csr->v_end > n)
    fail(GLP_ERR_INVALID_ARGUMENT, "owned row range [v_begin, v_end) invalid");
  if (csr->nnz_local < 0) fail(GLP_ERR_INVALID_ARGUMENT, "nnz_local < 0");
  if (!csr->row_offsets) fail(GLP_ERR_INVALID_ARGUMENT, "row_offsets is NULL");
  if (csr->nnz_local > 0 && !csr->col_idx) fail(GLP_ERR_INVALID_ARGUMENT, "col_idx is NULL");
  int rank = 0, nranks = 1;
  if (dist) {
    rank = dist->rank;
    nranks = dist->nranks;
    if (nranks < 1 || rank < 0 || rank >= nranks) fail(GLP_ERR_INVALID_ARGUMENT, "bad rank/nranks");
    if (nranks > 1 && !dist->nccl_unique_id && !dist->local_group)
      fail(GLP_ERR_INVALID_ARGUMENT, "nccl_unique_id or local_group required for nranks > 1");
    if (dist->nccl_unique_id && dist->local_group)
      fail(GLP_ERR_INVALID_ARGUMENT, "set nccl_unique_id or local_group, not both");
  }
  if (nranks == 1 && (csr->v_begin != 0 || csr->v_end != n))
    fail(GLP_ERR_INVALID_ARGUMENT, "single GPU: owned range must be [0, n_global)");

  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    fail(GLP_ERR_UNSUPPORTED, "no CUDA device visible (libglp has no CPU fallback)");
  }
  int dev = 0;
  if (dist) dev = dist->device;
  else CK(cudaGetDevice(&dev));
  if (dev < 0 || dev >= ndev) fail(GLP_ERR_INVALID_ARGUMENT, "device ordinal out of range");
  CK(cudaSetDevice(dev));
  cudaDeviceProp prop;
  CK(cudaGetDeviceProperties(&prop, dev));
  if (prop.major != 10)
    fail(GLP_ERR_UNSUPPORTED, std::string("libglp is built for sm_100a (B200); device is ") + prop.name);

  glp_graph* g = new glp_graph();
  try {
    g->device = dev;
    g->rank = rank;
    g->nranks = nranks;
    if (dist && dist->cuda_stream) {
      g->stream = (cudaStream_t)dist->cuda_stream;
    } else {
      CK(cudaStreamCreateWithFlags(&g->stream, cudaStreamNonBlocking));
      g->own_stream = true;
    }
    g->n = n;
    g->vb = csr->v_begin;
    g->ve = csr->v_end;
    g->nl = g->ve - g->vb;
    g->nnz = csr->nnz_local;
    g->symmetric = csr->symmetric ? 1 : 0;
    g->host_arcs = p.host_arcs != 0;
    if (g->host_arcs && csr->on_device) fail(GLP_ERR_INVALID_ARGUMENT, "host_arcs needs a host CSR (on_device = 0)");
    if (g->nnz >= ((int64_t)1 << 40)) fail(GLP_ERR_INVALID_ARGUMENT, "nnz_local too large");

    g->sms = prop.multiProcessorCount;
    side_streams(dev, g->xs);
    for (auto& e : g->xev) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    const int64_t* off_d = nullptr;
    const int32_t* col_d = nullptr;
    std::vector<void*> temps;  // caller-CSR staging freed after the relayout
    if (csr->on_device) {
      off_d = csr->row_offsets;
      col_d = csr->col_idx;
    } else if (g->host_arcs) {
      // hybrid mode: the caller's arcs stay in host memory (registered and
      // mapped for the relayout, which reads them over the host link); only
      // the offsets are staged on the device
      void* po = nullptr;
      if (pool_malloc(&po, (g->nl + 1) * sizeof(int64_t), g->stream) != cudaSuccess) {
        cudaGetLastError();
        fail(GLP_ERR_OUT_OF_MEMORY, "staging the row offsets on the device failed");
      }
      temps.push_back(po);
      CK(cudaMemcpyAsync(po, csr->row_offsets, (g->nl + 1) * sizeof(int64_t), cudaMemcpyHostToDevice, g->stream));
      off_d = (const int64_t*)po;
      if (g->nnz) {
        void* hp = (void*)csr->col_idx;
        void* dp = nullptr;
        // already pinned (cudaHostAlloc / registered by the caller): mapped
        // under UVA as it is; otherwise register it for the create
        cudaPointerAttributes pa;
        CK(cudaPointerGetAttributes(&pa, hp));
        if (pa.type != cudaMemoryTypeHost) {
          CK(cudaHostRegister(hp, g->nnz * sizeof(int32_t), cudaHostRegisterMapped | cudaHostRegisterReadOnly));
          g->registered = hp;
        }
        CK(cudaHostGetDevicePointer(&dp, hp, 0));
        col_d = (const int32_t*)dp;
      }
    } else {
      void *po = nullptr, *pc = nullptr;
      if (pool_malloc(&po, (g->nl + 1) * sizeof(int64_t), g->stream) != cudaSuccess ||
          pool_malloc(&pc, std::max<int64_t>(g->nnz, 1) * sizeof(int32_t), g->stream) != cudaSuccess) {
        cudaGetLastError();
        if (po) pool_free(po, g->stream);
        if (pc) pool_free(pc, g->stream);
        fail(GLP_ERR_OUT_OF_MEMORY, "staging the CSR on the device failed");
      }
      temps.push_back(po);
      temps.push_back(pc);
      CK(cudaMemcpyAsync(po, csr->row_offsets, (g->nl + 1) * sizeof(int64_t), cudaMemcpyHostToDevice, g->stream));
      off_d = (const int64_t*)po;
      col_d = (const int32_t*)pc;
      g->own_csr = true;
    }
    // The arcs (the bulk of a host CSR) are copied, and checked, on a side
    // stream while the layout is derived from the offsets alone; the arc
    // relayout waits for them (col_ready).
    int* dbad = dalloc<int>(g, 2);
    CK(cudaMemsetAsync(dbad, 0, 2 * sizeof(int), g->stream));
    CK(cudaEventRecord(g->xev[0], g->stream));
    CK(cudaStreamWaitEvent(g->xs[0], g->xev[0], 0));
    // row chunks of ~equal arcs (host offsets): copy + check chunk c, then
    // record its event; the relayout of chunk c waits for that event only
    g->arc_chunks.assign({0, g->nl});
    if (!csr->on_device && !g->host_arcs && g->nnz >= ((int64_t)1 << 26)) {
      const int K = 8;
      g->arc_chunks.clear();
      g->arc_chunks.push_back(0);
      for (int c = 1; c < K; ++c) {
        const int64_t target = g->nnz * c / K;
        const int64_t r = std::upper_bound(csr->row_offsets, csr->row_offsets + g->nl + 1, target) - csr->row_offsets - 1;
        if (r > g->arc_chunks.back() && r < g->nl) g->arc_chunks.push_back(r);
      }
      g->arc_chunks.push_back(g->nl);
    }
    // GLP_TRACE_CREATE: time the arc copy on the side stream
    cudaEvent_t tc0 = nullptr, tc1 = nullptr;
    if (g_trace && g_trace->on) {
      CK(cudaEventCreate(&tc0));
      CK(cudaEventCreate(&tc1));
      CK(cudaEventRecord(tc0, g->xs[0]));
    }
    for (size_t c = 0; c + 1 < g->arc_chunks.size(); ++c) {
      const int64_t a0 = csr->on_device || g->host_arcs ? 0 : csr->row_offsets[g->arc_chunks[c]];
      const int64_t a1 = csr->on_device || g->host_arcs ? g->nnz : csr->row_offsets[g->arc_chunks[c + 1]];
      if (!csr->on_device && !g->host_arcs && a1 > a0)
        CK(cudaMemcpyAsync((void*)(col_d + a0), csr->col_idx + a0, (a1 - a0) * sizeof(int32_t),
                           cudaMemcpyHostToDevice, g->xs[0]));
      if (p.validate && a1 > a0) k_validate_col<<<g->sms * 4, 256, 0, g->xs[0]>>>(col_d + a0, a1 - a0, g->n, dbad + 1);
      CK(cudaGetLastError());
      if (g->arc_chunks.size() > 2) {
        cudaEvent_t e;
        CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        g->arc_chunk_ev.push_back(e);
        CK(cudaEventRecord(e, g->xs[0]));
      }
    }
    CK(cudaEventRecord(g->xev[1], g->xs[0]));
    if (g_trace && g_trace->on) {
      CK(cudaEventRecord(tc1, g->xs[0]));
      CK(cudaEventSynchronize(tc1));
      float cms = 0.f;
      CK(cudaEventElapsedTime(&cms, tc0, tc1));
      fprintf(stderr, "[glp create] arc copy + check on the side stream: %.2f ms (%.1f GB/s)\n", cms,
              g->nnz * 4.0 / 1e6 / std::max(cms, 1e-3f));
      cudaEventDestroy(tc0);
      cudaEventDestroy(tc1);
    }
    struct TempGuard {
      std::vector<void*>& v;
      cudaStream_t s;
      cudaEvent_t col_ready;
      ~TempGuard() {
        cudaStreamWaitEvent(s, col_ready, 0);  // the side-stream copy may still read the staging
        for (void* p : v) pool_free(p, s);
      }
    } tg{temps, g->stream, g->xev[1]};
    // structural checks on the device: off[0] == 0, off[nl] == nnz, monotone
    // offsets (always); col in [0, n) (validate = 1, checked before the relayout)
    {
      k_validate_off<<<g->sms * 4, 256, 0, g->stream>>>(off_d, g->nl, g->nnz, dbad);
      CK(cudaGetLastError());
      int bad = 0;
      CK(cudaMemcpyAsync(&bad, dbad, sizeof(int), cudaMemcpyDeviceToHost, g->stream));
      CK(cudaStreamSynchronize(g->stream));
      trace("offsets checked");
      if (bad & 3) fail(GLP_ERR_INVALID_GRAPH, "row_offsets[0] must be 0 and row_offsets[last] == nnz_local");
      if (bad & 4) fail(GLP_ERR_INVALID_GRAPH, "row_offsets not non-decreasing");
    }
    g->col_bad = dbad + 1;
    // labels: replicated full arrays, padded to a multiple of nranks for the
    // in-place all-gather
    const int64_t npad = ((n + nranks - 1) / nranks) * nranks;
    g->npad = npad;
    g->nnz_global = g->nnz;
    // exchange for nranks > 1: an in-process local group, else NCCL; with
    // nranks == 1 a unique id or group still selects that path (a one-rank
    // communicator), which tests its plumbing on one GPU
    if (dist && dist->local_group) g->comm = new LocalComm(g, dist->local_group);
    else if (nranks > 1 || (dist && dist->nccl_unique_id)) g->comm = new NcclComm(g, dist->nccl_unique_id);
    if (g->comm) g->comm->setup(g);
    build_layout(g, off_d, col_d);
    if (csr->weights) {
      // weighted LP: validate and place the weights beside the arcs
      const uint32_t* w_d = csr->weights;
      if (!csr->on_device) {
        void* pw = nullptr;
        if (g->nnz && pool_malloc(&pw, g->nnz * sizeof(uint32_t), g->stream) != cudaSuccess) {
          cudaGetLastError();
          fail(GLP_ERR_OUT_OF_MEMORY, "staging the weights on the device failed");
        }
        if (pw) {
          temps.push_back(pw);
          CK(cudaMemcpyAsync(pw, csr->weights, g->nnz * sizeof(uint32_t), cudaMemcpyHostToDevice, g->stream));
        }
        w_d = (const uint32_t*)pw;
      }
      g->w2 = dalloc<uint32_t>(g, std::max<int64_t>(g->nnz2, 1));
      CK(cudaMemsetAsync(g->w2, 0, std::max<int64_t>(g->nnz2, 1) * sizeof(uint32_t), g->stream));
      if (g->nl && g->nnz) {
        k_validate_w<<<g->sms * 4, 256, 0, g->stream>>>(off_d, w_d, g->nl, dbad);
        k_relayout_w<<<g->sms * 8, 256, 0, g->stream>>>(off_d, w_d, g->ioff, g->pos, g->nl, g->vb, g->w2);
        if (g->relay_big)
          k_relayout_w_big<<<g->sms * 8, 256, 0, g->stream>>>(off_d, w_d, g->ioff, g->pos, g->vb, g->w2, g->relay_big,
                                                             g->relay_nbig);
        CK(cudaGetLastError());
      }
      int bad = 0;
      CK(cudaMemcpyAsync(&bad, dbad, sizeof(int), cudaMemcpyDeviceToHost, g->stream));
      CK(cudaStreamSynchronize(g->stream));
      if (bad & 16) fail(GLP_ERR_INVALID_GRAPH, "weights must be in [1, 2^31) with every row total < 2^31");
      g->weighted = true;
      // giant rows whose weight totals fit the giant tables' count field are
      // counted by the segmented giant kernels (else one block per row)
      const char* wg = getenv("GLP_WT_GIANT");
      if (g->n_giant > 0 && !(wg && wg[0] == '0')) {
        unsigned long long* dmx = nullptr;
        CK(cudaMallocAsync((void**)&dmx, sizeof(unsigned long long), g->stream));
        CK(cudaMemsetAsync(dmx, 0, sizeof(unsigned long long), g->stream));
        k_giant_wsum_max<<<std::min(g->n_giant, g->sms * 4), 256, 0, g->stream>>>(g->rows, g->n_giant, g->w2, dmx);
        unsigned long long mx = 0;
        CK(cudaMemcpyAsync(&mx, dmx, sizeof(mx), cudaMemcpyDeviceToHost, g->stream));
        CK(cudaFreeAsync(dmx, g->stream));
        CK(cudaStreamSynchronize(g->stream));
        g->wt_giant = mx < (1ull << kGCountBits);
      }
      const char* wl = getenv("GLP_WT_LOW");
      g->wt_low_off = wl && wl[0] == '0';
    }
    if (g->registered) {  // the caller's arcs are not read after the relayout
      CK(cudaStreamSynchronize(g->stream));
      cudaHostUnregister(g->registered);
      g->registered = nullptr;
    }

    g->L[0] = dalloc<int32_t>(g, npad);
    g->L[1] = dalloc<int32_t>(g, npad);
    g->so = dalloc<int2>(g, g->nl);
    g->V = dalloc<int32_t>(g, std::max<int64_t>(n, 1));
    if (g->comm) g->Vloc = dalloc<int32_t>(g, std::max<int64_t>(n, 1));
    g->is_seed = dalloc<uint8_t>(g, g->nl);
    g->flag[0] = dalloc<uint8_t>(g, npad);
    g->flag[1] = dalloc<uint8_t>(g, npad);
    CK(cudaMemsetAsync(g->flag[0], 0, std::max<int64_t>(npad, 1), g->stream));
    CK(cudaMemsetAsync(g->flag[1], 0, std::max<int64_t>(npad, 1), g->stream));
    g->d_cnt = dalloc<Counters>(g, kNumCounters);
    g->push_big = dalloc<int32_t>(g, std::max<int64_t>(g->nl, 1));  // frontier push: long changed rows
    g->push_nbig = dalloc<unsigned>(g, 1);
    CK(cudaMallocHost(&g->h_cnt, kNumCounters * sizeof(Counters)));
    CK(cudaEventCreate(&g->ev_a));
    CK(cudaEventCreate(&g->ev_b));
    {
      const char* ser = getenv("GLP_SERIAL");
      g->concurrent = !(ser && ser[0] == '1');
      const char* novl = getenv("GLP_NO_VL");
      g->use_vl = !(novl && novl[0] == '1');
      const char* nomono = getenv("GLP_NO_MONO");
      g->use_mono = !(nomono && nomono[0] == '1');
      // device-driven loop: opt-in (GLP_DEVICE_LOOP=1).  A/B, median ms/run:
      // karate 0.47 -> 0.59, SBM 5.38 -> 5.44, R24 18.19 -> 17.98, TaoBao
      // 109.1 -> 108.5, R24 LLP 177.7 -> 178.1: the kernels it must enqueue
      // unconditionally (push, mark clearing, decide) cost about what the
      // host round trip saved
      const char* dl = getenv("GLP_DEVICE_LOOP");
      g->dev_loop = dl && dl[0] == '1';
      const char* l2w = getenv("GLP_L2_WINDOW");
      if (l2w && l2w[0] == '1') {
        // persisting L2 set-aside up to the device maximum
        int maxp = 0, maxw = 0;
        CK(cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev));
        CK(cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, dev));
        CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)maxp));
        g->l2_window = maxp > 0 && maxw > 0;
        g->l2_window_max = (size_t)maxw;
      }
    }

    const int sms = g->sms;
    const int ms_ = kMSlots * 8, ls_ = kLSlots * 8;
    CK(cudaFuncSetAttribute(GLP_M_KERNEL(V_CLASSIC), cudaFuncAttributeMaxDynamicSharedMemorySize, ms_));
    CK(cudaFuncSetAttribute(GLP_M_KERNEL(V_SEEDED), cudaFuncAttributeMaxDynamicSharedMemorySize, ms_));
    CK(cudaFuncSetAttribute(GLP_M_KERNEL(V_LLP), cudaFuncAttributeMaxDynamicSharedMemorySize, ms_));
    // (+ the CMS counters of the §8(f)2 HT + CMS mode)
    const int lsc_ = ls_ + (int)kCmsCounters * 4;
    CK(cudaFuncSetAttribute(GLP_L_KERNEL(V_CLASSIC), cudaFuncAttributeMaxDynamicSharedMemorySize, lsc_));
    CK(cudaFuncSetAttribute(GLP_L_KERNEL(V_SEEDED), cudaFuncAttributeMaxDynamicSharedMemorySize, lsc_));
    CK(cudaFuncSetAttribute(GLP_L_KERNEL(V_LLP), cudaFuncAttributeMaxDynamicSharedMemorySize, lsc_));
    g->grid_low = grid_for(sms, (const void*)mfl_low<V_LLP>, kLowBlock, 0);
    const int ws_ = (kWBlock / 32) * kWSlots * 8;
    CK(cudaFuncSetAttribute(mfl_warp<V_CLASSIC>, cudaFuncAttributeMaxDynamicSharedMemorySize, ws_));
    CK(cudaFuncSetAttribute(mfl_warp<V_SEEDED>, cudaFuncAttributeMaxDynamicSharedMemorySize, ws_));
    CK(cudaFuncSetAttribute(mfl_warp<V_LLP>, cudaFuncAttributeMaxDynamicSharedMemorySize, ws_));
    CK(cudaFuncSetAttribute(mfl_warp<V_CLASSIC, 3>, cudaFuncAttributeMaxDynamicSharedMemorySize, ws_));
    CK(cudaFuncSetAttribute(mfl_warp<V_SEEDED, 3>, cudaFuncAttributeMaxDynamicSharedMemorySize, ws_));
    CK(cudaFuncSetAttribute(mfl_warp<V_LLP, 3>, cudaFuncAttributeMaxDynamicSharedMemorySize, ws_));
    g->grid_w = g->w_short ? grid_for(sms, (const void*)mfl_warp<V_LLP, 3>, kWBlock, ws_)
                           : grid_for(sms, (const void*)mfl_warp<V_LLP>, kWBlock, ws_);
    g->grid_m = grid_for(sms, (const void*)GLP_M_KERNEL(V_LLP), kMBlock, ms_);
    g->grid_mono = grid_for(sms, (const void*)mfl_mono<V_LLP>, kMonoBlock, 0);
    const int wtw_ = (kWtBlock / 32) * kWtWarpSlots * 8, wtb_ = kWtSlots * 8;
    CK(cudaFuncSetAttribute(mfl_wt_warp<V_CLASSIC>, cudaFuncAttributeMaxDynamicSharedMemorySize, wtw_));
    CK(cudaFuncSetAttribute(mfl_wt_warp<V_SEEDED>, cudaFuncAttributeMaxDynamicSharedMemorySize, wtw_));
    CK(cudaFuncSetAttribute(mfl_wt_block<V_CLASSIC>, cudaFuncAttributeMaxDynamicSharedMemorySize, wtb_));
    CK(cudaFuncSetAttribute(mfl_wt_block<V_SEEDED>, cudaFuncAttributeMaxDynamicSharedMemorySize, wtb_));
    g->grid_wtw = grid_for(sms, (const void*)mfl_wt_warp<V_CLASSIC>, kWtBlock, wtw_);
    g->grid_wtb = grid_for(sms, (const void*)mfl_wt_block<V_CLASSIC>, kWtBBlock, wtb_);
    g->grid_l = grid_for(sms, (const void*)GLP_L_KERNEL(V_LLP), kLBlock, ls_);
    const int gs_ = GLP_GIANT_SMEM ? kGSlots * 8 : 0;
    CK(cudaFuncSetAttribute(mfl_giant_count<V_CLASSIC>, cudaFuncAttributeMaxDynamicSharedMemorySize, gs_));
    CK(cudaFuncSetAttribute(mfl_giant_count<V_SEEDED>, cudaFuncAttributeMaxDynamicSharedMemorySize, gs_));
    CK(cudaFuncSetAttribute(mfl_giant_count<V_LLP>, cudaFuncAttributeMaxDynamicSharedMemorySize, gs_));
    CK(cudaFuncSetAttribute(mfl_giant_count<V_CLASSIC, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, gs_));
    CK(cudaFuncSetAttribute(mfl_giant_count<V_SEEDED, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, gs_));
    g->grid_g = grid_for(sms, (const void*)mfl_giant_count<V_LLP>, kGBlock, gs_);
    g->grid_aux = sms * 8;
    if (g->n_rows > 0) {
      // L staging: two row-sized buffers per resident L block, in two regions:
      // the static L launch (side stream) and the redo L launch (main stream)
      // may run at the same time, so each has its own (a shared
      // region let a redo row overwrite a static row's staged labels).
      // L never takes giant rows (deg > kGiantMin)
      g->stage_stride = (std::min<int64_t>(g->max_deg, kGiantMin) + 3) & ~(int64_t)3;
      g->stage = dalloc<int32_t>(g, (size_t)g->stage_stride * 4 * g->grid_l);
    }
    CK(cudaStreamSynchronize(g->stream));
    trace("done");
  } catch (const Err& e) {
    if (g->comm) g->comm->abort(e.msg);  // release the other ranks of a local group
    free_graph(g);
    throw;
  } catch (...) {
    if (g->comm) g->comm->abort("rank failed in glp_graph_create");
    free_graph(g);
    throw;
  }
  *out = g;
}

// ---------------------------------------------------------------- profiling
struct Pending {
  int kid;
  cudaEvent_t a, b;
  int t;  // iteration of the launch
};

cudaEvent_t pool_event(glp_graph* g, size_t& used) {
  if (used == g->ev_pool.size()) {
    cudaEvent_t e;
    CK(cudaEventCreate(&e));
    g->ev_pool.push_back(e);
  }
  return g->ev_pool[used++];
}

const char* kKernelNames[] = {"mfl_low", "mfl_warp", "mfl_block_m", "mfl_block_l", "push", "llp_hist", "exchange",
                              "mfl_giant", "mfl_mono", "mfl_wt_warp", "mfl_wt_block"};
constexpr int kNumKernelNames = 11;
// counter slot of each MFL kernel id (glp_internal.cuh kNumCounters)
inline int counter_of(int kid) { return kid == 7 ? 4 : kid == 8 ? 5 : kid == 9 ? 1 : kid == 10 ? 3 : kid; }

template <class F>
void timed(glp_graph* g, bool prof, int kid, std::vector<Pending>& pend, size_t& used, cudaStream_t st, F f) {
  if (!prof) {
    f();
    CK(cudaGetLastError());
    return;
  }
  // events on the launching stream: with concurrent class kernels the time is
  // the launch's duration while it shares the GPU with the others
  cudaEvent_t a = pool_event(g, used), b = pool_event(g, used);
  CK(cudaEventRecord(a, st));
  f();
  CK(cudaGetLastError());
  CK(cudaEventRecord(b, st));
  pend.push_back({kid, a, b, g->cur_t});
}

// ---------------------------------------------------------------- run
// frontier push of the vertices changed at t (k_push + its long-row pass)
void push(glp_graph* g, int32_t t, uint8_t* flag, const int* ctl = nullptr, int* dirty = nullptr) {
  cudaStream_t s = g->stream;
  CK(cudaMemsetAsync(g->push_nbig, 0, sizeof(unsigned), s));
  k_push<<<g->grid_aux, 256, 0, s>>>(g->ioff, g->ideg, g->col2, g->so, g->nl, g->vb, t, flag, g->push_big,
                                     g->push_nbig, ctl, dirty);
  if (g->max_deg >= kPushBig)
    k_push_big<<<g->sms * 4, 256, 0, s>>>(g->ioff, g->ideg, g->col2, g->push_big, g->push_nbig, flag, ctl);
  CK(cudaGetLastError());
}

template <int VAR>
int launch_mfl(glp_graph* g, MflArgs a, bool prof, std::vector<Pending>& pend, size_t& used) {
  Counters* c = g->d_cnt;
  Sched* sc = g->d_sched;
  int n = 0;
  const size_t ms_ = kMSlots * 8, ls_ = kLSlots * 8 + (a.cms ? kCmsCounters * 4 : 0);
  MflArgs r = a;
  r.items = g->rows; r.big_prefix = g->n_ge8k; r.pred = g->pred[g->pb]; r.pred_prev = g->pred[(g->pb + 2) % 3];
  r.pred_next = g->pred[(g->pb + 1) % 3];
  r.stage = g->stage; r.stage_stride = g->stage_stride;
  // The class kernels of one iteration touch disjoint rows, so they run
  // concurrently (filling each other's tails) unless profiling or GLP_SERIAL:
  // giant | L | M | low on their own streams, W -> redo M -> redo L on the
  // main stream (redo L also waits for the static M, which feeds its queue).
  const bool cc = g->concurrent && !prof;  // profiled runs serialise: clean per-kernel durations
  cudaStream_t s0 = g->stream;
  bool used_x[4] = {false, false, false, false};
  auto S = [&](int i) -> cudaStream_t {
    if (!cc) return s0;
    used_x[i] = true;
    return g->xs[i];
  };
  if (cc) {
    CK(cudaEventRecord(g->xev[0], s0));
    for (auto x : g->xs) CK(cudaStreamWaitEvent(x, g->xev[0], 0));
  }
  if (g->l2_window) {
    // A/B (GLP_L2_WINDOW=1): an L2 persisting access-policy window on the
    // array every arc gathers from (L_{t-1}, or LV for LLP), on every stream
    // that runs an MFL kernel of this iteration
    cudaStreamAttrValue av;
    memset(&av, 0, sizeof(av));
    const void* base = a.LV ? (const void*)a.LV : (const void*)a.R;
    const size_t bytes = (size_t)g->npad * (a.LV ? sizeof(int2) : sizeof(int32_t));
    av.accessPolicyWindow.base_ptr = const_cast<void*>(base);
    av.accessPolicyWindow.num_bytes = std::min(bytes, g->l2_window_max);
    av.accessPolicyWindow.hitRatio = 1.0f;
    av.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    av.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    CK(cudaStreamSetAttribute(s0, cudaStreamAttributeAccessPolicyWindow, &av));
    for (auto x : g->xs) CK(cudaStreamSetAttribute(x, cudaStreamAttributeAccessPolicyWindow, &av));
  }
  if (g->n_giant) {  // giant rows: all blocks count segments into per-row global tables
    MflArgs b = r;
    b.cnt = c + 4; b.work = &sc->work_g;
    b.gsegs = g->gsegs; b.n_gsegs = g->n_gsegs; b.gtab = g->gtab; b.gtab_off = g->gtab_off;
    b.gcand_key = g->gcand_key; b.gcand_lab = g->gcand_lab; b.gdistinct = g->gdistinct; b.epoch = g->gepoch;
    timed(g, prof, 7, pend, used, cc ? g->xs[0] : s0, [&] {
      mfl_giant_count<VAR><<<std::min(g->grid_g, g->n_gsegs), kGBlock, GLP_GIANT_SMEM ? kGSlots * 8 : 0, S(0)>>>(b);
      mfl_giant_finish<VAR><<<g->n_giant, 256, 0, S(0)>>>(b, g->gseg_first);
    });
    n += 2;
  }
  if (g->n_gt2048) {  // L, static: rows of class L (a prefix of deg > 2048)
    MflArgs b = r;
    b.n_items = g->n_gt2048; b.cnt = c + 3; b.work = &sc->work_l;
    const int grid = std::min<int>(g->grid_l, g->n_ge8k + (g->n_gt2048 - g->n_ge8k + 31) / 32);
    timed(g, prof, 3, pend, used, cc ? g->xs[1] : s0, [&] { GLP_L_KERNEL(VAR)<<<grid, kLBlock, ls_, S(1)>>>(b); });
    ++n;
  }
  if (g->n_gt256) {  // M, static; overflowing rows -> L redo list
    MflArgs b = r;
    b.n_items = g->n_gt256; b.cnt = c + 2; b.redo_out = g->redo_l; b.redo_out_n = &sc->n_redo_l;
    b.work = &sc->work_m;
    const int grid = std::min<int>(g->grid_m, g->n_ge8k + (g->n_gt256 - g->n_ge8k + 31) / 32);
    timed(g, prof, 2, pend, used, cc ? g->xs[2] : s0, [&] { GLP_M_KERNEL(VAR)<<<grid, kMBlock, ms_, S(2)>>>(b); });
    if (cc) CK(cudaEventRecord(g->xev[1], g->xs[2]));
    ++n;
  }
  if (g->n_rows && a.mono_kernel) {  // t = 1: sorted-row candidates, table-free; unsorted rows -> M redo list
    MflArgs b = r;
    b.n_items = g->n_rows; b.cnt = c + 5; b.redo_out = g->redo_m; b.redo_out_n = &sc->n_redo_m;
    const int grid = std::min<int>(g->grid_mono, (g->n_rows + kMonoBlock - 1) / kMonoBlock);
    timed(g, prof, 8, pend, used, s0, [&] { mfl_mono<VAR><<<grid, kMonoBlock, 0, s0>>>(b); });
    ++n;
  }
  if (g->n_rows) {  // W: every row of class W; overflowing rows -> M redo list
    MflArgs b = r;
    b.n_items = g->n_rows; b.cnt = c + 1; b.redo_out = g->redo_m; b.redo_out_n = &sc->n_redo_m;
    const int grid = std::min<int>(g->grid_w, (g->n_rows + kWBlock - 1) / kWBlock);
    timed(g, prof, 1, pend, used, s0,
          [&] {
            if (g->w_short) mfl_warp<VAR, 3><<<grid, kWBlock, (kWBlock / 32) * kWSlots * 8, s0>>>(b);
            else mfl_warp<VAR><<<grid, kWBlock, (kWBlock / 32) * kWSlots * 8, s0>>>(b);
          });
    ++n;
  }
  if (g->n_chunks) {
    MflArgs b = a;
    b.low_base = g->low_base; b.chunks = g->chunks; b.cflag = g->cflag; b.n_chunks = g->n_chunks; b.cnt = c + 0;
    const int grid = std::min<int>(g->grid_low, (g->n_chunks + kLowBlock - 1) / kLowBlock);
    timed(g, prof, 0, pend, used, cc ? g->xs[3] : s0, [&] { mfl_low<VAR><<<grid, kLowBlock, 0, S(3)>>>(b); });
    ++n;
  }
  if (g->n_rows) {
    // re-queued rows (their labels overflowed the smaller table): W -> M -> L.
    // The redo launches read the queue length on the device and exit at once
    // when it is empty.
    MflArgs b = r;
    b.mode = 1; b.cnt = c + 2; b.redo_in = g->redo_m; b.redo_in_n = &sc->n_redo_m; b.work = &sc->work_mr;
    b.redo_out = g->redo_l; b.redo_out_n = &sc->n_redo_l;
    timed(g, prof, 2, pend, used, s0, [&] { GLP_M_KERNEL(VAR)<<<g->grid_m, kMBlock, ms_, s0>>>(b); });
    if (used_x[2]) CK(cudaStreamWaitEvent(s0, g->xev[1], 0));
    MflArgs q = r;
    q.mode = 1; q.cnt = c + 3; q.redo_in = g->redo_l; q.redo_in_n = &sc->n_redo_l; q.work = &sc->work_lr;
    q.stage = g->stage + (size_t)g->stage_stride * 2 * g->grid_l;  // redo region (runs beside static L)
    timed(g, prof, 3, pend, used, s0, [&] { GLP_L_KERNEL(VAR)<<<g->grid_l, kLBlock, ls_, s0>>>(q); });
    n += 2;
  }
  if (cc) {
    // join: the main stream waits for every side stream used
    const int xe[4] = {2, 3, 1, 4};
    for (int i = 0; i < 4; ++i)
      if (used_x[i] && i != 2) {
        CK(cudaEventRecord(g->xev[xe[i]], g->xs[i]));
        CK(cudaStreamWaitEvent(s0, g->xev[xe[i]], 0));
      }
    if (used_x[2] && !g->n_rows) CK(cudaStreamWaitEvent(s0, g->xev[1], 0));
  }
  return n;
}

// weighted LP (§8(f)3): long rows block-per-row, the rest warp-per-vertex
template <int VAR>
int launch_wt(glp_graph* g, MflArgs a, bool prof, std::vector<Pending>& pend, size_t& used) {
  Counters* c = g->d_cnt;
  Sched* sc = g->d_sched;
  cudaStream_t s0 = g->stream;
  a.w2 = g->w2; a.ioff = g->ioff; a.ideg = g->ideg;
  int n = 0;
  // giant rows (deg > kGiantMin): segments over all blocks, weights added
  // into the per-row global tables (mfl_giant_count), when their totals fit
  const int g0 = g->wt_giant ? g->n_giant : 0;
  if (g0) {
    MflArgs b = a;
    b.items = g->rows; b.pred = g->pred[g->pb]; b.pred_next = g->pred[(g->pb + 1) % 3];
    b.cnt = c + 4; b.work = &sc->work_g;
    b.gsegs = g->gsegs; b.n_gsegs = g->n_gsegs; b.gtab = g->gtab; b.gtab_off = g->gtab_off;
    b.gcand_key = g->gcand_key; b.gcand_lab = g->gcand_lab; b.gdistinct = g->gdistinct; b.epoch = g->gepoch;
    timed(g, prof, 7, pend, used, s0, [&] {
      mfl_giant_count<VAR, true><<<std::min(g->grid_g, g->n_gsegs), kGBlock, GLP_GIANT_SMEM ? kGSlots * 8 : 0, s0>>>(b);
      mfl_giant_finish<VAR><<<g->n_giant, 256, 0, s0>>>(b, g->gseg_first);
    });
    n += 2;
  }
  if (g->n_gt512 > g0) {
    MflArgs b = a;
    b.items = g->rows + g0; b.n_items = g->n_gt512 - g0; b.cnt = c + 3; b.work = &sc->work_l;
    b.pred = g->pred[g->pb] + g0; b.pred_next = g->pred[(g->pb + 1) % 3] + g0;
    const int grid = std::min(g->grid_wtb, g->n_gt512 - g0);
    timed(g, prof, 10, pend, used, s0,
          [&] { mfl_wt_block<VAR><<<grid, kWtBBlock, kWtSlots * 8, s0>>>(b); });
    ++n;
  }
  // low-degree vertices (deg <= 32): the packed-warp kernel with weight sums
  if (g->n_chunks && !g->wt_low_off) {
    MflArgs b = a;
    b.low_base = g->low_base; b.chunks = g->chunks; b.cflag = g->cflag; b.n_chunks = g->n_chunks; b.cnt = c + 0;
    const int grid = std::min<int>(g->grid_low, (g->n_chunks + kLowBlock - 1) / kLowBlock);
    timed(g, prof, 0, pend, used, s0, [&] { mfl_low<VAR, true><<<grid, kLowBlock, 0, s0>>>(b); });
    ++n;
  }
  const int64_t lo = g->n_gt512, hi = (int64_t)g->n_rows + (g->wt_low_off ? g->n_low : 0);
  if (hi > lo) {
    MflArgs b = a;
    b.wt_lo = lo; b.wt_hi = hi; b.cnt = c + 1;
    const int grid = (int)std::min<int64_t>(g->grid_wtw, (hi - lo + kWtBlock - 1) / kWtBlock);
    timed(g, prof, 9, pend, used, s0,
          [&] { mfl_wt_warp<VAR><<<grid, kWtBlock, (kWtBlock / 32) * kWtWarpSlots * 8, s0>>>(b); });
    ++n;
  }
  return n;
}

void run_impl(glp_graph* g, glp_variant variant, int32_t max_iters, const int32_t* seeds, int64_t n_seeds,
              const glp_params* prm, glp_run_info* info) {
  if (!g) fail(GLP_ERR_INVALID_ARGUMENT, "graph is NULL");
  glp_params p = get_params(prm);
  if (variant < GLP_VARIANT_CLASSIC || variant > GLP_VARIANT_SLP) fail(GLP_ERR_INVALID_ARGUMENT, "unknown variant");
  const bool slp = variant == GLP_VARIANT_SLP;
  const int slp_k = p.slp_max_labels > 0 ? p.slp_max_labels : 5;
  if (slp) {
    if (slp_k > 16) fail(GLP_ERR_INVALID_ARGUMENT, "slp_max_labels must be in [1, 16]");
    if (!(p.slp_threshold >= 0.0) || !std::isfinite(p.slp_threshold))
      fail(GLP_ERR_INVALID_ARGUMENT, "slp_threshold must be finite and >= 0");
    if (g->weighted) fail(GLP_ERR_UNSUPPORTED, "SLP on a weighted graph is not supported");
  }
  if (max_iters < 0) fail(GLP_ERR_INVALID_ARGUMENT, "max_iters < 0");
  if (variant == GLP_VARIANT_LLP) {
    if (!std::isfinite(p.gamma) || p.gamma < 0) fail(GLP_ERR_INVALID_ARGUMENT, "gamma must be finite and >= 0");
    if (p.frontier == 1) fail(GLP_ERR_INVALID_ARGUMENT, "the frontier is not exact for LLP (frontier=1 rejected)");
    if (g->weighted) fail(GLP_ERR_UNSUPPORTED, "weighted LP supports CLASSIC and SEEDED (not LLP)");
  }
  if (variant != GLP_VARIANT_SEEDED && (seeds != nullptr || n_seeds != 0))
    fail(GLP_ERR_INVALID_ARGUMENT, "seeds are only valid for GLP_VARIANT_SEEDED");
  if (n_seeds < 0 || (n_seeds > 0 && !seeds)) fail(GLP_ERR_INVALID_ARGUMENT, "bad seeds/n_seeds");
  for (int64_t i = 0; i < n_seeds; ++i)
    if (seeds[i] < 0 || seeds[i] >= g->n) fail(GLP_ERR_INVALID_ARGUMENT, "seed id out of range");
  if (p.frontier == 1 && !g->symmetric)
    fail(GLP_ERR_INVALID_ARGUMENT, "frontier=1 needs a symmetric graph (glp_csr.symmetric)");
  // SLP: the speakers change by the memory rule, not by the neighbours alone:
  // full sweeps (R19)
  const bool use_frontier = variant != GLP_VARIANT_LLP && !slp && g->symmetric && p.frontier != 0;
  const bool prof = p.profile != 0;

  CK(cudaSetDevice(g->device));
  cudaStream_t s = g->stream;
  const int ga = g->grid_aux;
  // PickLabel
  g->init_launches = 1;
  k_init_labels<<<ga, 256, 0, s>>>(g->L[0], g->L[1], g->orig, g->npad, variant == GLP_VARIANT_SEEDED);
  CK(cudaGetLastError());
  CK(cudaMemsetAsync(g->so, 0x80, std::max<int64_t>(g->nl, 1) * sizeof(int2), s));  // stamp = INT_MIN-ish
  CK(cudaMemsetAsync(g->is_seed, 0, std::max<int64_t>(g->nl, 1), s));
  for (int f = 0; f < 2; ++f)
    if (!g->flag_clean[f]) {
      CK(cudaMemsetAsync(g->flag[f], 0, std::max<int64_t>(g->npad, 1), s));
      g->flag_clean[f] = true;
    }
  // SEEDED presence filter (mfl_kernels.cuh lbit_clear): one rank, label
  // array larger than ~3/4 of L2 (GLP_LBITS=0 off, =1 forced)
  const char* lbenv = getenv("GLP_LBITS");
  const bool use_lbits = variant == GLP_VARIANT_SEEDED && !g->comm && !(lbenv && lbenv[0] == '0') &&
                         ((lbenv && lbenv[0] == '1') || g->npad * (int64_t)sizeof(int32_t) >= (96ll << 20));
  if (use_lbits) {
    const int64_t words = (g->npad + 31) / 32;
    if (!g->lbits) g->lbits = dalloc<uint32_t>(g, std::max<int64_t>(words, 1));
    CK(cudaMemsetAsync(g->lbits, 0, std::max<int64_t>(words, 1) * sizeof(uint32_t), s));
  }
  if (variant == GLP_VARIANT_SEEDED && n_seeds > 0) {
    if (n_seeds > g->seeds_cap) {
      g->d_seeds = dalloc<int32_t>(g, n_seeds);
      g->seeds_cap = n_seeds;
    }
    CK(cudaMemcpyAsync(g->d_seeds, seeds, n_seeds * sizeof(int32_t), cudaMemcpyHostToDevice, s));
    k_init_seeds<<<ga, 256, 0, s>>>(g->d_seeds, n_seeds, g->pos, g->L[0], g->L[1], g->is_seed, g->so, g->vb,
                                     g->ve, use_lbits ? g->lbits : nullptr);
    g->init_launches += 1;
    CK(cudaGetLastError());
  }
  // LLP histogram with several ranks: sharded (each rank counts its rows,
  // all-reduce, all-gather of the owned (label, V) pairs) or replicated
  const bool llp_shard = variant == GLP_VARIANT_LLP && g->comm && g->use_vl && p.llp_hist != 1;
  if (variant == GLP_VARIANT_LLP) {
    // V[l] = #{w : L_0[w] = l} = 1 for every l (L_0 is a permutation): t = 1
    // reads no V (v_ones), and LV = (L_0[q], 1) needs no histogram
    if (g->use_vl) {
      if (!g->LV) g->LV = dalloc<int2>(g, std::max<int64_t>(g->npad, 1));  // npad: equal-slice all-gather
      k_lv_ones<<<ga, 256, 0, s>>>(g->L[0], g->n, g->LV);
      g->init_launches += 1;
    }
    CK(cudaGetLastError());
  }
  if (g->n_rows) {
    // predicted distinct labels per row for t = 1: deg (all labels distinct)
    // for CLASSIC/LLP, at most the number of seeds for SEEDED
    g->pb = 0;
    k_init_pred<<<ga, 256, 0, s>>>(g->rows, g->n_rows, g->pred[0], g->pred[1], g->pred[2],
                                   variant == GLP_VARIANT_SEEDED ? (unsigned)std::min<int64_t>(n_seeds, 1 << 30) : 0u);
    CK(cudaGetLastError());
    g->init_launches += 1;
  }
  // change lists of t-1 and t for the sparse exchange (CLASSIC / SEEDED, P > 1)
  const bool track_changes = g->comm && variant != GLP_VARIANT_LLP && !slp && p.sparse_exchange != 0;
  if (slp) {
    // memory M^0: slot 0 = (own label, 1); the speakers of t = 1 are L_0
    if (g->slp_cap < slp_k) {
      g->slp_l = dalloc<int32_t>(g, std::max<int64_t>(g->nl * slp_k, 1));
      g->slp_c = dalloc<int32_t>(g, std::max<int64_t>(g->nl * slp_k, 1));
      g->slp_cap = slp_k;
    }
    g->slp_k = slp_k;
    if (g->nl) k_slp_init<<<ga, 256, 0, s>>>(g->slp_l, g->slp_c, g->orig, g->nl, g->vb, slp_k);
    CK(cudaGetLastError());
    g->init_launches += 1;
  }
  g->slp_valid = false;
  if (track_changes) {
    if (!g->chg[0]) {
      g->chg[0] = dalloc<int2>(g, std::max<int64_t>(g->nl, 1));
      g->chg[1] = dalloc<int2>(g, std::max<int64_t>(g->nl, 1));
      g->chg_n = dalloc<unsigned>(g, 2);
    }
    CK(cudaMemsetAsync(g->chg_n, 0, 2 * sizeof(unsigned), s));  // nothing changed at t = 0 (seeds are in L0 and L1)
  }
  int rb = 0;  // R = L[rb], W = L[1-rb]
  int fb = 0;  // flags read this iteration
  bool dense = true;
  if (variant == GLP_VARIANT_SEEDED) {
    // frontier of t = 1 is N(S) (+ S): push from the seeds (stamped t = 0)
    if (use_frontier) {
      push(g, 0, g->flag[fb]);
      g->init_launches += g->max_deg >= kPushBig ? 2 : 1;
      CK(cudaGetLastError());
      g->flag_clean[fb] = false;
      if (g->comm) g->comm->merge_flags(g, g->flag[fb]);
      if (g->n_chunks) {
        k_chunk_flags<<<ga, 256, 0, s>>>(g->chunks, g->n_chunks, g->low_base, g->flag[fb], g->vb, g->cflag);
        g->init_launches += 1;
      }
      dense = false;
    }
  }

  g->iter_stats.clear();
  g->kstats.assign(kNumKernelNames, KStat());
  for (int k = 0; k < kNumKernelNames; ++k) g->kstats[k].name = kKernelNames[k];
  std::vector<Pending> pend;
  size_t used = 0;
  cudaEvent_t ev_run0 = pool_event(g, used);
  CK(cudaEventRecord(ev_run0, s));
  // drain profiled launches (stream must be synchronised); counters attach
  // algorithmic bytes to the MFL kernels (SURVEY §8(d) model)
  auto drain = [&](bool with_counters) {
    const int cur_t = g->cur_t;
    bool credited[kNumKernelNames] = {false};  // M and L launch twice (static + redo): credit once
    for (auto& pe : pend) {
      float kms = 0;
      CK(cudaEventElapsedTime(&kms, pe.a, pe.b));
      KStat& ks = g->kstats[pe.kid];
      ks.launches += 1;
      ks.ms += kms;
      if (with_counters && (pe.kid < 4 || pe.kid >= 7) && pe.t == cur_t && !credited[pe.kid]) {
        credited[pe.kid] = true;
        const Counters& c = g->h_cnt[counter_of(pe.kid)];
        ks.arcs += (double)c.arcs;
        // 4 B/arc (col_idx) + 8 B/active vertex (row offsets) + 4 B/changed label
        ks.bytes += 4.0 * (double)c.arcs + 8.0 * (double)c.verts + 4.0 * (double)c.changed;
      }
    }
    pend.clear();
  };

  int32_t iters = 0;
  int reason = GLP_STOP_MAX_ITERS;
  int64_t changed_last = 0, arcs_total = 0;
  int64_t labelled_bound = variant == GLP_VARIANT_SEEDED ? n_seeds : g->n;  // presence filter: vertices that may hold a label
  int64_t launches = 0;  // kernels of this run (excluding memsets/copies)

  // ---- device-driven loop (one rank, not profiled): the stop rule and the
  // frontier decision run on the device (k_decide), so the host never waits
  // for an iteration to finish before enqueueing the next; it looks two
  // iterations back through a mapped stop flag, and iterations enqueued past
  // the stop return at once (every kernel checks ctl).  Opt-in
  // (GLP_DEVICE_LOOP=1); the host-driven loop below is the default.
  if (!prof && !g->comm && g->dev_loop && max_iters > 0) {
    if (g->rec_cap < max_iters) {
      g->d_rec = dalloc<IterRec>(g, max_iters);
      g->rec_cap = max_iters;
    }
    if (!g->d_ctl) {
      g->d_ctl = dalloc<int>(g, 8);  // {stopped, dense, reason, iters}, dirty[2]
      CK(cudaHostAlloc((void**)&g->h_stop, sizeof(int), cudaHostAllocMapped));
      CK(cudaHostGetDevicePointer((void**)&g->d_hstop, (void*)g->h_stop, 0));
    }
    *g->h_stop = 0;
    const int ctl0[8] = {0, dense ? 1 : 0, 0, 0, use_frontier ? 1 : 0, 0, 0, 0};  // dirty[fb = 0]: seeded push
    g->h_ctl_init[0] = ctl0[0];
    for (int i = 0; i < 8; ++i) g->h_ctl_init[i] = ctl0[i];
    CK(cudaMemcpyAsync(g->d_ctl, g->h_ctl_init, 8 * sizeof(int), cudaMemcpyHostToDevice, s));
    CK(cudaMemsetAsync(g->d_cnt, 0, kNumCounters * sizeof(Counters), s));
    CK(cudaMemsetAsync(g->d_sched, 0, sizeof(Sched), s));
    int* dirty = g->d_ctl + 4;
    std::vector<cudaEvent_t> e0v, e1v;
    std::vector<int64_t> lv;  // launches per enqueued iteration
    int32_t enq = 0;
    for (int32_t t = 1; t <= max_iters; ++t) {
      if (t >= 3) {  // look-ahead of two iterations
        CK(cudaEventSynchronize(e1v[t - 3]));
        if (*(volatile int*)g->h_stop) break;
      }
      int64_t lt = 0;
      cudaEvent_t e0 = pool_event(g, used), e1 = pool_event(g, used);
      e0v.push_back(e0);
      e1v.push_back(e1);
      CK(cudaEventRecord(e0, s));
      g->cur_t = t;
      if (g->n_giant) {
        if (++g->gepoch >= (1ull << kGEpochBits)) {
          CK(cudaMemsetAsync(g->gtab, 0, g->gtab_slots * sizeof(unsigned long long), s));
          g->gepoch = 1;
        }
      }
      MflArgs a;
      memset(&a, 0, sizeof(a));
      a.col = g->col2; a.R = g->L[rb]; a.W = g->L[1 - rb]; a.so = g->so;
      a.V = g->V; a.is_seed = g->is_seed; a.flag = g->flag[fb];
      a.vb = g->vb; a.gamma = p.gamma; a.t = t; a.dense = 1;
      a.ctl = g->d_ctl;
      a.pred_cap = p.debug_pred_cap > 0 ? (unsigned)p.debug_pred_cap : 0u;
      a.v_ones = (variant == GLP_VARIANT_LLP && t == 1) ? 1 : 0;
      a.LV = (variant == GLP_VARIANT_LLP && g->use_vl) ? g->LV : nullptr;
      a.mono_kernel = (t == 1 && variant != GLP_VARIANT_SEEDED && g->use_mono) ? 1 : 0;
      a.cms = p.tail_cms ? 1 : 0;
      a.cms_ht = p.cms_ht_slots > 0 ? (unsigned)p.cms_ht_slots : 0u;
      a.cms_depth = p.cms_depth > 0 ? (unsigned)p.cms_depth : 4u;
      if (g->weighted) {
        lt += variant == GLP_VARIANT_SEEDED ? launch_wt<V_SEEDED>(g, a, false, pend, used)
                                            : launch_wt<V_CLASSIC>(g, a, false, pend, used);
      } else switch (variant) {
        case GLP_VARIANT_CLASSIC: lt += launch_mfl<V_CLASSIC>(g, a, false, pend, used); break;
        case GLP_VARIANT_SEEDED: lt += launch_mfl<V_SEEDED>(g, a, false, pend, used); break;
        case GLP_VARIANT_SLP: lt += launch_mfl<V_CLASSIC>(g, a, false, pend, used); break;
        default: lt += launch_mfl<V_LLP>(g, a, false, pend, used); break;
      }
      if (slp && g->nl) {
        k_slp_listen_speak<<<ga, 256, 0, s>>>(g->slp_l, g->slp_c, g->L[1 - rb], g->ideg, g->nl, g->vb, slp_k,
                                              p.slp_threshold * (double)(t + 1));
        lt += 1;
      }
      k_decide<<<1, 32, 0, s>>>(g->d_cnt, kNumCounters, (unsigned long long*)g->d_sched,
                                (int)(sizeof(Sched) / sizeof(unsigned long long)), g->d_ctl, g->d_rec, g->d_hstop,
                                t, (long long)g->nnz_global, p.dense_divisor, p.stop_on_2cycle, use_frontier ? 1 : 0,
                                slp ? 1 : 0);
      CK(cudaGetLastError());
      lt += 1;
      CK(cudaEventRecord(e1, s));
      const int nf = 1 - fb;
      if (use_frontier && t < max_iters) {
        // the marks of t+1 (skipped on the device when t+1 is dense or the
        // run stopped); the marks just read are cleared if a push wrote them
        CK(cudaMemsetAsync(dirty + nf, 0, sizeof(int), s));
        push(g, t, g->flag[nf], g->d_ctl, dirty + nf);
        lt += g->max_deg >= kPushBig ? 2 : 1;
        if (g->n_chunks) {
          k_chunk_flags<<<ga, 256, 0, s>>>(g->chunks, g->n_chunks, g->low_base, g->flag[nf], g->vb, g->cflag, g->d_ctl);
          lt += 1;
        }
      }
      if (use_frontier) {
        k_clear_flags<<<ga, 256, 0, s>>>(g->flag[fb], g->npad, dirty + fb);
        k_reset_dirty<<<1, 1, 0, s>>>(dirty + fb);
        lt += 2;
      }
      if (t < max_iters && variant == GLP_VARIANT_LLP) {
        CK(cudaMemsetAsync(g->V, 0, std::max<int64_t>(g->n, 1) * sizeof(int32_t), s));
        k_hist<<<ga, 256, 0, s>>>(g->L[1 - rb], g->n, g->V);
        if (g->use_vl) k_vl<<<ga, 256, 0, s>>>(g->L[1 - rb], g->V, g->n, g->LV);
        lt += g->use_vl ? 2 : 1;
      }
      CK(cudaGetLastError());
      lv.push_back(lt);
      g->pb = (g->pb + 1) % 3;
      rb = 1 - rb;
      fb = nf;
      enq = t;
    }
    CK(cudaStreamSynchronize(s));
    int ctl_h[8];
    CK(cudaMemcpy(ctl_h, g->d_ctl, sizeof(ctl_h), cudaMemcpyDeviceToHost));
    iters = ctl_h[3];
    reason = ctl_h[0] ? ctl_h[2] : GLP_STOP_MAX_ITERS;
    std::vector<IterRec> rec(std::max(iters, 1));
    if (iters > 0) CK(cudaMemcpy(rec.data(), g->d_rec, iters * sizeof(IterRec), cudaMemcpyDeviceToHost));
    for (int32_t t = 1; t <= iters; ++t) {
      const IterRec& r = rec[t - 1];
      glp_iter_stat st;
      memset(&st, 0, sizeof(st));
      st.changed = (int64_t)r.changed; st.d2 = (int64_t)r.d2;
      st.active_vertices = (int64_t)r.verts; st.active_arcs = (int64_t)r.arcs;
      st.dense = r.dense;
      st.cms_rows = (int64_t)r.cms0; st.cms_rescans = (int64_t)r.cms1; st.cms_fallbacks = (int64_t)r.cms2;
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, e0v[t - 1], e1v[t - 1]));
      st.ms = ms;
      g->iter_stats.push_back(st);
      changed_last = st.changed;
      arcs_total += st.active_arcs;
      launches += lv[t - 1];
    }
    (void)enq;
    // stale flags of a buffer a skipped iteration would have cleared
    g->flag_clean[0] = g->flag_clean[1] = false;
    cudaEvent_t ev_run1 = pool_event(g, used);
    CK(cudaEventRecord(ev_run1, s));
    CK(cudaStreamSynchronize(s));
    float run_ms = 0;
    CK(cudaEventElapsedTime(&run_ms, ev_run0, ev_run1));
    g->cur = iters & 1;
    g->has_run = true;
    g->slp_valid = slp;
    if (info) {
      info->iterations = iters;
      info->stop_reason = reason;
      info->changed_last = changed_last;
      info->arcs_processed = arcs_total;
      info->elapsed_ms = run_ms;
      info->kernel_launches = launches + g->init_launches;
    }
    return;
  }

  for (int32_t t = 1; t <= max_iters; ++t) {
    cudaEvent_t e0 = pool_event(g, used), e1 = pool_event(g, used);
    CK(cudaEventRecord(e0, s));
    CK(cudaMemsetAsync(g->d_cnt, 0, kNumCounters * sizeof(Counters), s));
    CK(cudaMemsetAsync(g->d_sched, 0, sizeof(Sched), s));
    g->cur_t = t;
    if (g->n_giant) {
      // giant-table epoch: slots of other epochs are free; clear on wrap
      if (++g->gepoch >= (1ull << kGEpochBits)) {
        CK(cudaMemsetAsync(g->gtab, 0, g->gtab_slots * sizeof(unsigned long long), s));
        g->gepoch = 1;
      }
    }
    MflArgs a;
    memset(&a, 0, sizeof(a));
    a.col = g->col2; a.R = g->L[rb]; a.W = g->L[1 - rb]; a.so = g->so;
    a.V = g->V; a.is_seed = g->is_seed; a.flag = g->flag[fb];
    a.vb = g->vb; a.gamma = p.gamma; a.t = t; a.dense = dense ? 1 : 0;
    a.pred_cap = p.debug_pred_cap > 0 ? (unsigned)p.debug_pred_cap : 0u;
    // L_0 = PickLabel's identity labelling (a permutation): its histogram V is
    // all ones (k_hist still writes it), so t = 1 needs no V gathers
    a.v_ones = (variant == GLP_VARIANT_LLP && t == 1) ? 1 : 0;
    a.LV = (variant == GLP_VARIANT_LLP && g->use_vl) ? g->LV : nullptr;
    a.lv_labels = llp_shard ? 1 : 0;  // non-owned labels live only in LV
    // t = 1: every row is a sorted-row candidate (unique labels); they go to
    // the table-free mono kernel (SEEDED never takes the sorted path)
    a.mono_kernel = (t == 1 && variant != GLP_VARIANT_SEEDED && g->use_mono) ? 1 : 0;
    a.cms = p.tail_cms ? 1 : 0;
    a.cms_ht = p.cms_ht_slots > 0 ? (unsigned)p.cms_ht_slots : 0u;
    a.cms_depth = p.cms_depth > 0 ? (unsigned)p.cms_depth : 4u;
    // the filter pays while at most half the vertices can hold a label
    // (bound: seeds + every change so far; it only grows, so once off the
    // bitmap is never read again and need not be maintained)
    if (use_lbits && 2.0 * (double)labelled_bound < (double)g->n) { a.lbits = g->lbits; a.lbits_w = g->lbits; }
    if (g->weighted) {
      launches += variant == GLP_VARIANT_SEEDED ? launch_wt<V_SEEDED>(g, a, prof, pend, used)
                                                : launch_wt<V_CLASSIC>(g, a, prof, pend, used);
    } else switch (variant) {
      case GLP_VARIANT_CLASSIC: launches += launch_mfl<V_CLASSIC>(g, a, prof, pend, used); break;
      case GLP_VARIANT_SEEDED: launches += launch_mfl<V_SEEDED>(g, a, prof, pend, used); break;
      case GLP_VARIANT_SLP: launches += launch_mfl<V_CLASSIC>(g, a, prof, pend, used); break;
      default: launches += launch_mfl<V_LLP>(g, a, prof, pend, used); break;
    }
    if (slp) {
      // listener update + threshold + the speakers of t+1, written to W
      // before the exchange replicates W
      if (g->nl)
        k_slp_listen_speak<<<ga, 256, 0, s>>>(g->slp_l, g->slp_c, g->L[1 - rb], g->ideg, g->nl, g->vb, slp_k,
                                              p.slp_threshold * (double)(t + 1));
      CK(cudaGetLastError());
      launches += 1;
    }
    int exch = 0;
    if (g->comm) {
      // sharded LLP replicates (label, V) pairs after the histogram instead;
      // CLASSIC / SEEDED may exchange only the changed vertices (§8(f)1)
      if (track_changes) {
        const int ct = t & 1;
        CK(cudaMemsetAsync(g->chg_n + ct, 0, sizeof(unsigned), s));
        if (g->nl) k_collect_changes<<<ga, 256, 0, s>>>(g->so, g->L[1 - rb], g->nl, g->vb, t, g->chg[ct], g->chg_n + ct);
        CK(cudaGetLastError());
        launches += 1;
      }
      const bool sparse = track_changes && (p.sparse_exchange == 1 ||
                                            (p.sparse_exchange < 0 && t >= 2 &&
                                             (double)changed_last * 4.0 * g->nranks < (double)g->n));
      if (sparse) {
        const int ct = t & 1;
        const int2* lists[2] = {g->chg[1 - ct], g->chg[ct]};
        const unsigned* counts[2] = {g->chg_n + (1 - ct), g->chg_n + ct};
        timed(g, prof, 6, pend, used, s, [&] { g->comm->exchange_changes(g, g->L[1 - rb], lists, counts); });
        exch = 2;
      } else if (!llp_shard) {
        timed(g, prof, 6, pend, used, s, [&] { g->comm->allgather(g, g->L[1 - rb], sizeof(int32_t)); });
        exch = 1;
      } else {
        exch = 3;
      }
      g->comm->allreduce_u64(g, (unsigned long long*)g->d_cnt, kNumCounters * sizeof(Counters) / sizeof(unsigned long long));
    }
    CK(cudaMemcpyAsync(g->h_cnt, g->d_cnt, kNumCounters * sizeof(Counters), cudaMemcpyDeviceToHost, s));
    CK(cudaEventRecord(e1, s));
    CK(cudaStreamSynchronize(s));
    Counters tot;
    memset(&tot, 0, sizeof(tot));
    for (int b = 0; b < kNumCounters; ++b) {
      tot.changed += g->h_cnt[b].changed; tot.d2 += g->h_cnt[b].d2; tot.chdeg += g->h_cnt[b].chdeg;
      tot.arcs += g->h_cnt[b].arcs; tot.verts += g->h_cnt[b].verts;
      tot.pad0 += g->h_cnt[b].pad0; tot.pad[0] += g->h_cnt[b].pad[0]; tot.pad[1] += g->h_cnt[b].pad[1];
    }
    glp_iter_stat st;
    memset(&st, 0, sizeof(st));
    st.changed = (int64_t)tot.changed;
    st.d2 = (int64_t)tot.d2;
    st.active_vertices = (int64_t)tot.verts;
    st.active_arcs = (int64_t)tot.arcs;
    st.dense = dense ? 1 : 0;
    st.exchange = exch;
    st.cms_rows = (int64_t)tot.pad0;
    st.cms_rescans = (int64_t)tot.pad[0];
    st.cms_fallbacks = (int64_t)tot.pad[1];
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    st.ms = ms;
    // every kernel launched so far has completed: drain the profile events
    // (this iteration's MFL kernels and the previous iteration's push/hist)
    drain(true);
    used = 1;  // ev_run0 stays; everything else is recycled
    iters = t;
    changed_last = st.changed;
    labelled_bound += st.changed;
    arcs_total += st.active_arcs;
    // stop rule (R8): fixed point, or L_t == L_{t-2} (d2 == 0) with changes
    bool stop = false;
    // (SLP runs max_iters iterations: its memories keep changing)
    if (slp) {
    } else if (st.changed == 0) { reason = GLP_STOP_FIXED_POINT; stop = true; }
    else if (p.stop_on_2cycle && t >= 2 && st.d2 == 0) { reason = GLP_STOP_TWO_CYCLE; stop = true; }
    // frontier of t+1: dense when the changed vertices touch > nnz/divisor arcs
    const int nf = 1 - fb;
    bool next_dense = true;
    // nothing of t+1 is prepared after the last iteration (stop or max_iters)
    const bool last = stop || t == max_iters;
    if (!last && use_frontier)
      next_dense = (double)tot.chdeg * (double)p.dense_divisor > (double)g->nnz_global;
    if (!last && !next_dense) {
      launches += g->max_deg >= kPushBig ? 2 : 1;
      timed(g, prof, 4, pend, used, s, [&] {
        push(g, t, g->flag[nf]);
        if (g->comm) g->comm->merge_flags(g, g->flag[nf]);
        if (g->n_chunks)
          k_chunk_flags<<<ga, 256, 0, s>>>(g->chunks, g->n_chunks, g->low_base, g->flag[nf], g->vb, g->cflag);
      });
      launches += g->n_chunks ? 1 : 0;
      g->flag_clean[nf] = false;
    }
    if (!dense && !g->flag_clean[fb]) {
      CK(cudaMemsetAsync(g->flag[fb], 0, std::max<int64_t>(g->npad, 1), s));
      g->flag_clean[fb] = true;
    }
    if (!last && variant == GLP_VARIANT_LLP) {
      launches += 1;
      if (llp_shard) {
        // this rank's rows only: V = sum over ranks of the owned counts, then
        // LV of the owned rows, all-gathered (replaces the label all-gather)
        timed(g, prof, 5, pend, used, s, [&] {
          CK(cudaMemsetAsync(g->Vloc, 0, std::max<int64_t>(g->n, 1) * sizeof(int32_t), s));
          if (g->nl) k_hist<<<ga, 256, 0, s>>>(g->L[1 - rb] + g->vb, g->nl, g->Vloc);
          CK(cudaGetLastError());
          g->comm->allreduce_i32(g, g->Vloc, g->V, (size_t)g->n);
          if (g->nl) k_vl<<<ga, 256, 0, s>>>(g->L[1 - rb] + g->vb, g->V, g->nl, g->LV + g->vb);
        });
        timed(g, prof, 6, pend, used, s, [&] { g->comm->allgather(g, g->LV, sizeof(int2)); });
        launches += 1;
        g->kstats[5].arcs += (double)g->nl;  // labels histogrammed by this rank
      } else {
        timed(g, prof, 5, pend, used, s, [&] {
          CK(cudaMemsetAsync(g->V, 0, std::max<int64_t>(g->n, 1) * sizeof(int32_t), s));
          k_hist<<<ga, 256, 0, s>>>(g->L[1 - rb], g->n, g->V);
          if (g->use_vl) k_vl<<<ga, 256, 0, s>>>(g->L[1 - rb], g->V, g->n, g->LV);
        });
        launches += g->use_vl ? 1 : 0;
        g->kstats[5].arcs += (double)g->n;
      }
    }
    g->iter_stats.push_back(st);
    g->pb = (g->pb + 1) % 3;
    rb = 1 - rb;
    fb = nf;
    dense = next_dense;
    if (stop) break;
  }
  // sharded LLP exchanged (label, V) pairs only: replicate the final labels
  if (llp_shard && iters > 0) g->comm->allgather(g, g->L[rb], sizeof(int32_t));
  if (!pend.empty()) {
    CK(cudaStreamSynchronize(s));
    drain(false);
  }
  cudaEvent_t ev_run1 = pool_event(g, used);
  CK(cudaEventRecord(ev_run1, s));
  CK(cudaStreamSynchronize(s));
  float run_ms = 0;
  CK(cudaEventElapsedTime(&run_ms, ev_run0, ev_run1));
  g->cur = rb;
  g->has_run = true;
  g->slp_valid = slp;
  if (info) {
    info->iterations = iters;
    info->stop_reason = reason;
    info->changed_last = changed_last;
    info->arcs_processed = arcs_total;
    info->elapsed_ms = run_ms;
    info->kernel_launches = launches + g->init_launches;
  }
}

}  // namespace

// ================================================================ C ABI
extern "C" {

glp_status glp_graph_create(const glp_csr* csr, const glp_dist* dist, const glp_params* params, glp_graph** out) {
  return guard([&] { create_impl(csr, dist, params, out); });
}

glp_status glp_run(glp_graph* g, glp_variant variant, int32_t max_iters, const int32_t* seeds, int64_t n_seeds,
                   const glp_params* params, glp_run_info* info) {
  const glp_status st = guard([&] { run_impl(g, variant, max_iters, seeds, n_seeds, params, info); });
  // a failed rank releases the others of its local group (they would wait
  // at the next exchange forever)
  if (st != GLP_OK && g && g->comm) g->comm->abort(g_last_error);
  return st;
}

glp_status glp_local_group_create(int32_t nranks, glp_local_group** out) {
  return guard([&] {
    if (!out) fail(GLP_ERR_INVALID_ARGUMENT, "out is NULL");
    *out = nullptr;
    if (nranks < 1 || nranks > kMaxLocalRanks) fail(GLP_ERR_INVALID_ARGUMENT, "nranks must be in [1, 16]");
    *out = new glp_local_group(nranks);
  });
}

glp_status glp_local_group_destroy(glp_local_group* grp) {
  return guard([&] { delete grp; });
}

glp_status glp_labels_get(const glp_graph* g, int32_t* out, int64_t out_len, int32_t out_on_device) {
  return guard([&] {
    if (!g) fail(GLP_ERR_INVALID_ARGUMENT, "graph is NULL");
    if (!g->has_run) fail(GLP_ERR_STATE, "glp_labels_get before glp_run");
    if (out_len < g->n) fail(GLP_ERR_INVALID_ARGUMENT, "out_len < n_global");
    if (g->n == 0) return;
    if (!out) fail(GLP_ERR_INVALID_ARGUMENT, "out is NULL");
    CK(cudaSetDevice(g->device));
    // back to original vertex order; the dead buffer L_{t-1} is the staging
    // area of a host copy
    int32_t* dst = out_on_device ? out : g->L[1 - g->cur];
    k_unpermute<<<g->grid_aux, 256, 0, g->stream>>>(g->L[g->cur], g->pos, g->n, dst);
    CK(cudaGetLastError());
    if (!out_on_device)
      CK(cudaMemcpyAsync(out, dst, g->n * sizeof(int32_t), cudaMemcpyDeviceToHost, g->stream));
    CK(cudaStreamSynchronize(g->stream));
  });
}

glp_status glp_slp_memory_get(const glp_graph* g, int32_t* labels_out, int32_t* counts_out, int64_t out_len,
                              int32_t out_on_device) {
  return guard([&] {
    if (!g) fail(GLP_ERR_INVALID_ARGUMENT, "graph is NULL");
    if (!g->slp_valid) fail(GLP_ERR_STATE, "the last run was not an SLP run");
    const int64_t need = g->nl * g->slp_k;
    if (out_len < need) fail(GLP_ERR_INVALID_ARGUMENT, "out_len < (v_end - v_begin) * slp_max_labels");
    if (need == 0) return;
    if (!labels_out || !counts_out) fail(GLP_ERR_INVALID_ARGUMENT, "output is NULL");
    CK(cudaSetDevice(g->device));
    int32_t* dl = labels_out;
    int32_t* dc = counts_out;
    std::vector<void*> tmp;
    if (!out_on_device) {
      void *a = nullptr, *b = nullptr;
      CK(cudaMalloc(&a, need * sizeof(int32_t)));
      tmp.push_back(a);
      CK(cudaMalloc(&b, need * sizeof(int32_t)));
      tmp.push_back(b);
      dl = (int32_t*)a;
      dc = (int32_t*)b;
    }
    k_slp_unpermute<<<g->grid_aux, 256, 0, g->stream>>>(g->slp_l, g->slp_c, g->pos, g->vb, g->ve, g->slp_k, dl, dc);
    CK(cudaGetLastError());
    if (!out_on_device) {
      CK(cudaMemcpyAsync(labels_out, dl, need * sizeof(int32_t), cudaMemcpyDeviceToHost, g->stream));
      CK(cudaMemcpyAsync(counts_out, dc, need * sizeof(int32_t), cudaMemcpyDeviceToHost, g->stream));
    }
    CK(cudaStreamSynchronize(g->stream));
    for (void* p : tmp) cudaFree(p);
  });
}

glp_status glp_iter_stats(const glp_graph* g, glp_iter_stat* out, int32_t max_entries, int32_t* n_out) {
  return guard([&] {
    if (!g || !n_out || max_entries < 0 || (max_entries > 0 && !out)) fail(GLP_ERR_INVALID_ARGUMENT, "bad arguments");
    const int32_t k = std::min<int32_t>(max_entries, (int32_t)g->iter_stats.size());
    for (int32_t i = 0; i < k; ++i) out[i] = g->iter_stats[i];
    *n_out = (int32_t)g->iter_stats.size();
  });
}

glp_status glp_kernel_stats(const glp_graph* g, glp_kernel_stat* out, int32_t max_entries, int32_t* n_out) {
  return guard([&] {
    if (!g || !n_out || max_entries < 0 || (max_entries > 0 && !out)) fail(GLP_ERR_INVALID_ARGUMENT, "bad arguments");
    const int32_t k = std::min<int32_t>(max_entries, (int32_t)g->kstats.size());
    for (int32_t i = 0; i < k; ++i) {
      memset(&out[i], 0, sizeof(glp_kernel_stat));
      strncpy(out[i].name, g->kstats[i].name.c_str(), sizeof(out[i].name) - 1);
      out[i].launches = g->kstats[i].launches;
      out[i].ms = g->kstats[i].ms;
      out[i].bytes = g->kstats[i].bytes;
      out[i].arcs = g->kstats[i].arcs;
    }
    *n_out = (int32_t)g->kstats.size();
  });
}

glp_status glp_graph_info(const glp_graph* g, int64_t* out, int32_t max_entries) {
  return guard([&] {
    if (!g || (max_entries > 0 && !out)) fail(GLP_ERR_INVALID_ARGUMENT, "bad arguments");
    std::vector<int64_t> v = {g->n, g->nnz};
    for (int b = 0; b < NBINS; ++b) { v.push_back(g->bin_verts[b]); v.push_back(g->bin_arcs[b]); }
    v.push_back(g->max_deg);
    v.push_back(g->n_chunks);
    for (int i = 0; i < max_entries && i < (int)v.size(); ++i) out[i] = v[i];
  });
}

glp_status glp_partition(const int64_t* row_offsets_host, int64_t n, int32_t nranks, int32_t edge_balanced,
                         int64_t* bounds_out) {
  return guard([&] {
    if (n < 0 || nranks < 1 || !bounds_out) fail(GLP_ERR_INVALID_ARGUMENT, "bad arguments");
    if (edge_balanced && !row_offsets_host) fail(GLP_ERR_INVALID_ARGUMENT, "row_offsets_host required");
    bounds_out[0] = 0;
    if (!edge_balanced) {
      const int64_t per = (n + nranks - 1) / nranks;
      for (int r = 1; r <= nranks; ++r) bounds_out[r] = std::min<int64_t>(n, per * r);
    } else {
      const int64_t m = row_offsets_host[n];
      for (int r = 1; r < nranks; ++r) {
        const int64_t target = (int64_t)((double)m * r / nranks);
        const int64_t* it = std::lower_bound(row_offsets_host, row_offsets_host + n + 1, target);
        bounds_out[r] = std::max<int64_t>(bounds_out[r - 1], std::min<int64_t>(n, it - row_offsets_host));
      }
      bounds_out[nranks] = n;
    }
  });
}

glp_status glp_nccl_unique_id(uint8_t out[128]) {
  return guard([&] {
    if (!out) fail(GLP_ERR_INVALID_ARGUMENT, "out is NULL");
    nccl_unique_id(out);
  });
}

glp_status glp_graph_destroy(glp_graph* g) {
  return guard([&] { free_graph(g); });
}

glp_status glp_struct_sizes(int64_t* out, int32_t max_entries) {
  return guard([&] {
    if (!out && max_entries > 0) fail(GLP_ERR_INVALID_ARGUMENT, "out is NULL");
    const int64_t v[6] = {(int64_t)sizeof(glp_csr),      (int64_t)sizeof(glp_dist),
                          (int64_t)sizeof(glp_params),   (int64_t)sizeof(glp_run_info),
                          (int64_t)sizeof(glp_iter_stat), (int64_t)sizeof(glp_kernel_stat)};
    for (int i = 0; i < max_entries && i < 6; ++i) out[i] = v[i];
  });
}

const char* glp_last_error(void) { return g_last_error.c_str(); }
const char* glp_version(void) { return "glp-b200 0.1 (sm_100a)"; }

}  // extern "C"
