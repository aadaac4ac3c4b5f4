// mfl_kernels.cuh -- most-frequent-label (MFL) kernels for sm_100a.
//
// One synchronous LP iteration [P:68 §2.1]: every processed vertex v gathers
// the labels of N(v) from R = L_{t-1} (LoadNeighbor [P:110]), counts them,
// scores them (LabelScore [P:111]; LLP: k - gamma*(V-k) [P:119]) and writes
// the best label (score desc, label asc: R4) to W = L_t (UpdateVertex [P:112],
// Lnext [P:143]).
//
// Kernels by degree bin:
//   mfl_low   deg <= 32: one warp serves several vertices whose arcs are
//             contiguous ("one-warp-multi-vertices" [P:227-234 §4.2]):
//             activemask/vmask/lmask + popc, then a segmented redux arg-max.
//   mfl_mid   deg <= 256: one warp per vertex, per-warp shared-memory table.
//   mfl_high  deg <= 4096: one block per vertex, shared-memory table
//             ("SharedMemBigNodes" HT [P:132-182 §4.1]).
//   mfl_huge  deg > 4096: as high with a 192 KB table; when a label finds no
//             slot within kHugeProbe probes the vertex is recounted exactly in a
//             per-block global-memory table (GlobalInsert/GHT [P:166, P:182]).
//
// Exactness of the running arg-max (the paper's ht_score taken from the
// atomicAdd return value [P:150-156]): a label's count only grows, and its
// score is non-decreasing in its count (gamma >= 0), so the maximum over every
// (post-increment score, label) observation equals the maximum over final
// scores, and the labels attaining it at an observation are exactly those whose
// final score is maximal.  No table scan is needed.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "glp_internal.cuh"

namespace glp {

constexpr unsigned kFull = 0xffffffffu;
constexpr unsigned long long kEmpty = ~0ull;  // table slot: (label << 32) | count
constexpr unsigned kNoLabel = 0xffffffffu;

enum Variant { V_CLASSIC = 0, V_SEEDED = 1, V_LLP = 2 };

__device__ __forceinline__ int ld_stream(const int32_t* p) {
  int r;
  asm volatile("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ int ld_label(const int32_t* p) { return __ldg(p); }

// LLP score val = k - gamma * (v - k) [P:119], double, no contraction (R11).
__device__ __forceinline__ double llp_score(unsigned k, int v, double gamma) {
  double kd = (double)k;
  double diff = __dsub_rn((double)v, kd);
  double prod = __dmul_rn(gamma, diff);
  return __dsub_rn(kd, prod);
}

// Order-preserving map double -> u64 (finite and infinite values).
__device__ __forceinline__ unsigned long long dkey(double x) {
  unsigned long long b = (unsigned long long)__double_as_longlong(x);
  return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}

// Score key of label `lab` with count `k`: larger is better.
template <int VAR>
__device__ __forceinline__ unsigned long long score_key(unsigned k, unsigned lab, const MflArgs& a) {
  if (VAR == V_LLP) return dkey(llp_score(k, ld_label(a.V + lab), a.gamma));
  return (unsigned long long)k;
}

struct Best {
  unsigned long long key;  // 0 = none
  unsigned lab;
};
__device__ __forceinline__ bool better(unsigned long long k1, unsigned l1, unsigned long long k2, unsigned l2) {
  return k1 > k2 || (k1 == k2 && l1 < l2);
}
__device__ __forceinline__ void best_update(Best& b, unsigned long long k, unsigned l) {
  if (better(k, l, b.key, b.lab)) { b.key = k; b.lab = l; }
}
__device__ __forceinline__ Best warp_best(Best b) {
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) {
    unsigned long long k = __shfl_xor_sync(kFull, b.key, s);
    unsigned l = __shfl_xor_sync(kFull, b.lab, s);
    best_update(b, k, l);
  }
  return b;
}

__device__ __forceinline__ unsigned slot_hash(unsigned lab, unsigned tsz) {
  return __umulhi(lab * 0x9E3779B1u, tsz);
}

// Insert `c` occurrences of `lab` into an open-addressing table of `tsz` slots
// (shared or global memory).  Returns the post-increment count, or 0 when no
// slot was found within `max_probe` probes (overflow).
__device__ __forceinline__ unsigned ht_add(unsigned long long* tab, unsigned tsz, unsigned lab,
                                           unsigned c, unsigned max_probe) {
  unsigned h = slot_hash(lab, tsz);
  for (unsigned p = 0; p < max_probe; ++p) {
    unsigned long long e = *((volatile unsigned long long*)(tab + h));
    if (e == kEmpty) {
      unsigned long long prev = atomicCAS(tab + h, kEmpty, ((unsigned long long)lab << 32) | c);
      if (prev == kEmpty) return c;
      e = prev;
    }
    if ((unsigned)(e >> 32) == lab) {
      unsigned long long old = atomicAdd(tab + h, (unsigned long long)c);
      return (unsigned)old + c;
    }
    if (++h == tsz) h = 0;
  }
  return 0;
}

// Per-thread iteration statistics, block-reduced once at kernel exit.
struct Tally {
  unsigned long long changed = 0, d2 = 0, chdeg = 0, arcs = 0, verts = 0;
};

__device__ __forceinline__ void tally_flush(Tally t, Counters* cnt) {
  __shared__ unsigned long long red[5][32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) {
    t.changed += __shfl_xor_sync(kFull, t.changed, s);
    t.d2 += __shfl_xor_sync(kFull, t.d2, s);
    t.chdeg += __shfl_xor_sync(kFull, t.chdeg, s);
    t.arcs += __shfl_xor_sync(kFull, t.arcs, s);
    t.verts += __shfl_xor_sync(kFull, t.verts, s);
  }
  if (lane == 0) {
    red[0][wid] = t.changed; red[1][wid] = t.d2; red[2][wid] = t.chdeg;
    red[3][wid] = t.arcs; red[4][wid] = t.verts;
  }
  __syncthreads();
  if (wid == 0) {
#pragma unroll
    for (int i = 0; i < 5; ++i) {
      unsigned long long x = lane < nw ? red[i][lane] : 0ull;
#pragma unroll
      for (int s = 16; s > 0; s >>= 1) x += __shfl_xor_sync(kFull, x, s);
      if (lane == 0 && x) atomicAdd(&((unsigned long long*)cnt)[i], x);
    }
  }
}

// UpdateVertex [P:101, P:112] for local vertex v with MFL result.
//   r   = L_{t-1}[v];  have = some neighbour voted;  best = winning label.
// Writes W[v] unconditionally (the frontier invariant of DESIGN.md §Frontier),
// and records (t, r) in so[v] when the label changed.
template <int VAR>
__device__ __forceinline__ void update_vertex(const MflArgs& a, int v, int deg, bool have, unsigned best,
                                              Tally& ty) {
  const int64_t gv = a.vb + v;
  const int r = ld_label(a.R + gv);
  int nw = have ? (int)best : r;
  if (VAR == V_SEEDED && a.is_seed[v]) nw = r;  // clamped seed (R12)
  const int2 so = a.so[v];
  const int l2 = (so.x == a.t - 1) ? so.y : r;  // L_{t-2}[v]
  a.W[gv] = nw;
  ty.verts += 1;
  ty.d2 += (nw != l2);
  if (nw != r) {
    ty.changed += 1;
    ty.chdeg += (unsigned long long)deg;
    a.so[v] = make_int2(a.t, r);
  }
}

// ---------------------------------------------------------------------------
// mfl_low: one warp, up to 32 arcs of several consecutive low-degree vertices
// (a static "chunk" of the low list with sum of degrees <= 32).
// Fig. 3 / [P:229-232]: activemask = ballot(valid label); vmask = lanes of the
// same vertex (from the chunk's segment starts); lmask = match_any(label) &
// vmask; frequency = popc(lmask).  Arg-max: redux max(count), then redux
// min(label) over the lanes of the vertex (R4).
template <int VAR>
__global__ void __launch_bounds__(kLowBlock) mfl_low(MflArgs a) {
  const int lane = threadIdx.x & 31;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  Tally ty;
  for (int c = gw; c < a.n_chunks; c += nwarps) {
    const int k0 = a.chunk[c];
    const int nv = a.chunk[c + 1] - k0;
    int v = 0, d = 0;
    int64_t o = 0;
    if (lane < nv) {
      v = a.list[k0 + lane];
      o = a.off[v];
      d = (int)(a.off[v + 1] - o);
    }
    if (!a.dense) {
      const bool act = lane < nv && a.flag[a.vb + v];
      if (__ballot_sync(kFull, act) == 0) continue;  // whole chunk inactive
    }
    // exclusive prefix of degrees -> segment starts
    int incl = d;
#pragma unroll
    for (int s = 1; s < 32; s <<= 1) {
      int x = __shfl_up_sync(kFull, incl, s);
      if (lane >= s) incl += x;
    }
    const int start = incl - d;
    const int total = __shfl_sync(kFull, incl, 31);
    const unsigned segstarts = __reduce_or_sync(kFull, lane < nv ? (1u << start) : 0u);
    const bool valid = lane < total;
    const int seg = max(__popc(segstarts & (kFull >> (31 - lane))) - 1, 0);
    const int64_t vo = __shfl_sync(kFull, o, seg);
    const int vstart = __shfl_sync(kFull, start, seg);
    const int vd = __shfl_sync(kFull, d, seg);
    int lab = -1;
    if (valid) {
      const int u = ld_stream(a.col + vo + (lane - vstart));
      lab = ld_label(a.R + u);
    }
    const bool vote = valid && (VAR != V_SEEDED || lab >= 0);
    // vmask: lanes of this lane's vertex [P:230]; idle lanes form singleton groups
    const unsigned vmask = valid ? ((vd == 32 ? kFull : ((1u << vd) - 1u)) << vstart) : (1u << lane);
    const unsigned activemask = __ballot_sync(kFull, vote);  // [P:229]
    const unsigned key = vote ? (unsigned)lab : kNoLabel;
    const unsigned lmask = __match_any_sync(kFull, key) & vmask & activemask;  // [P:231]
    const unsigned k = __popc(lmask);                                           // [P:232]
    unsigned bestlab;
    if (VAR == V_LLP) {
      const unsigned long long sk = vote ? score_key<VAR>(k, (unsigned)lab, a) : 0ull;
      const unsigned hi = (unsigned)(sk >> 32), lo = (unsigned)sk;
      const unsigned mhi = __reduce_max_sync(vmask, hi);
      const unsigned mlo = __reduce_max_sync(vmask, (vote && hi == mhi) ? lo : 0u);
      bestlab = __reduce_min_sync(vmask, (vote && hi == mhi && lo == mlo) ? (unsigned)lab : kNoLabel);
    } else {
      const unsigned cnt = vote ? k : 0u;
      const unsigned maxc = __reduce_max_sync(vmask, cnt);
      bestlab = __reduce_min_sync(vmask, (vote && cnt == maxc) ? (unsigned)lab : kNoLabel);
    }
    if (lane == 0) ty.arcs += (unsigned long long)total;
    // the first lane of each segment updates its vertex
    const int vv = __shfl_sync(kFull, v, seg);
    if (valid && lane == vstart) {
      const bool have = (activemask & vmask) != 0u;
      update_vertex<VAR>(a, vv, vd, have, bestlab, ty);
    }
  }
  tally_flush(ty, a.cnt);
}

// ---------------------------------------------------------------------------
// mfl_mid: one warp per vertex (33..256 arcs), per-warp shared table of
// 2*deg slots.  Labels of a 32-arc round are warp-aggregated with
// match_any before the table insert (hot keys after communities form [P:130]).
constexpr int kMidUnroll = 8;  // 8 x 32 = 256 arcs in flight per warp

template <int VAR>
__global__ void __launch_bounds__(kMidBlock) mfl_mid(MflArgs a) {
  __shared__ unsigned long long tabs[kMidBlock / 32][kMidSlots];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  unsigned long long* tab = tabs[wid];
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  Tally ty;
  for (int i = gw; i < a.list_len; i += nwarps) {
    const int v = a.list[i];
    if (!a.dense && !a.flag[a.vb + v]) continue;
    const int64_t o = a.off[v];
    const int d = (int)(a.off[v + 1] - o);
    const unsigned tsz = 2u * (unsigned)d;
    for (unsigned j = lane; j < tsz; j += 32) tab[j] = kEmpty;
    __syncwarp();
    Best b{0ull, kNoLabel};
    for (int base = 0; base < d; base += 32 * kMidUnroll) {
      int u[kMidUnroll], lab[kMidUnroll];
#pragma unroll
      for (int j = 0; j < kMidUnroll; ++j) {
        const int idx = base + j * 32 + lane;
        u[j] = idx < d ? ld_stream(a.col + o + idx) : -1;
      }
#pragma unroll
      for (int j = 0; j < kMidUnroll; ++j) lab[j] = u[j] >= 0 ? ld_label(a.R + u[j]) : -1;
#pragma unroll
      for (int j = 0; j < kMidUnroll; ++j) {
        if (base + j * 32 >= d) break;  // warp-uniform
        const bool vote = u[j] >= 0 && lab[j] >= 0;
        const unsigned key = vote ? (unsigned)lab[j] : kNoLabel;
        const unsigned m = __match_any_sync(kFull, key);
        if (vote && lane == __ffs(m) - 1) {
          const unsigned cnt = ht_add(tab, tsz, (unsigned)lab[j], __popc(m), tsz);
          best_update(b, score_key<VAR>(cnt, (unsigned)lab[j], a), (unsigned)lab[j]);
        }
      }
    }
    b = warp_best(b);
    if (lane == 0) {
      ty.arcs += (unsigned long long)d;
      update_vertex<VAR>(a, v, d, b.key != 0ull, b.lab, ty);
    }
    __syncwarp();
  }
  tally_flush(ty, a.cnt);
}

// ---------------------------------------------------------------------------
// Block-per-vertex counting shared by mfl_high and mfl_huge.
template <int VAR, int BLOCK, int UNROLL>
__device__ __forceinline__ bool block_count(const MflArgs& a, int64_t o, int d, unsigned long long* tab,
                                            unsigned tsz, unsigned max_probe, volatile int* overflow,
                                            Best& b) {
  const int lane = threadIdx.x & 31;
  for (int base = 0; base < d; base += BLOCK * UNROLL) {
    int u[UNROLL], lab[UNROLL];
#pragma unroll
    for (int j = 0; j < UNROLL; ++j) {
      const int idx = base + j * BLOCK + (int)threadIdx.x;
      u[j] = idx < d ? ld_stream(a.col + o + idx) : -1;
    }
#pragma unroll
    for (int j = 0; j < UNROLL; ++j) lab[j] = u[j] >= 0 ? ld_label(a.R + u[j]) : -1;
#pragma unroll
    for (int j = 0; j < UNROLL; ++j) {
      const bool vote = u[j] >= 0 && lab[j] >= 0;
      const unsigned key = vote ? (unsigned)lab[j] : kNoLabel;
      const unsigned m = __match_any_sync(kFull, key);
      if (vote && lane == __ffs(m) - 1) {
        const unsigned cnt = ht_add(tab, tsz, (unsigned)lab[j], __popc(m), max_probe);
        if (cnt == 0) {
          *overflow = 1;
        } else {
          best_update(b, score_key<VAR>(cnt, (unsigned)lab[j], a), (unsigned)lab[j]);
        }
      }
    }
    if (overflow != nullptr && __any_sync(kFull, *overflow != 0)) return false;  // warp-uniform exit
  }
  return true;
}

template <int BLOCK>
__device__ __forceinline__ Best block_best(Best b) {
  __shared__ unsigned long long rk[BLOCK / 32];
  __shared__ unsigned rl[BLOCK / 32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  b = warp_best(b);
  if (lane == 0) { rk[wid] = b.key; rl[wid] = b.lab; }
  __syncthreads();
  if (wid == 0) {
    Best x{0ull, kNoLabel};
    if (lane < BLOCK / 32) { x.key = rk[lane]; x.lab = rl[lane]; }
    x = warp_best(x);
    b = x;
  }
  return b;  // valid in thread 0
}

constexpr int kHighUnroll = 4;

template <int VAR>
__global__ void __launch_bounds__(kHighBlock) mfl_high(MflArgs a) {
  extern __shared__ unsigned long long tab[];  // kHighSlots
  Tally ty;
  for (int i = blockIdx.x; i < a.list_len; i += gridDim.x) {
    const int v = a.list[i];
    if (!a.dense && !a.flag[a.vb + v]) continue;  // block-uniform
    const int64_t o = a.off[v];
    const int d = (int)(a.off[v + 1] - o);
    const unsigned tsz = 2u * (unsigned)d;
    for (unsigned j = threadIdx.x; j < tsz; j += kHighBlock) tab[j] = kEmpty;
    __syncthreads();
    Best b{0ull, kNoLabel};
    block_count<VAR, kHighBlock, kHighUnroll>(a, o, d, tab, tsz, tsz, nullptr, b);
    __syncthreads();
    b = block_best<kHighBlock>(b);
    if (threadIdx.x == 0) {
      ty.arcs += (unsigned long long)d;
      update_vertex<VAR>(a, v, d, b.key != 0ull, b.lab, ty);
    }
    __syncthreads();
  }
  tally_flush(ty, a.cnt);
}

constexpr int kHugeUnroll = 4;

template <int VAR>
__global__ void __launch_bounds__(kHugeBlock) mfl_huge(MflArgs a) {
  extern __shared__ unsigned long long tab[];  // kHugeSlots
  __shared__ int s_i, s_over;
  unsigned long long* gtab = a.ght + (int64_t)blockIdx.x * a.ght_slots;
  Tally ty;
  for (;;) {
    if (threadIdx.x == 0) {
      s_i = (int)atomicAdd(&a.cnt->huge_next, 1ull);
      s_over = 0;
    }
    __syncthreads();
    const int i = s_i;
    if (i >= a.list_len) break;
    const int v = a.list[i];
    if (!a.dense && !a.flag[a.vb + v]) { __syncthreads(); continue; }
    const int64_t o = a.off[v];
    const int d = (int)(a.off[v + 1] - o);
    const unsigned tsz = min(2u * (unsigned)d, (unsigned)kHugeSlots);
    for (unsigned j = threadIdx.x; j < tsz; j += kHugeBlock) tab[j] = kEmpty;
    __syncthreads();
    Best b{0ull, kNoLabel};
    block_count<VAR, kHugeBlock, kHugeUnroll>(a, o, d, tab, tsz, kHugeProbe, &s_over, b);
    __syncthreads();
    if (s_over) {
      // GlobalInsert [P:166]: exact recount of the whole neighbourhood in a
      // per-block global table of 2*deg slots (labels never split between the
      // two tables, so the shared-memory observations are discarded).
      const unsigned gsz = 2u * (unsigned)d;
      for (unsigned j = threadIdx.x; j < gsz; j += kHugeBlock) gtab[j] = kEmpty;
      __syncthreads();
      b = Best{0ull, kNoLabel};
      block_count<VAR, kHugeBlock, kHugeUnroll>(a, o, d, gtab, gsz, gsz, nullptr, b);
      __syncthreads();
    }
    b = block_best<kHugeBlock>(b);
    if (threadIdx.x == 0) {
      ty.arcs += (unsigned long long)d;
      update_vertex<VAR>(a, v, d, b.key != 0ull, b.lab, ty);
    }
    __syncthreads();
  }
  tally_flush(ty, a.cnt);
}

}  // namespace glp
