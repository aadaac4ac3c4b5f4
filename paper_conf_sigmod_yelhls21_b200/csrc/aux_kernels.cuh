// aux_kernels.cuh -- setup / frontier / histogram kernels (non-MFL steps).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "glp_internal.cuh"

namespace glp {

// CSR validation [P:97]: off[0]==0, off non-decreasing, off[nl]==nnz, col in [0,n).
__global__ void k_validate_off(const int64_t* __restrict__ off, int64_t nl, int64_t nnz, int* bad) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= nl; v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = off[v];
    if (v == 0 && x != 0) atomicOr(bad, 1);
    if (v == nl && x != nnz) atomicOr(bad, 2);
    if (v < nl && off[v + 1] < x) atomicOr(bad, 4);
  }
}
__global__ void k_validate_col(const int32_t* __restrict__ col, int64_t nnz, int64_t n, int* bad) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t u = col[e];
    if (u < 0 || (int64_t)u >= n) atomicOr(bad, 8);
  }
}

// PickLabel [P:99, P:109]: L[v] = v (CLASSIC, LLP) or UNLABELED (SEEDED, R12).
// Arrays are indexed by internal id q (layout.cuh); the label value is the
// original id orig[q].
__global__ void k_init_labels(int32_t* __restrict__ L0, int32_t* __restrict__ L1, const int32_t* __restrict__ orig,
                              int64_t n, int seeded) {
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
    const int32_t x = seeded ? -1 : orig[q];
    L0[q] = x;
    L1[q] = x;
  }
}

// glp_labels_get: out[v] = L[pos[v]] (original order)
__global__ void k_unpermute(const int32_t* __restrict__ L, const int32_t* __restrict__ pos, int64_t n,
                            int32_t* __restrict__ out) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    out[v] = L[pos[v]];
}

// Seeds carry their own id; owned seeds are marked and recorded as "changed at
// t = 0" so that the first frontier is N(S) (exact: every other vertex has no
// labelled neighbour and keeps -1, R5).
__global__ void k_init_seeds(const int32_t* __restrict__ seeds, int64_t ns, const int32_t* __restrict__ pos,
                             int32_t* __restrict__ L0, int32_t* __restrict__ L1, uint8_t* __restrict__ is_seed,
                             int2* __restrict__ so, int64_t vb, int64_t ve, uint32_t* __restrict__ lbits) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < ns; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t s = seeds[i];
    const int32_t q = pos[s];
    L0[q] = s;
    L1[q] = s;
    if (lbits) atomicOr(lbits + (q >> 5), 1u << (q & 31));
    if (q >= vb && q < ve) {
      is_seed[q - vb] = 1;
      so[q - vb] = make_int2(0, s);
    }
  }
}

// Frontier push: for every owned vertex changed at iteration t (so.x == t),
// mark itself and its neighbours (global ids) active for t+1 (DESIGN.md
// §Frontier: marking the changed vertex itself keeps the unconditional-write
// invariant).  One warp scans 32 stamps, then walks each changed row; rows of
// at least kPushBig arcs are only listed, and k_push_big spreads each of them
// over the whole grid (a changed hub -- TaoBao's 10.9M-arc item -- would
// otherwise keep one warp busy for milliseconds).
constexpr int kPushBig = 8192;
// GLP_PUSH_CHECK: read a mark before writing it (most marks of a large push
// are already set: a read costs less than a partial-sector write)
#ifndef GLP_PUSH_CHECK
#define GLP_PUSH_CHECK 1
#endif
__device__ __forceinline__ void mark(uint8_t* flag, int32_t x) {
  if (!GLP_PUSH_CHECK || !flag[x]) flag[x] = 1;
}
// ctl (device-driven loop): {stopped, dense of t+1}; the push is skipped when
// the run stopped or t+1 is a full sweep, and marks its flags dirty.
__device__ __forceinline__ bool push_off(const int* ctl) { return ctl && (ctl[0] || ctl[1]); }
__global__ void k_push(const int64_t* __restrict__ ioff, const int32_t* __restrict__ ideg,
                       const int32_t* __restrict__ col2, const int2* __restrict__ so, int64_t nl, int64_t vb,
                       int32_t t, uint8_t* __restrict__ flag, int32_t* __restrict__ big, unsigned* __restrict__ n_big,
                       const int* __restrict__ ctl = nullptr, int* __restrict__ dirty = nullptr) {
  if (push_off(ctl)) return;
  if (dirty && blockIdx.x == 0 && threadIdx.x == 0) *dirty = 1;
  const int lane = threadIdx.x & 31;
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t base = gw * 32; base < nl; base += nw * 32) {
    const int64_t v = base + lane;
    const bool ch = v < nl && so[v].x == t;
    unsigned m = __ballot_sync(0xffffffffu, ch);
    if (ch) flag[vb + v] = 1;
    const bool isbig = ch && ideg[v] >= kPushBig;
    if (isbig) big[atomicAdd(n_big, 1u)] = (int32_t)v;
    m &= ~__ballot_sync(0xffffffffu, isbig);
    while (m) {
      const int j = __ffs(m) - 1;
      m &= m - 1;
      const int64_t u = base + j;
      const int64_t e0 = ioff[u], e1 = e0 + ideg[u];
      for (int64_t e = e0 + lane; e < e1; e += 32) mark(flag, col2[e]);  // global ids
    }
  }
}
// the listed long rows: every thread of the grid takes a stride of each row
__global__ void k_push_big(const int64_t* __restrict__ ioff, const int32_t* __restrict__ ideg,
                           const int32_t* __restrict__ col2, const int32_t* __restrict__ big,
                           const unsigned* __restrict__ n_big, uint8_t* __restrict__ flag,
                           const int* __restrict__ ctl = nullptr) {
  if (push_off(ctl)) return;
  const unsigned nb = *n_big;
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t nth = (int64_t)gridDim.x * blockDim.x;
  for (unsigned i = 0; i < nb; ++i) {
    const int32_t u = big[i];
    const int64_t e0 = ioff[u];
    const int32_t d = ideg[u];
    for (int64_t e = tid; e < d; e += nth) mark(flag, col2[e0 + e]);
  }
}

// Weighted LP: the largest weight total of the giant rows (one block per
// row): giant tables hold counts in kGCountBits bits.
__global__ void k_giant_wsum_max(const BinItem* __restrict__ rows, int32_t n_giant, const uint32_t* __restrict__ w2,
                                 unsigned long long* __restrict__ out) {
  __shared__ unsigned long long red[32];
  for (int i = blockIdx.x; i < n_giant; i += gridDim.x) {
    const BinItem it = rows[i];
    unsigned long long s = 0;
    for (int e = threadIdx.x; e < it.d; e += blockDim.x) s += w2[it.start + e];
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long t = 0;
      for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += red[w];
      atomicMax(out, t);
    }
    __syncthreads();
  }
}

// Sparse iterations: a low-degree chunk is active if any of its vertices is.
__global__ void k_chunk_flags(const LowChunk* __restrict__ chunks, int32_t n_chunks, int64_t low_base,
                              const uint8_t* __restrict__ flag, int64_t vb, uint8_t* __restrict__ cflag,
                              const int* __restrict__ ctl = nullptr) {
  if (push_off(ctl)) return;
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n_chunks; c += (int64_t)gridDim.x * blockDim.x) {
    const LowChunk ch = chunks[c];
    const int nv = __popc(ch.segmask);
    uint8_t act = 0;
    for (int j = 0; j < nv && !act; ++j) act = flag[vb + low_base + ch.vbase + j];
    cflag[c] = act ? 1 : 0;
  }
}

// Build the bin-major arc copy: row v of the caller's CSR (local original id)
// -> col2[ioff[pos[vb + v] - vb] ...], each arc renamed to its internal id.
// Arc order within a row is kept.
// Rows [v0, v1) only (the create pipelines the relayout with the arcs' host
// copy chunk by chunk); an out-of-range column (rejected after the relayout
// by the validation flag) is written as -1 instead of indexing pos with it.
// Rows longer than kRelayBig arcs are only listed (big / n_big) and copied
// by k_relayout_big with the whole grid: one warp per row left a
// 10.9M-arc TaoBao item copying for ~0.4 s.
constexpr int64_t kRelayBig = 32768;
__global__ void k_relayout(const int64_t* __restrict__ off, const int32_t* __restrict__ col,
                           const int64_t* __restrict__ ioff, const int32_t* __restrict__ pos, int64_t v0, int64_t v1,
                           int64_t vb, int64_t n, int32_t* __restrict__ col2, int32_t* __restrict__ big,
                           unsigned* __restrict__ n_big) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t v = v0 + gw; v < v1; v += nw) {
    const int64_t s = off[v], d = off[v + 1] - s;
    if (big != nullptr && d > kRelayBig) {
      if (lane == 0) big[atomicAdd(n_big, 1u)] = (int32_t)v;
      continue;
    }
    const int64_t o = ioff[pos[vb + v] - vb];
    for (int64_t j = lane; j < d; j += 32) {
      const int32_t u = col[s + j];
      col2[o + j] = (u >= 0 && (int64_t)u < n) ? pos[u] : -1;
    }
  }
}
// the listed long rows, one after the other, each strided over the grid
__global__ void k_relayout_big(const int64_t* __restrict__ off, const int32_t* __restrict__ col,
                               const int64_t* __restrict__ ioff, const int32_t* __restrict__ pos, int64_t vb,
                               int64_t n, int32_t* __restrict__ col2, const int32_t* __restrict__ big,
                               const unsigned* __restrict__ n_big) {
  const unsigned nb = *n_big;
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t nth = (int64_t)gridDim.x * blockDim.x;
  for (unsigned i = 0; i < nb; ++i) {
    const int64_t v = big[i];
    const int64_t s = off[v], d = off[v + 1] - s, o = ioff[pos[vb + v] - vb];
    for (int64_t j = tid; j < d; j += nth) {
      const int32_t u = col[s + j];
      col2[o + j] = (u >= 0 && (int64_t)u < n) ? pos[u] : -1;
    }
  }
}

// Weighted LP: the arc weights beside the relayouted arcs (same positions).
__global__ void k_relayout_w(const int64_t* __restrict__ off, const uint32_t* __restrict__ w,
                             const int64_t* __restrict__ ioff, const int32_t* __restrict__ pos, int64_t nl, int64_t vb,
                             uint32_t* __restrict__ w2) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t v = gw; v < nl; v += nw) {
    const int64_t s = off[v], d = off[v + 1] - s;
    if (d > kRelayBig) continue;  // listed by k_relayout: k_relayout_w_big
    const int64_t o = ioff[pos[vb + v] - vb];
    for (int64_t j = lane; j < d; j += 32) w2[o + j] = w[s + j];
  }
}
__global__ void k_relayout_w_big(const int64_t* __restrict__ off, const uint32_t* __restrict__ w,
                                 const int64_t* __restrict__ ioff, const int32_t* __restrict__ pos, int64_t vb,
                                 uint32_t* __restrict__ w2, const int32_t* __restrict__ big,
                                 const unsigned* __restrict__ n_big) {
  const unsigned nb = *n_big;
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t nth = (int64_t)gridDim.x * blockDim.x;
  for (unsigned i = 0; i < nb; ++i) {
    const int64_t v = big[i];
    const int64_t s = off[v], d = off[v + 1] - s, o = ioff[pos[vb + v] - vb];
    for (int64_t j = tid; j < d; j += nth) w2[o + j] = w[s + j];
  }
}
// weights in [1, 2^31) and every row's total < 2^31 (exact 32-bit sums)
__global__ void k_validate_w(const int64_t* __restrict__ off, const uint32_t* __restrict__ w, int64_t nl,
                             int* __restrict__ bad) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t v = gw; v < nl; v += nw) {
    unsigned long long sum = 0;
    bool zero = false;
    for (int64_t e = off[v] + lane; e < off[v + 1]; e += 32) {
      const uint32_t x = w[e];
      sum += x;
      zero |= x == 0u || x >= 0x80000000u;
    }
    for (int s = 16; s > 0; s >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, s);
    if (__any_sync(0xffffffffu, zero) || sum >= 0x80000000ull) {
      if (lane == 0) atomicOr(bad, 16);
    }
  }
}

// Predicted distinct labels of each row at t = 1 (performance hint only).
__global__ void k_init_pred(const BinItem* __restrict__ rows, int32_t n_rows, unsigned* __restrict__ pred0,
                            unsigned* __restrict__ pred1, unsigned* __restrict__ pred2, unsigned seed_cap) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n_rows; i += (int64_t)gridDim.x * blockDim.x) {
    const unsigned d = (unsigned)rows[i].d;
    const unsigned p = seed_cap ? max(1u, min(d, seed_cap)) : d;
    pred0[i] = p;
    pred1[i] = p;
    pred2[i] = p;
  }
}

// LLP: V[l] = #{w : L[w] = l} [P:119].
// LLP: LV[q] = (L[q], V[L[q]]): each vertex's label next to its histogram
// value, so that the MFL kernels read a neighbour's label and V with one
// 8-byte gather at the neighbour's index (one random V gather per vertex here
// instead of one per candidate label there).
__global__ void k_vl(const int32_t* __restrict__ L, const int32_t* __restrict__ V, int64_t n, int2* __restrict__ LV) {
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
    const int32_t l = L[q];
    LV[q] = make_int2(l, l >= 0 ? V[l] : 0);
  }
}

// device-driven loop: clear a mark buffer after the iteration that read it,
// if a push wrote it
__global__ void k_clear_flags(uint8_t* __restrict__ flag, int64_t n, int* __restrict__ dirty) {
  if (!*dirty) return;
  uint4* f4 = (uint4*)flag;
  const int64_t n16 = n / 16;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n16; i += (int64_t)gridDim.x * blockDim.x)
    f4[i] = make_uint4(0u, 0u, 0u, 0u);
  for (int64_t i = n16 * 16 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    flag[i] = 0;
}
__global__ void k_reset_dirty(int* dirty) { *dirty = 0; }

// One iteration's record of the device-driven loop (glp_iter_stat fields).
struct IterRec {
  unsigned long long changed, d2, chdeg, arcs, verts, cms0, cms1, cms2;
  int dense, pad;
};
// End of iteration t (device-driven loop; one thread): totals of the per-kernel
// counters -> rec[t-1]; the stop rule R8 (fixed point / two-cycle); the
// frontier decision for t+1 (dense when the changed vertices touch more than
// nnz / dense_div arcs); the counters and tickets are zeroed for t+1, and the
// stop flag is mirrored to mapped host memory for the host's look-ahead.
// ctl = {stopped, dense, reason, iters}.
__global__ void k_decide(Counters* __restrict__ cnt, int ncnt, unsigned long long* __restrict__ sched, int nsched,
                         int* __restrict__ ctl, IterRec* __restrict__ rec, volatile int* __restrict__ h_stop, int t,
                         long long nnz_global, int dense_div, int stop_2c, int use_frontier, int never_stop) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  if (ctl[0]) return;
  Counters tot;
  memset(&tot, 0, sizeof(tot));
  for (int b = 0; b < ncnt; ++b) {
    tot.changed += cnt[b].changed; tot.d2 += cnt[b].d2; tot.chdeg += cnt[b].chdeg;
    tot.arcs += cnt[b].arcs; tot.verts += cnt[b].verts;
    tot.pad0 += cnt[b].pad0; tot.pad[0] += cnt[b].pad[0]; tot.pad[1] += cnt[b].pad[1];
  }
  IterRec r;
  r.changed = tot.changed; r.d2 = tot.d2; r.chdeg = tot.chdeg; r.arcs = tot.arcs; r.verts = tot.verts;
  r.cms0 = tot.pad0; r.cms1 = tot.pad[0]; r.cms2 = tot.pad[1];
  r.dense = ctl[1]; r.pad = 0;
  rec[t - 1] = r;
  int reason = 0;
  if (!never_stop) {
    if (tot.changed == 0) reason = 1;
    else if (stop_2c && t >= 2 && tot.d2 == 0) reason = 2;
  }
  ctl[3] = t;
  if (reason) { ctl[0] = 1; ctl[2] = reason; }
  ctl[1] = (!use_frontier || (double)tot.chdeg * (double)dense_div > (double)nnz_global) ? 1 : 0;
  for (int b = 0; b < ncnt; ++b) memset(&cnt[b], 0, sizeof(Counters));
  for (int i = 0; i < nsched; ++i) sched[i] = 0ull;
  *h_stop = ctl[0];
  __threadfence_system();
}

// LLP at t = 0: L_0 is a permutation, so V[L_0[q]] = 1 for every q.
__global__ void k_lv_ones(const int32_t* __restrict__ L, int64_t n, int2* __restrict__ LV) {
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x)
    LV[q] = make_int2(L[q], 1);
}

__global__ void k_hist(const int32_t* __restrict__ L, int64_t n, int32_t* __restrict__ V) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const int32_t l = L[v];
    if (l >= 0) atomicAdd(V + l, 1);
  }
}

// ---- SLP (§8(f)3, speaker-listener LP [P:120]; readings R19).  Memory of
// owned vertex q (local internal id): K slots (label, count), label -1 = empty.
__device__ __forceinline__ int slp_argmax(const int32_t* l, const int32_t* c, int K) {
  int b = -1;
  for (int k = 0; k < K; ++k) {
    if (l[k] < 0) continue;
    if (b < 0 || c[k] > c[b] || (c[k] == c[b] && l[k] < l[b])) b = k;
  }
  return b;
}
__global__ void k_slp_init(int32_t* __restrict__ ml, int32_t* __restrict__ mc, const int32_t* __restrict__ orig,
                           int64_t nl, int64_t vb, int K) {
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nl; q += (int64_t)gridDim.x * blockDim.x)
    for (int k = 0; k < K; ++k) {
      ml[q * K + k] = k == 0 ? orig[vb + q] : -1;
      mc[q * K + k] = k == 0 ? 1 : 0;
    }
}
// listener: the MFL heard (W, written by the classic MFL kernels from the
// speakers) joins the candidates of every owned vertex with neighbours; then
// the threshold; then the speaker of t+1 (the most frequent candidate, min
// label on ties) is written to W for every owned vertex
__global__ void k_slp_listen_speak(int32_t* __restrict__ ml, int32_t* __restrict__ mc, int32_t* __restrict__ W,
                                   const int32_t* __restrict__ ideg, int64_t nl, int64_t vb, int K, double thr) {
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nl; q += (int64_t)gridDim.x * blockDim.x) {
    int32_t* l = ml + q * K;
    int32_t* c = mc + q * K;
    if (ideg[q] > 0) {
      const int32_t m = W[vb + q];
      int hit = -1, empty = -1, low = -1;
      for (int k = 0; k < K; ++k) {
        if (l[k] == m) hit = k;
        if (l[k] < 0 && empty < 0) empty = k;
        if (l[k] >= 0 && (low < 0 || c[k] < c[low] || (c[k] == c[low] && l[k] > l[low]))) low = k;
      }
      if (hit >= 0) c[hit] += 1;
      else if (empty >= 0) { l[empty] = m; c[empty] = 1; }
      else { l[low] = m; c[low] = 1; }
    }
    const int keep = slp_argmax(l, c, K);
    for (int k = 0; k < K; ++k)
      if (k != keep && l[k] >= 0 && (double)c[k] < thr) { l[k] = -1; c[k] = 0; }
    W[vb + q] = l[keep];
  }
}
// glp_slp_memory_get: original order, owned rows [vb, ve)
__global__ void k_slp_unpermute(const int32_t* __restrict__ ml, const int32_t* __restrict__ mc,
                                const int32_t* __restrict__ pos, int64_t vb, int64_t ve, int K,
                                int32_t* __restrict__ ol, int32_t* __restrict__ oc) {
  for (int64_t v = vb + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < ve; v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = pos[v] - vb;
    for (int k = 0; k < K; ++k) {
      ol[(v - vb) * K + k] = ml[q * K + k];
      oc[(v - vb) * K + k] = mc[q * K + k];
    }
  }
}

// L2 flush helper for benchmarks (writes a buffer larger than L2).
__global__ void k_fill(uint4* __restrict__ p, int64_t n16, unsigned x) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n16; i += (int64_t)gridDim.x * blockDim.x)
    p[i] = make_uint4(x, x, x, x);
}

}  // namespace glp
