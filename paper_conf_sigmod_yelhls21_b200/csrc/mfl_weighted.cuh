// mfl_weighted.cuh -- weighted MFL (§8(f)3, the paper's LoadNeighbor weight).
//
// LoadNeighbor returns (l, weight) [P:110, P:145] and the SharedMemBigNodes
// procedure adds the weight, not 1, into the hash table (atomicAdd(HT, l,
// weight) [P:150-156]).  A label's frequency is the sum of the weights of the
// arcs carrying it; the score is that sum (CLASSIC / SEEDED); ties go to the
// smallest label (R4).  Weights are integers in [1, 2^31) and every row's
// total is < 2^31 (checked at create), so sums are exact in 32 bits and the
// running arg-max over post-add sums is exact (sums only grow: mfl_kernels.cuh
// header).
//
// Two kernels over the library's layout (ioff / ideg per local vertex; the
// weights w2 sit beside the arcs of col2):
//   mfl_wt_warp   vertices with 1 <= deg <= kWtWarpMax: one warp per vertex,
//                 per-warp shared table of pow2 >= 2 deg slots (never full)
//   mfl_wt_block  longer rows: one block per row.  A row whose labels are
//                 strictly increasing (t = 1) needs no table; otherwise an
//                 8192-slot shared table, and a row with more labels than half
//                 the table (predicted from its last distinct count) is
//                 counted in label-hash partitions (every pass re-reads the
//                 row and counts only its part's labels), doubling the parts
//                 when a part overflows -- exact by construction
#pragma once
#include "mfl_kernels.cuh"

namespace glp {

constexpr int kWtWarpMax = 512;
constexpr int kWtWarpSlots = 1024;
constexpr int kWtBlock = 256;
constexpr int kWtSlots = 8192;

template <int VAR>
__global__ void __launch_bounds__(kWtBlock) mfl_wt_warp(MflArgs a) {
  GLP_CTL_PROLOGUE(a)
  extern __shared__ __align__(16) unsigned long long wts_tab[];  // [8][kWtWarpSlots]
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  Tally ty;
  for (int64_t base = a.wt_lo + (int64_t)gw * 32; base < a.wt_hi; base += (int64_t)nwarps * 32) {
    const int64_t v = base + lane;
    int deg = 0;
    bool ok = v < a.wt_hi;
    if (ok) {
      deg = a.ideg[v];
      ok = deg >= 1 && deg <= kWtWarpMax && (dense_ || a.flag[a.vb + v]);
    }
    unsigned todo = __ballot_sync(kFull, ok);
    bool rdone = false;
    unsigned long long rkey = 0ull;
    unsigned rlab = kNoLabel;
    while (todo) {
      const int j = __ffs(todo) - 1;
      todo &= todo - 1;
      const int64_t start = __shfl_sync(kFull, ok ? a.ioff[v] : 0, j);
      const int d = __shfl_sync(kFull, deg, j);
      const unsigned tsz = min(max(64u, 1u << (32 - __clz(2u * (unsigned)d - 1u))), (unsigned)kWtWarpSlots);
      const Table tab{wts_tab + (size_t)wid * kWtWarpSlots, tsz};
      tab.clear(lane, 32);
      __syncwarp();
      Best<VAR> b;
      unsigned fresh = 0;
      for (int off = lane; off < d; off += 32) {
        const int u = a.col[start + off];
        const int l = gather(a, u);
        if (l >= 0) {
          // at most d <= tsz / 2 labels: the full probe always finds a slot
          const unsigned c = ht_add(tab, (unsigned)l, a.w2[start + off], tsz, &fresh);
          b.observe(c, (unsigned)l, a);
        }
      }
      b.warp_reduce();
      __syncwarp();
      if (lane == j) {
        rdone = true;
        rkey = b.key;
        rlab = b.lab;
      }
    }
    if (rdone) {
      Best<VAR> r;
      r.key = rkey;
      r.lab = rlab;
      update_vertex<VAR>(a, (int)v, deg, r.have(), r.label(), ty, deg);
    }
  }
  tally_flush(ty, a.cnt);
}

template <int VAR>
__global__ void __launch_bounds__(kWtBlock) mfl_wt_block(MflArgs a) {
  GLP_CTL_PROLOGUE(a)
  extern __shared__ __align__(16) unsigned long long wtb_tab[];  // kWtSlots
  __shared__ int s_k, s_over, s_distinct;
  Tally ty;
  for (;;) {
    if (threadIdx.x == 0) s_k = (int)atomicAdd(a.work, 1ull);
    __syncthreads();
    const int k = s_k;
    if (k >= a.n_items) break;
    const BinItem it = a.items[k];
    const unsigned raw = a.pred[k];
    if (!dense_ && !a.flag[a.vb + it.v]) {
      if (threadIdx.x == 0) a.pred_next[k] = raw;  // inactive: carry the count forward
      __syncthreads();  // s_k is rewritten by the next ticket
      continue;
    }
    const int d = it.d;
    Best<VAR> b;
    unsigned distinct = 0;
    bool done = false;
    // Sorted-row fast path (t = 1's unique labels on sorted rows, checked on
    // the data): labels strictly increasing along the row occur once each, so
    // a label's weight sum is its arc's weight -- no table, one pass.
    if (mono_cand<VAR>(raw, a.pred_cap, d, a.t)) {
      bool inc = true;
      for (int e = threadIdx.x; e < d; e += kWtBlock) {
        const int l = gather(a, a.col[it.start + e]);
        const int lp = e > 0 ? gather(a, a.col[it.start + e - 1]) : -1;
        inc = inc && l >= 0 && lp < l;
        if (inc) b.observe(a.w2[it.start + e], (unsigned)l, a);
      }
      done = __syncthreads_and(inc ? 1 : 0) != 0;
      if (done) distinct = (unsigned)d;
      else b = Best<VAR>();
    }
    if (!done) {
      // table passes: parts sized from the last distinct count (a row that
      // took the sorted path last time: 40 % of it -- labels collapse
      // [P:130]); an overflowing part doubles the parts (exact recount)
      const unsigned pr = raw & kPredMask;
      const unsigned est = (raw & kMonoTried) ? max(1u, (unsigned)(((unsigned long long)pr * 40ull) / 100ull)) : max(pr, 1u);
      unsigned nparts = max(1u, (2u * min(est, (unsigned)d) + kWtSlots - 1) / kWtSlots);
      if (2u * (unsigned)d <= (unsigned)kWtSlots) nparts = 1u;
      for (;;) {
        b = Best<VAR>();
        if (threadIdx.x == 0) s_distinct = 0;
        bool over = false;
        for (unsigned p = 0; p < nparts && !over; ++p) {
          const Table tab{wtb_tab, (unsigned)kWtSlots};
          tab.clear(threadIdx.x, kWtBlock);
          if (threadIdx.x == 0) s_over = 0;
          __syncthreads();
          // the whole row at half load: a full probe never fails
          const unsigned probe = 2u * (unsigned)d <= (unsigned)kWtSlots ? (unsigned)kWtSlots : (unsigned)kLProbe;
          unsigned fresh = 0;
          for (int e = threadIdx.x; e < d; e += kWtBlock) {
            const int l = gather(a, a.col[it.start + e]);
            if (l < 0 || (nparts > 1u && label_part((unsigned)l, nparts) != p)) continue;
            const unsigned c = ht_add(tab, (unsigned)l, a.w2[it.start + e], probe, &fresh);
            if (c == 0u) {
              s_over = 1;
              break;
            }
            b.observe(c, (unsigned)l, a);
          }
          fresh = __reduce_add_sync(kFull, fresh);
          if ((threadIdx.x & 31) == 0 && fresh) atomicAdd(&s_distinct, (int)fresh);
          __syncthreads();
          over = s_over != 0;
          __syncthreads();  // the next part clears the table
        }
        if (!over) break;
        nparts *= 2u;
      }
      distinct = (unsigned)s_distinct;
    }
    b = block_best<VAR, kWtBlock>(b);
    if (threadIdx.x == 0) {
      a.pred_next[k] = max(distinct, 1u) | (done ? kMonoTried : 0u);
      update_vertex<VAR>(a, it.v, d, b.have(), b.label(), ty, d);
    }
    __syncthreads();
  }
  tally_flush(ty, a.cnt);
}

}  // namespace glp
