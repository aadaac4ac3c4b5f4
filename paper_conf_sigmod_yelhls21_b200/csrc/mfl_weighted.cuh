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
#ifndef GLP_WTB_BLOCK
#define GLP_WTB_BLOCK 512  // A/B R24 weighted (128 / 256 / 512 threads): 67.0 / 56.5 / 51.5 ms/run
#endif
#ifndef GLP_WTB_SLOTS
#define GLP_WTB_SLOTS 8192
#endif
constexpr int kWtBBlock = GLP_WTB_BLOCK;  // mfl_wt_block threads
constexpr int kWtSlots = GLP_WTB_SLOTS;

// Lean weighted insert of four (label, weight) pairs per lane (the
// lean_insert4 scheme of mfl_kernels.cuh: valid pairs compacted to the front
// of a shift register, one shared CAS per probe, a hit adds the weight).
// The table holds at least twice the row's arcs, so a full probe never fails.
template <int VAR>
__device__ __forceinline__ unsigned lean_insert4w(const MflArgs& a, const Table& t, int q0, int q1, int q2, int q3,
                                                  unsigned w0, unsigned w1, unsigned w2, unsigned w3, Best<VAR>& b,
                                                  unsigned max_probe = 0xffffffffu, volatile int* overflow = nullptr) {
  auto cswap = [&](int& x, int& y, unsigned& wx, unsigned& wy) {
    const bool s = x < 0;
    const int tx = x;
    const unsigned tw = wx;
    x = s ? y : x;
    y = s ? tx : y;
    wx = s ? wy : wx;
    wy = s ? tw : wy;
  };
  unsigned fresh = 0u, np = 0u;
  // hot label of the warp (lane 0's best so far, else its first label): every
  // lane sums the weights of its copies, one warp sum, one shared add by lane
  // 0 -- a collapsed row does not serialise on one slot
  {
    const int cand = b.have() ? (int)b.label() : (q0 >= 0 ? q0 : q1 >= 0 ? q1 : q2 >= 0 ? q2 : q3);
    const int hot = __shfl_sync(kFull, cand, 0);
    if (hot >= 0) {
      unsigned hc = 0u;
      hc += q0 == hot ? w0 : 0u; q0 = q0 == hot ? -1 : q0;
      hc += q1 == hot ? w1 : 0u; q1 = q1 == hot ? -1 : q1;
      hc += q2 == hot ? w2 : 0u; q2 = q2 == hot ? -1 : q2;
      hc += q3 == hot ? w3 : 0u; q3 = q3 == hot ? -1 : q3;
      const unsigned tot = __reduce_add_sync(kFull, hc);
      if ((threadIdx.x & 31) == 0 && tot) {
        const unsigned c = ht_add(t, (unsigned)hot, tot, max_probe < t.tsz ? max_probe : t.tsz, &fresh);
        if (c) b.observe(c, (unsigned)hot, a);
        else flag_set(overflow);
      }
    }
  }
  cswap(q0, q1, w0, w1);
  cswap(q2, q3, w2, w3);
  cswap(q0, q2, w0, w2);
  cswap(q1, q3, w1, w3);
  cswap(q1, q2, w1, w2);
  unsigned h = slot_hash((unsigned)q0, t.tsz);
  const unsigned mask = t.tsz - 1u;
  while (__any_sync(kFull, q0 >= 0)) {
    if (q0 >= 0) {
      const unsigned k = atomicCAS(t.key + h, kFree, (unsigned)q0);
      if (k == kFree || k == (unsigned)q0) {
        const unsigned c = atomicAdd(t.cnt + h, w0) + w0;
        fresh += k == kFree ? 1u : 0u;
        b.observe(c, (unsigned)q0, a);
        q0 = q1; q1 = q2; q2 = q3; q3 = -1;
        w0 = w1; w1 = w2; w2 = w3;
        h = slot_hash((unsigned)q0, t.tsz);
        np = 0u;
      } else if (++np >= max_probe) {  // part overflowed: the caller recounts in finer parts
        flag_set(overflow);
        q0 = q1 = q2 = q3 = -1;
      } else {
        h = (h + 1u) & mask;
      }
    }
  }
  return fresh;
}

// One warp per vertex with 33 <= deg <= kWtWarpMax (rows start 16-B aligned,
// padded with -1 / weight 0): rounds of 128 arcs, one 128-bit load of arcs
// and one of weights per lane, lean weighted insert into a per-warp table of
// pow2 >= 2 deg slots.  (Low rows, deg <= 32, go to mfl_low with weights
// unless GLP_WT_LOW=0 keeps them here, one per warp.)
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
      if (d > kLowMax) {
        for (int off = 0; off < d; off += 128) {
          int4 u = make_int4(-1, -1, -1, -1), w = make_int4(0, 0, 0, 0);
          if (off + 4 * lane < d) {
            u = ld_stream4(a.col + start + off + 4 * lane);
            w = ld_stream4((const int32_t*)a.w2 + start + off + 4 * lane);
          }
          lean_insert4w<VAR>(a, tab, gather(a, u.x), gather(a, u.y), gather(a, u.z), gather(a, u.w), (unsigned)w.x,
                             (unsigned)w.y, (unsigned)w.z, (unsigned)w.w, b);
        }
      } else {  // low rows (GLP_WT_LOW=0): contiguous, not aligned
        const int u = lane < d ? a.col[start + lane] : -1;
        const unsigned w = lane < d ? a.w2[start + lane] : 0u;
        lean_insert4w<VAR>(a, tab, gather(a, u), -1, -1, -1, w, 0u, 0u, 0u, b);
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
__global__ void __launch_bounds__(kWtBBlock) mfl_wt_block(MflArgs a) {
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
    // a label's weight sum is its arc's weight -- no table, one pass.  Rows
    // start 16-B aligned (padded with -1 / weight 0): 128-bit loads, element
    // e = 4 * thread + j of each 4 * kWtBBlock-arc round.
    if (mono_cand<VAR>(raw, a.pred_cap, d, a.t)) {
      bool inc = true;
      for (int base = 0; base < d; base += 4 * kWtBBlock) {
        const int e0 = base + 4 * (int)threadIdx.x;
        if (e0 < d) {
          const int4 u = ld_stream4(a.col + it.start + e0);
          const int4 w = ld_stream4((const int32_t*)a.w2 + it.start + e0);
          const int l[4] = {gather(a, u.x), gather(a, u.y), gather(a, u.z), gather(a, u.w)};
          const unsigned wv[4] = {(unsigned)w.x, (unsigned)w.y, (unsigned)w.z, (unsigned)w.w};
          int lp = e0 > 0 ? gather(a, a.col[it.start + e0 - 1]) : -1;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            if (e0 + j < d) {
              inc = inc && l[j] >= 0 && lp < l[j];
              if (inc) b.observe(wv[j], (unsigned)l[j], a);
              lp = l[j];
            }
          }
        }
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
          // the whole row at half load: a full probe never fails
          const unsigned tsz = nparts == 1u ? min(max(64u, 1u << (32 - __clz(2u * (unsigned)d - 1u))), (unsigned)kWtSlots)
                                            : (unsigned)kWtSlots;
          const Table tab{wtb_tab, tsz};
          tab.clear(threadIdx.x, kWtBBlock);
          if (threadIdx.x == 0) s_over = 0;
          __syncthreads();
          const unsigned probe = 2u * (unsigned)d <= tsz ? tsz : (unsigned)kLProbe;
          unsigned fresh = 0;
          for (int base = 0; base < d; base += 4 * kWtBBlock) {
            const int e0 = base + 4 * (int)threadIdx.x;
            int4 u = make_int4(-1, -1, -1, -1), w = make_int4(0, 0, 0, 0);
            if (e0 < d) {
              u = ld_stream4(a.col + it.start + e0);
              w = ld_stream4((const int32_t*)a.w2 + it.start + e0);
            }
            int l[4] = {gather(a, u.x), gather(a, u.y), gather(a, u.z), gather(a, u.w)};
            if (nparts > 1u) {
#pragma unroll
              for (int j = 0; j < 4; ++j)
                if (l[j] >= 0 && label_part((unsigned)l[j], nparts) != p) l[j] = -1;
            }
            fresh += lean_insert4w<VAR>(a, tab, l[0], l[1], l[2], l[3], (unsigned)w.x, (unsigned)w.y, (unsigned)w.z,
                                        (unsigned)w.w, b, probe, &s_over);
            if (warp_flag(&s_over)) break;
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
    b = block_best<VAR, kWtBBlock>(b);
    if (threadIdx.x == 0) {
      a.pred_next[k] = max(distinct, 1u) | (done ? kMonoTried : 0u);
      update_vertex<VAR>(a, it.v, d, b.have(), b.label(), ty, d);
    }
    __syncthreads();
  }
  tally_flush(ty, a.cnt);
}

}  // namespace glp
