// mfl_kernels.cuh -- most-frequent-label (MFL) kernels for sm_100a.
//
// One synchronous LP iteration [P:68 §2.1]: every processed vertex v gathers
// the labels of N(v) from R = L_{t-1} (LoadNeighbor [P:110]), counts them,
// scores them (LabelScore [P:111]; LLP: k - gamma*(V-k) [P:119]) and writes
// the best label (score desc, label asc: R4) to W = L_t (UpdateVertex [P:112],
// Lnext [P:143]).
//
// Arcs are read from the library's bin-major copy `col2`:
// the arcs of each low-degree chunk are contiguous, and every mid/high/huge row
// starts 16-byte aligned and is padded with -1 to a multiple of 4, so rows are
// streamed with one 128-bit load per lane.
//
// Kernels by degree bin:
//   mfl_low   deg <= 32: one warp serves several vertices whose arcs fill its
//             32 lanes ("one-warp-multi-vertices" [P:227-234 §4.2]): lane
//             masks from the chunk's segment-start bitmap, label frequency per
//             segment, shuffle-tree arg-max per segment.
//   deg > 32: a row goes to one of three kernels by its predicted
//             distinct-label count (glp_internal.cuh row_class):
//   mfl_warp  W: one warp per row, per-warp shared-memory table;
//   mfl_block M/L: one block per row with a shared-memory hash table
//             ("SharedMemBigNodes" HT [P:132-182 §4.1]); L recounts rows whose
//             distinct labels overflow the table in hash partitions
//             (replacing GlobalInsert/GHT [P:166, P:182]).
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

#include <climits>
#include <type_traits>

#include "glp_internal.cuh"

namespace glp {

constexpr unsigned kFull = 0xffffffffu;
constexpr unsigned kNoLabel = 0xffffffffu;

enum Variant { V_CLASSIC = 0, V_SEEDED = 1, V_LLP = 2 };

// L2 policy of the two access streams: the arcs `col2`
// are read once per iteration and must not evict the label array L_{t-1},
// which every arc gathers from (64 MiB at RMAT-24, < 126 MB of L2), so arc
// loads carry an L2 evict_first hint.  GLP_GATHER_POLICY selects the gathers'
// hint: 0 none, 1 evict_last.
#ifndef GLP_STREAM_POLICY
#define GLP_STREAM_POLICY 0
#endif
#ifndef GLP_GATHER_POLICY
#define GLP_GATHER_POLICY 0
#endif
// kernel A/B switches (tools/build_variants.py)
#ifndef GLP_LOW_REDUX
#define GLP_LOW_REDUX 0
#endif
#ifndef GLP_LOW_MATCH
#define GLP_LOW_MATCH 6  // low segments of at least this degree count with match.any (33 = never);
                         // A/B: 6 / 12 / 17 all -2.8 % per R24 run vs never (shuffle loop)
#endif
#ifndef GLP_L_OPT
#define GLP_L_OPT 0
#endif
#ifndef GLP_L_IPF
#define GLP_L_IPF 0
#endif
#ifndef GLP_L_FILTER
#define GLP_L_FILTER 4  // L rows split into at most this many label parts count by filtering, not scattering
#endif
#ifndef GLP_L_STAGE1
#define GLP_L_STAGE1 0
#endif
#ifndef GLP_L_MAJ
#define GLP_L_MAJ 1
#endif
#ifndef GLP_M_EST
#define GLP_M_EST 100  // M rows after a sorted-row pass: table sized for this % of the degree (x GLP_M_LOAD)
#endif
#ifndef GLP_L_EST
#define GLP_L_EST 40
#endif
#ifndef GLP_M_LOAD
#define GLP_M_LOAD 4
#endif
#ifndef GLP_FEWER_BARRIERS
#define GLP_FEWER_BARRIERS 1
#endif
#ifndef GLP_ADD_ALWAYS
#define GLP_ADD_ALWAYS 1
#endif
#ifndef GLP_W_LOAD
#define GLP_W_LOAD 4
#endif

__device__ __forceinline__ int ld_stream(const int32_t* p) {
  int r;
#if GLP_STREAM_POLICY
  asm volatile("{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_first.b64 pol, 1.0;\n\t"
               "ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], pol;\n\t}"
               : "=r"(r) : "l"(p));
#else
  asm volatile("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(r) : "l"(p));
#endif
  return r;
}
__device__ __forceinline__ int4 ld_stream4(const int32_t* p) {
  int4 r;
#if GLP_STREAM_POLICY
  asm volatile("{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_first.b64 pol, 1.0;\n\t"
               "ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], pol;\n\t}"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
#else
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
#endif
  return r;
}
__device__ __forceinline__ int ld_label(const int32_t* p) {
#if GLP_GATHER_POLICY
  int r;
  asm volatile("{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_last.b64 pol, 1.0;\n\t"
               "ld.global.nc.L2::cache_hint.b32 %0, [%1], pol;\n\t}" : "=r"(r) : "l"(p));
  return r;
#else
  return __ldg(p);
#endif
}
// SEEDED presence filter (a.lbits): bit u is set for
// every vertex whose label in L_{t-1} is valid (seeds at PickLabel, a vertex
// when it first takes a label), so a clear bit means L_{t-1}[u] = -1 without
// reading it.  The bitmap (n/8 bytes) stays in L2 when the label array does
// not (TaoBao-100M: 12.5 MB vs 400 MB), and early seeded iterations gather
// mostly unlabelled neighbours.  A set bit only sends the load on.
__device__ __forceinline__ bool lbit_clear(const MflArgs& a, int u) {
  return a.lbits != nullptr && !((__ldg(a.lbits + (u >> 5)) >> (u & 31)) & 1u);
}
__device__ __forceinline__ int gather(const MflArgs& a, int u) {
  if (u < 0 || lbit_clear(a, u)) return -1;
  return a.lv_labels ? __ldg(&a.LV[u].x) : ld_label(a.R + u);
}

// LLP: (L_{t-1}[u], V[L_{t-1}[u]]) interleaved in a.LV (rebuilt once per
// vertex after the histogram): one 8-byte gather at the neighbour's index
// returns its label and the label's V, so a candidate's V arrives with it
// instead of a random V[l] gather per label.  Without LV: the plain label.
__device__ __forceinline__ int gather_lv(const MflArgs& a, int u, bool use_v, int& lv) {
  if (u < 0) { lv = -1; return -1; }
  if (use_v) {
    const int2 x = __ldg(a.LV + u);
    lv = x.y;
    return x.x;
  }
  lv = -1;
  if (lbit_clear(a, u)) return -1;
  return ld_label(a.R + u);
}

// Device-driven iteration loop: a.ctl = {stopped, dense} written by k_decide
// at the end of the previous iteration (null: host-driven, a.dense).  An
// iteration enqueued after the stop rule fired does nothing.
#define GLP_CTL_PROLOGUE(a)                 \
  int dense_ = (a).dense;                   \
  if ((a).ctl) {                            \
    if ((a).ctl[0]) return;                 \
    dense_ = (a).ctl[1];                    \
  }

// LLP score val = k - gamma * (v - k) [P:119], double, no contraction (R11).
__device__ __forceinline__ double llp_score(unsigned k, int v, double gamma) {
  double kd = (double)k;
  double diff = __dsub_rn((double)v, kd);
  double prod = __dmul_rn(gamma, diff);
  return __dsub_rn(kd, prod);
}

// Order-preserving map double -> u64 (finite and infinite values); 0 = none.
__device__ __forceinline__ unsigned long long dkey(double x) {
  unsigned long long b = (unsigned long long)__double_as_longlong(x);
  return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}

// Running best (score desc, label asc).  CLASSIC/SEEDED pack (count, ~label)
// into one u64 so "better" is a single 64-bit max; LLP keeps (score key, label).
template <int VAR>
struct Best {
  unsigned long long key = 0ull;
  unsigned lab = kNoLabel;
  int bv = -1;  // LLP: V of the best label
  // vl: V[l] when the caller has it (carried with the label, a.LV), else -1
  __device__ __forceinline__ void observe(unsigned cnt, unsigned l, const MflArgs& a, int vl = -1) {
    if (VAR == V_LLP) {
      // V of a permutation labelling is all ones (t = 1)
      const int v = vl >= 0 ? vl : (a.v_ones ? 1 : ld_label(a.V + l));
      const unsigned long long k = dkey(llp_score(cnt, v, a.gamma));
      if (k > key || (k == key && l < lab)) { key = k; lab = l; bv = v; }
    } else {
      const unsigned long long k = ((unsigned long long)cnt << 32) | (unsigned long long)(~l);
      key = k > key ? k : key;
    }
  }
  __device__ __forceinline__ void merge(unsigned long long k, unsigned l) {
    if (VAR == V_LLP) {
      if (k > key || (k == key && l < lab)) { key = k; lab = l; }
    } else {
      key = k > key ? k : key;
    }
  }
  __device__ __forceinline__ bool have() const { return key != 0ull; }
  __device__ __forceinline__ unsigned label() const { return VAR == V_LLP ? lab : ~(unsigned)key; }
  __device__ __forceinline__ void warp_reduce() {
#pragma unroll
    for (int s = 16; s > 0; s >>= 1) {
      const unsigned long long k = __shfl_xor_sync(kFull, key, s);
      const unsigned l = VAR == V_LLP ? __shfl_xor_sync(kFull, lab, s) : 0u;
      merge(k, l);
    }
  }
};

// Majority early exit (CLASSIC/SEEDED): a label observed with a count above
// d/2 is the strict maximum of the row's final counts (any other label has at
// most d - count < count votes), so it is the MFL whatever the unread arcs
// hold, and min-label ties cannot arise.  Counts in the shared table are
// row totals, so one lane's observation suffices.  Exact; saves reading the
// rest of collapsed rows (labels concentrate as communities form [P:130]).
#ifndef GLP_MAJORITY
#define GLP_MAJORITY 1
#endif
template <int VAR>
__device__ __forceinline__ bool strict_majority(const Best<VAR>& b, int d) {
  const unsigned k = (unsigned)(b.key >> 32);
  return __any_sync(kFull, 2ull * k > (unsigned long long)d);
}

// Monotone shared flags (overflow, strict majority) are polled by other warps
// while they are being set; both sides use atomics, so the polling is a
// synchronised read (compute-sanitizer racecheck clean) and a stale 0 only
// delays an exit by one round.  One lane reads and broadcasts.
__device__ __forceinline__ void flag_set(volatile int* f) { atomicExch((int*)f, 1); }
__device__ __forceinline__ bool warp_flag(volatile int* f) {
  int v = 0;
  if ((threadIdx.x & 31) == 0) v = atomicOr((int*)f, 0);
  return __shfl_sync(kFull, v, 0) != 0;
}

__device__ __forceinline__ unsigned slot_hash(unsigned lab, unsigned tsz) {
  return __umulhi(lab * 0x9E3779B1u, tsz);
}

// Open-addressing count table in shared memory: tsz (a power of two) slots
// in the storage of tsz u64 words -- key[tsz] (u32 label, kFree when free)
// then cnt[tsz] (u32) -- with linear probing.  A new label claims its key with
// a 32-bit CAS; every occurrence (the claimer's included) then adds to the
// count with a native 32-bit shared atomic, so counts start from the cleared 0.
constexpr unsigned kFree = 0xffffffffu;
struct Table {
  unsigned* key;
  unsigned* cnt;
  unsigned tsz;
  __device__ __forceinline__ Table(unsigned long long* storage, unsigned tsz_)
      : key((unsigned*)storage), cnt((unsigned*)storage + tsz_), tsz(tsz_) {}
  // cooperative clear by `nthr` threads starting at thread `tid` (16-B stores)
  __device__ __forceinline__ void clear(unsigned tid, unsigned nthr) const {
    uint4* k4 = (uint4*)key;
    uint4* c4 = (uint4*)cnt;
    for (unsigned j = tid; j < tsz / 4; j += nthr) {
      k4[j] = make_uint4(kFree, kFree, kFree, kFree);
      c4[j] = make_uint4(0u, 0u, 0u, 0u);
    }
  }
};

__device__ __forceinline__ unsigned ld_key(const Table& t, unsigned h) { return *((volatile unsigned*)(t.key + h)); }

// LLP scores each distinct label once, from the final table (one V[l] gather
// per distinct label), instead of at every insert: the table
// inserts skip `observe` for LLP, and the counting threads scan the table after
// the barrier that ends the count.  (CLASSIC/SEEDED keep the running arg-max
// of the insert observations, which needs no scan.)
template <int VAR>
__device__ __forceinline__ void table_scan(const Table& t, unsigned tid, unsigned nthr, const MflArgs& a,
                                           Best<VAR>& b) {
  if constexpr (VAR == V_LLP) {
    for (unsigned j = tid; j < t.tsz; j += nthr) {
      const unsigned k = t.key[j];
      if (k != kFree) b.observe(t.cnt[j], k, a);
    }
  }
}

// One probe of slot h (whose key was read as k) for `c` occurrences of label
// l: returns the post-add count, or 0 when the slot holds another label.
// *fresh counts a slot claimed by this call.
__device__ __forceinline__ unsigned slot_try(const Table& t, unsigned h, unsigned l, unsigned c, unsigned k,
                                             unsigned* fresh) {
  if (k == kFree) {
    const unsigned p = atomicCAS(t.key + h, kFree, l);
    *fresh += p == kFree ? 1u : 0u;
    k = p == kFree ? l : p;
  }
#if GLP_ADD_ALWAYS
  // the add is issued by every lane (a lane whose slot holds another label
  // adds 0): one divergent region less per label
  const bool hit = k == l;
  const unsigned old = atomicAdd(t.cnt + h, hit ? c : 0u);
  return hit ? old + c : 0u;
#else
  return k == l ? atomicAdd(t.cnt + h, c) + c : 0u;
#endif
}

// Probe from slot h + 1 on (the home slot h held another label).  Returns the
// post-add count, or 0 when no slot was found within `max_probe` probes in
// total (overflow).
__device__ __forceinline__ unsigned ht_probe_from(const Table& t, unsigned lab, unsigned c, unsigned h,
                                                  unsigned max_probe, unsigned* fresh) {
  for (unsigned p = 1; p < max_probe; ++p) {
    h = (h + 1) & (t.tsz - 1);
    const unsigned r = slot_try(t, h, lab, c, ld_key(t, h), fresh);
    if (r) return r;
  }
  return 0u;
}

// Insert `c` occurrences of `lab` (home slot first).
__device__ __forceinline__ unsigned ht_add(const Table& t, unsigned lab, unsigned c, unsigned max_probe,
                                           unsigned* fresh) {
  const unsigned h = slot_hash(lab, t.tsz);
  const unsigned r = slot_try(t, h, lab, c, ld_key(t, h), fresh);
  return r ? r : ht_probe_from(t, lab, c, h, max_probe, fresh);
}

// Batched insert of N labels per lane (-1 = no vote).  First the warp's
// "hot" label -- lane 0's best label so far, else its first label of this
// batch -- is taken out: every lane counts its copies locally, one warp
// reduction sums them and lane 0 adds the sum with a single shared atomic, so a
// collapsed neighbourhood (most neighbours share a community label [P:130])
// costs a few ALU ops per arc instead of same-address atomics.  The remaining
// labels are inserted one by one: the N home-slot keys are read as
// independent shared loads, then each label takes its home slot (claim or
// match) with predicated atomics; only labels whose home slot holds another
// label fall back to the probing loop.  Returns this lane's count of newly
// claimed slots.
// ---------------------------------------------------------------------------
// Count-Min Sketch beside the hash table (§8(f)2, PAPER §4.1 Procedure
// SharedMemBigNodes [P:132-182]): a label whose insertion into the shared HT
// fails (its probe chain is full) is counted in a CMS of `depth` rows x
// `width` u32 counters in shared memory instead, and flags `used`.  A label is
// wholly in HT or wholly in the CMS (HT slots are never freed, so once a
// label's chain is full it stays full), so HT counts are exact.
constexpr unsigned kCmsCounters = 8192;  // u32 sketch counters per block (32 KB)
struct Cms {
  unsigned* c;      // depth * width counters (shared memory)
  unsigned depth, width;
  volatile int* used;
  __device__ __forceinline__ unsigned slot(unsigned l, unsigned i) const {
    // row i: an independent multiplicative hash (odd multipliers)
    return __umulhi((l ^ (0x9E3779B9u * (i + 1u))) * (0x85EBCA6Bu + 2u * i * 0x27D4EB2Du), width);
  }
  __device__ __forceinline__ void add(unsigned l, unsigned k) const {
    for (unsigned i = 0; i < depth; ++i) atomicAdd(c + i * width + slot(l, i), k);
    flag_set(used);
  }
  // estimate g(l) = min over rows (read after a barrier: an upper bound of
  // l's count, exact for every label that went to the sketch [P:134, Lemma 2])
  __device__ __forceinline__ unsigned estimate(unsigned l) const {
    unsigned g = 0xffffffffu;
    for (unsigned i = 0; i < depth; ++i) g = min(g, c[i * width + slot(l, i)]);
    return g;
  }
};

// Rows predicted to hold more than d / GLP_HOT_DIV distinct labels (few
// repeats per label: t = 2..3) skip the hot-label pass, whose single-lane
// insert costs more than it saves there (0 = always take it).
#ifndef GLP_HOT_DIV
#define GLP_HOT_DIV 0
#endif
// GLP_MATCH_INSERT: 1 = equal labels of one batch slot are merged across the
// warp with match.any (the lowest lane inserts the group's count); 2 = the
// same without the hot-label pass
#ifndef GLP_MATCH_INSERT
#define GLP_MATCH_INSERT 0
#endif
// GLP_LEAN: the label columns left after the hot pass are inserted by a
// persistent per-lane probe loop (warp_insert_n); GLP_LEAN_PEEK: each probe
// reads the key before the CAS
#ifndef GLP_LEAN
#define GLP_LEAN 1
#endif
#ifndef GLP_LEAN_PEEK
#define GLP_LEAN_PEEK 0  // A/B (R24 ms/run): 0 17.29, 1 17.27, 2 17.72, 3 17.80; LLP 174.5 / 182.6 / 180.4 / 174.5.  0 never, 1 always, 2 rows predicted to repeat labels, 3 = 2 but not LLP
#endif
template <int VAR>
__device__ __forceinline__ bool peek_pass(unsigned pred, int d) {
  if (GLP_LEAN_PEEK == 0 || (GLP_LEAN_PEEK == 3 && VAR == V_LLP)) return false;
  return GLP_LEAN_PEEK == 1 || 2ull * pred <= (unsigned long long)d;
}
__device__ __forceinline__ bool hot_pass(unsigned pred, int d) {
  return GLP_HOT_DIV == 0 || (unsigned long long)pred * GLP_HOT_DIV <= (unsigned long long)d;
}
// Lean insert of four labels per lane (-1 = none), count 1 each.  The lane's
// valid labels are first compacted to the front of a 4-entry shift register
// (five compare-swaps); then a persistent probe loop takes one probe per trip
// for the register's head: one shared CAS claims a free slot or returns its
// occupant; on a hit the count is added and the register shifts.  A lane
// whose label probes does not hold up the other lanes' labels: the warp runs
// max over lanes of the lane's summed probes, not the sum over label columns
// of the longest chain.  Returns the lane's number of newly claimed slots.
template <int VAR>
__device__ __forceinline__ unsigned lean_insert4(const MflArgs& a, const Table& t, unsigned max_probe, int q0, int q1,
                                                 int q2, int q3, int v0, int v1, int v2, int v3, Best<VAR>& b,
                                                 volatile int* overflow, bool use_v, bool obs, const Cms* cms,
                                                 bool peek) {
  constexpr bool kV = VAR == V_LLP;  // labels carry V (LLP with a.LV)
  auto cswap = [&](int& x, int& y, int& vx, int& vy) {
    const bool s = x < 0;
    const int tx = x, tv = vx;
    x = s ? y : x;
    y = s ? tx : y;
    if (kV) {
      vx = s ? vy : vx;
      vy = s ? tv : vy;
    }
  };
  cswap(q0, q1, v0, v1);
  cswap(q2, q3, v2, v3);
  cswap(q0, q2, v0, v2);
  cswap(q1, q3, v1, v3);
  cswap(q1, q2, v1, v2);
  unsigned fresh = 0u, np = 0u;
  unsigned h = slot_hash((unsigned)q0, t.tsz);
  const unsigned mask = t.tsz - 1u;
  while (__any_sync(kFull, q0 >= 0)) {
    if (q0 >= 0) {
      // peek (rows predicted to repeat labels): read the key first, so a
      // repeated label (its slot already claimed) costs a shared load instead
      // of a CAS serialised with its copies; otherwise one CAS per probe
      unsigned k = peek ? ld_key(t, h) : kFree;
      bool claimed = false;
      if (k == kFree) {
        k = atomicCAS(t.key + h, kFree, (unsigned)q0);
        claimed = k == kFree;
        k = claimed ? (unsigned)q0 : k;
      }
      bool next = false;
      if (k == (unsigned)q0) {
        const unsigned c = atomicAdd(t.cnt + h, 1u) + 1u;
        fresh += claimed ? 1u : 0u;
        if (obs) b.observe(c, (unsigned)q0, a, (kV && use_v) ? v0 : -1);
        next = true;
      } else if (++np >= max_probe) {
        if (cms) {
          cms->add((unsigned)q0, 1u);
          next = true;
        } else {
          flag_set(overflow);
          q0 = q1 = q2 = q3 = -1;
        }
      } else {
        h = (h + 1u) & mask;
      }
      if (next) {
        q0 = q1; q1 = q2; q2 = q3; q3 = -1;
        if (kV) { v0 = v1; v1 = v2; v2 = v3; }
        h = slot_hash((unsigned)q0, t.tsz);
        np = 0u;
      }
    }
  }
  return fresh;
}

template <int VAR, int N>
__device__ __forceinline__ unsigned warp_insert_n(const MflArgs& a, const Table& t, unsigned max_probe,
                                                  const int (&labin)[N], Best<VAR>& b, volatile int* overflow,
                                                  const int (&vin)[N], bool use_v, bool hot_ok = true,
                                                  const Cms* cms = nullptr, bool peek = false) {
  // use_v (LLP with a.LV): labels carry their V, so LLP observes at insert
  // like CLASSIC; otherwise LLP scores from the final table (table_scan)
  const bool obs = VAR != V_LLP || use_v;
  const int lane = threadIdx.x & 31;
  int lab[N];
#pragma unroll
  for (int j = 0; j < N; ++j) lab[j] = labin[j];
  unsigned nfresh = 0;
  // hot candidate: the lane's best so far, else its first label of this batch
  int cand = b.have() ? (int)b.label() : -1;
  int candv = b.have() ? b.bv : -1;
#pragma unroll
  for (int j = N - 1; j >= 0; --j) {
    candv = (cand < 0 && lab[j] >= 0) ? (use_v ? vin[j] : -1) : candv;
    cand = (cand < 0 && lab[j] >= 0) ? lab[j] : cand;
  }
  const int hot = (hot_ok && GLP_MATCH_INSERT != 2) ? __shfl_sync(kFull, cand, 0) : -1;
  const int hotv = __shfl_sync(kFull, candv, 0);
  if (hot >= 0) {  // warp-uniform
    unsigned hc = 0;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      hc += lab[j] == hot ? 1u : 0u;
      lab[j] = lab[j] == hot ? -1 : lab[j];
    }
    const unsigned tot = __reduce_add_sync(kFull, hc);
    if (lane == 0 && tot) {
      const unsigned cnt = ht_add(t, (unsigned)hot, tot, max_probe, &nfresh);
      if (cnt == 0u) {
        if (cms) cms->add((unsigned)hot, tot);  // HT full: the sketch counts it
        else flag_set(overflow);
      } else if (obs) {
        b.observe(cnt, (unsigned)hot, a, hotv);
      }
    }
  }
#if GLP_LEAN && !GLP_MATCH_INSERT
#pragma unroll
  for (int j0 = 0; j0 < N; j0 += 4)
    nfresh += lean_insert4<VAR>(a, t, max_probe, lab[j0], lab[j0 + 1], lab[j0 + 2], lab[j0 + 3], vin[j0], vin[j0 + 1],
                                vin[j0 + 2], vin[j0 + 3], b, overflow, use_v, obs, cms, peek);
#else
  unsigned mc[N];  // occurrences this lane inserts for slot j
#pragma unroll
  for (int j = 0; j < N; ++j) {
    mc[j] = 1u;
    if (GLP_MATCH_INSERT) {
      const unsigned m = __match_any_sync(kFull, lab[j]);
      const bool lead = (m & ((1u << lane) - 1u)) == 0u;
      mc[j] = __popc(m);
      lab[j] = lead ? lab[j] : -1;
    }
  }
  unsigned h[N], k[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    h[j] = slot_hash((unsigned)lab[j], t.tsz);
    k[j] = lab[j] >= 0 ? ld_key(t, h[j]) : 0u;
  }
  unsigned cnt[N];
#pragma unroll
  for (int j = 0; j < N; ++j) cnt[j] = lab[j] >= 0 ? slot_try(t, h[j], (unsigned)lab[j], mc[j], k[j], &nfresh) : 0u;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    if (lab[j] >= 0 && cnt[j] == 0u) {
      cnt[j] = ht_probe_from(t, (unsigned)lab[j], mc[j], h[j], max_probe, &nfresh);
      if (cnt[j] == 0u) {
        if (cms) cms->add((unsigned)lab[j], mc[j]);
        else flag_set(overflow);
      }
    }
  }
  if (obs) {
#pragma unroll
    for (int j = 0; j < N; ++j)
      if (cnt[j]) b.observe(cnt[j], (unsigned)lab[j], a, use_v ? vin[j] : -1);
  }
#endif
  return nfresh;
}

// Predicted distinct labels of a row this iteration (steers the row class and
// table sizes only; overflow always triggers an exact recount).  Labels
// collapse geometrically as communities form [P:130], so the count of t-1 is
// extrapolated with the row's own ratio: p_{t-1}^2 / p_{t-2} (GLP_PRED_EXTRAP).
#ifndef GLP_PRED_EXTRAP
#define GLP_PRED_EXTRAP 1
#endif
// LLP does not converge: with gamma > 0 the labels oscillate with period 2
// (the distinct counts alternate spread / collapsed), so the count of t-2 is
// the prediction (GLP_PRED_LLP 1), or the larger of t-1 and t-2 (2); 0 =
// the converging extrapolation above.
#ifndef GLP_PRED_LLP
#define GLP_PRED_LLP 2  // A/B (0 / 1 / 2): R24 LLP 194.6 / 185.0 / 175.2 ms, R28 LLP 4103 / - / 3860 ms per run
#endif
template <int VAR>
__device__ __forceinline__ unsigned pred_est(unsigned raw, unsigned rawprev, unsigned cap) {
  unsigned p = raw & kPredMask;
  const unsigned q = rawprev & kPredMask;
  if (VAR == V_LLP && GLP_PRED_LLP == 1) p = q > 0 ? q : p;
  else if (VAR == V_LLP && GLP_PRED_LLP == 2) p = max(p, q);
  else if (GLP_PRED_EXTRAP && q > p) p = (unsigned)(((unsigned long long)p * p) / q);
  if (cap) p = min(p, cap);
  return max(p, 1u);
}
// Sorted-row candidate: all labels were distinct last time and the fast path
// has not been tried on them (every row at t = 1); never for SEEDED (R12).
// Only at t = 1: sorted labels come from PickLabel's identity labelling
// [P:68] on sorted rows; a row whose labels were all distinct at t >= 2 is not
// sorted (retrying it cost SBM 0.3 ms at t = 3).
template <int VAR>
__device__ __forceinline__ bool mono_cand(unsigned raw, unsigned cap, int d, int t) {
  const unsigned p = cap ? min(raw & kPredMask, cap) : (raw & kPredMask);
  return VAR != V_SEEDED && t <= 1 && !(raw & kMonoTried) && p >= (unsigned)d;
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
// `scanned` = arcs whose labels were gathered (< deg after a majority exit);
// `deg` feeds the frontier-size estimate (sum of changed degrees).
template <int VAR>
__device__ __forceinline__ void update_vertex(const MflArgs& a, int v, int deg, bool have, unsigned best,
                                              Tally& ty, int scanned) {
  const int64_t gv = a.vb + v;
  const int r = ld_label(a.R + gv);
  int nw = have ? (int)best : r;
  if (VAR == V_SEEDED && a.is_seed[v]) nw = r;  // clamped seed (R12)
  const int2 so = a.so[v];
  const int l2 = (so.x == a.t - 1) ? so.y : r;  // L_{t-2}[v]
  a.W[gv] = nw;
  if (VAR == V_SEEDED && a.lbits_w != nullptr && r < 0 && nw >= 0) atomicOr(a.lbits_w + (gv >> 5), 1u << (gv & 31));
  ty.verts += 1;
  ty.arcs += (unsigned long long)scanned;
  ty.d2 += (nw != l2);
  if (nw != r) {
    ty.changed += 1;
    ty.chdeg += (unsigned long long)deg;
    a.so[v] = make_int2(a.t, r);
  }
}

// ---------------------------------------------------------------------------
// mfl_low: one warp per chunk = floor(32/deg) low-degree vertices of one
// degree `deg`, their arcs filling lanes [j*deg, (j+1)*deg) ("one-warp-multi-
// vertices" [P:227-234 §4.2]).  activemask = lanes holding a valid label;
// vmask = the deg lanes of a vertex; frequency of a lane's label = number of
// vmask lanes with the same label (a shuffle loop of deg steps: match.any.sync
// costs ~60 SM cycles per warp on distinct keys on sm_100, tools/ubench);
// arg-max = two segmented warp reductions (redux.sync over the vmask: max
// count, then min label among the maximal ones; LLP: a shuffle tree over the
// double scores toward the segment head), then lane j updates vertex j.  Loads
// of the next chunk are issued before the current chunk is counted (software
// pipelining across the warp's chunks).  Chunk rows are consecutive internal
// ids, so no vertex table is read.
template <int VAR>
__device__ __forceinline__ void update_vertex_pre(const MflArgs& a, int v, int deg, bool have, unsigned best, int r,
                                                  int2 so, Tally& ty) {
  const int64_t gv = a.vb + v;
  int nw = have ? (int)best : r;
  if (VAR == V_SEEDED && a.is_seed[v]) nw = r;  // clamped seed (R12)
  const int l2 = (so.x == a.t - 1) ? so.y : r;  // L_{t-2}[v]
  a.W[gv] = nw;
  if (VAR == V_SEEDED && a.lbits_w != nullptr && r < 0 && nw >= 0) atomicOr(a.lbits_w + (gv >> 5), 1u << (gv & 31));
  ty.verts += 1;
  ty.arcs += (unsigned long long)deg;
  ty.d2 += (nw != l2);
  if (nw != r) {
    ty.changed += 1;
    ty.chdeg += (unsigned long long)deg;
    a.so[v] = make_int2(a.t, r);
  }
}

// WT: weighted LP (a.w2), a separate instantiation so the unweighted kernel
// carries no weight code
template <int VAR, bool WT = false>
__global__ void __launch_bounds__(kLowBlock) mfl_low(MflArgs a) {
  GLP_CTL_PROLOGUE(a)
  const int lane = threadIdx.x & 31;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  Tally ty;
  // each warp takes 32 consecutive chunks at a time; in sparse iterations the
  // inactive ones are skipped with one coalesced read of their chunk flags
  for (int c0 = gw * 32; c0 < a.n_chunks; c0 += nwarps * 32) {
    const int cl = c0 + lane;
    LowChunk mine;
    mine.st = 0ull; mine.vbase = 0; mine.segmask = 0u;
    bool act = cl < a.n_chunks;
    if (act) {
      mine = a.chunks[cl];
      if (!dense_) act = a.cflag[cl] != 0;
    }
    unsigned todo = __ballot_sync(kFull, act);
    if (!todo) continue;
    // issue the arc and vertex-id loads of chunk j
    // weighted LP (§8(f)3, a.w2): each lane also loads its arc's weight
    auto issue = [&](int j, int& u, int& v, int& total, int& d, unsigned& segs, unsigned& wt) {
      const unsigned long long st = __shfl_sync(kFull, mine.st, j);
      const int vbase = __shfl_sync(kFull, mine.vbase, j);
      segs = __shfl_sync(kFull, mine.segmask, j);
      total = (int)(st >> 56);
      d = (int)((st >> 48) & 0xffull);
      const int64_t start = (int64_t)(st & ((1ull << 48) - 1));
      u = lane < total ? ld_stream(a.col + start + lane) : -1;
      v = lane < __popc(segs) ? (int)(a.low_base + vbase + lane) : -1;
      wt = (WT && lane < total) ? (unsigned)ld_stream((const int32_t*)a.w2 + start + lane) : 1u;
    };
    int j = __ffs(todo) - 1;
    todo &= todo - 1;
    int u, v, total, d;
    unsigned segs, wt;
    issue(j, u, v, total, d, segs, wt);
    for (;;) {
      // prefetch the next chunk while this one is counted
      int nu = -1, nvid = -1, ntotal = 0, nd = 1;
      unsigned nsegs = 0u, nwt = 1u;
      const bool more = todo != 0;
      if (more) {
        const int nj = __ffs(todo) - 1;
        todo &= todo - 1;
        issue(nj, nu, nvid, ntotal, nd, nsegs, nwt);
      }
      // every vertex of the chunk has degree d; nv vertices, lanes [0, total)
      const int nv = __popc(segs);
      int lv;
      int lab = gather_lv(a, u, VAR == V_LLP && a.LV != nullptr, lv);
      int r = 0;
      int2 so = make_int2(0, 0);
      if (lane < nv) {
        r = ld_label(a.R + a.vb + v);
        so = a.so[v];
      }
      const bool vote = lane < total && lab >= 0;
      if (!vote) lab = -1;
      // first lane of this lane's segment (vmask [P:230])
      const int sstart = 31 - __clz(segs & ((2u << lane) - 1u));
      const int head = (lane < nv ? lane * d : 0) & 31;  // lane jv takes segment jv
      Best<VAR> h;
      // Every segment's labels valid and strictly increasing (t = 1's unique
      // labels on sorted rows): all counts are 1, so the MFL is the segment
      // head's label (R4) and nothing needs counting.  CLASSIC/SEEDED at any
      // t; LLP only while V == 1 (equal scores).
      const int up = __shfl_up_sync(kFull, lab, 1);
      const bool inc = lane >= total || (vote && (lane == sstart || up < lab));
      constexpr bool wtd = WT;  // weighted: counts are weight sums (no shortcut, no match.any)
      if ((VAR != V_LLP || a.v_ones) && !wtd && __all_sync(kFull, inc)) {
        const int hl = __shfl_sync(kFull, lab, head);
        h.observe(1u, (unsigned)hl, a, 1);
      } else {
      // label frequency inside the vertex's lanes [P:231-232]
      unsigned k = 0;
      bool first = true;  // LLP: only a label's first lane scores it (one V[l] gather per distinct label)
      if (d >= GLP_LOW_MATCH && !wtd) {
        // long segments: one match.any over the warp, restricted to the
        // segment's lanes (d warp-uniform), instead of d shuffles
        const unsigned segm = d >= 32 ? kFull : (((1u << d) - 1u) << sstart);
        const unsigned m = __match_any_sync(kFull, lab) & segm;
        k = __popc(m);
        if (VAR == V_LLP) first = (m & ((1u << lane) - 1u)) == 0u;
      } else {
#pragma unroll 4
        for (int i = 0; i < d; ++i) {
          const bool eq = __shfl_sync(kFull, lab, sstart + i) == lab;
          const unsigned wi = wtd ? __shfl_sync(kFull, wt, sstart + i) : 1u;
          k += eq ? wi : 0u;
          if (VAR == V_LLP) first = first && !(eq && sstart + i < lane);
        }
      }
      if (VAR == V_LLP || !GLP_LOW_REDUX) {
        Best<VAR> b;
        if (vote && first) b.observe(k, (unsigned)lab, a, lv);
        // segmented arg-max toward the segment head: ceil(log2 d) steps (d is
        // warp-uniform)
        const int send = sstart + d;
        for (int s2 = 1; s2 < d; s2 <<= 1) {
          const unsigned long long ok = __shfl_down_sync(kFull, b.key, s2);
          const unsigned ol = VAR == V_LLP ? __shfl_down_sync(kFull, b.lab, s2) : 0u;
          if (lane + s2 < send) b.merge(ok, ol);
        }
        h.key = __shfl_sync(kFull, b.key, head);
        h.lab = __shfl_sync(kFull, b.lab, head);
      } else {
        // segmented arg-max with two warp reductions over the segment's lanes
        // (max count, then min label among the maximal ones: R4); lanes past
        // the last segment form their own group
        const unsigned segm = lane < total ? (d >= 32 ? kFull : ((1u << d) - 1u) << sstart)
                                           : (kFull << (total & 31));
        const unsigned kmax = __reduce_max_sync(segm, vote ? k : 0u);
        const unsigned lmin = __reduce_min_sync(segm, (vote && k == kmax) ? (unsigned)lab : kNoLabel);
        const unsigned hk = __shfl_sync(kFull, kmax, head);
        const unsigned hl = __shfl_sync(kFull, lmin, head);
        h.key = hk ? (((unsigned long long)hk << 32) | (unsigned long long)(~hl)) : 0ull;
      }
      }  // counted
      if (lane < nv) update_vertex_pre<VAR>(a, v, d, h.have(), h.label(), r, so, ty);
      if (!more) break;
      u = nu;
      v = nvid;
      total = ntotal;
      d = nd;
      segs = nsegs;
      wt = nwt;
    }
  }
  tally_flush(ty, a.cnt);
}

// ---------------------------------------------------------------------------
// Sorted-row fast path.  If the labels of a row, read in arc order, are all
// valid and strictly increasing, every label occurs exactly once: each count is
// 1 and no table is needed (the scores are observed directly).  This is the
// case at t = 1 (unique labels L0[u] = u [P:68]) whenever the CSR rows are
// sorted, and is checked on the data, never assumed.  Rows only try it when
// their predicted distinct count equals their degree.
//
// Lane-local part: labels x[0..3] at arcs idx0..idx0+3 (valid while < d).
__device__ __forceinline__ bool quad_increasing(const int (&x)[4], int idx0, int d) {
  bool ok = true;
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    if (idx0 + k < d) {
      ok &= x[k] >= 0;
      if (k > 0) ok &= x[k - 1] < x[k];
    }
  }
  return ok;
}

// Warp-level check of one 128-arc quad row (lane l holds arcs base+4l..+3);
// `prev` is the label of the arc just before `base` (-1 at the row start).
// Returns the warp-uniform verdict and the last valid label in *last.
__device__ __forceinline__ bool warp_quads_increasing(const int (&x)[4], int base, int d, int prev, int* last) {
  const int lane = threadIdx.x & 31;
  const int idx0 = base + 4 * lane;
  bool ok = quad_increasing(x, idx0, d);
  const int nxt = __shfl_down_sync(kFull, x[0], 1);
  if (lane < 31 && idx0 + 4 < d) ok &= x[3] < nxt;   // lane boundary
  const int first = __shfl_sync(kFull, x[0], 0);
  if (base < d) ok &= prev < first;                   // boundary with the previous quad row
  // last valid label of this quad row
  const int lastidx = min(d, base + 128) - 1 - base;   // >= 0 when base < d
  const int src = max(lastidx, 0) >> 2, k = max(lastidx, 0) & 3;
  const int mine = k == 0 ? x[0] : k == 1 ? x[1] : k == 2 ? x[2] : x[3];
  const int lv = __shfl_sync(kFull, mine, src);
  *last = base < d ? lv : prev;
  return __all_sync(kFull, ok);
}

// ---------------------------------------------------------------------------
// Sort-and-count of one short row held by a warp (<= 128 arcs, 4 per lane:
// element i = 4 * lane + j, the load_round layout).  For rows whose labels are
// mostly distinct (t = 2..3) this replaces ~25 instructions of hash insert
// per label by a bitonic sort in registers (28 compare-exchange stages, 15 of
// them across lanes) plus a run-length scan: the per-row count the paper's
// segmented-sort baseline computes [P:126], kept in registers instead of a
// global neighbour-label array.  Invalid arcs (-1 label, padding) sort last as
// INT_MAX and never vote.  Observes every run (count, label) into b, returns
// this lane's number of runs (distinct labels).
#ifndef GLP_W_SORT
#define GLP_W_SORT 1
#endif
#ifndef GLP_W_PAIR
#define GLP_W_PAIR 1  // rows of <= 64 arcs: two per warp, sort-and-count per half (half_sort_count)
#endif
#ifndef GLP_W_SORT_MAX
#define GLP_W_SORT_MAX 64  // rows up to this many arcs (<= kWRound) take the sort path
                          // A/B (sort 64 / 128 / off): SBM 5.33 / 5.35 / 5.60 ms, R24 17.99 / 17.97 / 18.0-18.4,
                          // R24 LLP 194.7 / 196.7 / 194.1 ms per run
#endif
template <int VAR, int K>
__device__ __forceinline__ unsigned warp_sort_count(int (&v)[K], const MflArgs& a, Best<VAR>& b) {
  constexpr int N = 32 * K;
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int j = 0; j < K; ++j) v[j] = v[j] < 0 ? INT_MAX : v[j];
  // bitonic sort of N keys, ascending in i = K * lane + j
#pragma unroll
  for (int k = 2; k <= N; k <<= 1) {
#pragma unroll
    for (int st = k >> 1; st > 0; st >>= 1) {
      if (st >= K) {
        const int ls = st / K;  // partner lane = lane ^ ls, same j
#pragma unroll
        for (int j = 0; j < K; ++j) {
          const int o = __shfl_xor_sync(kFull, v[j], ls);
          const int i = K * lane + j;
          const bool up = (i & k) == 0;
          const bool low = (lane & ls) == 0;  // this element has the smaller index of the pair
          v[j] = (low == up) ? min(v[j], o) : max(v[j], o);
        }
      } else {
#pragma unroll
        for (int j = 0; j < K; ++j) {
          const int pj = j ^ st;
          if (pj > j) {
            const int i = K * lane + j;
            const bool up = (i & k) == 0;
            const int x = v[j], y = v[pj];
            v[j] = up ? min(x, y) : max(x, y);
            v[pj] = up ? max(x, y) : min(x, y);
          }
        }
      }
    }
  }
  // run starts: element differs from its predecessor
  const int prev_last = __shfl_up_sync(kFull, v[K - 1], 1);
  bool start[K];
  start[0] = v[0] != INT_MAX && (lane == 0 || prev_last != v[0]);
#pragma unroll
  for (int j = 1; j < K; ++j) start[j] = v[j] != INT_MAX && v[j] != v[j - 1];
  // end of each run = position of the next start (or of the first INT_MAX)
  int nvalid = 0;
#pragma unroll
  for (int j = 0; j < K; ++j) nvalid += __popc(__ballot_sync(kFull, v[j] != INT_MAX));
  int first_start = K;
#pragma unroll
  for (int j = K - 1; j >= 0; --j) first_start = start[j] ? j : first_start;
  const unsigned lanes_with = __ballot_sync(kFull, first_start < K);
  const unsigned after = lane < 31 ? (lanes_with >> (lane + 1)) : 0u;
  const int nl = after ? lane + __ffs(after) : 32;             // next lane holding a start
  const int nfs = __shfl_sync(kFull, first_start, nl & 31);  // its first start
  const int next_lane_pos = nl < 32 ? K * nl + nfs : nvalid;
  unsigned distinct = 0;
  int nxt = next_lane_pos;
#pragma unroll
  for (int j = K - 1; j >= 0; --j) {
    if (start[j]) {
      const unsigned cnt = (unsigned)(nxt - (K * lane + j));
      b.observe(cnt, (unsigned)v[j], a);  // LLP: V[l] gathered once per distinct label
      ++distinct;
      nxt = K * lane + j;
    }
  }
  return distinct;  // this lane's runs (the caller reduces over the warp)
}

// Two short rows per warp (GLP_W_PAIR): each half-warp sorts and counts one
// row of <= 64 arcs, 4 per lane (element i = 4 * (lane & 15) + j, the int4
// load layout), with one 64-key bitonic network whose cross-lane stages stay
// inside the half (partner lane ^ st / 4 <= 8): every instruction serves both
// rows ("one-warp-multi-vertices" [P:227-234] for rows past the low bin).
// Invalid arcs (-1, padding) sort last as INT_MAX.  Observes every run
// (count, label) into b (the lane's half), returns the lane's runs.
template <int VAR, int K>
__device__ __forceinline__ unsigned half_sort_count(int (&v)[K], const MflArgs& a, Best<VAR>& b) {
  constexpr int NH = 16 * K;  // keys per half
  const int lane = threadIdx.x & 31, hl = lane & 15;
#pragma unroll
  for (int j = 0; j < K; ++j) v[j] = v[j] < 0 ? INT_MAX : v[j];
#pragma unroll
  for (int k = 2; k <= NH; k <<= 1) {
#pragma unroll
    for (int st = k >> 1; st > 0; st >>= 1) {
      if (st >= K) {
        const int ls = st / K;
#pragma unroll
        for (int j = 0; j < K; ++j) {
          const int o = __shfl_xor_sync(kFull, v[j], ls);
          const int i = K * hl + j;
          const bool up = (i & k) == 0;
          const bool low = (hl & ls) == 0;
          v[j] = (low == up) ? min(v[j], o) : max(v[j], o);
        }
      } else {
#pragma unroll
        for (int j = 0; j < K; ++j) {
          const int pj = j ^ st;
          if (pj > j) {
            const int i = K * hl + j;
            const bool up = (i & k) == 0;
            const int x = v[j], y = v[pj];
            v[j] = up ? min(x, y) : max(x, y);
            v[pj] = up ? max(x, y) : min(x, y);
          }
        }
      }
    }
  }
  const unsigned half = lane < 16 ? 0x0000ffffu : 0xffff0000u;
  const int prev_last = __shfl_up_sync(kFull, v[K - 1], 1);
  bool start[K];
  start[0] = v[0] != INT_MAX && (hl == 0 || prev_last != v[0]);
#pragma unroll
  for (int j = 1; j < K; ++j) start[j] = v[j] != INT_MAX && v[j] != v[j - 1];
  int nvalid = 0;
#pragma unroll
  for (int j = 0; j < K; ++j) nvalid += __popc(__ballot_sync(kFull, v[j] != INT_MAX) & half);
  int first_start = K;
#pragma unroll
  for (int j = K - 1; j >= 0; --j) first_start = start[j] ? j : first_start;
  const unsigned with = __ballot_sync(kFull, first_start < K) & half;
  const unsigned after = lane < 31 ? (with >> (lane + 1)) << (lane + 1) : 0u;  // later lanes of the half
  const int nl = after ? __ffs(after) - 1 : -1;                                 // next lane holding a start
  const int nfs = __shfl_sync(kFull, first_start, nl < 0 ? lane : nl);
  const int base = K * hl;
  int nxt = nl >= 0 ? K * (nl & 15) + nfs : nvalid;
  unsigned distinct = 0;
#pragma unroll
  for (int j = K - 1; j >= 0; --j) {
    if (start[j]) {
      b.observe((unsigned)(nxt - (base + j)), (unsigned)v[j], a);
      ++distinct;
      nxt = base + j;
    }
  }
  return distinct;
}

// ---------------------------------------------------------------------------
// mfl_warp: one warp per row of class W (few distinct labels): per-warp shared
// table of pow2 >= 4*pred slots (<= 512), one 128-bit load per lane per
// round (128 arcs per warp; 256-arc rounds measured 2 % slower: most W rows
// have < 128 arcs, and the smaller round frees registers for a 4th block per
// SM), no block barriers.  Rows whose labels overflow the
// table are re-queued to the block kernel M.
//   * 32 rows per warp at a time: the class / frontier test of the batch is
//     lane-parallel; rows are degree-sorted, so a warp's batch is strided
//     across the list (lane l of warp w takes row base + l * nwarps + w);
//   * software pipeline: the arcs of the next round -- of this row, or the
//     first round of the next selected row -- are loaded while the current
//     round is gathered and counted;
//   * lane j keeps the result of batch row j, and the batch's vertices are
//     updated lane-parallel at the end.
#ifndef GLP_W_ROUND
#define GLP_W_ROUND 128
#endif
constexpr int kWRound = GLP_W_ROUND;  // arcs per warp round: 256 (two 128-bit loads per lane) or 128
__device__ __forceinline__ void load_round(const int32_t* col, int64_t start, int off, int d, int4& u0, int4& u1) {
  const int lane = threadIdx.x & 31;
  u0 = make_int4(-1, -1, -1, -1);
  u1 = u0;
  if (off + 4 * lane < d) u0 = ld_stream4(col + start + off + 4 * lane);
  if (kWRound == 256 && off + 128 + 4 * lane < d) u1 = ld_stream4(col + start + off + 128 + 4 * lane);
}

#ifndef GLP_W_MINB
#define GLP_W_MINB 4
#endif
// MINB: resident blocks per SM.  4 (64 registers, the pair path spills) by
// default; 3 (no spills) when most arcs of the deg > 32 rows are in rows of
// <= 64 arcs (glp_graph::w_short: SBM -6 %, while R24 / LLP lose 1.3 % at 3)
template <int VAR, int MINB = GLP_W_MINB>
__global__ void __launch_bounds__(kWBlock, MINB) mfl_warp(MflArgs a) {
  GLP_CTL_PROLOGUE(a)
  extern __shared__ __align__(16) unsigned long long wtabs[];  // [kWBlock / 32][kWSlots] (dynamic)
  __shared__ int s_over[kWBlock / 32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  Tally ty;
  for (int base = 0; base < a.n_items; base += nwarps * 32) {
    const int il = base + lane * nwarps + gw;
    BinItem mine;
    mine.start = 0; mine.v = 0; mine.d = 0;
    unsigned mpred = 0;
    bool ok = il < a.n_items;
    if (ok) {
      mine = a.items[il];
      const unsigned raw = a.pred[il];
      // in this kernel bit 31 of mpred marks a sorted-row candidate
      const bool cand = mono_cand<VAR>(raw, a.pred_cap, mine.d, a.t);
      mpred = pred_est<VAR>(raw, a.pred_prev[il], a.pred_cap) | (cand ? kMonoTried : 0u);
      ok = row_class(mpred & kPredMask, mine.d, cand, a.mono_kernel) == CLS_W;
      if (ok && !dense_ && !a.flag[a.vb + mine.v]) {
        ok = false;
        a.pred_next[il] = raw;  // inactive: carry the prediction forward
      }
    }
    unsigned todo = __ballot_sync(kFull, ok);
    if (!todo) continue;
    // per-lane result of batch row `lane`
    bool rdone = false;
    unsigned long long rkey = 0ull;
    unsigned rlab = kNoLabel, rpred = 0u;
    int rscan = 0;
    // rows of <= 64 (<= 128: GLP_W_PAIR 2) arcs, not sorted-row candidates:
    // two per warp, one per half, sort-and-count (half_sort_count)
    auto pair_pass = [&](auto kc) {
      constexpr int K = decltype(kc)::value;
      unsigned shortm =
          __ballot_sync(kFull, ok && mine.d <= 16 * K && mine.d > (K == 4 ? 0 : 64) && !(mpred & kMonoTried)) & todo;
      todo &= ~shortm;
      const int hl = lane & 15;
      // pop the next pair of rows (ja: lower half, jb: upper half; -1: none)
      auto pop = [&](int& ja, int& jb) {
        ja = shortm ? __ffs(shortm) - 1 : -1;
        if (ja >= 0) shortm &= shortm - 1;
        jb = shortm ? __ffs(shortm) - 1 : -1;
        if (jb >= 0) shortm &= shortm - 1;
      };
      // the arcs of this lane's half of a pair (every lane shuffles)
      auto load_pair = [&](int ja, int jb, int4 (&u)[K / 4]) {
        const int jm = lane < 16 ? ja : jb;
        const int64_t st = __shfl_sync(kFull, mine.start, jm < 0 ? 0 : jm);
        const int dsrc = __shfl_sync(kFull, mine.d, jm < 0 ? 0 : jm);
        const int dd = jm < 0 ? 0 : dsrc;
#pragma unroll
        for (int q = 0; q < K / 4; ++q)
          u[q] = K * hl + 4 * q < dd ? ld_stream4(a.col + st + K * hl + 4 * q) : make_int4(-1, -1, -1, -1);
      };
      auto gather_pair = [&](const int4 (&u)[K / 4], int (&v)[K]) {
#pragma unroll
        for (int q = 0; q < K / 4; ++q) {
          v[4 * q] = gather(a, u[q].x); v[4 * q + 1] = gather(a, u[q].y);
          v[4 * q + 2] = gather(a, u[q].z); v[4 * q + 3] = gather(a, u[q].w);
        }
      };
      // the arcs of pair p+1 are loaded ahead (a software pipeline that also
      // gathered pair p+1's labels during pair p's sort measured no gain)
      int ja0, jb0, ja1, jb1;
      int4 u0[K / 4], u1[K / 4];
      int v0[K];
      pop(ja0, jb0);
      load_pair(ja0, jb0, u0);
      gather_pair(u0, v0);
      pop(ja1, jb1);
      load_pair(ja1, jb1, u1);
      while (ja0 >= 0) {
        int ja2, jb2;
        int4 u2[K / 4];
        int v1[K];
        Best<VAR> b;
        unsigned fr = half_sort_count<VAR, K>(v0, a, b);
#pragma unroll
        for (int s2 = 8; s2 > 0; s2 >>= 1) {  // reduce within the half
          const unsigned long long k2 = __shfl_xor_sync(kFull, b.key, s2);
          const unsigned l2 = VAR == V_LLP ? __shfl_xor_sync(kFull, b.lab, s2) : 0u;
          b.merge(k2, l2);
          fr += __shfl_xor_sync(kFull, fr, s2);
        }
        const unsigned long long ka = __shfl_sync(kFull, b.key, 0), kb = __shfl_sync(kFull, b.key, 16);
        const unsigned la = __shfl_sync(kFull, b.lab, 0), lb = __shfl_sync(kFull, b.lab, 16);
        const unsigned fa = __shfl_sync(kFull, fr, 0), fb = __shfl_sync(kFull, fr, 16);
        if (lane == ja0 || lane == jb0) {
          const bool isa = lane == ja0;
          rdone = true;
          rkey = isa ? ka : kb;
          rlab = isa ? la : lb;
          rscan = mine.d;
          rpred = max(isa ? fa : fb, 1u);
        }
        pop(ja2, jb2);
        load_pair(ja2, jb2, u2);
        gather_pair(u1, v1);
        ja0 = ja1; jb0 = jb1; ja1 = ja2; jb1 = jb2;
#pragma unroll
        for (int q = 0; q < K; ++q) v0[q] = v1[q];
#pragma unroll
        for (int q = 0; q < K / 4; ++q) u1[q] = u2[q];
      }
    };
    if (GLP_W_PAIR >= 1) pair_pass(std::integral_constant<int, 4>());
    if (GLP_W_PAIR >= 2) pair_pass(std::integral_constant<int, 8>());
    if (!todo) {
      if (rdone) {
        Best<VAR> r;
        r.key = rkey;
        r.lab = rlab;
        a.pred_next[il] = rpred;
        update_vertex<VAR>(a, mine.v, mine.d, r.have(), r.label(), ty, rscan);
      }
      continue;
    }
    int jl = __ffs(todo) - 1;
    todo &= todo - 1;
    int64_t start = __shfl_sync(kFull, mine.start, jl);
    int d = __shfl_sync(kFull, mine.d, jl);
    unsigned pred = __shfl_sync(kFull, mpred, jl);
    int4 x0, x1;
    load_round(a.col, start, 0, d, x0, x1);
    for (;;) {
      // the next selected row of the batch (its first round is prefetched)
      const int njl = todo ? __ffs(todo) - 1 : -1;
      if (todo) todo &= todo - 1;
      int64_t nstart = 0;
      int nd = 0;
      unsigned npred = 0u;
      if (njl >= 0) {
        nstart = __shfl_sync(kFull, mine.start, njl);
        nd = __shfl_sync(kFull, mine.d, njl);
        npred = __shfl_sync(kFull, mpred, njl);
      }
      const unsigned tsz =
          min(max(64u, 1u << (32 - __clz(GLP_W_LOAD * max(pred & kPredMask, 1u) - 1u))), (unsigned)kWSlots);
      const Table tab{wtabs + (size_t)wid * kWSlots, tsz};
      // rows of <= 128 arcs predicted mostly distinct: sort-and-count, no table
      const bool wsort = GLP_W_SORT && d <= GLP_W_SORT_MAX && !(pred & kMonoTried) && 4u * (pred & kPredMask) > (unsigned)d;
      if (!wsort) tab.clear(lane, 32);
      if (lane == 0) s_over[wid] = 0;
      __syncwarp();
      Best<VAR> b;
      unsigned fresh = 0;
      bool over = false;
      bool mono = (pred & kMonoTried) != 0;  // sorted-row candidate
      const bool tried = mono;
      int prev = -1;
      bool next_loaded = false;  // x0/x1 hold the next row's first round
      bool major = false;        // a strict-majority label was observed: the rest of the row cannot change the MFL
      int scanned = 0;           // arcs gathered so far
      const bool hot = hot_pass(pred & kPredMask, d);
      const bool pk = peek_pass<VAR>(pred & kPredMask, d);
      for (int off = 0; off < d && !over && !major; off += kWRound) {
        scanned = min(d, off + kWRound);
        int4 p0, p1;
        if (off + kWRound < d) {
          load_round(a.col, start, off + kWRound, d, p0, p1);
        } else {
          load_round(a.col, nstart, 0, nd, p0, p1);  // nd == 0: no loads
          next_loaded = true;
        }
        int l[8], lv[8];
        const bool use_v = VAR == V_LLP && a.LV != nullptr;
        l[0] = gather_lv(a, x0.x, use_v, lv[0]); l[1] = gather_lv(a, x0.y, use_v, lv[1]);
        l[2] = gather_lv(a, x0.z, use_v, lv[2]); l[3] = gather_lv(a, x0.w, use_v, lv[3]);
        lv[4] = lv[5] = lv[6] = lv[7] = -1;
        if (kWRound == 256) {
          l[4] = gather(a, x1.x); l[5] = gather(a, x1.y); l[6] = gather(a, x1.z); l[7] = gather(a, x1.w);
        } else {
          l[4] = l[5] = l[6] = l[7] = -1;
        }
        x0 = p0;
        x1 = p1;
        if (mono) {
          const int q0[4] = {l[0], l[1], l[2], l[3]}, q1[4] = {l[4], l[5], l[6], l[7]};
          int mid = -1, end = -1;
          bool okm = warp_quads_increasing(q0, off, d, prev, &mid);
          if (kWRound == 256) okm = okm && warp_quads_increasing(q1, off + 128, d, mid, &end);
          else end = mid;
          if (okm) {  // every label of this round occurs once in the row so far
#pragma unroll
            for (int j = 0; j < 8; ++j)
              if (l[j] >= 0) { b.observe(1u, (unsigned)l[j], a, lv[j]); ++fresh; }
            prev = end;
            continue;
          }
          // not sorted: count this row with the table, re-inserting the rounds
          // already observed (their count-1 observations stay valid lower bounds)
          mono = false;
          fresh = 0;
          for (int b2 = 0; b2 < off; b2 += kWRound) {
            int4 v0, v1;
            load_round(a.col, start, b2, d, v0, v1);
            int m8[8], mv8[8];
            m8[0] = gather_lv(a, v0.x, use_v, mv8[0]); m8[1] = gather_lv(a, v0.y, use_v, mv8[1]);
            m8[2] = gather_lv(a, v0.z, use_v, mv8[2]); m8[3] = gather_lv(a, v0.w, use_v, mv8[3]);
            m8[4] = gather_lv(a, v1.x, use_v, mv8[4]); m8[5] = gather_lv(a, v1.y, use_v, mv8[5]);
            m8[6] = gather_lv(a, v1.z, use_v, mv8[6]); m8[7] = gather_lv(a, v1.w, use_v, mv8[7]);
            fresh += warp_insert_n<VAR, 8>(a, tab, kTabProbe, m8, b, &s_over[wid], mv8, use_v, hot, nullptr, pk);
          }
        }
        if (wsort) {  // the whole row is this round (d <= kWRound)
          if (d <= 64) {
            // 2 per lane: lane L takes arcs 2L, 2L+1 from lane L/2's quad
            const int src = lane >> 1;
            const int q0 = __shfl_sync(kFull, l[0], src), q1 = __shfl_sync(kFull, l[1], src);
            const int q2 = __shfl_sync(kFull, l[2], src), q3 = __shfl_sync(kFull, l[3], src);
            int l2[2] = {(lane & 1) ? q2 : q0, (lane & 1) ? q3 : q1};
            fresh = warp_sort_count<VAR, 2>(l2, a, b);
          } else {
            int l4[4] = {l[0], l[1], l[2], l[3]};
            fresh = warp_sort_count<VAR, 4>(l4, a, b);
          }
          break;
        }
        if (kWRound == 256 && d - off > 128) {  // warp-uniform
          fresh += warp_insert_n<VAR, 8>(a, tab, kTabProbe, l, b, &s_over[wid], lv, use_v, hot, nullptr, pk);
        } else {
          const int l4[4] = {l[0], l[1], l[2], l[3]};
          const int v4[4] = {lv[0], lv[1], lv[2], lv[3]};
          fresh += warp_insert_n<VAR, 4>(a, tab, kTabProbe, l4, b, &s_over[wid], v4, use_v, hot, nullptr, pk);
        }
        __syncwarp();
        over = warp_flag(&s_over[wid]);
        if (GLP_MAJORITY && VAR != V_LLP && !over && off + kWRound < d) major = strict_majority(b, d);
      }
      if ((over || major) && !next_loaded) load_round(a.col, nstart, 0, nd, x0, x1);
      if (over) {
        if (lane == 0) a.redo_out[atomicAdd(a.redo_out_n, 1u)] = base + jl * nwarps + gw;
      } else {
        if (a.LV == nullptr && !wsort) table_scan<VAR>(tab, lane, 32, a, b);  // LLP (s_over's __syncwarp ended the count)
        b.warp_reduce();
        fresh = __reduce_add_sync(kFull, fresh);
        if (lane == jl) {
          rdone = true;
          rkey = b.key;
          rlab = b.lab;
          rscan = scanned;
          // a row that just took the sorted fast path is not retried next time
          // (a majority exit saw part of the row: keep the old prediction if larger)
          rpred = max(major ? max(fresh, pred & kPredMask) : fresh, 1u) | (tried && mono ? kMonoTried : 0u);
        }
      }
      __syncwarp();
      if (njl < 0) break;
      jl = njl;
      start = nstart;
      d = nd;
      pred = npred;
    }
    if (rdone) {
      Best<VAR> r;
      r.key = rkey;
      r.lab = rlab;
      a.pred_next[il] = rpred;
      update_vertex<VAR>(a, mine.v, mine.d, r.have(), r.label(), ty, rscan);
    }
  }
  tally_flush(ty, a.cnt);
}

// ---------------------------------------------------------------------------
// mfl_mono: the sorted-row fast path alone (t = 1: unique labels L0[u] = u
// [P:68]), without the W kernel's shared tables, so it runs at full occupancy
// with two rounds of label gathers in flight per lane (the path is bound by
// gather latency, not by counting).  One warp per sorted-row candidate of at
// most kMonoWMax arcs; a row whose labels turn out not to be strictly
// increasing (unsorted input rows, repeated arcs) is re-queued to the M
// kernel's redo list, which counts it exactly.
#ifndef GLP_MONO_MINB
#define GLP_MONO_MINB 6
#endif
constexpr int kMonoBlock = 256;
template <int VAR>
__global__ void __launch_bounds__(kMonoBlock, GLP_MONO_MINB) mfl_mono(MflArgs a) {
  GLP_CTL_PROLOGUE(a)
  const int lane = threadIdx.x & 31;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  Tally ty;
  for (int base = 0; base < a.n_items; base += nwarps * 32) {
    const int il = base + lane * nwarps + gw;
    BinItem mine;
    mine.start = 0; mine.v = 0; mine.d = 0;
    bool ok = il < a.n_items;
    if (ok) {
      mine = a.items[il];
      const unsigned raw = a.pred[il];
      ok = mono_cand<VAR>(raw, a.pred_cap, mine.d, a.t) &&
           row_class(raw & kPredMask, mine.d, true, true) == CLS_MONO;
      if (ok && !dense_ && !a.flag[a.vb + mine.v]) {
        ok = false;
        a.pred_next[il] = raw;
      }
    }
    unsigned todo = __ballot_sync(kFull, ok);
    bool rdone = false;
    unsigned long long rkey = 0ull;
    unsigned rlab = kNoLabel, rpred = 0u;
    while (todo) {
      const int jl = __ffs(todo) - 1;
      todo &= todo - 1;
      const int64_t start = __shfl_sync(kFull, mine.start, jl);
      const int d = __shfl_sync(kFull, mine.d, jl);
      Best<VAR> b;
      unsigned fresh = 0;
      int prev = -1;
      bool sorted = true;
      // round r's labels in l[], round r+1's gathers in flight in nl[]
      int4 x = make_int4(-1, -1, -1, -1);
      if (4 * lane < d) x = ld_stream4(a.col + start + 4 * lane);
      int l[4] = {gather(a, x.x), gather(a, x.y), gather(a, x.z), gather(a, x.w)};
      for (int off = 0; off < d; off += 128) {
        int nl[4] = {-1, -1, -1, -1};
        if (off + 128 < d) {
          int4 y = make_int4(-1, -1, -1, -1);
          if (off + 128 + 4 * lane < d) y = ld_stream4(a.col + start + off + 128 + 4 * lane);
          nl[0] = gather(a, y.x); nl[1] = gather(a, y.y); nl[2] = gather(a, y.z); nl[3] = gather(a, y.w);
        }
        int end = -1;
        if (!warp_quads_increasing(l, off, d, prev, &end)) {
          sorted = false;
          break;
        }
#pragma unroll
        for (int j = 0; j < 4; ++j)
          if (l[j] >= 0) { b.observe(1u, (unsigned)l[j], a); ++fresh; }  // (t = 1: V == 1, v_ones)
        prev = end;
#pragma unroll
        for (int j = 0; j < 4; ++j) l[j] = nl[j];
      }
      if (!sorted) {
        if (lane == 0) a.redo_out[atomicAdd(a.redo_out_n, 1u)] = base + jl * nwarps + gw;
        continue;
      }
      b.warp_reduce();
      fresh = __reduce_add_sync(kFull, fresh);
      if (lane == jl) {
        rdone = true;
        rkey = b.key;
        rlab = b.lab;
        rpred = max(fresh, 1u) | kMonoTried;
      }
    }
    if (rdone) {
      Best<VAR> r;
      r.key = rkey;
      r.lab = rlab;
      a.pred_next[il] = rpred;
      update_vertex<VAR>(a, mine.v, mine.d, r.have(), r.label(), ty, mine.d);
    }
  }
  tally_flush(ty, a.cnt);
}

// ---------------------------------------------------------------------------
// Block-per-vertex counting of one row into `tab` (UNROLL 128-bit loads per
// thread in flight).  Only labels of hash partition `part` of `nparts` vote
// (multi-pass counting of rows with more distinct labels than the table
// holds).  Stops early (warp-uniformly) once a label overflowed.
__device__ __forceinline__ unsigned label_part(unsigned lab, unsigned nparts) {
  return __umulhi(lab * 0x85EBCA77u + 0x165667B1u, nparts);
}

// Round `base` of a row for the block kernels: UNROLL 128-bit loads per thread.
template <int BLOCK, int UNROLL>
__device__ __forceinline__ void block_load_round(const int32_t* col, int64_t start, int d, int base,
                                                 int4 (&u)[UNROLL]) {
#pragma unroll
  for (int j = 0; j < UNROLL; ++j) {
    const int idx = base + (j * BLOCK + (int)threadIdx.x) * 4;
    u[j] = idx < d ? ld_stream4(col + start + idx) : make_int4(-1, -1, -1, -1);
  }
}

// `u` holds round 0 of the row (loaded ahead by the caller); each round loads
// the next one before gathering its own labels.
// IPF = false: rounds after the first are loaded in place (register-capped L).
template <int VAR, int BLOCK, int UNROLL, bool IPF>
__device__ __forceinline__ void block_count(const MflArgs& a, int64_t start, int d, const Table& tab,
                                            unsigned max_probe, int4 (&u)[UNROLL], int32_t* stage_out,
                                            volatile int* overflow, int* distinct, Best<VAR>& b,
                                            volatile int* major, unsigned fparts = 1u, int* scanned = nullptr,
                                            bool hot = true, const Cms* cms = nullptr, bool peek = false) {
  constexpr int STEP = BLOCK * 4 * UNROLL;
  unsigned fresh = 0;
  int base = 0;
  for (; base < d; base += STEP) {
    int4 un[UNROLL];
    if (!IPF && base > 0) block_load_round<BLOCK, UNROLL>(a.col, start, d, base, u);
    if (IPF) block_load_round<BLOCK, UNROLL>(a.col, start, d, base + STEP, un);
    int lab[4 * UNROLL], lv[4 * UNROLL];
    const bool use_v = VAR == V_LLP && a.LV != nullptr;
#pragma unroll
    for (int j = 0; j < UNROLL; ++j) {
      lab[4 * j + 0] = gather_lv(a, u[j].x, use_v, lv[4 * j + 0]);
      lab[4 * j + 1] = gather_lv(a, u[j].y, use_v, lv[4 * j + 1]);
      lab[4 * j + 2] = gather_lv(a, u[j].z, use_v, lv[4 * j + 2]);
      lab[4 * j + 3] = gather_lv(a, u[j].w, use_v, lv[4 * j + 3]);
      const int idx = base + (j * BLOCK + (int)threadIdx.x) * 4;
      if (stage_out != nullptr && idx < d)
        __stcg((int4*)(stage_out + idx), make_int4(lab[4 * j], lab[4 * j + 1], lab[4 * j + 2], lab[4 * j + 3]));
    }
    if (fparts > 1u) {  // filtered count: only labels of hash partition 0 vote (the row is staged whole)
#pragma unroll
      for (int k = 0; k < 4 * UNROLL; ++k)
        lab[k] = (lab[k] >= 0 && label_part((unsigned)lab[k], fparts) == 0u) ? lab[k] : -1;
    }
    if (IPF) {
#pragma unroll
      for (int j = 0; j < UNROLL; ++j) u[j] = un[j];
    }
    fresh += warp_insert_n<VAR, 4 * UNROLL>(a, tab, max_probe, lab, b, overflow, lv, use_v, hot, cms, peek);
    if (GLP_MAJORITY && VAR != V_LLP && major != nullptr && base + STEP < d) {
      // a strict-majority observation ends the row for every warp (they poll the flag)
      const bool m = strict_majority(b, d);
      if (m && (threadIdx.x & 31) == 0) flag_set(major);
      if (m || warp_flag(major)) break;
    }
    if (warp_flag(overflow)) break;  // warp-uniform exit
  }
  fresh = __reduce_add_sync(kFull, fresh);
  if ((threadIdx.x & 31) == 0) {
    if (fresh) atomicAdd(distinct, (int)fresh);
    // arcs this warp gathered: rounds up to the one it stopped in
    if (scanned != nullptr) atomicMax(scanned, min(d, base + STEP));
  }
}

// Block-level sorted-row fast path (see warp_quads_increasing): rounds of
// UNROLL 128-bit loads per thread (the block_load_round layout; `u` holds round
// 0, loaded ahead by the caller, and each round loads the next before
// gathering).  A round is a sequence of 128-arc quad rows q = j*NW + warp; each
// warp checks its own, then warp 0 checks the NW*UNROLL boundaries between
// consecutive quad rows lane-parallel.  Returns the block-uniform verdict; on
// success every label has been observed with count 1 and *fresh counts them.
template <int VAR, int BLOCK, int UNROLL>
__device__ __forceinline__ bool block_mono(const MflArgs& a, int64_t start, int d, int4 (&u)[UNROLL], Best<VAR>& b,
                                           unsigned* fresh) {
  constexpr int NW = BLOCK / 32, NQ = NW * UNROLL, STEP = 4 * BLOCK * UNROLL;
  __shared__ int s_first[NQ], s_last[NQ], s_ok, s_prev;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int prev_round = -1;
  for (int base = 0; base < d; base += STEP) {
    int4 un[UNROLL];
    block_load_round<BLOCK, UNROLL>(a.col, start, d, base + STEP, un);
    int x[UNROLL][4];
#pragma unroll
    for (int j = 0; j < UNROLL; ++j) {
      x[j][0] = gather(a, u[j].x); x[j][1] = gather(a, u[j].y); x[j][2] = gather(a, u[j].z);
      x[j][3] = gather(a, u[j].w);
      u[j] = un[j];
    }
    bool okw = true;
#pragma unroll
    for (int j = 0; j < UNROLL; ++j) {
      const int wb = base + j * 4 * BLOCK + 128 * wid;
      int lastw = -1;
      okw &= warp_quads_increasing(x[j], wb, d, INT_MIN, &lastw);
      if (lane == 0) {
        s_first[j * NW + wid] = x[j][0];
        s_last[j * NW + wid] = lastw;
      }
    }
    const int ok_all = __syncthreads_and(okw ? 1 : 0);
    if (wid == 0) {
      const int nq = min(NQ, (d - base + 127) / 128);  // quad rows holding arcs
      bool ok = ok_all != 0;
      for (int q = lane; q < nq; q += 32) ok &= (q == 0 ? prev_round : s_last[q - 1]) < s_first[q];
      ok = __all_sync(kFull, ok);
      if (lane == 0) {
        s_ok = ok ? 1 : 0;
        s_prev = s_last[nq - 1];
      }
    }
    __syncthreads();
    if (!s_ok) return false;
    prev_round = s_prev;
#pragma unroll
    for (int j = 0; j < UNROLL; ++j) {
      const int wb = base + j * 4 * BLOCK + 128 * wid;
#pragma unroll
      for (int k = 0; k < 4; ++k)
        if (wb + 4 * lane + k < d) { b.observe(1u, (unsigned)x[j][k], a); ++*fresh; }  // (V gathered: t = 1 has v_ones)
    }
  }
  return true;
}

template <int VAR, int BLOCK>
__device__ __forceinline__ Best<VAR> block_best(Best<VAR> b) {
  __shared__ unsigned long long rk[BLOCK / 32];
  __shared__ unsigned rl[BLOCK / 32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  b.warp_reduce();
  if (lane == 0) { rk[wid] = b.key; rl[wid] = b.lab; }
  __syncthreads();
  if (wid == 0) {
    Best<VAR> x;
    if (lane < BLOCK / 32) { x.key = rk[lane]; x.lab = rl[lane]; }
    x.warp_reduce();
    b = x;
  }
  return b;  // valid in thread 0
}

// Count the labels lab[off .. off + cnt) of stage (one hash partition of a
// huge row) into `tab`; every non-negative label votes.
template <int VAR, int BLOCK>
__device__ __forceinline__ void count_staged(const MflArgs& a, const int32_t* stage, int cnt, const Table& tab,
                                             unsigned max_probe, volatile int* overflow, int* distinct,
                                             Best<VAR>& b, unsigned fparts = 1u, unsigned part = 0u) {
  unsigned fresh = 0;
  for (int j0 = 0; j0 < cnt; j0 += 4 * BLOCK) {
    int lab[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int j = j0 + k * BLOCK + (int)threadIdx.x;
      lab[k] = j < cnt ? __ldcg(stage + j) : -1;
      // filtered count: only labels of hash partition `part` of `fparts` vote
      if (fparts > 1u && lab[k] >= 0 && label_part((unsigned)lab[k], fparts) != part) lab[k] = -1;
    }
    const int nov[4] = {-1, -1, -1, -1};
    fresh += warp_insert_n<VAR, 4>(a, tab, max_probe, lab, b, overflow, nov, false, GLP_HOT_DIV == 0);
    if (warp_flag(overflow)) break;
  }
  fresh = __reduce_add_sync(kFull, fresh);
  if ((threadIdx.x & 31) == 0 && fresh) atomicAdd(distinct, (int)fresh);
}

// Linear-probe lookup (post-count, read only): is l in the HT?
__device__ __forceinline__ bool ht_has(const Table& t, unsigned l, unsigned max_probe) {
  unsigned h = slot_hash(l, t.tsz);
  for (unsigned p = 0; p < max_probe; ++p) {
    const unsigned k = t.key[h];
    if (k == l) return true;
    if (k == kFree) return false;
    h = (h + 1) & (t.tsz - 1);
  }
  return false;
}

// Block-wide max of a u64 key (every thread gets it).
template <int BLOCK>
__device__ __forceinline__ unsigned long long block_max_u64(unsigned long long x) {
  __shared__ unsigned long long red[BLOCK / 32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) x = max(x, __shfl_xor_sync(kFull, x, s));
  __syncthreads();
  if (lane == 0) red[wid] = x;
  __syncthreads();
  unsigned long long y = 0;
  for (int w = 0; w < BLOCK / 32; ++w) y = max(y, red[w]);
  return y;
}

// HT + CMS count of one L row (§8(f)2).  The shared table region holds the HT
// (a.cms_ht slots, default all SLOTS) and, after it, the sketch counters.
// Returns true when the HT's best is the row's MFL (b then holds it in the
// usual running-max form); false when the row must be recounted exactly.
// Decision, all post-barrier (R15):
//   1. no label reached the sketch: the HT holds every label (exact);
//   2. a strict majority was observed in the HT: it is the MFL;
//   3. s(HT) > bound, bound = min over rows of the row's largest counter (an
//      upper bound of every sketch label's count) -- no rescan;
//   4. s(HT) > s(CMS) = max over sketch labels of their estimate g(l) =
//      min_i C[i][h_i(l)] (Lemma 2's quantity), found by rescanning the row
//      for labels not in the HT;
//   else fallback.  Scores compare strictly: a sketch label tying the HT's
//   best could be smaller (min-label ties, R4).  Stats go to cnt->pad0
//   (rows that used the sketch), pad[0] (rescans), pad[1] (fallbacks).
template <int VAR, int BLOCK, int SLOTS, int UNROLL>
__device__ __forceinline__ bool cms_count(const MflArgs& a, int64_t start, int d, int4 (&cur)[UNROLL], Best<VAR>& b,
                                          volatile int* s_over, int* s_distinct, volatile int* s_major, int* s_scan,
                                          bool hot) {
  extern __shared__ __align__(16) unsigned long long smem_tab[];
  __shared__ int s_used;
  const unsigned hs = a.cms_ht ? min((unsigned)SLOTS, 1u << (31 - __clz(max(a.cms_ht, 2u)))) : (unsigned)SLOTS;
  const Table tab{smem_tab, hs};
  const unsigned depth = min(max(a.cms_depth, 1u), 8u);
  const unsigned width = kCmsCounters / depth;
  unsigned* ctr = (unsigned*)(smem_tab + SLOTS);
  const Cms cm{ctr, depth, width, &s_used};
  tab.clear(threadIdx.x, BLOCK);
  for (unsigned j = threadIdx.x; j < kCmsCounters / 4; j += BLOCK) ((uint4*)ctr)[j] = make_uint4(0u, 0u, 0u, 0u);
  if (threadIdx.x == 0) s_used = 0;
  __syncthreads();
  // the probe limit marks an HT insertion as failed (chain full); with a tiny
  // HT (a.cms_ht) it is "the HT is full" of the paper
  block_count<VAR, BLOCK, UNROLL, GLP_L_IPF>(a, start, d, tab, kLProbe, cur, nullptr, s_over, s_distinct, b, s_major,
                                             1u, s_scan, hot, &cm);
  __syncthreads();
  if (a.LV == nullptr) table_scan<VAR>(tab, threadIdx.x, BLOCK, a, b);  // LLP without carried V
  if (s_used == 0) return true;
  Counters* st = a.cnt;
  if (threadIdx.x == 0) atomicAdd(&st->pad0, 1ull);
  if (*s_major) return true;  // (never set for LLP)
  // s(HT) as an order-preserving key: CLASSIC/SEEDED count<<32 | ~label,
  // LLP dkey(score)
  Best<VAR> hb = b;
  hb.warp_reduce();
  const unsigned long long hkey = block_max_u64<BLOCK>(hb.key);
  // 3. cheap bound
  unsigned long long rowmin = ~0ull;
  for (unsigned i = 0; i < depth; ++i) {
    unsigned m = 0;
    for (unsigned j = threadIdx.x; j < width; j += BLOCK) m = max(m, ctr[i * width + j]);
    rowmin = min(rowmin, block_max_u64<BLOCK>(m));
  }
  auto score_key = [&](unsigned g, int v) -> unsigned long long {
    // the best key a sketch label with count <= g and histogram v could reach
    if (VAR == V_LLP) return dkey(llp_score(g, v, a.gamma));
    return ((unsigned long long)g << 32) | 0xffffffffull;  // (label 0: the strongest tie-break)
  };
  const unsigned long long hcmp = VAR == V_LLP ? hkey : (hkey | 0xffffffffull);  // compare counts only
  // LLP: V[l] >= 1 for a present label, and the score falls with V
  if (hcmp > score_key((unsigned)rowmin, 1)) return true;
  // 4. per-label estimates of the sketch labels (rescan of the row)
  if (threadIdx.x == 0) atomicAdd(&st->pad[0], 1ull);
  unsigned long long ckey = 0ull;
  for (int e = threadIdx.x; e < d; e += BLOCK) {
    const int l = gather(a, a.col[start + e]);
    if (l < 0 || ht_has(tab, (unsigned)l, kLProbe)) continue;
    const unsigned g = cm.estimate((unsigned)l);
    const int v = VAR == V_LLP ? (a.v_ones ? 1 : (a.LV ? __ldg(&a.LV[a.col[start + e]].y) : ld_label(a.V + l))) : 0;
    ckey = max(ckey, score_key(g, v));
  }
  ckey = block_max_u64<BLOCK>(ckey);
  if (hcmp > ckey) return true;
  if (threadIdx.x == 0) atomicAdd(&st->pad[1], 1ull);
  return false;
}

// mfl_block: one block per row of class CLS (M or L).  mode 0 scans the
// degree-sorted row prefix and takes the rows of its class; mode 1 takes the
// rows another kernel re-queued this iteration.
//   M (PART = false): table of pow2 >= 4*pred slots (<= SLOTS); a row whose
//     labels overflow it is re-queued to L.
//   L (PART = true): rows with more distinct labels than the table holds are
//     radix-partitioned by a hash of the label into P parts (gather pass ->
//     per-block staging buffer + shared histogram, scatter pass ->
//     partition-contiguous copy), then each part is counted exactly in the
//     shared table; the best over the parts is the row's MFL.  A part that
//     still overflows (probe limit) restarts the row with 2P.  This replaces
//     the paper's global-memory fallback table [P:166]: on B200 re-streaming a
//     staged row costs less than clearing and probing a per-row global table.
// Both record the row's exact distinct-label count as the next `pred`.
template <int VAR, int BLOCK, int SLOTS, bool PART, int UNROLL, int CLS>
#ifndef GLP_M_MINB
#define GLP_M_MINB 5
#endif
#ifndef GLP_L_MINB
#define GLP_L_MINB 2
#endif
__global__ void __launch_bounds__(BLOCK, PART ? GLP_L_MINB : GLP_M_MINB) mfl_block(MflArgs a) {
  GLP_CTL_PROLOGUE(a)
  extern __shared__ __align__(16) unsigned long long smem_tab[];  // SLOTS
  __shared__ int s_over, s_distinct, s_major, s_scan;
  __shared__ int s_hist[PART ? 256 : 1], s_cur[PART ? 256 : 1];
  Tally ty;
  int32_t* stageA = PART ? a.stage + (int64_t)blockIdx.x * 2 * a.stage_stride : nullptr;
  int32_t* stageB = PART ? stageA + a.stage_stride : nullptr;
  __shared__ int s_k0, s_nsel, s_sel[32], s_cand[32];
  __shared__ BinItem s_item[32];
  __shared__ unsigned s_pe[32], s_raw[32];
  const int n_redo = a.mode ? (int)*a.redo_in_n : 0;
  if (a.mode && n_redo == 0) return;  // empty redo queue (block-uniform): no tally to flush
  const int lim = a.mode ? n_redo : a.n_items;
  for (;;) {
    // dynamic fetch of 32 rows (row costs vary by orders of magnitude); warp 0
    // selects the rows of this class (and, in sparse iterations, the active
    // ones) lane-parallel
    // (tickets below big_prefix -- the longest rows, and every re-queued row --
    // fetch one row each so long rows spread over blocks; later tickets 32)
    if (threadIdx.x == 0) s_k0 = (int)atomicAdd(a.work, 1ull);
    __syncthreads();
    const int tk = s_k0;
    const int big = a.mode ? lim : a.big_prefix;
    const int k0 = tk < big ? tk : big + (tk - big) * 32;
    const int kn = tk < big ? 1 : 32;
    if (k0 >= lim) break;
    if (threadIdx.x < 32) {
      // lane-parallel selection; the selected rows' descriptors and
      // predictions are staged in shared memory (no dependent global loads
      // in the per-row loop)
      const int k = k0 + (int)threadIdx.x;
      bool ok = (int)threadIdx.x < kn && k < lim;
      int ik = -1;
      BinItem itk;
      itk.start = 0; itk.v = 0; itk.d = 0;
      unsigned raw = 0u, pe = 1u;
      bool cnd = false;
      if (ok) {
        ik = a.mode ? a.redo_in[k] : k;
        itk = a.items[ik];
        raw = a.pred[ik];
        pe = pred_est<VAR>(raw, a.pred_prev[ik], a.pred_cap);
        cnd = mono_cand<VAR>(raw, a.pred_cap, itk.d, a.t);
        if (!a.mode) {
          ok = row_class(pe, itk.d, cnd, a.mono_kernel) == CLS;
          if (ok && !dense_ && !a.flag[a.vb + itk.v]) {
            ok = false;
            a.pred_next[ik] = raw;  // inactive: carry the prediction forward
          }
        }
      }
      const unsigned m = __ballot_sync(kFull, ok);
      if (ok) {
        const int pos = __popc(m & ((1u << threadIdx.x) - 1u));
        s_sel[pos] = ik;
        s_item[pos] = itk;
        s_pe[pos] = pe;
        s_raw[pos] = raw;
        s_cand[pos] = cnd ? 1 : 0;
      }
      if (threadIdx.x == 0) s_nsel = __popc(m);
    }
    __syncthreads();
    const int nsel = s_nsel;
    for (int q = 0; q < nsel; ++q) {
    const int i = s_sel[q];
    const BinItem it = s_item[q];
    int4 cur[UNROLL];
    block_load_round<BLOCK, UNROLL>(a.col, it.start, it.d, 0, cur);
    const unsigned praw = s_raw[q];
    const bool cand = s_cand[q] != 0;
    const unsigned pred = s_pe[q];
    const int d = it.d;
    Best<VAR> b;
    if (threadIdx.x == 0) { s_distinct = 0; s_over = 0; s_major = 0; s_scan = 0; }
    bool mono_done = false;
    if (!a.mode && cand) {
      __syncthreads();
      unsigned fr = 0;
      mono_done = block_mono<VAR, BLOCK, UNROLL>(a, it.start, d, cur, b, &fr);
      if (mono_done) {
        fr = __reduce_add_sync(kFull, fr);
        if ((threadIdx.x & 31) == 0 && fr) atomicAdd(&s_distinct, (int)fr);
        __syncthreads();
      } else {
        b = Best<VAR>();
        block_load_round<BLOCK, UNROLL>(a.col, it.start, d, 0, cur);  // table path restarts the row
      }
    }
    if (!mono_done) {
    // a re-queued row overflowed a smaller table: its pred is stale.
    // L: a row whose last count took the sorted fast path (all labels distinct
    // at t = 1) is sized at GLP_L_EST % of that count -- labels collapse
    // [P:130] (RMAT probe at t = 2: 26-36 % distinct for deg > 2048); the
    // labels are staged, so an overflow recounts them in partitions
    const unsigned est = a.mode ? (unsigned)d
                                : (praw & kMonoTried)
                                      ? max(1u, (unsigned)(((unsigned long long)pred * (PART ? GLP_L_EST : GLP_M_EST)) / 100ull))
                                      : pred;
    unsigned nparts = PART ? max(1u, (min(est, (unsigned)d) + SLOTS / 2 - 1) / (SLOTS / 2)) : 1u;
    bool staged = false;  // stageA holds the row's gathered labels
    bool over = false;
    if (PART && a.cms) {
      // §8(f)2 SharedMemBigNodes [P:132-182]: one scan, HT + CMS; the HT's
      // best is the MFL when it beats every sketch estimate strictly (R15),
      // else the row is recounted exactly in partitions (the paper's global
      // table fallback [P:166])
      over = !cms_count<VAR, BLOCK, SLOTS, UNROLL>(a, it.start, d, cur, b, &s_over, &s_distinct, &s_major, &s_scan,
                                                  hot_pass(est, d));
      if (over) nparts = min(max(2u, ((unsigned)d + SLOTS / 2 - 1) / (SLOTS / 2)), 255u);
      if (over) b = Best<VAR>();
      __syncthreads();
    } else if (nparts == 1u) {
      // single pass: gather + count.  Nothing is staged: an overflow stops the
      // count early, so the partition passes below gather the row again
      // (GLP_L_STAGE1 = 1 restores the old, never-read staging writes), and a
      // strict majority may end the row (GLP_L_MAJ)
      const unsigned want = PART ? 2u * (unsigned)d : GLP_M_LOAD * est;
      const unsigned tsz = min(max(64u, 1u << (32 - __clz(want - 1u))), (unsigned)SLOTS);
      const Table tab{smem_tab, tsz};
      tab.clear(threadIdx.x, BLOCK);
      __syncthreads();
      const bool may_over = PART && 2u * (unsigned)d > (unsigned)SLOTS;
      block_count<VAR, BLOCK, UNROLL, !PART || GLP_L_IPF>(a, it.start, d, tab, may_over ? kLProbe : (PART ? tsz : kTabProbe), cur,
                                      (GLP_L_STAGE1 && may_over) ? stageA : nullptr, &s_over, &s_distinct, b,
                                      (may_over && !GLP_L_MAJ) ? nullptr : &s_major, 1u, &s_scan,
                                      hot_pass(est, d), nullptr, peek_pass<VAR>(est, d));
      __syncthreads();
      over = s_over != 0;
      if (!over && a.LV == nullptr) table_scan<VAR>(tab, threadIdx.x, BLOCK, a, b);
      // (s_over is next reset by the partition passes below or at the next row,
      // which every thread reaches only through block_best's barrier)
      if (!GLP_FEWER_BARRIERS || (over && PART)) __syncthreads();
      if (over && PART) {
        nparts = min(max(2u, ((unsigned)d + SLOTS / 2 - 1) / (SLOTS / 2)), 255u);
        over = false;
      }
    }
    if (!PART && over) {
      if (threadIdx.x == 0) a.redo_out[atomicAdd(a.redo_out_n, 1u)] = i;
      __syncthreads();
      continue;
    }
    if (PART) {
      nparts = min(nparts, 255u);
      while (nparts > 1u) {
        if (nparts <= (unsigned)GLP_L_FILTER) {
          // Few parts: no partition histogram and scatter.  Part 0 is counted
          // while the row is gathered and staged (labels of other parts are
          // skipped), parts 1.. re-read the staged row and count only their
          // own labels.  Every label lives in exactly one part, so the best
          // over the parts is the row's MFL.
          b = Best<VAR>();
          bool pover = false;
          unsigned p = 0;
          for (; p < nparts && !pover; ++p) {
            const Table tab{smem_tab, (unsigned)SLOTS};
            tab.clear(threadIdx.x, BLOCK);
            if (threadIdx.x == 0) {
              s_over = 0;
              if (p == 0) s_distinct = 0;
            }
            __syncthreads();
            const bool gather_pass = p == 0 && !staged;
            if (gather_pass) {
              block_load_round<BLOCK, UNROLL>(a.col, it.start, d, 0, cur);
              block_count<VAR, BLOCK, UNROLL, GLP_L_IPF>(a, it.start, d, tab, kLProbe, cur, stageA, &s_over,
                                                         &s_distinct, b, nullptr, nparts, nullptr, GLP_HOT_DIV == 0);
            } else {
              count_staged<VAR, BLOCK>(a, stageA, d, tab, kLProbe, &s_over, &s_distinct, b, nparts, p);
            }
            __syncthreads();
            pover = s_over != 0;
            if (!pover && !(gather_pass && a.LV != nullptr)) table_scan<VAR>(tab, threadIdx.x, BLOCK, a, b);
            if (!pover && gather_pass) staged = true;  // a gather pass that did not overflow staged the whole row
            __syncthreads();
          }
          if (!pover) break;
          nparts = nparts * 2u;  // a part overflowed: finer partitions (exact recount)
          continue;
        }
        // (a) histogram of partitions (gathering + staging the row if needed)
        if (threadIdx.x < 256) s_hist[threadIdx.x] = 0;
        if (threadIdx.x == 0) { s_over = 0; s_distinct = 0; }
        __syncthreads();
        for (int base = 0; base < d; base += BLOCK * 4) {
          const int idx = base + (int)threadIdx.x * 4;
          if (idx < d) {
            int4 x;
            if (staged) {
              x = __ldcg((const int4*)(stageA + idx));
            } else {
              const int4 u = ld_stream4(a.col + it.start + idx);
              x = make_int4(gather(a, u.x), gather(a, u.y), gather(a, u.z), gather(a, u.w));
              __stcg((int4*)(stageA + idx), x);
            }
            if (x.x >= 0) atomicAdd(&s_hist[label_part((unsigned)x.x, nparts)], 1);
            if (x.y >= 0) atomicAdd(&s_hist[label_part((unsigned)x.y, nparts)], 1);
            if (x.z >= 0) atomicAdd(&s_hist[label_part((unsigned)x.z, nparts)], 1);
            if (x.w >= 0) atomicAdd(&s_hist[label_part((unsigned)x.w, nparts)], 1);
          }
        }
        staged = true;
        __syncthreads();
        // (b) exclusive scan -> cursors (one warp, nparts <= 255)
        if (threadIdx.x < 32) {
          int carry = 0;
          for (int p0 = 0; p0 < (int)nparts; p0 += 32) {
            const int p = p0 + (int)threadIdx.x;
            const int h = p < (int)nparts ? s_hist[p] : 0;
            int x = h;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
              const int y = __shfl_up_sync(kFull, x, o);
              if ((int)threadIdx.x >= o) x += y;
            }
            if (p < (int)nparts) s_cur[p] = carry + x - h;
            carry += __shfl_sync(kFull, x, 31);
          }
        }
        __syncthreads();
        // (c) scatter into partition-contiguous order
        for (int base = 0; base < d; base += BLOCK * 4) {
          const int idx = base + (int)threadIdx.x * 4;
          if (idx < d) {
            const int4 x = __ldcg((const int4*)(stageA + idx));
            if (x.x >= 0) __stcg(stageB + atomicAdd(&s_cur[label_part((unsigned)x.x, nparts)], 1), x.x);
            if (x.y >= 0) __stcg(stageB + atomicAdd(&s_cur[label_part((unsigned)x.y, nparts)], 1), x.y);
            if (x.z >= 0) __stcg(stageB + atomicAdd(&s_cur[label_part((unsigned)x.z, nparts)], 1), x.z);
            if (x.w >= 0) __stcg(stageB + atomicAdd(&s_cur[label_part((unsigned)x.w, nparts)], 1), x.w);
          }
        }
        __syncthreads();
        // (d) count each partition exactly (s_cur[p] now = end of part p)
        b = Best<VAR>();
        bool pover = false;
        for (unsigned p = 0; p < nparts && !pover; ++p) {
          const int end = s_cur[p];
          const int cnt = s_hist[p];
          const unsigned tsz = min(max(64u, 1u << (32 - __clz(2u * (unsigned)max(cnt, 1) - 1u))), (unsigned)SLOTS);
          const Table tab{smem_tab, tsz};
          tab.clear(threadIdx.x, BLOCK);
          __syncthreads();
          const unsigned probe = 2u * (unsigned)cnt <= (unsigned)SLOTS ? tsz : kLProbe;
          count_staged<VAR, BLOCK>(a, stageB + (end - cnt), cnt, tab, probe, &s_over, &s_distinct, b);
          __syncthreads();
          pover = s_over != 0;
          if (!pover) table_scan<VAR>(tab, threadIdx.x, BLOCK, a, b);
          __syncthreads();
        }
        if (!pover) break;
        nparts = min(nparts * 2u, 255u);  // a part overflowed: finer partitions (exact recount)
      }
    }
    }  // !mono_done
    b = block_best<VAR, BLOCK>(b);
    if (threadIdx.x == 0) {
      const unsigned dist = s_major ? max((unsigned)s_distinct, pred) : (unsigned)s_distinct;  // partial on a majority exit
      a.pred_next[i] = max(dist, 1u) | (mono_done ? kMonoTried : 0u);
      // arcs gathered: the whole row unless the single pass stopped on a majority
      update_vertex<VAR>(a, it.v, d, b.have(), b.label(), ty, s_major ? s_scan : d);
    }
    // No barrier here: every shared value of this row (table, flags, the
    // block_best scratch) was last read before block_best's barrier, and the
    // next row rewrites them only after its own clear barrier; thread 0 alone
    // reads s_distinct / s_major above and resets them itself.
    if (!GLP_FEWER_BARRIERS) __syncthreads();
    }  // selected rows
  }
  tally_flush(ty, a.cnt);
}

// ---------------------------------------------------------------------------
// Giant rows (deg > kGiantMin): one global-memory table per row, shared by all
// blocks that count the row's segments.  Slot = [epoch | label | count]; a slot
// whose epoch is not this iteration's is free, so tables are never cleared
// between iterations (only when the epoch counter wraps).
__device__ __forceinline__ unsigned giant_add(unsigned long long* tab, unsigned long long tsz, unsigned lab,
                                              unsigned c, unsigned long long epoch, bool* fresh) {
  constexpr int kShift = 31 + kGCountBits;
  const unsigned long long tag = (epoch << kShift) | ((unsigned long long)lab << kGCountBits);
  const unsigned long long keymask = ~((1ull << kGCountBits) - 1ull);
  const unsigned long long cmask = (1ull << kGCountBits) - 1ull;
  unsigned long long h = (unsigned long long)((lab * 0x9E3779B97F4A7C15ull) >> 20) & (tsz - 1ull);
  for (;;) {
    unsigned long long e = *((volatile unsigned long long*)(tab + h));
    for (;;) {
      if ((e & keymask) == tag) return (unsigned)((atomicAdd(tab + h, (unsigned long long)c) & cmask) + c);
      if ((e >> kShift) != epoch) {  // stale slot: claim it
        const unsigned long long prev = atomicCAS(tab + h, e, tag | c);
        if (prev == e) {
          *fresh = true;
          return c;
        }
        e = prev;  // re-examine the same slot
        continue;
      }
      break;  // another label of this iteration
    }
    h = (h + 1ull) & (tsz - 1ull);
  }
}

// Phase 1: blocks take segments (dynamic tickets).  A segment is first
// counted in a shared-memory table (the same open-addressing table as the
// block kernels, hot-label ballots included), then the table is flushed into
// the row's global table with ONE global atomic per distinct label of the
// segment instead of one per arc: a collapsed or seeded hub (few distinct
// labels, huge counts) no longer serialises all blocks on a few L2 atomic
// addresses.  Labels that do not fit the shared table go to the global table
// directly.  Only global post-add counts are observed (segment-local counts
// are partial), so each segment's best observation stays a valid candidate:
// the last add of every label returns its final row count.  (A/B, R24
// classic / LLP / TaoBao: always pre-aggregating cost +0.7 % / +2 % / -2 %
// per run; the per-row choice below keeps the gain only.)
#ifndef GLP_GIANT_SMEM
#define GLP_GIANT_SMEM 1
#endif
#ifndef GLP_GIANT_BATCH
#define GLP_GIANT_BATCH 1  // giant count: first probes of a lane's labels in flight together
#endif
#ifndef GLP_GIANT_PRE_DIV
#define GLP_GIANT_PRE_DIV 4ull  // pre-aggregate rows whose last distinct count is <= d / this (1: always)
#endif
constexpr int kGSlots = 8192;  // shared pre-aggregation table (64 KB)
#ifndef GLP_G_MINB
#define GLP_G_MINB 1  // 1: 56-64 registers, no spills (3: 32 registers + spills); A/B TaoBao 97.3 -> 94.2 ms/run, R24 17.51 -> 17.41
#endif
template <int VAR, bool WT = false>
__global__ void __launch_bounds__(kGBlock, GLP_G_MINB) mfl_giant_count(MflArgs a) {
  GLP_CTL_PROLOGUE(a)
  extern __shared__ __align__(16) unsigned long long gsm[];  // kGSlots (GLP_GIANT_SMEM)
  __shared__ int s_k;
  const int lane = threadIdx.x & 31;
  for (;;) {
    if (threadIdx.x == 0) s_k = (int)atomicAdd(a.work, 1ull);
    __syncthreads();
    const int k = s_k;
    __syncthreads();
    if (k >= a.n_gsegs) break;
    const GiantSeg sg = a.gsegs[k];
    const BinItem it = a.items[sg.row];
    if (!dense_ && !a.flag[a.vb + it.v]) continue;  // block-uniform
    unsigned long long* tab = a.gtab + a.gtab_off[sg.row];
    const unsigned long long tsz = (unsigned long long)(a.gtab_off[sg.row + 1] - a.gtab_off[sg.row]);
    const int end = min(sg.begin + kGiantSeg, it.d);
    Best<VAR> b;
    unsigned fresh = 0;
    const bool use_v = VAR == V_LLP && a.LV != nullptr;
    // rows predicted to repeat labels (last count <= d / 4: collapsed or
    // seeded hubs) pre-aggregate; distinct-heavy rows (t = 2, LLP's
    // oscillation) would only pay the shared insert and flush on top
    const bool pre = GLP_GIANT_SMEM && (unsigned long long)(a.pred[sg.row] & kPredMask) * GLP_GIANT_PRE_DIV <=
                                           (unsigned long long)it.d;
    if (pre) {
      const Table st{gsm, (unsigned)kGSlots};
      st.clear(threadIdx.x, kGBlock);
      __syncthreads();
      Best<VAR> hotb;  // steers the hot-label pass only (segment-local counts)
      unsigned lf = 0;
      for (int base = sg.begin; base < end; base += kGBlock * 4) {
        const int idx = base + (int)threadIdx.x * 4;
        const int4 u = idx < end ? ld_stream4(a.col + it.start + idx) : make_int4(-1, -1, -1, -1);
        int lab[4] = {gather(a, u.x), gather(a, u.y), gather(a, u.z), gather(a, u.w)};
        // weighted LP (§8(f)3): a label adds its arc's weight (w2 beside col2)
        unsigned w[4] = {1u, 1u, 1u, 1u};
        if (WT && idx < end) {
          const int4 wv = ld_stream4((const int32_t*)a.w2 + it.start + idx);
          w[0] = (unsigned)wv.x; w[1] = (unsigned)wv.y; w[2] = (unsigned)wv.z; w[3] = (unsigned)wv.w;
        }
        // hot label of the warp: one shared atomic for all its copies
        const int hot = __shfl_sync(kFull, hotb.have() ? (int)hotb.label() : lab[0] >= 0 ? lab[0] : lab[1], 0);
        if (hot >= 0) {
          unsigned hc = 0;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            hc += lab[j] == hot ? w[j] : 0u;
            lab[j] = lab[j] == hot ? -1 : lab[j];
          }
          const unsigned tot = __reduce_add_sync(kFull, hc);
          if (lane == 0 && tot) {
            const unsigned c = ht_add(st, (unsigned)hot, tot, kTabProbe, &lf);
            if (c) {
              hotb.observe(c, (unsigned)hot, a, 1);
            } else {  // shared table full: straight to the row's table
              bool fr = false;
              const unsigned gc = giant_add(tab, tsz, (unsigned)hot, tot, a.epoch, &fr);
              fresh += fr ? 1u : 0u;
              b.observe(gc, (unsigned)hot, a);
            }
          }
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          if (lab[j] < 0) continue;
          const unsigned c = ht_add(st, (unsigned)lab[j], w[j], kTabProbe, &lf);
          if (c == 0u) {
            bool fr = false;
            const unsigned gc = giant_add(tab, tsz, (unsigned)lab[j], w[j], a.epoch, &fr);
            fresh += fr ? 1u : 0u;
            b.observe(gc, (unsigned)lab[j], a);
          }
        }
        hotb.warp_reduce();  // every lane steers by the warp's best so far
      }
      __syncthreads();
      // flush: one global add per distinct label of the segment
      for (unsigned j = threadIdx.x; j < (unsigned)kGSlots; j += kGBlock) {
        const unsigned l = st.key[j];
        if (l == kFree) continue;
        bool fr = false;
        const unsigned gc = giant_add(tab, tsz, l, st.cnt[j], a.epoch, &fr);
        fresh += fr ? 1u : 0u;
        b.observe(gc, l, a);  // LLP: V[l] (or 1 at t = 1)
      }
    } else {
      for (int base = sg.begin; base < end; base += kGBlock * 4 * kGUnroll) {
        int lab[4 * kGUnroll], gv[4 * kGUnroll];
        unsigned wt[4 * kGUnroll];
#pragma unroll
        for (int j = 0; j < kGUnroll; ++j) {
          const int idx = base + (j * kGBlock + (int)threadIdx.x) * 4;
          const int4 u = idx < end ? ld_stream4(a.col + it.start + idx) : make_int4(-1, -1, -1, -1);
          int4 wv = make_int4(1, 1, 1, 1);
          if (WT && idx < end) wv = ld_stream4((const int32_t*)a.w2 + it.start + idx);
          wt[4 * j + 0] = (unsigned)wv.x; wt[4 * j + 1] = (unsigned)wv.y;
          wt[4 * j + 2] = (unsigned)wv.z; wt[4 * j + 3] = (unsigned)wv.w;
          lab[4 * j + 0] = gather_lv(a, u.x, use_v, gv[4 * j + 0]);
          lab[4 * j + 1] = gather_lv(a, u.y, use_v, gv[4 * j + 1]);
          lab[4 * j + 2] = gather_lv(a, u.z, use_v, gv[4 * j + 2]);
          lab[4 * j + 3] = gather_lv(a, u.w, use_v, gv[4 * j + 3]);
        }
        const int cand0 = b.have() ? (int)b.label() : -2;
        constexpr int NG = 4 * kGUnroll;
        unsigned cc[NG];
#pragma unroll
        for (int j = 0; j < NG; ++j) {
          const bool vote = lab[j] >= 0;
          const int hot = __shfl_sync(kFull, cand0 == -2 ? lab[j] : cand0, 0);
          const unsigned m = __ballot_sync(kFull, vote && lab[j] == hot);
          unsigned c = vote ? (lab[j] != hot ? 1u : (lane == __ffs(m) - 1 ? (unsigned)__popc(m) : 0u)) : 0u;
          if (WT) c = vote ? wt[j] : 0u;  // weighted: every arc adds its own weight
          cc[j] = c;
        }
#if GLP_GIANT_BATCH
        // The lane's NG inserts go to the row's table in L2 with their first
        // probes in flight together (home-slot loads, then the adds on slots
        // already holding the label and the claims of slots of older epochs,
        // each batch independent); only labels whose home slot holds another
        // label of this epoch, or whose claim lost a race, walk giant_add.
        // LLP only (A/B: R28 LLP -4 %; classic / seeded +0.5-1 %).
        if (VAR == V_LLP) {
          constexpr int kShift = 31 + kGCountBits;
          const unsigned long long keymask = ~((1ull << kGCountBits) - 1ull);
          const unsigned long long cmask = (1ull << kGCountBits) - 1ull;
          unsigned long long hh[NG], ee[NG];
#pragma unroll
          for (int j = 0; j < NG; ++j) {
            hh[j] = (unsigned long long)(((unsigned)lab[j] * 0x9E3779B97F4A7C15ull) >> 20) & (tsz - 1ull);
            ee[j] = cc[j] ? *((volatile unsigned long long*)(tab + hh[j])) : 0ull;
          }
#pragma unroll
          for (int j = 0; j < NG; ++j) {
            if (!cc[j]) continue;
            const unsigned long long tag = (a.epoch << kShift) | ((unsigned long long)(unsigned)lab[j] << kGCountBits);
            unsigned cnt = 0u;
            if ((ee[j] & keymask) == tag) {
              cnt = (unsigned)((atomicAdd(tab + hh[j], (unsigned long long)cc[j]) & cmask) + cc[j]);
            } else if ((ee[j] >> kShift) != a.epoch) {
              if (atomicCAS(tab + hh[j], ee[j], tag | cc[j]) == ee[j]) {
                cnt = cc[j];
                ++fresh;
              }
            }
            if (cnt) {
              b.observe(cnt, (unsigned)lab[j], a, use_v ? gv[j] : -1);
              cc[j] = 0u;
            }
          }
        }
#endif
#pragma unroll
        for (int j = 0; j < NG; ++j) {
          if (cc[j]) {
            bool fr = false;
            const unsigned cnt = giant_add(tab, tsz, (unsigned)lab[j], cc[j], a.epoch, &fr);
            fresh += fr ? 1u : 0u;
            b.observe(cnt, (unsigned)lab[j], a, use_v ? gv[j] : -1);
          }
        }
      }
    }
    fresh = __reduce_add_sync(kFull, fresh);
    if (lane == 0 && fresh) atomicAdd(a.gdistinct + sg.row, fresh);
    b = block_best<VAR, kGBlock>(b);
    if (threadIdx.x == 0) {
      a.gcand_key[k] = b.key;
      a.gcand_lab[k] = b.lab;
    }
  }
}

// Phase 2: one block per giant row reduces its segments' candidates (the best
// over all observations is exact, see the header) and updates the vertex.
template <int VAR>
__global__ void __launch_bounds__(256) mfl_giant_finish(MflArgs a, const int32_t* __restrict__ seg_first) {
  GLP_CTL_PROLOGUE(a)
  Tally ty;
  const int i = blockIdx.x;
  const BinItem it = a.items[i];
  const bool active = dense_ || a.flag[a.vb + it.v];
  if (active) {
    Best<VAR> b;
    for (int k = seg_first[i] + (int)threadIdx.x; k < seg_first[i + 1]; k += 256) b.merge(a.gcand_key[k], a.gcand_lab[k]);
    b = block_best<VAR, 256>(b);
    if (threadIdx.x == 0) {
      a.pred_next[i] = max(a.gdistinct[i], 1u);
      a.gdistinct[i] = 0u;
      update_vertex<VAR>(a, it.v, it.d, b.have(), b.label(), ty, it.d);
    }
  } else if (threadIdx.x == 0) {
    a.pred_next[i] = a.pred[i];
  }
  tally_flush(ty, a.cnt);
}

}  // namespace glp
