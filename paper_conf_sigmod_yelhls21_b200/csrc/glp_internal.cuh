// glp_internal.cuh -- internal types of libglp.so (not part of the ABI).
//
// Data layout in HBM:
//   col2  int32[nnz2]   bin-major copy of the owned arcs (global ids):
//                       low chunks contiguous, other rows 16-B aligned and
//                       padded with -1; streamed once per iteration   [P:97]
//   ioff/ideg [nl]      row start in col2 / degree (frontier push)
//   L[2]  int32[n]      labels, double-buffered (R = L_{t-1}, W = L_t) [P:143]
//   so    int2[nl]      (stamp, old): iteration of the last change and the
//                       label before it -> exact 2-cycle test (R8)
//   flag[2] u8[n]       frontier marks by global id (sparse iterations only)
//   V     int32[n]      LLP label histogram (LLP only)               [P:119]
//   pos/orig int32[n]   internal <-> original vertex ids (layout.cuh)
//   chunks              low-degree warp chunks
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/glp.h"

namespace glp {

struct Comm;     // comm.cuh: the exchange of the 1-D partition (NCCL or in-process)
struct IterRec;  // aux_kernels.cuh: one iteration's record of the device-driven loop

// Degree bin of the packed-warp kernel (PAPER §4.2): deg <= 32.
constexpr int kLowMax = 32;
constexpr int kLowBlock = 256;

// Rows with deg > 32 are counted in shared-memory hash tables (PAPER §4.1).
// Each iteration a row goes to one of three kernels by its *predicted*
// distinct-label count `pred` (the exact count of its previous iteration;
// deg at t = 1, when all labels are distinct) -- labels collapse as
// communities form [P:130], so most rows migrate to the warp path:
//   W  pred <= 256,  deg <= 4096  : one warp per row, 512-slot table per warp
//   M  pred <= 2048, deg <= 16384 : one 128-thread block per row, 4096 slots
//   L  otherwise                  : one 512-thread block per row (two per
//                                   SM), 8192 slots, hash-partitioned passes
// Sorted-row candidates (row_class `mono`) go to W whatever their size.
// A row whose labels overflow its table is re-queued to the next class in the
// same iteration (exact recount), so `pred` only steers performance.
#ifndef GLP_WPRED
#define GLP_WPRED 256
#endif
#ifndef GLP_WSLOTS
#define GLP_WSLOTS 512
#endif
constexpr unsigned kWPred = GLP_WPRED, kMPred = 2048;
#ifndef GLP_MMAXDEG
#define GLP_MMAXDEG 16384
#endif
constexpr int kWMaxDeg = 4096, kMMaxDeg = GLP_MMAXDEG;
#ifndef GLP_MONO_WMAX
#define GLP_MONO_WMAX 65536
#endif
constexpr int kMonoWMax = GLP_MONO_WMAX;  // sorted-row candidates longer than this use the block path (L)
constexpr int kWBlock = 256;
constexpr int kWSlots = GLP_WSLOTS;
constexpr int kMBlock = 128;
constexpr int kMSlots = 4096;
#ifndef GLP_MUNROLL
#define GLP_MUNROLL 2
#endif
constexpr int kMUnroll = GLP_MUNROLL;
#ifndef GLP_LBLOCK
#define GLP_LBLOCK 512
#endif
#ifndef GLP_LSLOTS
#define GLP_LSLOTS 8192
#endif
constexpr int kLBlock = GLP_LBLOCK;
constexpr int kLSlots = GLP_LSLOTS;
#ifndef GLP_LUNROLL
#define GLP_LUNROLL 1
#endif
constexpr int kLUnroll = GLP_LUNROLL;
constexpr int kLProbe = 32;  // probe limit before declaring a partition overflowed
// Probe limit of the W and M tables (sized >= 4x the predicted distinct
// labels, so a legitimate insert rarely probes far).  A row whose prediction
// was far too low (LLP's oscillating regime) fills its table; without a limit
// every further new label would probe the whole table before the overflow is
// noticed.  Hitting the limit re-queues the row to the next class (exact).
constexpr unsigned kTabProbe = 32;
// Giant rows (deg > kGiantMin) are split into segments of kGiantSeg arcs that
// many blocks count concurrently into one global-memory table per row
// (epoch-tagged slots, never cleared between iterations); a second kernel
// reduces the per-segment candidates of each row.
constexpr int kGiantMin = 65536;
constexpr int kGiantSeg = 32768;
constexpr int kGBlock = 512;
constexpr int kGUnroll = 2;
constexpr int kGCountBits = 25;  // count field of a giant-table slot (deg < 2^25)
constexpr int kGEpochBits = 64 - 31 - kGCountBits;
enum RowClass { CLS_W = 0, CLS_M = 1, CLS_L = 2, CLS_G = 3, CLS_MONO = 4 };
// pred word: low 31 bits = predicted distinct labels; bit 31 = the row took
// the sorted-row fast path last time (do not retry it)
constexpr unsigned kPredMask = 0x7fffffffu, kMonoTried = 0x80000000u;
// A sorted-row candidate (`mono`: its labels were all distinct last time and
// it has not tried the fast path yet, e.g. every row at t = 1) needs no table:
// it goes to the barrier-free warp kernel whatever its size (to the table-free
// mono kernel when that one is launched: mono_k, t = 1).
__host__ __device__ __forceinline__ int row_class(unsigned pred, int d, bool mono, bool mono_k = false) {
  if (d > kGiantMin) return CLS_G;
  if (mono) return d > kMonoWMax ? CLS_L : (mono_k ? CLS_MONO : CLS_W);
  if (pred <= kWPred && d <= kWMaxDeg) return CLS_W;
  if (pred <= kMPred && d <= kMMaxDeg) return CLS_M;
  return CLS_L;
}

// One segment of a giant row.
struct GiantSeg {
  int32_t row;    // index into the giant prefix of `rows`
  int32_t begin;  // arc offset within the row
};

// Per-iteration scheduling state (reset with the counters).
struct Sched {
  unsigned n_redo_m, n_redo_l;      // rows re-queued to M / L this iteration
  unsigned long long work_m, work_mr, work_l, work_lr;  // dynamic fetch counters (static / redo)
  unsigned long long work_g;
};

// A low-degree chunk: up to 32 consecutive arcs of consecutive low-list
// vertices.  st = arc start in col2 | (degree << 48) | (arc count << 56); bit i of segmask set
// iff a vertex's first arc is at lane i; vbase = index of its first vertex in
// the low list.
struct LowChunk {
  unsigned long long st;
  int32_t vbase;
  uint32_t segmask;
};

// A mid/high/huge row: arcs col2[start, start + d) (start 16-byte aligned,
// padded with -1 up to a multiple of 4).
struct BinItem {
  int64_t start;
  int32_t v;  // local vertex id
  int32_t d;
};

enum Bin { BIN_ISO = 0, BIN_LOW = 1, BIN_MID = 2, BIN_HIGH = 3, BIN_HUGE = 4, NBINS = 5 };

// Device counters of one iteration (reset per iteration).
struct Counters {
  unsigned long long changed;   // #{v : L_t != L_{t-1}}
  unsigned long long d2;        // #{v : L_t != L_{t-2}}
  unsigned long long chdeg;     // sum of deg over changed vertices
  unsigned long long arcs;      // arcs scanned
  unsigned long long verts;     // vertices scanned
  unsigned long long pad0;    // L rows that used the CMS (§8(f)2)
  unsigned long long pad[2];  // [0] of those, rows rescanned for estimates; [1] rows recounted (fallback)
};

// per-kernel iteration counters: low, W, M, L, giant, mono
constexpr int kNumCounters = 6;

// Arguments shared by the MFL kernels (passed by value).
struct MflArgs {
  const int32_t* __restrict__ col;      // col2: bin-major arcs (global ids, -1 = padding)
  const int32_t* __restrict__ R;        // L_{t-1}, global ids [n]
  int32_t* __restrict__ W;              // L_t, global ids [n]
  int2* __restrict__ so;                // [nl] (stamp, old label)
  const int32_t* __restrict__ V;        // LLP histogram [n] or null
  const uint8_t* __restrict__ is_seed;  // [nl] or null
  const uint8_t* __restrict__ flag;     // [npad] frontier marks by global id (sparse)
  int64_t low_base;                     // low bin: internal id of low-list entry 0
  const LowChunk* __restrict__ chunks;  // low bin
  const uint8_t* __restrict__ cflag;    // low bin: chunk has an active vertex (sparse)
  int32_t n_chunks;
  const BinItem* __restrict__ items;    // rows with deg > 32, degree-descending
  int32_t n_items;                      // prefix of items this launch scans
  int32_t big_prefix;                   // rows fetched one per ticket (longest rows)
  const unsigned* __restrict__ pred;    // per row: predicted distinct labels (this iteration)
  const unsigned* __restrict__ pred_prev;  // per row: distinct labels at t-2 (extrapolation)
  unsigned* __restrict__ pred_next;     // per row: distinct labels counted now (next iteration)
  unsigned pred_cap;                    // testing: clamp predictions (0 = off)
  int32_t mode;                         // 0: scan items by class, 1: redo list
  const int32_t* __restrict__ redo_in;  // mode 1: rows to process
  const unsigned* redo_in_n;
  int32_t* __restrict__ redo_out;       // rows re-queued to the next class
  unsigned* redo_out_n;
  unsigned long long* work;             // dynamic fetch counter (L)
  int32_t* __restrict__ stage;          // L: per-block staged row labels (2 x stride)
  int64_t stage_stride;
  const GiantSeg* __restrict__ gsegs;   // giant rows: segments, tables, candidates
  int32_t n_gsegs;
  unsigned long long* __restrict__ gtab;
  const int64_t* __restrict__ gtab_off; // per giant row: slot offset, table size = next - this
  unsigned long long* __restrict__ gcand_key;  // per segment
  unsigned* __restrict__ gcand_lab;
  unsigned* __restrict__ gdistinct;     // per giant row
  unsigned long long epoch;             // giant-table epoch of this iteration (1..2^kGEpochBits-1)
  Counters* cnt;
  int64_t vb;                           // global id of local row 0
  double gamma;
  int32_t t;                            // iteration number (1-based)
  int32_t dense;                        // 1: process every listed vertex (host-driven loop)
  const int* __restrict__ ctl;          // device-driven loop: {stopped, dense} (glp.cu k_decide), or null
  const int2* __restrict__ LV;          // LLP: (L_{t-1}[u], V[L_{t-1}[u]]) interleaved, or null
  int32_t v_ones;                       // LLP: V[l] == 1 for every l (L_{t-1} is PickLabel's permutation)
  int32_t lv_labels;                    // LLP sharded: neighbour labels are read from LV (R holds owned rows only)
  int32_t mono_kernel;                  // sorted-row candidates go to mfl_mono (launched this iteration)
  // weighted LP (mfl_weighted.cuh)
  const uint32_t* __restrict__ w2;      // arc weights beside col2
  const int64_t* __restrict__ ioff;     // [nl] row start in col2
  const int32_t* __restrict__ ideg;     // [nl] degree
  int64_t wt_lo, wt_hi;                 // local vertices of the warp kernel
  // §8(f)2 HT + CMS for L rows (mfl_kernels.cuh cms_count)
  int32_t cms;                          // 1: L rows count with HT + CMS
  unsigned cms_ht;                      // HT slots (0 = the whole L table)
  unsigned cms_depth;                   // sketch rows d (width = 8192 / d)
  // SEEDED presence filter (mfl_kernels.cuh lbit_clear): read / maintained bitmap, or null
  const uint32_t* __restrict__ lbits;
  uint32_t* lbits_w;
};

// Internal error: thrown inside the library, converted to glp_status at the ABI.
struct Err {
  glp_status st;
  std::string msg;
};

struct KStat {
  std::string name;
  int64_t launches = 0;
  double ms = 0, bytes = 0, arcs = 0;
};

}  // namespace glp

struct glp_graph {
  int device = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int rank = 0, nranks = 1;
  glp::Comm* comm = nullptr;  // exchange when nranks > 1 (or a one-rank NCCL comm)

  int64_t n = 0, vb = 0, ve = 0, nl = 0, nnz = 0;
  int64_t npad = 0;        // label arrays padded to a multiple of nranks
  int64_t nnz_global = 0;  // arcs of all ranks
  bool equal_slices = true;
  int sms = 0;
  const int64_t* off = nullptr;
  const int32_t* col = nullptr;
  bool own_csr = false;
  bool host_arcs = false;       // hybrid mode: col2 in pinned mapped host memory
  std::vector<int64_t> arc_chunks;         // create: row bounds of the arc copy chunks
  std::vector<cudaEvent_t> arc_chunk_ev;   // create: chunk c copied + checked
  bool weighted = false;        // weighted LP: w2 holds the arc weights
  uint32_t* w2 = nullptr;       // [nnz2] weights beside col2 (padding 0)
  int32_t n_gt512 = 0;          // prefix of rows with deg > kWtWarpMax
  int32_t* relay_big = nullptr;   // create: rows past kRelayBig arcs (listed by k_relayout)
  unsigned* relay_nbig = nullptr;
  bool wt_low_off = false;      // weighted low rows in mfl_wt_warp (GLP_WT_LOW=0) instead of mfl_low
  bool wt_giant = false;        // weighted giant rows go to the segmented giant kernels (totals fit kGCountBits)
  void* col2_host = nullptr;    // its host allocation
  void* registered = nullptr;   // caller's host arcs registered during create
  int symmetric = 1;
  int64_t max_deg = 0;

  // bin-major arc layout
  int32_t* col2 = nullptr;  int64_t nnz2 = 0;
  int64_t* ioff = nullptr;  // [nl] start of row v in col2
  int32_t* ideg = nullptr;  // [nl] degree of row v
  int32_t n_low = 0;
  int64_t low_base = 0;     // internal id of the first low row (= n_rows)
  int32_t* pos = nullptr;   // [npad] internal id of original vertex v (global)
  int32_t* orig = nullptr;  // [npad] original id of internal vertex q (global)
  glp::LowChunk* chunks = nullptr;   int32_t n_chunks = 0;
  uint8_t* cflag = nullptr;          // [n_chunks] chunk activity (sparse iterations)
  glp::BinItem* rows = nullptr; int32_t n_rows = 0;  // deg > 32, degree-descending
  int32_t n_gt256 = 0, n_gt2048 = 0;                 // prefixes with deg > 256 / > 2048
  int32_t n_ge8k = 0;                                // prefix with deg >= 8192
  bool w_short = false;                              // W kernel at 3 blocks/SM (mostly <= 64-arc rows)
  int32_t n_giant = 0;                               // prefix with deg > kGiantMin
  glp::GiantSeg* gsegs = nullptr; int32_t n_gsegs = 0;
  unsigned long long* gtab = nullptr; int64_t gtab_slots = 0;
  int64_t* gtab_off = nullptr;
  unsigned long long* gcand_key = nullptr;
  unsigned* gcand_lab = nullptr;
  unsigned* gdistinct = nullptr;
  int32_t* gseg_first = nullptr;                     // [n_giant+1]
  unsigned long long gepoch = 0;                     // last giant-table epoch used
  unsigned* pred[3] = {nullptr, nullptr, nullptr};   // [n_rows], distinct counts of t-1, t-2 and t
  int pb = 0;                                        // pred[pb] is read this iteration
  int32_t* redo_m = nullptr;                         // [n_rows]
  int32_t* redo_l = nullptr;                         // [n_rows]
  int32_t* push_big = nullptr;                       // [nl] changed rows of >= kPushBig arcs (push)
  int2* chg[2] = {nullptr, nullptr};                 // sparse exchange: (id, label) of owned changes, t-1 / t
  int32_t* slp_l = nullptr;                          // SLP candidates [nl * slp_k] (labels, counts)
  int32_t* slp_c = nullptr;
  int32_t slp_k = 0, slp_cap = 0;                    // K of the last SLP run, allocated K
  bool slp_valid = false;
  unsigned* chg_n = nullptr;                         // [2] their counts
  unsigned* push_nbig = nullptr;
  glp::Sched* d_sched = nullptr;
  int64_t bin_verts[glp::NBINS] = {0}, bin_arcs[glp::NBINS] = {0};

  // per-rank row bounds (all ranks), for the exchange
  std::vector<int64_t> bounds;

  // state
  int32_t* L[2] = {nullptr, nullptr};
  int2* so = nullptr;
  int32_t* V = nullptr;
  int32_t* Vloc = nullptr;  // LLP, sharded histogram: this rank's counts (summed into V)
  int2* LV = nullptr;  // LLP: (label, V of the label) of each vertex
  uint8_t* is_seed = nullptr;
  uint32_t* lbits = nullptr;  // SEEDED presence filter: bit q = L[q] >= 0 (single rank)
  uint8_t* flag[2] = {nullptr, nullptr};
  bool flag_clean[2] = {true, true};
  int32_t* stage = nullptr;  // huge bin staging buffers (grid_huge x stage_stride)
  int64_t stage_stride = 0;
  glp::Counters* d_cnt = nullptr;
  glp::Counters* h_cnt = nullptr;  // pinned
  int32_t* d_seeds = nullptr;
  int64_t seeds_cap = 0;

  // launch geometry
  int grid_low = 0, grid_w = 0, grid_m = 0, grid_l = 0, grid_g = 0, grid_aux = 0, grid_mono = 0;
  int grid_wtw = 0, grid_wtb = 0;

  int cur = 0;  // index of L holding the result of the last run
  int cur_t = 0;  // iteration being launched (profiling)
  int64_t init_launches = 0;
  bool has_run = false;
  std::vector<glp_iter_stat> iter_stats;
  std::vector<glp::KStat> kstats;
  cudaEvent_t ev_a = nullptr, ev_b = nullptr;
  // concurrent class kernels within an iteration (GLP_SERIAL=1 disables):
  // xs[0] giant, xs[1] L, xs[2] M, xs[3] low; W and the redo chain on `stream`
  bool concurrent = true;
  bool use_vl = true;  // LLP gathers (label, V[label]) pairs from LV (GLP_NO_VL=1 disables)
  bool use_mono = true;
  bool dev_loop = false;      // device-driven iteration loop (GLP_DEVICE_LOOP=1)
  int* d_ctl = nullptr;       // {stopped, dense, reason, iters, dirty[2]}
  volatile int* h_stop = nullptr;  // mapped host mirror of the stop flag
  int* d_hstop = nullptr;
  int h_ctl_init[8] = {0};
  glp::IterRec* d_rec = nullptr;
  int32_t rec_cap = 0;
  bool l2_window = false;     // A/B: persisting L2 window on the gathered array (GLP_L2_WINDOW=1)
  size_t l2_window_max = 0;  // t = 1 sorted-row candidates in mfl_mono (GLP_NO_MONO=1: in the W kernel)
  int* col_bad = nullptr;  // create: col_idx range check flag (side stream)
  cudaStream_t xs[4] = {nullptr, nullptr, nullptr, nullptr};
  cudaEvent_t xev[5] = {nullptr, nullptr, nullptr, nullptr, nullptr};
  std::vector<cudaEvent_t> ev_pool;

  // pooled device allocations (freed in destroy)
  std::vector<void*> allocs;
};
