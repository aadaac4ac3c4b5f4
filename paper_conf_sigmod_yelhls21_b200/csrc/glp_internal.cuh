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
//   lists int32         degree-bin vertex lists + low-degree warp chunks
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/glp.h"

namespace glp {

// Degree bins (thresholds are compile-time: each kernel's shared-memory table
// is sized for its bin).  low: packed warps (PAPER §4.2); mid: warp per vertex;
// high/huge: block per vertex with a shared-memory hash table (PAPER §4.1).
constexpr int kLowMax = 32;       // deg <= 32   -> mfl_low  (one warp, several vertices)
constexpr int kMidMax = 256;      // deg <= 256  -> mfl_mid  (one warp, one vertex)
constexpr int kHighMax = 2048;    // deg <= 2048 -> mfl_block<128 thr, 4096 slots>
                                  // deg >  2048 -> mfl_block<1024 thr, 16384 slots,
                                  //                 partitioned recount on overflow>
constexpr int kLowBlock = 256;
constexpr int kMidBlock = 256;
constexpr int kMidSlots = 2 * kMidMax;      // per-warp table slots (key+count u32), load <= 1/2
constexpr int kHighBlock = 128;
constexpr int kHighSlots = 2 * kHighMax;    // 32 KB table, load <= 1/2
constexpr int kHighUnroll = 2;
constexpr int kHugeBlock = 1024;
constexpr int kHugeSlots = 16384;           // 128 KB table
constexpr int kHugeUnroll = 2;
constexpr int kHugeProbe = 32;              // probe limit before declaring overflow

// A low-degree chunk: up to 32 consecutive arcs of consecutive low-list
// vertices.  st = arc start in col2 | (arc count << 56); bit i of segmask set
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
  unsigned long long work_next; // dynamic work counter (huge bin)
  unsigned long long pad[2];
};

// Arguments shared by the MFL kernels (passed by value).
struct MflArgs {
  const int32_t* __restrict__ col;      // col2: bin-major arcs (global ids, -1 = padding)
  const int32_t* __restrict__ R;        // L_{t-1}, global ids [n]
  int32_t* __restrict__ W;              // L_t, global ids [n]
  int2* __restrict__ so;                // [nl] (stamp, old label)
  const int32_t* __restrict__ V;        // LLP histogram [n] or null
  const uint8_t* __restrict__ is_seed;  // [nl] or null
  const uint8_t* __restrict__ flag;     // [npad] frontier marks by global id (sparse)
  const int32_t* __restrict__ list;     // low bin: vertex list (local ids)
  const LowChunk* __restrict__ chunks;  // low bin
  int32_t n_chunks;
  const BinItem* __restrict__ items;    // mid/high/huge bins
  int32_t n_items;
  uint8_t* __restrict__ ovf_hint;       // huge bin: hash partitions to start with
  int32_t* __restrict__ stage;          // huge bin: per-block staged row labels
  int64_t stage_stride;
  Counters* cnt;
  int64_t vb;                           // global id of local row 0
  double gamma;
  int32_t t;                            // iteration number (1-based)
  int32_t dense;                        // 1: process every listed vertex
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
  void* nccl = nullptr;  // ncclComm_t when nranks > 1

  int64_t n = 0, vb = 0, ve = 0, nl = 0, nnz = 0;
  int64_t npad = 0;        // label arrays padded to a multiple of nranks
  int64_t nnz_global = 0;  // arcs of all ranks
  bool equal_slices = true;
  int sms = 0;
  const int64_t* off = nullptr;
  const int32_t* col = nullptr;
  bool own_csr = false;
  int symmetric = 1;
  int64_t max_deg = 0;

  // bin-major arc layout
  int32_t* col2 = nullptr;  int64_t nnz2 = 0;
  int64_t* ioff = nullptr;  // [nl] start of row v in col2
  int32_t* ideg = nullptr;  // [nl] degree of row v
  int32_t* low_list = nullptr;  int32_t n_low = 0;
  glp::LowChunk* chunks = nullptr;   int32_t n_chunks = 0;
  glp::BinItem* mid_items = nullptr; int32_t n_mid = 0;
  glp::BinItem* high_items = nullptr; int32_t n_high = 0;
  glp::BinItem* huge_items = nullptr; int32_t n_huge = 0;
  uint8_t* ovf_hint = nullptr;
  std::vector<uint8_t> ovf_init;  // per-run initial hints (host)
  int64_t bin_verts[glp::NBINS] = {0}, bin_arcs[glp::NBINS] = {0};

  // per-rank row bounds (all ranks), for the exchange
  std::vector<int64_t> bounds;

  // state
  int32_t* L[2] = {nullptr, nullptr};
  int2* so = nullptr;
  int32_t* V = nullptr;
  uint8_t* is_seed = nullptr;
  uint8_t* flag[2] = {nullptr, nullptr};
  bool flag_clean[2] = {true, true};
  int32_t* stage = nullptr;  // huge bin staging buffers (grid_huge x stage_stride)
  int64_t stage_stride = 0;
  glp::Counters* d_cnt = nullptr;
  glp::Counters* h_cnt = nullptr;  // pinned
  int32_t* d_seeds = nullptr;
  int64_t seeds_cap = 0;

  // launch geometry
  int grid_low = 0, grid_mid = 0, grid_high = 0, grid_huge = 0, grid_aux = 0;

  int cur = 0;  // index of L holding the result of the last run
  int cur_t = 0;  // iteration being launched (profiling)
  int64_t init_launches = 0;
  bool has_run = false;
  std::vector<glp_iter_stat> iter_stats;
  std::vector<glp::KStat> kstats;
  cudaEvent_t ev_a = nullptr, ev_b = nullptr;
  std::vector<cudaEvent_t> ev_pool;

  // pooled device allocations (freed in destroy)
  std::vector<void*> allocs;
};
