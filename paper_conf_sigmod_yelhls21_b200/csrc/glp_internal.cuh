// glp_internal.cuh -- internal types of libglp.so (not part of the ABI).
//
// Data layout in HBM:
//   off   int64[nl+1]   CSR row offsets of the owned rows           [P:97]
//   col   int32[nnz]    global neighbour ids, streamed once/iter    [P:97]
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
constexpr int kHighMax = 4096;    // deg <= 4096 -> mfl_high (256-thread block per vertex)
                                  // deg >  4096 -> mfl_huge (1024-thread block, smem
                                  //                 table + global overflow table)
constexpr int kLowBlock = 256;
constexpr int kMidBlock = 256;
constexpr int kMidSlots = 2 * kMidMax;      // per-warp table slots (u64)
constexpr int kHighBlock = 256;
constexpr int kHighSlots = 2 * kHighMax;    // 64 KB table
constexpr int kHugeBlock = 1024;
constexpr int kHugeSlots = 24576;           // 192 KB table
constexpr int kHugeProbe = 32;              // probe limit before declaring overflow

enum Bin { BIN_ISO = 0, BIN_LOW = 1, BIN_MID = 2, BIN_HIGH = 3, BIN_HUGE = 4, NBINS = 5 };

// Device counters of one iteration (reset per iteration).
struct Counters {
  unsigned long long changed;   // #{v : L_t != L_{t-1}}
  unsigned long long d2;        // #{v : L_t != L_{t-2}}
  unsigned long long chdeg;     // sum of deg over changed vertices
  unsigned long long arcs;      // arcs scanned
  unsigned long long verts;     // vertices scanned
  unsigned long long huge_next; // dynamic work counter of mfl_huge
  unsigned long long pad[2];
};

// Arguments shared by the MFL kernels (passed by value).
struct MflArgs {
  const int64_t* __restrict__ off;      // [nl+1]
  const int32_t* __restrict__ col;      // [nnz]
  const int32_t* __restrict__ R;        // L_{t-1}, global ids [n]
  int32_t* __restrict__ W;              // L_t, global ids [n]
  int2* __restrict__ so;                // [nl] (stamp, old label)
  const int32_t* __restrict__ V;        // LLP histogram [n] or null
  const uint8_t* __restrict__ is_seed;  // [nl] or null
  const uint8_t* __restrict__ flag;     // [npad] frontier marks by global id (sparse)
  const int32_t* __restrict__ list;     // bin vertex list (local ids)
  int32_t list_len;
  const int32_t* __restrict__ chunk;    // low bin: chunk starts into list [nchunks+1]
  int32_t n_chunks;
  unsigned long long* __restrict__ ght; // huge: per-block global overflow tables
  int64_t ght_slots;                    // slots per block
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

  // degree bins (device lists of local ids)
  int32_t* low_list = nullptr;  int32_t n_low = 0;
  int32_t* low_chunk = nullptr; int32_t n_chunks = 0;
  int32_t* mid_list = nullptr;  int32_t n_mid = 0;
  int32_t* high_list = nullptr; int32_t n_high = 0;
  int32_t* huge_list = nullptr; int32_t n_huge = 0;
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
  unsigned long long* ght = nullptr;
  int64_t ght_slots = 0;
  glp::Counters* d_cnt = nullptr;
  glp::Counters* h_cnt = nullptr;  // pinned
  int32_t* d_seeds = nullptr;
  int64_t seeds_cap = 0;

  // launch geometry
  int grid_low = 0, grid_mid = 0, grid_high = 0, grid_huge = 0, grid_aux = 0;

  int cur = 0;  // index of L holding the result of the last run
  bool has_run = false;
  std::vector<glp_iter_stat> iter_stats;
  std::vector<glp::KStat> kstats;
  cudaEvent_t ev_a = nullptr, ev_b = nullptr;
  std::vector<cudaEvent_t> ev_pool;

  // pooled device allocations (freed in destroy)
  std::vector<void*> allocs;
};
