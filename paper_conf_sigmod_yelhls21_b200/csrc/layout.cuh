// layout.cuh -- device-side construction of the bin-major arc layout
// (DESIGN.md §Layout), run once by glp_graph_create.
//
//  * low rows (1 <= deg <= 32) are sorted by (deg, id); each chunk packs
//    floor(32/deg) rows of one degree, so a chunk's segments have equal length
//    and its arcs are contiguous in col2;
//  * rows with deg > 32 are sorted by (deg desc, id); each starts 16-B aligned
//    and is padded with -1 to a multiple of 4;
//  * ioff/ideg give every vertex's row in col2 (frontier push);
//  * vertices are renumbered into this layout order (internal ids, below).
//
// Internal vertex order.  The library numbers the owned vertices of a rank
// by their layout position: rows with deg > 32 in (deg desc, id) order, then
// the low rows in (deg, id) order, then the isolated vertices.  Row i of
// `rows` is internal vertex i and low-list entry q is internal vertex
// n_rows + q, so the kernels need no vertex-id tables, and the most gathered
// labels (hubs: an arc's target is a hub with probability proportional to
// its degree) sit together at the start of each rank's label slice, where
// their 32-B sectors are shared and stay cached.  Only ids are permuted:
// label VALUES remain original vertex ids (L0[pos[v]] = v), so scores, the
// min-label tie-break (R4) and every result are unchanged; glp_labels_get
// maps back.  A rank's owned range [vb, ve) maps onto itself.
// Sorting and scans use thrust (a library primitive, the CUDA analogue of the
// qsort the oracle uses); everything else is plain kernels.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <thrust/copy.h>
#include <thrust/count.h>
#include <thrust/device_ptr.h>
#include <thrust/execution_policy.h>
#include <thrust/iterator/counting_iterator.h>
#include <thrust/scan.h>
#include <thrust/sort.h>

#include "glp_internal.cuh"

namespace glp {

struct LayoutStats {
  unsigned long long verts[NBINS];
  unsigned long long arcs[NBINS];
  unsigned long long max_deg;
  unsigned long long low_hist[33];  // vertices per low degree 1..32
  unsigned long long n_low, n_rows;
};

__global__ void k_degree_stats(const int64_t* __restrict__ off, int64_t nl, int32_t* __restrict__ deg,
                               LayoutStats* st) {
  // per-thread sums, then shared-memory totals, then one global atomic per
  // counter per block (per-vertex global atomics on a handful of addresses
  // serialised this kernel: 23 ms at RMAT-24)
  __shared__ unsigned long long s_verts[NBINS], s_arcs[NBINS], s_max, s_hist[kLowMax + 1];
  for (int i = threadIdx.x; i < NBINS; i += blockDim.x) { s_verts[i] = 0ull; s_arcs[i] = 0ull; }
  for (int i = threadIdx.x; i <= kLowMax; i += blockDim.x) s_hist[i] = 0ull;
  if (threadIdx.x == 0) s_max = 0ull;
  __syncthreads();
  unsigned long long verts[NBINS] = {0ull}, arcs[NBINS] = {0ull}, mx = 0ull;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < nl; v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t d = off[v + 1] - off[v];
    deg[v] = (int32_t)min(d, (int64_t)0x7fffffff);
    const int b = d == 0 ? BIN_ISO : d <= kLowMax ? BIN_LOW : d <= 256 ? BIN_MID : d <= 2048 ? BIN_HIGH : BIN_HUGE;
#pragma unroll
    for (int i = 0; i < NBINS; ++i) {
      verts[i] += (b == i) ? 1ull : 0ull;
      arcs[i] += (b == i) ? (unsigned long long)d : 0ull;
    }
    mx = max(mx, (unsigned long long)d);
    if (d >= 1 && d <= kLowMax) atomicAdd(&s_hist[d], 1ull);
  }
#pragma unroll
  for (int i = 0; i < NBINS; ++i) {
    if (verts[i]) atomicAdd(&s_verts[i], verts[i]);
    if (arcs[i]) atomicAdd(&s_arcs[i], arcs[i]);
  }
  if (mx) atomicMax(&s_max, mx);
  __syncthreads();
  for (int i = threadIdx.x; i < NBINS; i += blockDim.x) {
    if (s_verts[i]) atomicAdd(&st->verts[i], s_verts[i]);
    if (s_arcs[i]) atomicAdd(&st->arcs[i], s_arcs[i]);
  }
  for (int i = threadIdx.x; i <= kLowMax; i += blockDim.x)
    if (s_hist[i]) atomicAdd(&st->low_hist[i], s_hist[i]);
  if (threadIdx.x == 0 && s_max) atomicMax(&st->max_deg, s_max);
}

struct IsLow {
  const int32_t* deg;
  __host__ __device__ bool operator()(int64_t v) const { return deg[v] >= 1 && deg[v] <= kLowMax; }
};
struct IsRow {
  const int32_t* deg;
  __host__ __device__ bool operator()(int64_t v) const { return deg[v] > kLowMax; }
};
struct IsIso {
  const int32_t* deg;
  __host__ __device__ bool operator()(int64_t v) const { return deg[v] == 0; }
};

// sort keys: low rows by (deg, id); other rows by (deg desc, id)
__global__ void k_make_keys(const int32_t* __restrict__ ids, int64_t n, const int32_t* __restrict__ deg, int desc,
                            unsigned long long* __restrict__ key) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const unsigned v = (unsigned)ids[i];
    const unsigned d = (unsigned)deg[v];
    key[i] = ((unsigned long long)(desc ? ~d : d) << 32) | v;
  }
}

__global__ void k_keys_to_ids(const unsigned long long* __restrict__ key, int64_t n, int32_t* __restrict__ ids) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    ids[i] = (int32_t)(key[i] & 0xffffffffull);
}

// Degree groups of the low list: group d holds low_hist[d] rows, packed
// k = 32/d per chunk.  Tables (index d = 1..32) are built on the host.
struct LowGroups {
  int64_t vbase[34];     // first low-list index of degree d
  int64_t cbase[34];     // first chunk of degree d
  int64_t abase[34];     // first arc (col2 position) of degree d
};

__global__ void k_low_chunks(LowGroups grp, int64_t n_chunks, int64_t n_low, LowChunk* __restrict__ chunks) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n_chunks; c += (int64_t)gridDim.x * blockDim.x) {
    int d = 1;
    while (d < 32 && grp.cbase[d + 1] <= c) ++d;
    const int k = 32 / d;
    const int64_t q = c - grp.cbase[d];
    const int64_t v0 = grp.vbase[d] + q * k;
    const int nv = (int)min((int64_t)k, grp.vbase[d + 1] - v0);
    unsigned mask = 0;
    for (int j = 0; j < nv; ++j) mask |= 1u << (j * d);
    LowChunk ch;
    ch.st = (unsigned long long)(grp.abase[d] + q * (int64_t)k * d) | ((unsigned long long)d << 48) |
            ((unsigned long long)(nv * d) << 56);
    ch.vbase = (int32_t)v0;
    ch.segmask = mask;
    chunks[c] = ch;
  }
}

// ioff/ideg of low-list entry q = internal vertex low_base + q
__global__ void k_low_place(LowGroups grp, const int32_t* __restrict__ low, int64_t n_low,
                            const int32_t* __restrict__ deg, int64_t low_base, int64_t* __restrict__ ioff,
                            int32_t* __restrict__ ideg) {
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < n_low; q += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = low[q];
    const int d = deg[v];
    const int k = 32 / d;
    const int64_t p = q - grp.vbase[d];
    ioff[low_base + q] = grp.abase[d] + (p / k) * (int64_t)k * d + (p % k) * d;
    ideg[low_base + q] = d;
  }
}

__global__ void k_padded_deg(const int32_t* __restrict__ rows, int64_t n, const int32_t* __restrict__ deg,
                             int64_t* __restrict__ pdeg) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    pdeg[i] = ((int64_t)deg[rows[i]] + 3) & ~(int64_t)3;
}

__global__ void k_row_place(const int32_t* __restrict__ rows, int64_t n, const int32_t* __restrict__ deg,
                            const int64_t* __restrict__ pstart, int64_t base, BinItem* __restrict__ items,
                            int64_t* __restrict__ ioff, int32_t* __restrict__ ideg) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = rows[i];
    BinItem it;
    it.start = base + pstart[i];
    it.v = (int32_t)i;  // internal id of row i
    it.d = deg[v];
    items[i] = it;
    ioff[i] = it.start;
    ideg[i] = it.d;
  }
}

// orig_local[p] -> pos/orig of the owned slice (global ids):
//   orig[vb + p] = vb + orig_local[p],  pos[vb + orig_local[p]] = vb + p
__global__ void k_perm(const int32_t* __restrict__ orig_local, int64_t nl, int64_t vb, int32_t* __restrict__ pos,
                       int32_t* __restrict__ orig) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < nl; p += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = orig_local[p];
    orig[vb + p] = (int32_t)(vb + v);
    pos[vb + v] = (int32_t)(vb + p);
  }
}

// identity on [a, b) (label-array padding beyond n_global)
__global__ void k_iota2(int32_t* __restrict__ x, int32_t* __restrict__ y, int64_t a, int64_t b) {
  for (int64_t i = a + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < b; i += (int64_t)gridDim.x * blockDim.x) {
    x[i] = (int32_t)i;
    y[i] = (int32_t)i;
  }
}

}  // namespace glp
