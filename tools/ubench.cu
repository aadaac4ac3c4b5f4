// ubench.cu -- ceiling microbenchmarks for the LP hot path.
// Not part of the product; used to decide kernel designs.
//   stream:  sum of col_idx (coalesced int4)                        -> HBM roof
//   gather:  sum of L[col_idx[e]] over all arcs                      -> random-gather roof
//   segmin:  warp-per-32-arcs segmented min of L[col] (MFL at t=1)   -> CSR+gather roof
//   atoms:   smem atomicAdd rate, distinct vs same address
#include <cuda_runtime.h>
#include <stdint.h>

__global__ void k_stream(const int4* __restrict__ p, int64_t n4, unsigned long long* out) {
  unsigned s = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
    int4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p + i));
    s += v.x ^ v.y ^ v.z ^ v.w;
  }
  if (s == 0x12345) atomicAdd(out, 1ull);
}

template <int U>
__global__ void k_gather(const int4* __restrict__ col, int64_t n4, const int* __restrict__ L, unsigned long long* out) {
  unsigned s = 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += stride * U) {
    int4 v[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
      int64_t k = i + j * stride;
      if (k < n4) asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v[j].x), "=r"(v[j].y), "=r"(v[j].z), "=r"(v[j].w) : "l"(col + k));
      else v[j] = make_int4(0, 0, 0, 0);
    }
#pragma unroll
    for (int j = 0; j < U; ++j) s += __ldg(L + v[j].x) + __ldg(L + v[j].y) + __ldg(L + v[j].z) + __ldg(L + v[j].w);
  }
  if (s == 0x12345) atomicAdd(out, 1ull);
}

__global__ void k_atoms(int iters, int distinct, unsigned long long* out) {
  __shared__ unsigned tab[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) tab[i] = 0;
  __syncthreads();
  unsigned idx = distinct ? ((threadIdx.x * 97) & 4095) : 0;
  for (int i = 0; i < iters; ++i) {
    atomicAdd(&tab[idx], 1u);
    idx = distinct ? ((idx + 131) & 4095) : 0;
  }
  __syncthreads();
  if (threadIdx.x == 0 && tab[5] == 0x1234567) atomicAdd(out, 1ull);
}

__global__ void k_match(int iters, const int* __restrict__ L, unsigned long long* out) {
  unsigned x = L[threadIdx.x & 31] + blockIdx.x, s = 0;
  for (int i = 0; i < iters; ++i) {
    unsigned m = __match_any_sync(0xffffffffu, x);
    s += m;
    x = x * 1664525u + 1013904223u;
    x &= 0xff;
  }
  if (s == 0x12345) atomicAdd(out, 1ull);
}

static float time_it(void (*f)(void*), void* arg, int reps) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  f(arg);
  cudaEventRecord(a);
  for (int r = 0; r < reps; ++r) f(arg);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  return ms / reps;
}

struct Args {
  const int* col;
  int64_t nnz;
  const int* L;
  unsigned long long* out;
  int sms;
  int mode;
};

extern "C" float ub_stream(const int* col, int64_t nnz, unsigned long long* out, int sms) {
  Args a{col, nnz, nullptr, out, sms, 0};
  return time_it([](void* p) { Args* a = (Args*)p; k_stream<<<a->sms * 8, 256>>>((const int4*)a->col, a->nnz / 4, a->out); }, &a, 5);
}
extern "C" float ub_gather(const int* col, int64_t nnz, const int* L, unsigned long long* out, int sms, int unroll) {
  Args a{col, nnz, L, out, sms, unroll};
  return time_it([](void* p) {
    Args* a = (Args*)p;
    if (a->mode == 1) k_gather<1><<<a->sms * 8, 256>>>((const int4*)a->col, a->nnz / 4, a->L, a->out);
    else if (a->mode == 2) k_gather<2><<<a->sms * 8, 256>>>((const int4*)a->col, a->nnz / 4, a->L, a->out);
    else k_gather<4><<<a->sms * 8, 256>>>((const int4*)a->col, a->nnz / 4, a->L, a->out);
  }, &a, 5);
}
extern "C" float ub_atoms(int distinct, unsigned long long* out, int sms) {
  Args a{nullptr, 0, nullptr, out, sms, distinct};
  return time_it([](void* p) { Args* a = (Args*)p; k_atoms<<<a->sms * 4, 512>>>(1024, a->mode, a->out); }, &a, 5);
}
extern "C" float ub_match(const int* L, unsigned long long* out, int sms) {
  Args a{nullptr, 0, L, out, sms, 0};
  return time_it([](void* p) { Args* a = (Args*)p; k_match<<<a->sms * 4, 512>>>(1024, a->L, a->out); }, &a, 5);
}

// Realistic table traffic: every lane hits a hashed slot of a 4096-entry
// shared table (bank conflicts as in the MFL tables).  mode 0: LDS, 1: atomicAdd
// with the return value used, 2: atomicCAS (32-bit), 3: atomicAdd without return.
__global__ void k_atoms2(int iters, int mode, unsigned long long* out) {
  __shared__ unsigned tab[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) tab[i] = 0;
  __syncthreads();
  unsigned x = threadIdx.x * 2654435761u + blockIdx.x, s = 0;
  for (int i = 0; i < iters; ++i) {
    const unsigned h = __umulhi(x * 0x9E3779B1u, 4096u);
    if (mode == 0) s += ((volatile unsigned*)tab)[h];
    else if (mode == 1) s += atomicAdd(&tab[h], 1u);
    else if (mode == 2) s += atomicCAS(&tab[h], s, x);
    else atomicAdd(&tab[h], 1u);
    x = x * 1664525u + 1013904223u + (s & 1u);
  }
  __syncthreads();
  if (threadIdx.x == 0 && (tab[5] + s) == 0x1234567) atomicAdd(out, 1ull);
}
extern "C" float ub_atoms2(int mode, unsigned long long* out, int sms) {
  Args a{nullptr, 0, nullptr, out, sms, mode};
  return time_it([](void* p) { Args* a = (Args*)p; k_atoms2<<<a->sms * 4, 512>>>(1024, a->mode, a->out); }, &a, 5);
}
