// csrc/rt/scan.cuh — block-wide prefix sum used by the instance bodies
// (XS bucket/hash offsets, Page-Rank CSR offsets).  Runs on the threads of
// one instance (the CTA, or its row with M instances per CTA).
#pragma once
#include "device_rt.cuh"

namespace ens {

// exclusive (or inclusive) prefix sum of a[0..n) (global or shared memory,
// 16-B aligned), block-wide, in coalesced tiles of 8 consecutive elements per
// thread (two 16-B loads)
template <bool INCL = false>
__device__ inline void global_exclusive_scan(uint32_t *a, long long n, Shared *sh) {
  const int tid = threadIdx.x, T = blockDim.x, lane = tid & 31, w = tid >> 5, nw = T >> 5;
  constexpr int V = 8;
  const bool vec = (reinterpret_cast<uintptr_t>(a) & 15) == 0;
  uint32_t carry = 0;
  for (long long base = 0; base < n; base += (long long)T * V) {
    const long long i0 = base + (long long)tid * V;
    uint32_t v[V];
    if (vec && i0 + V <= n) {
      const uint4 x = *reinterpret_cast<const uint4 *>(a + i0), y = *reinterpret_cast<const uint4 *>(a + i0 + 4);
      v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w; v[4] = y.x; v[5] = y.y; v[6] = y.z; v[7] = y.w;
    } else {
#pragma unroll
      for (int k = 0; k < V; k++) v[k] = i0 + k < n ? a[i0 + k] : 0u;
    }
    uint32_t sum = 0;
#pragma unroll
    for (int k = 0; k < V; k++) sum += v[k];
    uint32_t inc = sum;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += t;
    }
    if (lane == 31) sh->red_u[w] = inc;
    sub_sync();
    if (w == 0) {
      const unsigned long long t = lane < nw ? sh->red_u[lane] : 0ULL;
      unsigned long long ti = t;
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long u = __shfl_up_sync(0xffffffffu, ti, o);
        if (lane >= o) ti += u;
      }
      if (lane < nw) sh->red_u[lane] = ti - t;                         // exclusive warp offsets
      if (lane == 31) sh->red_d[0] = __longlong_as_double((long long)ti);  // tile total
    }
    sub_sync();
    uint32_t run = carry + (uint32_t)sh->red_u[w] + inc - sum;
    const uint32_t total = (uint32_t)__double_as_longlong(sh->red_d[0]);
#pragma unroll
    for (int k = 0; k < V; k++) {
      const uint32_t t = v[k];
      v[k] = INCL ? run + t : run;
      run += t;
    }
    if (vec && i0 + V <= n) {
      *reinterpret_cast<uint4 *>(a + i0) = make_uint4(v[0], v[1], v[2], v[3]);
      *reinterpret_cast<uint4 *>(a + i0 + 4) = make_uint4(v[4], v[5], v[6], v[7]);
    } else {
#pragma unroll
      for (int k = 0; k < V; k++)
        if (i0 + k < n) a[i0 + k] = v[k];
    }
    carry += total;
    sub_sync();
  }
}

// the same prefix sum of a shared-memory array in one pass: thread t owns the
// contiguous segment [tK, tK + K), K = ceil(n / T) rounded up to odd (the
// lanes' segments then start in distinct banks: no conflicts), so the whole
// array costs three barriers instead of three per 8T-element tile.  The
// caller has synchronised the array's producers; returns after a barrier.
template <bool INCL = false>
__device__ inline void smem_scan(uint32_t *a, int n, Shared *sh) {
  const int tid = threadIdx.x, T = blockDim.x, lane = tid & 31, w = tid >> 5, nw = T >> 5;
  const int K = ((n + T - 1) / T) | 1;
  const int b0 = tid * K;
  uint32_t sum = 0;
#pragma unroll 4
  for (int i = 0; i < K; i++) {
    const int x = b0 + i;
    if (x < n) sum += a[x];
  }
  uint32_t inc = sum;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += t;
  }
  if (lane == 31) sh->red_u[w] = inc;
  __syncthreads();
  if (w == 0) {
    const unsigned long long t = lane < nw ? sh->red_u[lane] : 0ULL;
    unsigned long long ti = t;
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long u = __shfl_up_sync(0xffffffffu, ti, o);
      if (lane >= o) ti += u;
    }
    if (lane < nw) sh->red_u[lane] = ti - t;  // exclusive warp offsets
  }
  __syncthreads();
  uint32_t run = (uint32_t)sh->red_u[w] + inc - sum;
#pragma unroll 4
  for (int i = 0; i < K; i++) {
    const int x = b0 + i;
    if (x < n) {
      const uint32_t t = a[x];
      a[x] = INCL ? run + t : run;
      run += t;
    }
  }
  __syncthreads();
}

}  // namespace ens
