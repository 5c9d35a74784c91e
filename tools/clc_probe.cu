#include <cstdio>
#include <cstdint>
__device__ __forceinline__ bool clc_steal(uint32_t *mbar_smem, uint4 *result_smem, uint32_t &phase, uint32_t &out_x) {
  // one thread: try to cancel a not-yet-launched CTA of this grid and take its id
  const uint32_t mbar = (uint32_t)__cvta_generic_to_shared(mbar_smem);
  const uint32_t res = (uint32_t)__cvta_generic_to_shared(result_smem);
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], 16;" :: "r"(mbar) : "memory");
  asm volatile("clusterlaunchcontrol.try_cancel.async.shared::cta.mbarrier::complete_tx::bytes.b128 [%0], [%1];"
               :: "r"(res), "r"(mbar) : "memory");
  uint32_t done = 0;
  while (!done) {
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                 : "=r"(done) : "r"(mbar), "r"(phase) : "memory");
  }
  phase ^= 1u;
  uint32_t ok = 0, x = 0;
  asm volatile("{ .reg .pred p; .reg .b128 r; ld.shared.b128 r, [%2];\n\t"
               "clusterlaunchcontrol.query_cancel.is_canceled.pred.b128 p, r;\n\t"
               "selp.u32 %0, 1, 0, p;\n\t"
               "@p clusterlaunchcontrol.query_cancel.get_first_ctaid::x.b32.b128 %1, r; }"
               : "=r"(ok), "=r"(x) : "r"(res) : "memory");
  out_x = x;
  return ok != 0;
}
__global__ void k(int n, unsigned *hits, unsigned *ctas) {
  __shared__ __align__(16) uint4 result;
  __shared__ __align__(8) uint64_t mbar;
  __shared__ uint32_t s_id, s_ok;
  uint32_t phase = 0;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"((uint32_t)__cvta_generic_to_shared(&mbar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    atomicAdd(ctas, 1u);
  }
  __syncthreads();
  uint32_t id = blockIdx.x;
  for (;;) {
    // "work"
    if (threadIdx.x == 0) atomicAdd(&hits[id], 1u);
    for (volatile int spin = 0; spin < 2000; spin++) {}
    __syncthreads();
    if (threadIdx.x == 0) { uint32_t x; s_ok = clc_steal((uint32_t*)&mbar, &result, phase, x); s_id = x; }
    __syncthreads();
    if (!s_ok) break;
    id = s_id;
    __syncthreads();
  }
}
int main() {
  int n = 100000; unsigned *hits, *ctas;
  cudaMalloc(&hits, n * 4); cudaMemset(hits, 0, n * 4); cudaMalloc(&ctas, 4); cudaMemset(ctas, 0, 4);
  k<<<n, 128>>>(n, hits, ctas);
  cudaError_t e = cudaDeviceSynchronize(); printf("err %s\n", cudaGetErrorString(e));
  unsigned *h = new unsigned[n]; cudaMemcpy(h, hits, n * 4, cudaMemcpyDeviceToHost); unsigned c; cudaMemcpy(&c, ctas, 4, cudaMemcpyDeviceToHost);
  int bad = 0; for (int i = 0; i < n; i++) bad += h[i] != 1; printf("bad %d launched CTAs %u of %d\n", bad, c, n);
}
