// csrc/tools/fp64_peak.cu — measurement tool, not part of the hot path.
//
// The FP64 denominator of the RSBench-style roofline (SURVEY.md §8(d) C3:
// "the FP64 denominator comes from a DFMA microbenchmark in the same run").
// Every thread runs kChains independent DFMA chains (enough to cover the
// pipe latency at full occupancy); grid = resident CTAs x SMs.  Reported as
// FLOP/s with one DFMA = 2 FLOP, and as DP-pipe instructions/s (what an
// FMA-free --fmad=false body can at most issue: one DMUL or DADD = 1 FLOP).
#include <cuda_runtime.h>

#include <cstdint>

namespace {
constexpr int kChains = 8;
constexpr int kThreads = 256;

__global__ void __launch_bounds__(kThreads) dfma_loop(double *out, int iters, double a, double b) {
  double x[kChains];
#pragma unroll
  for (int k = 0; k < kChains; k++) x[k] = 1.0 + 1e-3 * (threadIdx.x + k);
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int k = 0; k < kChains; k++) x[k] = fma(x[k], a, b);
  }
  double s = 0.0;
#pragma unroll
  for (int k = 0; k < kChains; k++) s += x[k];
  if (s == 12345.678) out[threadIdx.x] = s;  // keeps the chains live, never true
}
}  // namespace

extern "C" {
// Runs the DFMA loop on `stream` (cudaStream_t; NULL = legacy default) and
// returns the best of `reps` launches.  *flops = achieved FLOP/s (DFMA = 2),
// *ms = best launch time.  Returns 0, or the cudaError_t on failure.
int ens_tool_fp64_peak(void *stream, int reps, double *flops, float *ms) {
  cudaStream_t s = (cudaStream_t)stream;
  int dev = 0, sms = 0, per_sm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, dfma_loop, kThreads, 0);
  const int grid = sms * (per_sm > 0 ? per_sm : 1);
  const int iters = 1 << 14;
  double *out = nullptr;
  if (cudaMalloc(&out, kThreads * sizeof(double)) != cudaSuccess) return (int)cudaGetLastError();
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  dfma_loop<<<grid, kThreads, 0, s>>>(out, iters, 0.9999999, 1e-7);  // warm-up
  float best = 1e30f;
  for (int r = 0; r < (reps > 0 ? reps : 1); r++) {
    cudaEventRecord(e0, s);
    dfma_loop<<<grid, kThreads, 0, s>>>(out, iters, 0.9999999, 1e-7);
    cudaEventRecord(e1, s);
    cudaEventSynchronize(e1);
    float t = 0.f;
    cudaEventElapsedTime(&t, e0, e1);
    if (t < best) best = t;
  }
  const cudaError_t err = cudaGetLastError();
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFree(out);
  if (err != cudaSuccess) return (int)err;
  *ms = best;
  *flops = 2.0 * kChains * (double)iters * (double)grid * kThreads / (best * 1e-3);
  return 0;
}
}
