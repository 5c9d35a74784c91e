// csrc/tools/rs_math_check.cu — device self-checks of the RS body's scalar
// math (test tool, not part of the hot path): the SAME device functions the
// RS instance body compiles (apps/rsbench.cuh, built with the product's
// --fmad=false flags), evaluated on caller-given points and copied back, so
// tests/test_gpu_rs_math.py can compare them with the oracle and with IEEE
// arithmetic:
//   kind 0/1/2: dtrig sin / cos / atan (reading R-rs-trig) at x[k]
//   kind 3:     c_abs_lt6({x[2k], x[2k+1]}) as 1.0 / 0.0
//   kind 4:     div_y exactness: y[k] = the shared-reciprocal quotient of
//               x[2k] / x[2k+1] (c_div_x's path) — compared with n / den
#include <cuda_runtime.h>

#include <cstdint>

#include "../apps/rsbench.cuh"

namespace {
__global__ void rs_math_kernel(int kind, long n, const double *x, double *y) {
  for (long k = blockIdx.x * (long)blockDim.x + threadIdx.x; k < n; k += (long)gridDim.x * blockDim.x) {
    double s, c;
    switch (kind) {
      case 0: ens::dtrig::sincos_d(x[k], &s, &c); y[k] = s; break;
      case 1: ens::dtrig::sincos_d(x[k], &s, &c); y[k] = c; break;
      case 2: y[k] = ens::dtrig::atan_d(x[k]); break;
      case 3: y[k] = ens::c_abs_lt6(ens::Cx{x[2 * k], x[2 * k + 1]}) ? 1.0 : 0.0; break;
      default: {
        const double nu = x[2 * k], den = x[2 * k + 1];
        y[k] = ens::dq_safe(den) && ens::dq_safe(nu) ? ens::div_y(nu, den, __drcp_rn(den)) : nu / den;
      }
    }
  }
}
}  // namespace

// n outputs (kinds 3 and 4 read 2n inputs); host arrays; returns a cudaError_t
extern "C" int ens_tool_rs_math(int kind, long n, const double *x_host, double *y_host) {
  const long nin = (kind >= 3) ? 2 * n : n;
  double *dx = nullptr, *dy = nullptr;
  cudaError_t e = cudaMalloc(&dx, (size_t)(nin > 0 ? nin : 1) * 8);
  if (e == cudaSuccess) e = cudaMalloc(&dy, (size_t)(n > 0 ? n : 1) * 8);
  if (e == cudaSuccess && nin) e = cudaMemcpy(dx, x_host, (size_t)nin * 8, cudaMemcpyHostToDevice);
  if (e == cudaSuccess && n) {
    rs_math_kernel<<<1184, 256>>>(kind, n, dx, dy);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess && n) e = cudaMemcpy(y_host, dy, (size_t)n * 8, cudaMemcpyDeviceToHost);
  cudaFree(dx);
  cudaFree(dy);
  return (int)e;
}
