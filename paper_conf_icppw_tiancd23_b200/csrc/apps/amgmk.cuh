// csrc/apps/amgmk.cuh — N1 instance body: AMGmk-style CSR relax / matvec
// (the paper's HeCBench AMGmk relax benchmark, §4.1), as SURVEY.md
// §8(c) AMG-1..AMG-4 defines it: pure Jacobi (reading Q15), 7-point
// Laplacian rows in lexicographic order, entries diag-first then ascending
// columns (AMG-2), every row sum in CSR order (the order fixes the bits).
//
// B200 layout: SELL-32 (slices of 32 rows; entry e of the slice's 32 rows
// contiguous; rows padded to 7 entries, col = -1).  Thread = row, warp =
// slice, so every entry load of a warp is one coalesced 128-B (col) / 256-B
// (val) transaction — the fix for the paper's coalescing diagnosis
// inside an instance.  Entry order within a row is unchanged.
#pragma once
#include "../rt/device_rt.cuh"
#include "params.cuh"

namespace ens {

struct AmgApp {
  static constexpr uint32_t kId = APP_AMGMK;
  static constexpr int kMaxT = 1024;  // 64 registers suffice
  static constexpr bool kTeam = false;
  static constexpr bool kSub = true;  // runs as one of M instances per CTA (row threadIdx.y)

  __device__ static Result run(Ctx &c, int argc, char **argv) {
    Result R{};
    AmgParams p;
    const int bad = amg_parse(argc, argv, p);
    if (bad >= 0) {
      ens_printf(c, FMT_BADARG, (const char *)argv[0], (const char *)argv[bad]);
      ens_printf(c, FMT_USAGE_AMG, (const char *)argv[0]);
      R.exit_code = ENS_EXIT_USAGE;
      return R;
    }
    const AmgLayout L = amg_layout(p);
    if (L.total > c.arena_cap) {
      if (threadIdx.x == 0) ens_sh(c)->flags |= 2u;
      R.exit_code = ENS_EXIT_NOMEM;
      return R;
    }
    const int tid = threadIdx.x, T = blockDim.x;
    const long long n = L.n;
    const int nx = p.nx, ny = p.ny, nz = p.nz;
    int *col = (int *)(c.arena + L.col);
    double *val = (double *)(c.arena + L.val);
    double *f = (double *)(c.arena + L.f);
    double *u = (double *)(c.arena + L.u);
    double *u2 = (double *)(c.arena + L.u2);
    double *y = (double *)(c.arena + L.y);

    // ---- AMG-2: matrix (SELL-32), f = A*1, u0, y = 0 ----------------------
    const Affine JT = lcg_pow((uint64_t)T);
    uint64_t s = lcg_pow((uint64_t)tid)(p.seed);
    for (long long r = tid; r < n; r += T, s = JT(s)) {
      const long long ix = r % nx, iy = (r / nx) % ny, iz = r / ((long long)nx * ny);
      int cc[7];
      double vv[7];
      int k = 0;
      cc[k] = (int)r; vv[k++] = 6.0;
      if (iz > 0) { cc[k] = (int)(r - (long long)nx * ny); vv[k++] = -1.0; }
      if (iy > 0) { cc[k] = (int)(r - nx); vv[k++] = -1.0; }
      if (ix > 0) { cc[k] = (int)(r - 1); vv[k++] = -1.0; }
      if (ix < nx - 1) { cc[k] = (int)(r + 1); vv[k++] = -1.0; }
      if (iy < ny - 1) { cc[k] = (int)(r + nx); vv[k++] = -1.0; }
      if (iz < nz - 1) { cc[k] = (int)(r + (long long)nx * ny); vv[k++] = -1.0; }
      const long long base = (r >> 5) * 7 * 32 + (r & 31);
      double fs = 0.0;
#pragma unroll
      for (int e = 0; e < 7; e++) {
        col[base + 32 * e] = e < k ? cc[e] : -1;
        val[base + 32 * e] = e < k ? vv[e] : 0.0;
        if (e < k) fs += vv[e] * 1.0;
      }
      f[r] = fs;
      if (p.seed == 0) {
        u[r] = 1.0;
      } else {
        uint64_t t = s;
        u[r] = lcg_double(t);
      }
      y[r] = 0.0;
    }
    sub_sync();

    // ---- AMG-3: Jacobi sweeps and/or matvec -------------------------------
    for (int it = 0; it < p.iters; it++) {
      if (p.kind == 0 || p.kind == 2) {
        for (long long r = tid; r < n; r += T) {
          const long long base = (r >> 5) * 7 * 32 + (r & 31);
          const double a0 = ld_(val + base);
          double res = ld_(f + r);
#pragma unroll
          for (int e = 1; e < 7; e++) {
            const int cj = ld_(col + base + 32 * e);
            if (cj >= 0) res -= ld_(val + base + 32 * e) * ld_(u + cj);
          }
          u2[r] = res / a0;
        }
        sub_sync();
        double *t = u; u = u2; u2 = t;
      }
      if (p.kind == 1 || p.kind == 2) {
        for (long long r = tid; r < n; r += T) {
          const long long base = (r >> 5) * 7 * 32 + (r & 31);
          double acc = 0.0;
#pragma unroll
          for (int e = 0; e < 7; e++) {
            const int cj = ld_(col + base + 32 * e);
            if (cj >= 0) acc += ld_(val + base + 32 * e) * ld_(u + cj);
          }
          y[r] = acc;
        }
        sub_sync();
      }
    }

    // ---- AMG-4: checksums of the reported vector --------------------------
    const double *Rv = (p.kind == 0) ? u : y;
    unsigned long long bsum = 0;
    double fsum = 0.0, fabs_ = 0.0, mxe = 0.0;
    for (long long r = tid; r < n; r += T) {
      const double v = ld_(Rv + r);
      bsum += dbits(v);
      fsum += v;
      fabs_ += fabs(v);
      const double e = fabs(v - (p.kind == 0 ? 1.0 : ld_(f + r)));
      if (e > mxe) mxe = e;
      if (c.dump) dump_row(c.dump, c.dump_rows, r, (double)r, 0, &v, 1, -1);
    }
    bsum = block_sum_u64(ens_sh(c), bsum);
    fsum = block_sum_f64(ens_sh(c), fsum);
    fabs_ = block_sum_f64(ens_sh(c), fabs_);
    mxe = block_max_f64(ens_sh(c), mxe);
    R.vhash = bsum % 999983ULL;
    R.bitsum = bsum;
    R.fsum = fsum;
    R.fabs = fabs_;
    R.work = (uint64_t)n * (uint64_t)p.iters * (p.kind == 2 ? 2u : 1u);
    ens_printf(c, FMT_AMG, (int)n, (int)L.nnz, p.iters, mxe);
    R.exit_code = 0;
    return R;
  }

  __host__ static bool size(int argc, const char *const *argv, int, int, uint64_t *arena, uint32_t *smem) {
    AmgParams p;
    *smem = 0;
    if (amg_parse(argc, argv, p) >= 0) {
      *arena = 0;
      return false;
    }
    *arena = amg_layout(p).total;
    return true;
  }
};

}  // namespace ens
