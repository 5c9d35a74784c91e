// csrc/apps/pagerank.cuh — N1 instance body: Page-Rank-style propagation
// (the paper's fourth benchmark, HeCBench Page-Rank, §4.1 P:512-514;
// SURVEY.md §8(f) NEXT 3), on a synthetic graph (DESIGN.md R-pr-*):
//   PR-2  one LCG stream: n out-degrees 1 + LCG_int % (2e-1), then each
//         source's targets LCG_int % n in source order;
//   PR-3  r_0 = 1/n; per iteration r'[v] = (1-d)/n + d * sum over in-edges
//         (in (source, edge) order) of r[u] / deg[u], d = 0.85;
//   PR-4  checksums of r, node of maximal rank (first on ties).
// The paper could run only 2-4 Page-Rank instances on a 40 GB A100
// (P:568-570); with slot arenas the ensemble size is not bounded by memory.
//
// Block-parallel build: draw indices are computed (jump constants), the
// in-edge CSR is a counting sort by target whose per-target lists are then
// sorted by edge id — exactly the (source, edge) order the sum needs.
#pragma once
#include "../rt/device_rt.cuh"
#include "params.cuh"
#include "../rt/scan.cuh"

namespace ens {

struct PrApp {
  static constexpr uint32_t kId = APP_PAGERANK;
  static constexpr int kMaxT = 1024;
  static constexpr bool kTeam = false;
  static constexpr bool kSub = true;

  __device__ static Result run(Ctx &c, int argc, char **argv) {
    Result R{};
    PrParams p;
    const int bad = pr_parse(argc, argv, p);
    if (bad >= 0) {
      ens_printf(c, FMT_BADARG, (const char *)argv[0], (const char *)argv[bad]);
      ens_printf(c, FMT_USAGE_PR, (const char *)argv[0]);
      R.exit_code = ENS_EXIT_USAGE;
      return R;
    }
    const PrLayout L = pr_layout(p);
    if (L.total > c.arena_cap) {
      if (threadIdx.x == 0) ens_sh(c)->flags |= 2u;
      R.exit_code = ENS_EXIT_NOMEM;
      return R;
    }
    const int tid = threadIdx.x, T = blockDim.x;
    const long long n = p.n;
    uint32_t *deg = (uint32_t *)(c.arena + L.deg);
    uint32_t *dst = (uint32_t *)(c.arena + L.dstart);
    uint32_t *srce = (uint32_t *)(c.arena + L.src_of_edge);
    uint32_t *tgt = (uint32_t *)(c.arena + L.tgt);
    uint32_t *iptr = (uint32_t *)(c.arena + L.in_ptr);
    uint32_t *cur = (uint32_t *)(c.arena + L.cursor);
    uint32_t *ine = (uint32_t *)(c.arena + L.in_e);
    double *r = (double *)(c.arena + L.r);
    double *r2 = (double *)(c.arena + L.r2);

    // ---- PR-2: out-degrees (draws 1..n) --------------------------------------
    {
      const Affine JT = lcg_pow((uint64_t)T);
      uint64_t s = lcg_pow((uint64_t)tid)(p.gseed);
      for (long long u = tid; u < n; u += T, s = JT(s)) {
        uint64_t t = s;
        const uint32_t d = 1u + (uint32_t)(lcg_int(t) % (uint64_t)(2 * p.avg - 1));
        deg[u] = d;
        dst[u] = d;
        iptr[u] = 0;
      }
      if (tid == 0) {
        dst[n] = 0;
        iptr[n] = 0;
      }
    }
    sub_sync();
    global_exclusive_scan(dst, n + 1, ens_sh(c));  // dst[u] = first edge of u; dst[n] = edges
    const long long E = dst[n];
    // ---- PR-2: targets, source by source (draw n + e + 1 for edge e) --------
    for (long long u = tid; u < n; u += T) {
      const long long e0 = dst[u];
      uint64_t s = lcg_pow((uint64_t)(n + e0))(p.gseed);
      const uint32_t du = deg[u];
      for (uint32_t k = 0; k < du; k++) {
        const uint32_t v = (uint32_t)(lcg_int(s) % (uint64_t)n);
        tgt[e0 + k] = v;
        srce[e0 + k] = (uint32_t)u;
        atomicAdd(&iptr[v], 1u);
      }
    }
    sub_sync();
    global_exclusive_scan(iptr, n + 1, ens_sh(c));  // in-edge offsets
    for (long long v = tid; v < n; v += T) cur[v] = iptr[v];
    sub_sync();
    for (long long e = tid; e < E; e += T) ine[atomicAdd(&cur[tgt[e]], 1u)] = (uint32_t)e;
    sub_sync();
    // per-target lists sorted by edge id == (source, edge) order; then sources
    for (long long v = tid; v < n; v += T) {
      const uint32_t lo = iptr[v], hi = iptr[v + 1];
      for (uint32_t x = lo + 1; x < hi; x++) {
        const uint32_t key = ine[x];
        uint32_t y = x;
        while (y > lo && ine[y - 1] > key) {
          ine[y] = ine[y - 1];
          y--;
        }
        ine[y] = key;
      }
      for (uint32_t x = lo; x < hi; x++) ine[x] = srce[ine[x]];
    }
    // ---- PR-3: iterations ------------------------------------------------------
    const double d = 0.85;
    const double base = (1.0 - d) / (double)n;
    for (long long v = tid; v < n; v += T) r[v] = 1.0 / (double)n;
    sub_sync();
    for (int it = 0; it < p.iters; it++) {
      for (long long v = tid; v < n; v += T) {
        double acc = 0.0;
        for (uint32_t x = iptr[v]; x < iptr[v + 1]; x++) {
          const uint32_t u = ld_(ine + x);
          acc += ld_(r + u) / (double)ld_(deg + u);
        }
        r2[v] = base + d * acc;
      }
      sub_sync();
      double *t = r; r = r2; r2 = t;
    }
    // ---- PR-4 ---------------------------------------------------------------------
    unsigned long long bsum = 0;
    double fsum = 0.0, fabs_ = 0.0, best = -1.0;
    long long top = n;  // max rank, first index on ties
    for (long long v = tid; v < n; v += T) {
      const double x = ld_(r + v);
      bsum += dbits(x);
      fsum += x;
      fabs_ += fabs(x);
      if (x > best) {  // v increasing within a thread: keeps the first
        best = x;
        top = v;
      }
    }
    bsum = block_sum_u64(ens_sh(c), bsum);
    fsum = block_sum_f64(ens_sh(c), fsum);
    fabs_ = block_sum_f64(ens_sh(c), fabs_);
    const double bmax = block_max_f64(ens_sh(c), best);
    unsigned long long cand = (best == bmax) ? (unsigned long long)top : ~0ULL;
    for (int o = 16; o; o >>= 1) {
      const unsigned long long w = __shfl_xor_sync(0xffffffffu, cand, o);
      cand = w < cand ? w : cand;
    }
    sub_sync();
    if ((tid & 31) == 0) ens_sh(c)->red_u[tid >> 5] = cand;
    sub_sync();
    if (tid < 32) {
      unsigned long long m = tid < (T >> 5) ? ens_sh(c)->red_u[tid] : ~0ULL;
      for (int o = 16; o; o >>= 1) {
        const unsigned long long w = __shfl_xor_sync(0xffffffffu, m, o);
        m = w < m ? w : m;
      }
      if (tid == 0) ens_sh(c)->red_u[0] = m;
    }
    sub_sync();
    const long long topv = (long long)ens_sh(c)->red_u[0];
    R.vhash = bsum % 999983ULL;
    R.bitsum = bsum;
    R.fsum = fsum;
    R.fabs = fabs_;
    R.work = (uint64_t)E * (uint64_t)p.iters;
    ens_printf(c, FMT_PR, n, E, (long long)p.iters, topv);
    R.exit_code = 0;
    return R;
  }

  __host__ static bool size(int argc, const char *const *argv, int, int, uint64_t *arena, uint32_t *smem) {
    PrParams p;
    *smem = 0;
    if (pr_parse(argc, argv, p) >= 0) {
      *arena = 0;
      return false;
    }
    *arena = pr_layout(p).total;
    return true;
  }
};

}  // namespace ens
