// csrc/apps/xsbench.cuh — N1 instance body: XSBench-style macroscopic
// cross-section lookup (the paper's memory-bound benchmark, §4.1
// P:496-504), as SURVEY.md §8(c) XS-1..XS-11 defines it.  One instance runs
// on one thread block (one OpenMP team, §2.3); its parallel loops
// (grid generation, sort, index build, lookups) use the block's threads.
//
// Layout differences from upstream (results are identical):
//  * the hash index grid is stored nuclide-major [n_iso][bins+1] (bins+1-th
//    entry = n_gp-2 so u_high needs no branch): one nuclide's u_low/u_high
//    pair is 8 contiguous bytes and the init writes are coalesced;
//  * records are generated straight into per-nuclide scratch and scattered
//    once to their sorted position (no global sort pass).
#pragma once
#include "../rt/device_rt.cuh"
#include "params.cuh"

namespace ens {

// Hoogenboom-Martin material lists (SURVEY.md §8(c) "Materials").
__constant__ uint16_t kXsFuel34[34] = {58, 59, 60, 61, 40, 42, 43, 44, 45, 46, 1,  2,  3,  7,  8,  9,  10,
                                       29, 57, 47, 48, 0,  62, 15, 33, 34, 52, 53, 54, 55, 56, 18, 23, 41};
__constant__ uint16_t kXsClad[5] = {63, 64, 65, 66, 67};
__constant__ uint16_t kXsWater[4] = {24, 41, 4, 5};
__constant__ uint16_t kXsRpv[27] = {19, 20, 21, 22, 35, 36, 37, 38, 39, 25, 27, 28, 29, 30,
                                    31, 32, 26, 49, 50, 51, 11, 12, 13, 14, 6,  16, 17};
__constant__ uint16_t kXsRefl[21] = {24, 41, 4, 5, 19, 20, 21, 22, 35, 36, 37, 38, 39, 25, 49, 50, 51, 11, 12, 13, 14};
__constant__ uint16_t kXsFa[9] = {24, 41, 4, 5, 63, 64, 65, 66, 67};

__host__ __device__ __forceinline__ int hm_num_nucs(int n_iso, int m) {
  switch (m) {
    case 0: return n_iso == 68 ? 34 : 321;
    case 1: return 5;
    case 2: case 3: return 4;
    case 4: return 27;
    case 10: case 11: return 9;
    default: return 21;
  }
}
__device__ __forceinline__ int hm_nuc(int m, int j) {
  switch (m) {
    case 0: return j < 34 ? kXsFuel34[j] : 68 + (j - 34);  // large adds 68..354
    case 1: return kXsClad[j];
    case 2: case 3: return kXsWater[j];
    case 4: return kXsRpv[j];
    case 10: case 11: return kXsFa[j];
    default: return kXsRefl[j];
  }
}
// pick_mat thresholds: running sum of dist[j], j = i down to 1 (dist[0] never
// added, upstream quirk) in exactly that order.
__device__ __forceinline__ double hm_threshold(int i) {
  const double dist[12] = {0.140, 0.052, 0.275, 0.134, 0.154, 0.064, 0.066, 0.055, 0.008, 0.015, 0.025, 0.013};
  double running = 0;
  for (int j = i; j > 0; j--) running += dist[j];
  return running;
}

// Concentrations from CONC_SEED = 1070^2 (reading Q12; reproduces upstream's
// documented checksums) in m-major, j-minor order; draw d is the state after
// d+1 steps.  Also num_nucs, mats, pick_mat thresholds.  Shared with RS via
// the seed argument (RS draws its concentrations from its init stream).
__device__ inline void hm_tables(int n_iso, int mx, double *thr, int *nn, double *concs, uint16_t *mats) {
  const int tid = threadIdx.x, T = blockDim.x;
  if (tid < 12) {
    nn[tid] = hm_num_nucs(n_iso, tid);
    thr[tid] = hm_threshold(tid);
  }
  for (int x = tid; x < 12 * mx; x += T) {
    const int m = x / mx, j = x % mx;
    mats[x] = (uint16_t)(j < hm_num_nucs(n_iso, m) ? hm_nuc(m, j) : 0);
    concs[x] = 0.0;
  }
}
// concentration draw index of (m, j)
__device__ __forceinline__ int hm_draw(int n_iso, int m, int j) {
  int d = 0;
  for (int q = 0; q < m; q++) d += hm_num_nucs(n_iso, q);
  return d + j;
}
__device__ inline void hm_concs(int n_iso, int mx, double *concs, uint64_t seed0) {
  for (int x = threadIdx.x; x < 12 * mx; x += blockDim.x) {
    const int m = x / mx, j = x % mx;
    if (j < hm_num_nucs(n_iso, m)) {
      uint64_t s = lcg_pow((uint64_t)hm_draw(n_iso, m, j))(seed0);
      concs[x] = lcg_double(s);
    }
  }
}

__device__ __forceinline__ int pick_mat_thr(const double *thr, double roll) {
  for (int i = 0; i < 12; i++)
    if (roll < thr[i]) return i;
  return 0;
}

// bitonic sort of P2 (key, payload) pairs in shared memory, ascending keys
__device__ inline void smem_bitonic(uint64_t *keys, uint16_t *perm, int P2) {
  const int tid = threadIdx.x, T = blockDim.x;
  for (int k = 2; k <= P2; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int x = tid; x < (P2 >> 1); x += T) {
        const int i = ((x & ~(j - 1)) << 1) | (x & (j - 1));
        const int l = i + j;
        const bool up = (i & k) == 0;
        const uint64_t a = keys[i], b = keys[l];
        if ((a > b) == up) {
          keys[i] = b;
          keys[l] = a;
          const uint16_t t = perm[i];
          perm[i] = perm[l];
          perm[l] = t;
        }
      }
      __syncthreads();
    }
  }
}

// grid_search over sorted energies given as u64 bit patterns of doubles
__device__ __forceinline__ int gs_keys(const uint64_t *keys, double q, int lo, int hi) {
  int len = hi - lo;
  while (len > 1) {
    const int m = lo + len / 2;
    if (__longlong_as_double((long long)keys[m]) > q) hi = m;
    else lo = m;
    len = hi - lo;
  }
  return lo;
}
// grid_search over the energy field of 48-B records
__device__ __forceinline__ int gs_recs(const double *E6, double q, int lo, int hi) {
  int len = hi - lo;
  while (len > 1) {
    const int m = lo + len / 2;
    if (ld_(E6 + 6 * (size_t)m) > q) hi = m;
    else lo = m;
    len = hi - lo;
  }
  return lo;
}
__device__ __forceinline__ long long gs_u64(const uint64_t *A, double q, long long lo, long long hi) {
  long long len = hi - lo;
  while (len > 1) {
    const long long m = lo + len / 2;
    if (__longlong_as_double((long long)ld_((const unsigned long long *)A + m)) > q) hi = m;
    else lo = m;
    len = hi - lo;
  }
  return lo;
}

struct XsApp {
  static constexpr uint32_t kId = APP_XSBENCH;

  __device__ static Result run(Ctx &c, int argc, char **argv) {
    Result R{};
    XsParams p;
    const int bad = xs_parse(argc, argv, p);
    if (bad >= 0) {
      ens_printf(c, FMT_BADARG, (const char *)argv[0], (const char *)argv[bad]);
      ens_printf(c, FMT_USAGE_XS, (const char *)argv[0]);
      R.exit_code = ENS_EXIT_USAGE;
      return R;
    }
    const XsLayout L = xs_layout(p);
    if (L.total > c.arena_cap) {
      if (threadIdx.x == 0) c.sh->flags |= 2u;  // ENS_RF_NOMEM
      R.exit_code = ENS_EXIT_NOMEM;
      return R;
    }
    const int tid = threadIdx.x, T = blockDim.x;
    const int n_iso = p.n_iso, n_gp = p.n_gp, mx = xs_max_nucs(n_iso);
    const long long n_u = (long long)n_iso * n_gp;
    const XsSmem S = xs_smem(p);
    double *thr = (double *)(c.smem + S.thr);
    int *nn = (int *)(c.smem + S.nn);
    double *concs = (double *)(c.smem + S.concs);
    uint16_t *mats = (uint16_t *)(c.smem + S.mats);
    uint64_t *keys = (uint64_t *)(c.smem + S.keys);
    uint16_t *perm = (uint16_t *)(c.smem + S.perm);
    double *recs = (double *)(c.arena + L.recs);
    double *scr = (double *)(c.arena + L.scratch);
    int *ig = (int *)(c.arena + L.index);

    // ---- XS-2: materials, concentrations ---------------------------------
    hm_tables(n_iso, mx, thr, nn, concs, mats);
    __syncthreads();
    hm_concs(n_iso, mx, concs, 1070ULL * 1070ULL);

    // ---- XS-3/4/5: nuclide grid, per-nuclide sort, hash column / union run
    const int P2 = pow2_ceil(n_gp);
    const Affine J6T = lcg_pow(6ULL * T);
    const Affine Jnuc = lcg_pow(6ULL * n_gp);
    uint64_t s_nuc = lcg_pow(6ULL * tid)(p.gseed);  // record (i*n_gp + tid)
    uint64_t *uA = (uint64_t *)(c.arena + L.uenergy), *uB = (uint64_t *)(c.arena + L.utmp);
    uint16_t *oA = (uint16_t *)(c.arena + L.uown), *oB = (uint16_t *)(c.arena + L.uowntmp);
    int rounds = 0;
    while ((1 << rounds) < n_iso) rounds++;
    // merge rounds alternate buffers; start where the result ends in uA
    uint64_t *urun = (rounds & 1) ? uB : uA;
    uint16_t *orun = (rounds & 1) ? oB : oA;
    const double du = 1.0 / p.bins;
    for (int i = 0; i < n_iso; i++) {
      uint64_t s = s_nuc;
      for (int j = tid; j < P2; j += T) {
        if (j < n_gp) {
          uint64_t t = s;
          double v[6];
#pragma unroll
          for (int f = 0; f < 6; f++) v[f] = lcg_double(t);
          double2 *d = reinterpret_cast<double2 *>(scr + 6 * (size_t)j);
          d[0] = make_double2(v[0], v[1]);
          d[1] = make_double2(v[2], v[3]);
          d[2] = make_double2(v[4], v[5]);
          keys[j] = dbits(v[0]);
          perm[j] = (uint16_t)j;
          s = J6T(s);
        } else {
          keys[j] = ~0ULL;
          perm[j] = 0xFFFF;
        }
      }
      s_nuc = Jnuc(s_nuc);
      __syncthreads();
      smem_bitonic(keys, perm, P2);
      double *rec_i = recs + (size_t)i * n_gp * 6;
      for (int k = tid; k < n_gp; k += T) {
        const double2 *src = reinterpret_cast<const double2 *>(scr + 6 * (size_t)perm[k]);
        double2 *dst = reinterpret_cast<double2 *>(rec_i + 6 * (size_t)k);
        const double2 a = src[0], b = src[1], e = src[2];
        dst[0] = a;
        dst[1] = b;
        dst[2] = e;
      }
      if (p.grid == XS_HASH) {
        int *col = ig + (size_t)i * (p.bins + 1);
        for (int b = tid; b < p.bins; b += T) col[b] = gs_keys(keys, (double)b * du, 0, n_gp - 1);
        if (tid == 0) col[p.bins] = n_gp - 2;
      } else if (p.grid == XS_UNIONIZED) {
        for (int k = tid; k < n_gp; k += T) {
          urun[(size_t)i * n_gp + k] = keys[k];
          orun[(size_t)i * n_gp + k] = (uint16_t)i;
        }
      }
      __syncthreads();
    }

    if (p.grid == XS_UNIONIZED) {
      // ---- union: bottom-up merge of the n_iso sorted runs (merge path) ----
      uint64_t *src = urun, *dst = (urun == uA) ? uB : uA;
      uint16_t *osrc = orun, *odst = (orun == oA) ? oB : oA;
      const int CH = 16;
      for (long long w = n_gp; w < n_u; w <<= 1) {
        for (long long c0 = (long long)tid * CH; c0 < n_u; c0 += (long long)T * CH) {
          const long long c1 = (c0 + CH < n_u) ? c0 + CH : n_u;
          for (long long o0 = c0; o0 < c1;) {  // a chunk may straddle merge pairs
            const long long base = (o0 / (2 * w)) * (2 * w);
            const long long la = (base + w < n_u) ? w : n_u - base;
            const long long lb = (base + 2 * w < n_u) ? w : (n_u - base - la > 0 ? n_u - base - la : 0);
            const uint64_t *A = src + base, *B = src + base + la;
            const long long op = o0 - base;
            long long lo = op - lb > 0 ? op - lb : 0, hi = op < la ? op : la;
            while (lo < hi) {
              const long long mid = (lo + hi) >> 1;
              if (A[mid] < B[op - 1 - mid]) lo = mid + 1;
              else hi = mid;
            }
            long long ia = lo, ib = op - lo;
            const long long end = (c1 < base + la + lb) ? c1 : base + la + lb;
            for (long long o = o0; o < end; o++) {
              if (ia < la && (ib >= lb || A[ia] < B[ib])) {
                dst[o] = A[ia];
                odst[o] = osrc[base + ia];
                ia++;
              } else {
                dst[o] = B[ib];
                odst[o] = osrc[base + la + ib];
                ib++;
              }
            }
            o0 = end;
          }
        }
        __syncthreads();
        uint64_t *t = src; src = dst; dst = t;
        uint16_t *to = osrc; osrc = odst; odst = to;
      }
      // src == uA here. ---- index grid: ig[e][i] = clip(#{k>=1: E_i[k] <= u_e}, 0, n_gp-2)
      const int lane = tid & 31, warp = tid >> 5, nw = T >> 5;
      const long long C = (n_u + nw * 4 - 1) / (nw * 4) > 512 ? (n_u + nw * 4 - 1) / (nw * 4) : 512;
      const long long ntask = (n_u + C - 1) / C;
      for (long long task = warp; task < ntask; task += nw) {
        const long long e0 = task * C, e1 = (e0 + C < n_u) ? e0 + C : n_u;
        int cnt[12];
        const double ue0 = __longlong_as_double((long long)uA[e0]);
#pragma unroll
        for (int m = 0; m < 12; m++) {
          const int i = lane + 32 * m;
          cnt[m] = 0;
          if (i < n_iso) {  // #{k : E_i[k] < u[e0]}
            const double *E = recs + (size_t)i * n_gp * 6;
            int lo = 0, hi = n_gp;
            while (lo < hi) {
              const int mid = (lo + hi) >> 1;
              if (ld_(E + 6 * (size_t)mid) < ue0) lo = mid + 1;
              else hi = mid;
            }
            cnt[m] = lo;
          }
        }
        for (long long e = e0; e < e1; e++) {
          const int own = oA[e];
          int *row = ig + (size_t)e * n_iso;
#pragma unroll
          for (int m = 0; m < 12; m++) {
            const int i = lane + 32 * m;
            if (i < n_iso) {
              if (own == i) cnt[m]++;
              int v = cnt[m] - 1;
              v = v < 0 ? 0 : (v > n_gp - 2 ? n_gp - 2 : v);
              row[i] = v;
            }
          }
        }
      }
      __syncthreads();
    }

    // ---- XS-6..XS-10: lookups, thread per lookup ---------------------------
    unsigned long long ver = 0, bsum = 0;
    double fsum = 0.0, fabs_ = 0.0;
    const Affine J2T = lcg_pow(2ULL * T);
    uint64_t s = lcg_pow(2ULL * tid)(p.seed);
    for (long long li = tid; li < p.lookups; li += T, s = J2T(s)) {
      uint64_t t = s;
      const double pe = lcg_double(t);
      const int mat = pick_mat_thr(thr, lcg_double(t));
      long long idx = 0;
      if (p.grid == XS_UNIONIZED) {
        idx = gs_u64(uA, pe, 0, n_u - 1);
      } else if (p.grid == XS_HASH) {
        idx = (long long)(pe / du);
        if (idx > p.bins - 1) idx = p.bins - 1;  // reading Q14
      }
      double macro[5] = {0.0, 0.0, 0.0, 0.0, 0.0};
      const int nm = nn[mat];
      for (int j = 0; j < nm; j++) {
        const int nuc = mats[mat * mx + j];
        const double conc = concs[mat * mx + j];
        const double *E = recs + (size_t)nuc * n_gp * 6;
        int lo;
        if (p.grid == XS_NUCLIDE) {
          const int k = gs_recs(E, pe, 0, n_gp - 1);
          lo = (k == n_gp - 1) ? k - 1 : k;
        } else if (p.grid == XS_UNIONIZED) {
          const int k = ld_(ig + (size_t)idx * n_iso + nuc);
          lo = (k == n_gp - 1) ? k - 1 : k;
        } else {
          const int *col = ig + (size_t)nuc * (p.bins + 1) + idx;
          const int u_low = ld_(col), u_high = ld_(col + 1) + 1;
          const double e_low = ld_(E + 6 * (size_t)u_low), e_high = ld_(E + 6 * (size_t)u_high);
          int lower;
          if (pe <= e_low) lower = 0;
          else if (pe >= e_high) lower = n_gp - 1;
          else lower = gs_recs(E, pe, u_low, u_high);
          lo = (lower == n_gp - 1) ? lower - 1 : lower;
        }
        const double2 *r2 = reinterpret_cast<const double2 *>(E + 6 * (size_t)lo);
        const double2 a0 = ld_(r2 + 0), a1 = ld_(r2 + 1), a2 = ld_(r2 + 2);
        const double2 b0 = ld_(r2 + 3), b1 = ld_(r2 + 4), b2 = ld_(r2 + 5);
        // low = {a0.x=E, a0.y=total, a1.x=elastic, a1.y=absorption, a2.x=fission, a2.y=nu_fission}
        const double f = (b0.x - pe) / (b0.x - a0.x);
        macro[0] += (b0.y - f * (b0.y - a0.y)) * conc;
        macro[1] += (b1.x - f * (b1.x - a1.x)) * conc;
        macro[2] += (b1.y - f * (b1.y - a1.y)) * conc;
        macro[3] += (b2.x - f * (b2.x - a2.x)) * conc;
        macro[4] += (b2.y - f * (b2.y - a2.y)) * conc;
      }
      double mxv = -1.0;
      int am = 0;
#pragma unroll
      for (int q = 0; q < 5; q++)
        if (macro[q] > mxv) {
          mxv = macro[q];
          am = q;
        }
      ver += (unsigned long long)(am + 1);
      atomicAdd(&c.sh->tallies[am], 1u);
      atomicAdd(&c.sh->tallies[5 + mat], 1u);
#pragma unroll
      for (int q = 0; q < 5; q++) {
        bsum += dbits(macro[q]);
        fsum += macro[q];
        fabs_ += fabs(macro[q]);
      }
    }
    ver = block_sum_u64(c.sh, ver);
    bsum = block_sum_u64(c.sh, bsum);
    fsum = block_sum_f64(c.sh, fsum);
    fabs_ = block_sum_f64(c.sh, fabs_);
    R.vhash = ver % 999983ULL;
    R.bitsum = bsum;
    R.fsum = fsum;
    R.fabs = fabs_;
    R.work = (uint64_t)p.lookups;
    const char *grid = p.grid == XS_UNIONIZED ? "unionized" : p.grid == XS_NUCLIDE ? "nuclide" : "hash";
    ens_printf(c, FMT_XS_HDR, n_iso == 68 ? "small" : "large", n_iso, (long long)n_gp, grid, p.lookups,
               (unsigned long long)p.seed);
    ens_printf(c, FMT_VERIFY, (unsigned long long)R.vhash);
    R.exit_code = 0;
    return R;
  }

  __host__ static bool size(int argc, const char *const *argv, uint64_t *arena, uint32_t *smem) {
    XsParams p;
    if (xs_parse(argc, argv, p) >= 0) {
      *arena = 0;
      *smem = 0;
      return false;
    }
    *arena = xs_layout(p).total;
    *smem = xs_smem(p).total;
    return true;
  }
};

}  // namespace ens
