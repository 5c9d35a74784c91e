// csrc/apps/xsbench.cuh — N1 instance body: XSBench-style macroscopic
// cross-section lookup (the paper's memory-bound benchmark, §4.1
// P:496-504), as SURVEY.md §8(c) XS-1..XS-11 defines it.  One instance runs
// on one thread block (one OpenMP team, §2.3); its parallel loops
// (grid generation, sort, index build, lookups) use the block's threads.
//
// B200 design (results identical to the oracle):
//  * init keeps shared memory small (material tables + bucket counters) so
//    the L1 stays large for the lookup phase: each nuclide's records are
//    generated into an L2-resident scratch (LCG jump constants), sorted by a
//    bucket sort (energies are uniform in [0,1): counts -> scan -> scatter ->
//    insertion sort of ~1.4-element buckets), then scattered once to their
//    sorted position;
//  * the hash index grid is stored nuclide-major [n_iso][bins+1] (entry
//    `bins` = n_gp-2, so u_high needs no branch) and built by a merge walk;
//  * lookups run warp-cooperatively: lane = lookup for the sampling and the
//    union search (32 independent searches in flight), then lane = nuclide
//    for the bracket + record gathers of one lookup at a time (no divergence
//    between materials of 4 and 321 nuclides), and the macroscopic sum is a
//    shuffle fold in nuclide order (the oracle's summation order, so every
//    bit matches).
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

// num_nucs, mats (u16), pick_mat thresholds; concs zeroed.
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
// concentration draw index of (m, j): m-major, j-minor
__device__ __forceinline__ int hm_draw(int n_iso, int m, int j) {
  int d = 0;
  for (int q = 0; q < m; q++) d += hm_num_nucs(n_iso, q);
  return d + j;
}
// concs[m][j] = the (d+1)-th LCG double from seed0, d = hm_draw(m, j).
// XS: seed0 = CONC_SEED = 1070^2 (reading Q12); RS: its init stream.
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

// grid_search over the energy field of 48-B records (coherent loads: the
// arena is rewritten by the next instance of this block)
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
    if (__longlong_as_double((long long)ld_(A + m)) > q) hi = m;
    else lo = m;
    len = hi - lo;
  }
  return lo;
}

// exclusive prefix sum of a[0..n) in shared memory, block-wide (n >= 1)
__device__ inline void block_exclusive_scan(uint32_t *a, int n, Shared *sh) {
  const int tid = threadIdx.x, T = blockDim.x, lane = tid & 31, w = tid >> 5, nw = T >> 5;
  const int per = (n + T - 1) / T;
  const int b0 = tid * per < n ? tid * per : n, b1 = b0 + per < n ? b0 + per : n;
  uint32_t sum = 0;
  for (int i = b0; i < b1; i++) sum += a[i];
  uint32_t inc = sum;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t v = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += v;
  }
  if (lane == 31) sh->red_u[w] = inc;
  __syncthreads();
  if (w == 0) {
    unsigned long long t = lane < nw ? sh->red_u[lane] : 0ULL;
    unsigned long long ti = t;
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long v = __shfl_up_sync(0xffffffffu, ti, o);
      if (lane >= o) ti += v;
    }
    if (lane < nw) sh->red_u[lane] = ti - t;  // exclusive warp offsets
  }
  __syncthreads();
  uint32_t run = (uint32_t)sh->red_u[w] + inc - sum;
  for (int i = b0; i < b1; i++) {
    const uint32_t v = a[i];
    a[i] = run;
    run += v;
  }
  __syncthreads();
}

struct XsKey {
  unsigned long long key;  // energy bit pattern (positive doubles order as integers)
  unsigned int idx, pad;
};

struct XsApp {
  static constexpr uint32_t kId = APP_XSBENCH;
  // thread limit is an upper bound: 512 keeps 128 registers
  static constexpr int kMaxT = 512;
  static constexpr int kU = kXsU;

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
    const int n_iso = p.n_iso, mx = xs_max_nucs(n_iso);
    const XsSmem S = xs_smem(p, blockDim.x);
    double *thr = (double *)(c.smem + S.thr);
    int *nn = (int *)(c.smem + S.nn);
    double *concs = (double *)(c.smem + S.concs);
    uint16_t *mats = (uint16_t *)(c.smem + S.mats);

    // ---- XS-2: materials, concentrations ---------------------------------
    hm_tables(n_iso, mx, thr, nn, concs, mats);
    __syncthreads();
    hm_concs(n_iso, mx, concs, 1070ULL * 1070ULL);
    init(c, p, L, S);
    if (p.grid == XS_HASH) lookups<XS_HASH>(c, p, L, thr, nn, concs, mats, R);
    else if (p.grid == XS_UNIONIZED) lookups<XS_UNIONIZED>(c, p, L, thr, nn, concs, mats, R);
    else lookups<XS_NUCLIDE>(c, p, L, thr, nn, concs, mats, R);
    const char *grid = p.grid == XS_UNIONIZED ? "unionized" : p.grid == XS_NUCLIDE ? "nuclide" : "hash";
    ens_printf(c, FMT_XS_HDR, n_iso == 68 ? "small" : "large", n_iso, (long long)p.n_gp, grid, p.lookups,
               (unsigned long long)p.seed);
    ens_printf(c, FMT_VERIFY, (unsigned long long)R.vhash);
    R.exit_code = 0;
    return R;
  }

  // ---- XS-3/4/5: nuclide grid, per-nuclide sort, acceleration structure --
  __device__ static __noinline__ void init(Ctx &c, const XsParams &p, const XsLayout &L, const XsSmem &S) {
    const int tid = threadIdx.x, T = blockDim.x;
    const int n_iso = p.n_iso, n_gp = p.n_gp;
    const long long n_u = (long long)n_iso * n_gp;
    const int NB = xs_nb(n_gp);
    uint32_t *bkt = (uint32_t *)(c.smem + S.bkt);
    double *recs = (double *)(c.arena + L.recs);
    double *scr = (double *)(c.arena + L.scratch);
    XsKey *keys = (XsKey *)(c.arena + L.keys);
    int *ig = (int *)(c.arena + L.index);
    uint64_t *uA = (uint64_t *)(c.arena + L.uenergy), *uB = (uint64_t *)(c.arena + L.utmp);
    uint16_t *oA = (uint16_t *)(c.arena + L.uown), *oB = (uint16_t *)(c.arena + L.uowntmp);
    int rounds = 0;
    while ((1 << rounds) < n_iso) rounds++;
    uint64_t *urun = (rounds & 1) ? uB : uA;  // merge rounds alternate; end in uA
    uint16_t *orun = (rounds & 1) ? oB : oA;
    const double du = 1.0 / p.bins;
    const Affine J6T = lcg_pow(6ULL * T);
    const Affine Jnuc = lcg_pow(6ULL * n_gp);
    uint64_t s_nuc = lcg_pow(6ULL * tid)(p.gseed);  // before record (i*n_gp + tid)

    for (int i = 0; i < n_iso; i++) {
      for (int b = tid; b < NB; b += T) bkt[b] = 0;
      __syncthreads();
      // (a) generate: record r = i*n_gp + j takes draws 6r+1 .. 6r+6 (XS-3)
      uint64_t s = s_nuc;
      for (int j = tid; j < n_gp; j += T, s = J6T(s)) {
        uint64_t t = s;
        double v[6];
#pragma unroll
        for (int f = 0; f < 6; f++) v[f] = lcg_double(t);
        double2 *d = reinterpret_cast<double2 *>(scr + 6 * (size_t)j);
        d[0] = make_double2(v[0], v[1]);
        d[1] = make_double2(v[2], v[3]);
        d[2] = make_double2(v[4], v[5]);
        const int b = min((int)(v[0] * NB), NB - 1);
        atomicAdd(&bkt[b], 1u);
      }
      s_nuc = Jnuc(s_nuc);
      __syncthreads();
      // (b) XS-4 sort: bucket offsets, scatter, per-bucket insertion sort
      block_exclusive_scan(bkt, NB, c.sh);
      for (int j = tid; j < n_gp; j += T) {
        const double e = ld_(scr + 6 * (size_t)j);
        const int b = min((int)(e * NB), NB - 1);
        const uint32_t pos = atomicAdd(&bkt[b], 1u);
        XsKey k;
        k.key = dbits(e);
        k.idx = (unsigned)j;
        k.pad = 0;
        keys[pos] = k;
      }
      __syncthreads();
      for (int b = tid; b < NB; b += T) {  // bkt[b] is now the end of bucket b
        const int lo = b ? (int)bkt[b - 1] : 0, hi = (int)bkt[b];
        for (int x = lo + 1; x < hi; x++) {
          XsKey v = keys[x];
          int y = x - 1;
          while (y >= lo && keys[y].key > v.key) {
            keys[y + 1] = keys[y];
            y--;
          }
          keys[y + 1] = v;
        }
      }
      __syncthreads();
      // (c) scatter the records to their sorted position
      double *rec_i = recs + (size_t)i * n_gp * 6;
      for (int k = tid; k < n_gp; k += T) {
        const unsigned j = keys[k].idx;
        const double2 *src = reinterpret_cast<const double2 *>(scr + 6 * (size_t)j);
        double2 *dst = reinterpret_cast<double2 *>(rec_i + 6 * (size_t)k);
        const double2 a = src[0], b = src[1], e = src[2];
        dst[0] = a;
        dst[1] = b;
        dst[2] = e;
      }
      // (d) XS-5
      if (p.grid == XS_HASH) {
        // ig[i][b] = grid_search(E_i, b*du, 0, n_gp-1) = min(#{k>=1: E_k <= b*du}, n_gp-2),
        // a merge walk over the sorted keys per contiguous chunk of bins
        int *col = ig + (size_t)i * (p.bins + 1);
        const int C = (p.bins + T - 1) / T;
        const int b0 = tid * C, b1 = min(b0 + C, p.bins);
        if (b0 < b1) {
          const double q0 = (double)b0 * du;
          int lo = 1, hi = n_gp;  // first k >= 1 with E_k > q0
          while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (__longlong_as_double((long long)keys[mid].key) <= q0) lo = mid + 1;
            else hi = mid;
          }
          int cnt = lo - 1;  // #{k >= 1 : E_k <= q0}
          for (int b = b0; b < b1; b++) {
            const double q = (double)b * du;
            while (cnt < n_gp - 1 && __longlong_as_double((long long)keys[cnt + 1].key) <= q) cnt++;
            col[b] = cnt < n_gp - 2 ? cnt : n_gp - 2;
          }
        }
        if (tid == 0) col[p.bins] = n_gp - 2;
      } else if (p.grid == XS_UNIONIZED) {
        for (int k = tid; k < n_gp; k += T) {
          urun[(size_t)i * n_gp + k] = keys[k].key;
          orun[(size_t)i * n_gp + k] = (uint16_t)i;
        }
      }
      __syncthreads();
    }

    if (p.grid != XS_UNIONIZED) return;
    // ---- union: bottom-up merge of the n_iso sorted runs (merge path) ------
    {
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
    }
    // ---- index grid: ig[e][i] = clip(#{k>=1: E_i[k] <= u_e}, 0, n_gp-2), a
    // warp sweeps a chunk of rows, lanes own nuclides (coalesced row stores)
    {
      const int lane = tid & 31, warp = tid >> 5, nw = T >> 5;
      const long long per = (n_u + nw * 4 - 1) / (nw * 4);
      const long long C = per > 512 ? per : 512;
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
  }

  // ---- XS-6..XS-10: lookups ----------------------------------------------
  // Batches of K*T lookups: (A) every thread samples its K lookups (XS-6),
  // the batch is counting-sorted by material into shared memory; (B) thread
  // t takes sorted slots t, t+T, t+2T, ...: a warp's lanes share a material
  // (same nuclide count: no divergence), every thread gets the same mix of
  // materials (balanced), and each lane sums its lookup's nuclides in list
  // order (XS-9's order, bit-exact), kU nuclides' gathers in flight at once.
  template <int GRID>
  __device__ static __forceinline__ void lookups(Ctx &c, const XsParams &p, const XsLayout &L, const double *thr,
                                              const int *nn, const double *concs, const uint16_t *mats,
                                              Result &R) {
    const int tid = threadIdx.x, T = blockDim.x;
    const int n_iso = p.n_iso, n_gp = p.n_gp, mx = xs_max_nucs(n_iso);
    const long long n_u = (long long)n_iso * n_gp, nL = p.lookups;
    const double *recs = (const double *)(c.arena + L.recs);
    const int *ig = (const int *)(c.arena + L.index);
    const uint64_t *uA = (const uint64_t *)(c.arena + L.uenergy);
    const XsSmem S = xs_smem(p, T);
    const int K = xs_batch_k(n_iso);
    double *slot_pe = (double *)(c.smem + S.slot);
    int *slot_idx = (int *)(c.smem + S.slot + (size_t)K * T * 8);
    uint32_t *mcnt = (uint32_t *)(c.smem + S.mcnt);  // [12] counts -> cursors, [16..28] offsets
    const double du = 1.0 / p.bins;
    unsigned long long ver = 0, bsum = 0;
    double fsum = 0.0, fabs_ = 0.0;
    const long long NBt = (long long)K * T;
    const Affine JT = lcg_pow(2ULL * T);
    for (long long b0 = 0; b0 < nL; b0 += NBt) {
      const int nb = (int)((nL - b0 < NBt) ? nL - b0 : NBt);
      if (tid < 12) mcnt[tid] = 0;
      __syncthreads();
      // (A1) count the batch's materials; lookup li = b0 + tid + r*T
      const uint64_t s0 = lcg_pow(2ULL * (uint64_t)(b0 + tid))(p.seed);
      {
        uint64_t s = s0;
        for (int r = 0; r < K; r++, s = JT(s)) {
          if (tid + r * T >= nb) break;
          uint64_t t = s;
          (void)lcg_double(t);
          atomicAdd(&mcnt[pick_mat_thr(thr, lcg_double(t))], 1u);
        }
      }
      __syncthreads();
      if (tid == 0) {  // offsets (material order 0..11) and cursors; tallies
        uint32_t o = 0;
        for (int m = 0; m < 12; m++) {
          const uint32_t cm = mcnt[m];
          mcnt[16 + m] = o;
          c.sh->tallies[5 + m] += cm;
          mcnt[m] = o;
          o += cm;
        }
        mcnt[28] = o;
      }
      __syncthreads();
      // (A2) re-sample, scatter energies (and union indices) to sorted slots
      {
        uint64_t s = s0;
        for (int r = 0; r < K; r++, s = JT(s)) {
          if (tid + r * T >= nb) break;
          uint64_t t = s;
          const double pe = lcg_double(t);
          const int mat = pick_mat_thr(thr, lcg_double(t));
          const uint32_t pos = atomicAdd(&mcnt[mat], 1u);
          slot_pe[pos] = pe;
          if (GRID == XS_UNIONIZED) slot_idx[pos] = (int)gs_u64(uA, pe, 0, n_u - 1);
        }
      }
      __syncthreads();
      // (B) thread-per-lookup over sorted slots
      for (int sl = tid; sl < nb; sl += T) {
        int mat = 0;
#pragma unroll
        for (int m = 1; m < 12; m++) mat += (sl >= (int)mcnt[16 + m]) ? 1 : 0;
        const double pe = slot_pe[sl];
        int idx = 0;
        if (GRID == XS_UNIONIZED) idx = slot_idx[sl];
        else if (GRID == XS_HASH) {
          const long long bb = (long long)(pe / du);
          idx = bb > p.bins - 1 ? p.bins - 1 : (int)bb;  // reading Q14
        }
        const int nm = nn[mat];
        const uint16_t *mrow = mats + mat * mx;
        const double *crow = concs + mat * mx;
        double m0 = 0.0, m1 = 0.0, m2 = 0.0, m3 = 0.0, m4 = 0.0;
        for (int j0 = 0; j0 < nm; j0 += kU) {
          int nuc[kU], lo[kU];
          bool on[kU];
          double2 a0[kU], a1[kU], a2[kU], b0v[kU], b1[kU], b2[kU];
#pragma unroll
          for (int u = 0; u < kU; u++) {  // XS-7 step 1: index entries
            on[u] = j0 + u < nm;
            nuc[u] = on[u] ? mrow[j0 + u] : 0;
            lo[u] = 0;
            if (on[u]) {
              if (GRID == XS_HASH) lo[u] = ld_(ig + (size_t)nuc[u] * (p.bins + 1) + idx);
              else if (GRID == XS_UNIONIZED) {
                const int k = ld_(ig + (size_t)idx * n_iso + nuc[u]);
                lo[u] = (k == n_gp - 1) ? k - 1 : k;
              } else {
                const int k = gs_recs(recs + (size_t)nuc[u] * n_gp * 6, pe, 0, n_gp - 1);
                lo[u] = (k == n_gp - 1) ? k - 1 : k;
              }
            }
          }
#pragma unroll
          for (int u = 0; u < kU; u++) {  // step 2: record pair at lo (hash: at u_low)
            if (on[u]) {
              const double2 *r2 = reinterpret_cast<const double2 *>(recs + ((size_t)nuc[u] * n_gp + lo[u]) * 6);
              a0[u] = ld_(r2 + 0); a1[u] = ld_(r2 + 1); a2[u] = ld_(r2 + 2);
              b0v[u] = ld_(r2 + 3); b1[u] = ld_(r2 + 4); b2[u] = ld_(r2 + 5);
            }
          }
          if (GRID == XS_HASH) {
#pragma unroll
            for (int u = 0; u < kU; u++) {
              // E[u_low] < pe < E[u_low+1] is exactly grid_search's answer
              // u_low on [u_low, u_high]; otherwise the full upstream logic
              if (on[u] && !(a0[u].x < pe && pe < b0v[u].x)) {
                const double *E = recs + (size_t)nuc[u] * n_gp * 6;
                const int u_low = lo[u];
                const int u_high = ld_(ig + (size_t)nuc[u] * (p.bins + 1) + idx + 1) + 1;
                const double e_high = ld_(E + 6 * (size_t)u_high);
                int lower;
                if (pe <= a0[u].x) lower = 0;
                else if (pe >= e_high) lower = n_gp - 1;
                else lower = gs_recs(E, pe, u_low, u_high);
                const int l2 = lower == n_gp - 1 ? lower - 1 : lower;
                const double2 *r2 = reinterpret_cast<const double2 *>(E + 6 * (size_t)l2);
                a0[u] = ld_(r2 + 0); a1[u] = ld_(r2 + 1); a2[u] = ld_(r2 + 2);
                b0v[u] = ld_(r2 + 3); b1[u] = ld_(r2 + 4); b2[u] = ld_(r2 + 5);
              }
            }
          }
#pragma unroll
          for (int u = 0; u < kU; u++) {  // XS-8, XS-9 in nuclide order
            if (on[u]) {
              const double conc = crow[j0 + u];
              // low = {E, total, elastic, absorption, fission, nu_fission}
              const double f = (b0v[u].x - pe) / (b0v[u].x - a0[u].x);
              m0 += (b0v[u].y - f * (b0v[u].y - a0[u].y)) * conc;
              m1 += (b1[u].x - f * (b1[u].x - a1[u].x)) * conc;
              m2 += (b1[u].y - f * (b1[u].y - a1[u].y)) * conc;
              m3 += (b2[u].x - f * (b2[u].x - a2[u].x)) * conc;
              m4 += (b2[u].y - f * (b2[u].y - a2[u].y)) * conc;
            }
          }
        }
        // XS-10
        double mxv = -1.0;
        int am = 0;
        if (m0 > mxv) { mxv = m0; am = 0; }
        if (m1 > mxv) { mxv = m1; am = 1; }
        if (m2 > mxv) { mxv = m2; am = 2; }
        if (m3 > mxv) { mxv = m3; am = 3; }
        if (m4 > mxv) { mxv = m4; am = 4; }
        ver += (unsigned long long)(am + 1);
        atomicAdd(&c.sh->tallies[am], 1u);
        bsum += dbits(m0) + dbits(m1) + dbits(m2) + dbits(m3) + dbits(m4);
        fsum += m0; fsum += m1; fsum += m2; fsum += m3; fsum += m4;
        fabs_ += fabs(m0); fabs_ += fabs(m1); fabs_ += fabs(m2); fabs_ += fabs(m3); fabs_ += fabs(m4);
      }
      __syncthreads();  // slots reused by the next batch
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
  }

  __host__ static bool size(int argc, const char *const *argv, int T, uint64_t *arena, uint32_t *smem) {
    XsParams p;
    if (xs_parse(argc, argv, p) >= 0) {
      *arena = 0;
      *smem = 0;
      return false;
    }
    *arena = xs_layout(p).total;
    *smem = xs_smem(p, T).total;
    return true;
  }
};

}  // namespace ens
