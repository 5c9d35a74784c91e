// csrc/apps/xsbench.cuh — N1 instance body: XSBench-style macroscopic
// cross-section lookup (the paper's memory-bound benchmark, §4.1
// P:496-504), as SURVEY.md §8(c) XS-1..XS-11 defines it.  One instance runs
// on one thread block (one OpenMP team, §2.3); its parallel loops
// (grid generation, sort, index build, lookups) use the block's threads.
//
// B200 design (results identical to the oracle):
//  * init keeps shared memory small (material tables + bucket counters) so
//    the L1 stays large for the lookup phase: only record ids are sorted, by
//    energy (uniform in [0,1): counts -> scan -> scatter -> sort of ~4-record
//    buckets, energies re-drawn from the ids); each record is then written
//    once, at its sorted position, its cross sections re-drawn from the LCG
//    through jump tables (no generation-order copy);
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
#include "../rt/scan.cuh"
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

#ifdef ENS_XS_STOP  // profiling builds only: stop init after phase k
#define XS_STOP(k) do { if (ENS_XS_STOP == (k)) { __syncthreads(); return; } } while (0)
#else
#define XS_STOP(k) phase_mark_if(trc, c, (k))  // tracing (ENS_F_PHASES): end of init phase k
#endif

// init-sort bucket of record r with energy e in [0, 1]: by energy alone
// (unionized) or by (nuclide, energy); nb / nbn are powers of two, so
// e * nb is exact and floor() is monotone in e.
__device__ __forceinline__ long long bucket_of(double e, long long r, int n_gp, bool uni, long long nb, int nbn) {
  if (uni) {
    const long long b = (long long)(e * (double)nb);
    return b < nb - 1 ? b : nb - 1;
  }
  const long long b = (long long)(e * (double)nbn);
  return (r / n_gp) * nbn + (b < nbn - 1 ? b : nbn - 1);
}

struct XsApp {
  static constexpr uint32_t kId = APP_XSBENCH;
  // thread limit is an upper bound: 512 keeps 128 registers
  // (measured: a 1024-thread build at 64 registers spills and runs C2's
  // lookups 1.8x slower)
  static constexpr int kMaxT = 512;
  static constexpr bool kTeam = true;  // splits nuclides and lookup batches over a cluster
  static constexpr bool kSub = false;

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
    const XsLayout L = xs_layout(p, c.csize);
    if (L.total > c.arena_cap) {
      if (threadIdx.x == 0) ens_sh(c)->flags |= 2u;  // ENS_RF_NOMEM
      R.exit_code = ENS_EXIT_NOMEM;
      return R;
    }
    const int n_iso = p.n_iso, mx = xs_max_nucs(n_iso);
    const XsSmem S = xs_smem(p, blockDim.x);
    double *thr = (double *)(ens_smem(c) + S.thr);
    int *nn = (int *)(ens_smem(c) + S.nn);
    double *concs = (double *)(ens_smem(c) + S.concs);
    uint16_t *mats = (uint16_t *)(ens_smem(c) + S.mats);

    // ---- XS-2: materials, concentrations ---------------------------------
    hm_tables(n_iso, mx, thr, nn, concs, mats);
    {  // LCG jump tables for XS-3's record draws (see jump6)
      Affine *jt = (Affine *)(ens_smem(c) + S.jmp);
      for (int x = threadIdx.x; x < 320; x += blockDim.x)
        jt[x] = lcg_pow((6ULL * (uint64_t)(x & 63)) << (6 * (x >> 6)));
    }
    __syncthreads();
    hm_concs(n_iso, mx, concs, 1070ULL * 1070ULL);
    phase_mark(c, 0);
    // split phases: a hash / nuclide instance's per-nuclide tables are built
    // by the init-item kernel (kernels_items.cu) running beside this kernel
    const bool init_items = c.desc && xs_split_ok(p) && p.grid != XS_UNIONIZED;
    if (init_items) {
    } else if (p.grid == XS_UNIONIZED) {
      const bool warp_path = xs_warp_union(p) && !(c.flags & ENS_F_GENERIC);
      if (!warp_path && !xs_smem_nb(p)) {
        init(c, p, L, S, c.csize > 1);  // block-wide, striped over the team
      } else {
        // the warp path striped over the team's CTAs (team-uniform result); on a
        // chunk overflow, or with shared-memory counters, one CTA builds the union
        const bool ok = warp_path && init_warp(c, p, L, S);
        if (!ok && c.crank == 0) init(c, p, L, S, false);
      }
    } else {
      init_nuc(c, p, L, S);  // nuclides striped over the team's CTAs
    }
    team_sync(c);
    if (c.desc && xs_split_ok(p)) {  // split phases: sort the lookups, hand them to phase 2
      if (init_items) {  // the init-item kernel builds the tables, sorts and writes the descriptor
        R.deferred = 1;
        return R;
      }
      split_sort(c, p, L, S, thr);
      R.deferred = 1;
      return R;
    }
    if (p.history) {
      if (p.grid == XS_HASH) lookups_history<XS_HASH>(c, p, L, thr, nn, concs, mats, R);
      else if (p.grid == XS_UNIONIZED) lookups_history<XS_UNIONIZED>(c, p, L, thr, nn, concs, mats, R);
      else lookups_history<XS_NUCLIDE>(c, p, L, thr, nn, concs, mats, R);
    } else {
      if (p.grid == XS_HASH) lookups_hash(c, p, L, thr, nn, concs, mats, R);
      else if (p.grid == XS_UNIONIZED) lookups<XS_UNIONIZED>(c, p, L, thr, nn, concs, mats, R);
      else lookups<XS_NUCLIDE>(c, p, L, thr, nn, concs, mats, R);
    }
    const char *grid = p.grid == XS_UNIONIZED ? "unionized" : p.grid == XS_NUCLIDE ? "nuclide" : "hash";
    if (p.history)
      ens_printf(c, FMT_XS_HIST, n_iso == 68 ? "small" : "large", n_iso, (long long)p.n_gp, grid, p.particles,
                 p.lookups, (unsigned long long)p.seed);
    else
      ens_printf(c, FMT_XS_HDR, n_iso == 68 ? "small" : "large", n_iso, (long long)p.n_gp, grid, p.lookups,
                 (unsigned long long)p.seed);
    ens_printf(c, FMT_VERIFY, (unsigned long long)R.vhash);
    R.exit_code = 0;
    return R;
  }

  // split phases, phase 1 (unionized): sort the lookups and leave the
  // descriptor; out of line, so the fused path's registers are its own
  __device__ static __noinline__ void split_sort(Ctx &c, const XsParams &p, const XsLayout &L, const XsSmem &S,
                                                 const double *thr) {
    uint32_t *mcnt = (uint32_t *)(ens_smem(c) + S.mcnt);
    lookup_sort(c, p, L, thr, mcnt, 0, p.lookups);
    if (c.crank == 0 && threadIdx.x == 0) write_desc(c, p, L, mcnt);
  }

  // split phases: the instance's phase-2 descriptor (one thread)
  __device__ static void write_desc(const Ctx &c, const XsParams &p, const XsLayout &L, const uint32_t *mcnt) {
    XsDesc *d = reinterpret_cast<XsDesc *>(c.desc);
    d->recs = (uint64_t)(c.arena + L.recs);
    d->index = (uint64_t)(c.arena + L.index);
    d->uenergy = (uint64_t)(c.arena + L.uenergy);
    d->ufind = (uint64_t)(c.arena + L.ufind);
    d->lk_pe = (uint64_t)(c.arena + L.lk_pe);
    d->lookups = (uint64_t)p.lookups;
    d->seed = p.seed;
    d->ubins = xs_ubins(p);
    for (int m = 0; m < 13; m++) d->mcnt[m] = mcnt[16 + m];
    d->n_iso = p.n_iso;
    d->n_gp = p.n_gp;
    d->grid = p.grid;
    d->bins = p.bins;
    d->k = c.k;
    d->line = c.id;
    d->t_start = c.t_start;
  }

  // the LCG state s advanced by 6r draws (record r's draws are 6r+1..6r+6,
  // XS-3), from the smem tables jt[64 l + d] = A^(6 d 64^l): four affine
  // steps instead of a 6r-step walk, a fifth for r >= 2^24 (n_u <= 355 *
  // 65536 < 2^30)
  __device__ static __forceinline__ uint64_t jump6(const Affine *jt, uint32_t r, uint64_t s) {
    s = jt[r & 63u](s);
    s = jt[64 + ((r >> 6) & 63u)](s);
    s = jt[128 + ((r >> 12) & 63u)](s);
    s = jt[192 + ((r >> 18) & 63u)](s);
    if (r >> 24) s = jt[256 + ((r >> 24) & 63u)](s);
    return s;
  }
  // sort the record ids ids[lo, hi) by (energy, record id), each energy
  // re-drawn once from its id (draw 6r+1): <= 8 in registers, <= 64 in a
  // local array (~2 % of the buckets at ~4 records each), else in place with
  // the energies re-drawn per comparison (never at these bucket sizes)
  __device__ static __forceinline__ void sort_bucket(uint32_t *ids, long long lo, long long hi, const Affine *jt,
                                                     uint64_t gseed) {
    const int cnt = (int)(hi - lo);
    if (cnt <= 1) return;
    if (cnt <= 8) {
      unsigned long long kk[8];
      unsigned ii[8];
#pragma unroll
      for (int q = 0; q < 8; q++)
        if (q < cnt) {
          ii[q] = ids[lo + q];
          kk[q] = dbits(rec_energy(jt, ii[q], gseed));
        }
#pragma unroll
      for (int x = 1; x < 8; x++) {
#pragma unroll
        for (int y = x; y > 0; y--) {
          if (x < cnt && (kk[y - 1] > kk[y] || (kk[y - 1] == kk[y] && ii[y - 1] > ii[y]))) {
            const unsigned long long tk = kk[y - 1];
            kk[y - 1] = kk[y];
            kk[y] = tk;
            const unsigned ti = ii[y - 1];
            ii[y - 1] = ii[y];
            ii[y] = ti;
          }
        }
      }
#pragma unroll
      for (int q = 0; q < 8; q++)
        if (q < cnt) ids[lo + q] = ii[q];
      return;
    }
    if (cnt <= 64) {
      unsigned long long kk[64];
      unsigned ii[64];
      for (int x = 0; x < cnt; x++) {
        const unsigned v = ids[lo + x];
        const unsigned long long ve = dbits(rec_energy(jt, v, gseed));
        int y = x - 1;
        while (y >= 0 && (kk[y] > ve || (kk[y] == ve && ii[y] > v))) {
          kk[y + 1] = kk[y];
          ii[y + 1] = ii[y];
          y--;
        }
        kk[y + 1] = ve;
        ii[y + 1] = v;
      }
      for (int x = 0; x < cnt; x++) ids[lo + x] = ii[x];
      return;
    }
    for (long long x = lo + 1; x < hi; x++) {
      const unsigned v = ids[x];
      const unsigned long long ve = dbits(rec_energy(jt, v, gseed));
      long long y = x - 1;
      for (; y >= lo; y--) {
        const unsigned w = ids[y];
        const unsigned long long we = dbits(rec_energy(jt, w, gseed));
        if (!(we > ve || (we == ve && w > v))) break;
        ids[y + 1] = w;
      }
      ids[y + 1] = v;
    }
  }

  // Unionized index grid sweep: a warp per chunk of union rows, the chunk's
  // current row in the warp's shared memory: counts cnt_i(e) = #{k: E_i[k]
  // <= u_e} and row values clip(cnt_i(e) - 1, 0, n_gp-2).  Each union row
  // changes exactly one count (its owner's): the owner's lane updates it,
  // then the warp copies the row out as 16-B vectors.  The owner's count
  // before its increment is the sorted position s of that record: the
  // record id goes to inv[s] (each owner's positions are written in order),
  // so that (R) writes the records in sorted order.
  __device__ static __forceinline__ void sweep(const uint32_t *ids, uint32_t *inv, const uint32_t *chist, int *ig,
                                               int *sw, long long n_u,
                                               int n_iso, int n_gp, long long nch, int crank, int csize) {
    const int tid = threadIdx.x, T = blockDim.x, lane = tid & 31, warp = tid >> 5, nw = T >> 5;
    const int ip = xs_iso_pad(n_iso), ng4 = ip >> 2;
    int *cnt = sw + (size_t)warp * 2 * ip, *val = cnt + ip;
    auto clip = [&](int c) { const int v = c - 1; return v < 0 ? 0 : (v > n_gp - 2 ? n_gp - 2 : v); };
    for (long long ch = warp + (long long)crank * nw; ch < nch; ch += (long long)nw * csize) {
      const long long e0 = ch * kXsSweepRows, e1 = (e0 + kXsSweepRows < n_u) ? e0 + kXsSweepRows : n_u;
      for (int i = lane; i < ip; i += 32) {
        const int c = i < n_iso ? (int)chist[ch * n_iso + i] : 0;
        cnt[i] = c;
        val[i] = clip(c);
      }
      __syncwarp();
      // record ids of the next 32 rows are prefetched while this group is swept
      unsigned id_next = e0 + lane < e1 ? ids[e0 + lane] : 0u;
      for (long long g = e0; g < e1; g += 32) {
        const int own_cur = (int)(id_next / (unsigned)n_gp);
        id_next = g + 32 + lane < e1 ? ids[g + 32 + lane] : 0u;
        const int ng = (int)(e1 - g < 32 ? e1 - g : 32);
        int4 *row = reinterpret_cast<int4 *>(ig + (size_t)g * ip);
        for (int sl = 0; sl < ng; sl++, row += ng4) {
          if (lane == sl) {  // the row's owner
            const int c = cnt[own_cur];
            cnt[own_cur] = c + 1;
            val[own_cur] = clip(c + 1);
            inv[(size_t)own_cur * n_gp + c] = ids[g + sl];
          }
          __syncwarp();
          for (int q = lane; q < ng4; q += 32) __stcs(row + q, reinterpret_cast<const int4 *>(val)[q]);  // evict-first
        }
        __syncwarp();
      }
    }
  }

  // ---- XS-3/4/5, hash and nuclide grids: one nuclide at a time -------------
  // Nuclide i's n_gp energies (draw 6r+1 of record r = i*n_gp + j; XS-3)
  // are bucket-sorted as {energy, j} keys in an L2-resident buffer (XS-4:
  // shared-memory counts -> scan -> scatter -> per-bucket sort), each record
  // is written once in sorted order (coalesced) with its draws 6r+2..6r+6
  // re-generated, and (hash) the nuclide's index column is built by a merge
  // walk over the sorted energies, each bin written once (XS-5: ig[i][b] = grid_search(E_i, b*du) = min(#{k>=1: E_k <= b*du}, n_gp-2)).
  // SMK: the sort's keys and counters in shared memory (n_gp <= kXsSmemGp),
  // else in this CTA's arena scratch (L2 atomics; the same algorithm)
  // The team's CTAs take nuclides crank, crank + csize, ... with per-CTA
  // scratch in the arena; init_nuc_range runs nuclides [i0, i1) with the
  // caller's scratch (split phases: one nuclide per work item, kernels_items.cu)
  __device__ static void init_nuc(Ctx &c, const XsParams &p, const XsLayout &L, const XsSmem &S) {
    char *ekey = c.arena + L.keys + (size_t)c.crank * p.n_gp * 8;
    char *col = c.arena + L.hcol + (size_t)c.crank * (p.bins + 1) * 4;
    char *gscr = c.arena + L.nscr + (size_t)c.crank * xs_nscr_bytes(p);
    init_nuc_range(c, p, L, S, (int)c.crank, p.n_iso, (int)c.csize, ekey, col, gscr);
  }
  __device__ static void init_nuc_range(Ctx &c, const XsParams &p, const XsLayout &L, const XsSmem &S, int i0,
                                        int i1, int istep, char *ekey, char *col, char *gscr) {
    if (xs_nuc_smem(p)) init_nuc_t<true>(c, p, L, S, i0, i1, istep, ekey, col, gscr);
    else init_nuc_t<false>(c, p, L, S, i0, i1, istep, ekey, col, gscr);
  }
  // per-CTA scratch bytes of init_nuc_range: sorted energies, hash column, sort scratch
  ENS_HD static uint64_t nuc_scratch_bytes(const XsParams &p) {
    return align_up((uint64_t)p.n_gp * 8, 256) + align_up((uint64_t)(p.bins + 1) * 4, 256) + xs_nscr_bytes(p);
  }
  template <bool SMK>
  __device__ static __noinline__ void init_nuc_t(Ctx &c, const XsParams &p, const XsLayout &L, const XsSmem &S,
                                                 int i0, int i1, int istep, char *ekey_scr, char *col_scr,
                                                 char *gscr) {
    const bool trc = tracing(c);  // tracing (ENS_F_PHASES) thread, cached
    const int tid = threadIdx.x, T = blockDim.x;
    const int n_gp = p.n_gp;
    const int nbn = SMK ? xs_nbn_smem(n_gp) : xs_nbn(n_gp);
    uint32_t *nb = SMK ? (uint32_t *)(ens_smem(c) + S.nbkt) : (uint32_t *)gscr;
    const Affine *jt = (const Affine *)(ens_smem(c) + S.jmp);
    double *recs = (double *)(c.arena + L.recs);
    unsigned long long *ekey = (unsigned long long *)ekey_scr;  // sorted energies (this CTA's)
    const size_t kofs = SMK ? 0 : align_up((uint64_t)nbn * 4, 256);
    uint32_t *K = SMK ? (uint32_t *)(ens_smem(c) + S.nkey) : (uint32_t *)(gscr + kofs);  // sort keys, then
    uint16_t *J = SMK ? (uint16_t *)(ens_smem(c) + S.njdx)                               // record indices j
                      : (uint16_t *)(gscr + kofs + align_up((uint64_t)n_gp * 4, 256));
    int *ig = (int *)(c.arena + L.index);
    const bool hash = p.grid == XS_HASH;
    int kbits = 0;
    while ((1 << kbits) < nbn) kbits++;
    auto nkey_bkt = [&](uint32_t key) { return kbits ? (int)(key >> (32 - kbits)) : 0; };
    const double du = 1.0 / p.bins;
    const Affine J6T = lcg_pow(6ULL * T), J24T = lcg_pow(24ULL * T);
    for (int i = i0; i < i1; i += istep) {
      int *col = (int *)col_scr;  // this CTA's column
      XsHashEnt *ent = (XsHashEnt *)ig + (size_t)i * (p.bins + 1);
      const uint32_t r0 = (uint32_t)i * (uint32_t)n_gp;  // record i*n_gp + j
      for (int b = tid; b < nbn; b += T) nb[b] = 0;
      __syncthreads();
      {  // count the energies' buckets (energy = draw 6r+1; bucket = top bits of its sort key)
        uint64_t s = jump6(jt, r0 + (uint32_t)tid, p.gseed);
        for (int j = tid; j < n_gp; j += T, s = J6T(s)) atomicAdd(&nb[nkey_bkt((uint32_t)(lcg_next(s) >> 31))], 1u);
      }
      __syncthreads();
      phase_mark_if(trc, c, 1);
      if (SMK) smem_scan(nb, nbn, ens_sh(c));
      else global_exclusive_scan(nb, nbn, ens_sh(c));
      phase_mark_if(trc, c, 2);
      {  // scatter {key, j} in shared memory, four atomics in flight
        uint64_t s = jump6(jt, r0 + (uint32_t)tid, p.gseed);
        for (int j0 = tid; j0 < n_gp; j0 += 4 * T, s = J24T(s)) {
          uint32_t key[4];
          uint64_t sq = s;
#pragma unroll
          for (int q = 0; q < 4; q++, sq = J6T(sq)) key[q] = (uint32_t)(lcg_next(sq) >> 31);
#pragma unroll
          for (int q = 0; q < 4; q++) {
            const int j = j0 + q * T;
            if (j < n_gp) {
              const uint32_t pos = atomicAdd(&nb[nkey_bkt(key[q])], 1u);
              K[pos] = key[q];
              J[pos] = (uint16_t)j;
            }
          }
        }
      }
      __syncthreads();
      phase_mark_if(trc, c, 3);
      // sort within buckets: in shared memory, a thread per key counts the
      // keys of its bucket that sort before it — (energy, j) order: equal
      // 32-bit keys (rare) compare the re-drawn energies, then j — and
      // places its record index there (J2: sorted order); in arena scratch,
      // an insertion sort per bucket in place
      uint16_t *Js = J;
      if (SMK) {
        Js = (uint16_t *)(ens_smem(c) + S.njdx2);
        for (int x = tid; x < n_gp; x += T) {
          const uint32_t vk = K[x];
          const uint16_t vj = J[x];
          const int b = nkey_bkt(vk);
          const int lo = b ? (int)nb[b - 1] : 0, hi = (int)nb[b];
          // buckets of <= 8 keys (~4 on average): eight independent predicated
          // loads (the key at x counts itself as "not before"); equal keys or
          // a larger bucket take the exact loop
          int rank = 0;
          bool slow = hi - lo > 8;
#pragma unroll
          for (int q = 0; q < 8; q++) {
            const int y = lo + q;
            const uint32_t yk = K[y < n_gp ? y : n_gp - 1];
            const bool in = y < hi;
            rank += (in && yk < vk) ? 1 : 0;
            slow |= in && yk == vk && y != x;
          }
          if (slow) {
            rank = 0;
            for (int y = lo; y < hi; y++) {
              const uint32_t yk = K[y];
              if (yk < vk) {
                rank++;
              } else if (yk == vk && y != x) {
                const uint16_t yj = J[y];
                const double ey = rec_energy(jt, r0 + yj, p.gseed), ev = rec_energy(jt, r0 + vj, p.gseed);
                rank += (ey < ev || (ey == ev && yj < vj)) ? 1 : 0;
              }
            }
          }
          ENS_CHECK(lo + rank < hi);
          Js[lo + rank] = vj;
        }
      } else {
        for (int b = tid; b < nbn; b += T) isort_keys(K, J, b ? (int)nb[b - 1] : 0, (int)nb[b], jt, r0, p.gseed);
      }
      __syncthreads();
      phase_mark_if(trc, c, 4);
      // records written in sorted order (coalesced, evict-first), their draws
      // re-generated from the jump tables.  Hash grid: bin b's column entry
      // is #{k >= 1: E_k <= b*du} (XS-5), i.e. k on [bfirst(E_k),
      // bfirst(E_k+1)); with the column in shared memory (sm_col) each
      // record's bfirst and its quantization key are computed here, while its
      // energy is in a register, into the dead sort keys: W[k] = bin(E_k) << 16
      // | q15(E_k) << 1 | (bfirst(E_k) - bin(E_k)) (that difference is 0 or 1
      // unless E_k sits within a few ulps of a bin edge; any other value sends
      // the nuclide's column pass back to the exact energies in the records);
      // otherwise the sorted energies go to `ekey` (arena scratch)
      auto bfirst = [&](double e) {  // first bin b with e <= b*du (bins if none; bins <= 10^7: int)
        int bb = (int)(e * p.bins);
        // the usual answer is bb or bb+1: the three edge tests are independent
        // (no compare-then-multiply chain); anything else takes the walk
        const bool dn = bb > 0 && (double)(bb - 1) * du >= e;
        const bool u0 = bb < p.bins && (double)bb * du < e;
        const bool u1 = bb + 1 < p.bins && (double)(bb + 1) * du < e;
        if (!dn && !u1) return bb + (u0 ? 1 : 0);
        while (bb > 0 && (double)(bb - 1) * du >= e) bb--;
        while (bb < p.bins && (double)bb * du < e) bb++;
        return bb;
      };
      const uint32_t col_b = (uint32_t)align_up((uint64_t)(p.bins + 1) * 4, 16);
      const bool sm_col = SMK && hash && p.bins < 65536 && col_b <= S.total - S.nbkt;
      uint32_t *W = K;
      double *rec_i = recs + (size_t)i * n_gp * 6;
      int anom = 0;
#pragma unroll 2
      for (int k = tid; k < n_gp; k += T) {
        double x[6];  // draws 6r+1..6r+6: energy, five cross sections
        lcg_doubles6(jump6(jt, r0 + Js[k], p.gseed), x);
        const double e = x[0], x1 = x[1], x2 = x[2], x3 = x[3], x4 = x[4], x5 = x[5];
        double2 *d = reinterpret_cast<double2 *>(rec_i + 6 * (size_t)k);
        __stcs(d, make_double2(e, x1));
        __stcs(d + 1, make_double2(x2, x3));
        __stcs(d + 2, make_double2(x4, x5));
        if (sm_col) {  // the entry pass's (e * bins - b) * 2^16 at b = bin(e), as integers
          const double y = e * (double)p.bins;
          int be = (int)y;
          be = be < p.bins ? be : p.bins;
          const double x = (y - (double)be) * 65536.0;
          const int q = x < 0.0 ? 0 : (x >= 65535.0 ? 65535 : (int)x);
          const int db = bfirst(e) - be;
          anom |= db < 0 || db > 1;
          W[k] = ((uint32_t)be << 16) | ((uint32_t)(q >> 1) << 1) | (uint32_t)(db & 1);
        } else {
          ekey[k] = dbits(e);
        }
      }
      const bool anomaly = __syncthreads_or(anom) != 0;
      phase_mark_if(trc, c, 8);
      if (hash) {
        int *colp = sm_col ? (int *)(ens_smem(c) + S.nbkt) : col;  // overlays the dead counters and J
        constexpr int U = 4;  // independent iterations per thread (loads first)
        if (sm_col) {
          auto bf_at = [&](int k) {
            if (anomaly) return bfirst(ld_(rec_i + 6 * (size_t)k));  // this CTA's records (bar.sync-ordered)
            const uint32_t w = W[k];
            return (int)(w >> 16) + (int)(w & 1u);
          };
          // bin b's column entry min(#{k >= 1: bfirst(E_k) <= b}, n_gp-2): a
          // histogram of bfirst (shared atomics), then an inclusive scan
          // (the clamp is applied where the entries read it)
          for (int b = tid; b <= p.bins; b += T) colp[b] = 0;
          __syncthreads();
          for (int k = 1 + tid; k < n_gp; k += T) {
            const int bf = bf_at(k);
            if (bf < p.bins) atomicAdd(&colp[bf], 1);
          }
          __syncthreads();
          smem_scan<true>(reinterpret_cast<uint32_t *>(colp), p.bins, ens_sh(c));
        } else {
          for (int k0 = tid; k0 < n_gp; k0 += U * T) {
            unsigned long long ek[U], ek1[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
              const int k = k0 + u * T;
              ek[u] = k < n_gp ? ld_(ekey + k) : 0ull;
              ek1[u] = k + 1 < n_gp ? ld_(ekey + k + 1) : 0ull;
            }
#pragma unroll
            for (int u = 0; u < U; u++) {
              const int k = k0 + u * T;
              if (k < n_gp) {
                const int lo = k == 0 ? 0 : bfirst(__longlong_as_double((long long)ek[u]));
                const int hi = k + 1 < n_gp ? bfirst(__longlong_as_double((long long)ek1[u])) : p.bins;
                const int v = k < n_gp - 2 ? k : n_gp - 2;
                for (int b = lo; b < hi; b++) colp[b] = v;
              }
            }
          }
        }
        if (tid == 0) colp[p.bins] = n_gp - 2;
        __syncthreads();
        if (sm_col) {
          // entries {u_low, u_high, q(E[u_low+1..u_low+6])} from shared memory:
          // q = 0 below bin b, 65535 above it or past the grid
          for (int b = tid; b <= p.bins; b += T) {
            const int c0 = colp[b], c1 = b < p.bins ? colp[b + 1] : n_gp - 2;
            const int ul = c0 < n_gp - 2 ? c0 : n_gp - 2, uh = c1 < n_gp - 2 ? c1 : n_gp - 2;
            XsHashEnt h;
            h.u_low = (uint16_t)ul;
            h.u_high = (uint16_t)(uh + 1);
#pragma unroll
            for (int k = 0; k < 6; k++) {
              uint32_t q15 = 32767u;
              if (ul + 1 + k <= n_gp - 1) {
                const uint32_t w = W[ul + 1 + k];
                const int fb = (int)(w >> 16);
                q15 = fb == b ? (w >> 1) & 0x7fffu : (fb > b ? 32767u : 0u);
              }
              h.q[k] = (uint16_t)q15;  // 15-bit quanta (SWAR compare in guess)
            }
            __stcs(reinterpret_cast<uint4 *>(ent + b), *reinterpret_cast<const uint4 *>(&h));
          }
        } else {
        for (int b0 = tid; b0 <= p.bins; b0 += U * T) {  // entries {u_low, u_high, q(E[u_low+1..u_low+6])}
          int ul[U], uh[U];
#pragma unroll
          for (int u = 0; u < U; u++) {
            const int b = b0 + u * T;
            ul[u] = b <= p.bins ? ld_(col + b) : 0;
            uh[u] = b < p.bins ? ld_(col + b + 1) : n_gp - 2;
          }
          unsigned long long e6[U][6];
#pragma unroll
          for (int u = 0; u < U; u++)
#pragma unroll
            for (int k = 0; k < 6; k++)
              e6[u][k] = ul[u] + 1 + k <= n_gp - 1 && b0 + u * T <= p.bins ? ld_(ekey + ul[u] + 1 + k) : 0ull;
#pragma unroll
          for (int u = 0; u < U; u++) {
            const int b = b0 + u * T;
            if (b > p.bins) continue;
            XsHashEnt h;
            h.u_low = (uint16_t)ul[u];
            h.u_high = (uint16_t)(uh[u] + 1);
#pragma unroll
            for (int k = 0; k < 6; k++) {
              int q = 65535;
              if (ul[u] + 1 + k <= n_gp - 1) {
                const double e = __longlong_as_double((long long)e6[u][k]);
                const double x = (e * (double)p.bins - (double)b) * 65536.0;
                q = x < 0.0 ? 0 : (x >= 65535.0 ? 65535 : (int)x);
              }
              h.q[k] = (uint16_t)(q >> 1);  // 15-bit quanta (SWAR compare in guess)
            }
            __stcs(reinterpret_cast<uint4 *>(ent + b), *reinterpret_cast<const uint4 *>(&h));
          }
        }
        }
        __syncthreads();
        phase_mark_if(trc, c, 9);
      }
    }
  }

  // ---- XS-3/4/5, unionized grid: one block-wide sort of all records ------
  // One bucket sort of all n_u records by energy replaces n_iso per-nuclide
  // sorts and the union merge: (G) count each record's energy bucket (energy
  // = draw 6r+1, XS-3); (S) scan; (P) scatter the record ids (4 B: the
  // energies are re-drawn where needed); (B) sort each ~4-record bucket by
  // (energy, id).  The sorted records ARE the union
  // (XS-5) and a nuclide's records in union order are its sorted records
  // (XS-4).  Ties are measure-zero (reading Q13) and broken by record id.
  // (U) union tables, (W) index sweep, (R) every record written once to its
  // sorted position, its five cross sections re-drawn via the jump tables.
  __device__ static __noinline__ void init(Ctx &c, const XsParams &p, const XsLayout &L, const XsSmem &S,
                                          bool team) {
    const bool trc = tracing(c);  // tracing (ENS_F_PHASES) thread, cached
    const int tid = threadIdx.x, T = blockDim.x;
    // team: the cluster's CTAs stripe every pass (cluster barrier between
    // passes; the counters live in the arena); else this CTA runs it alone
    const long long g0 = team ? (long long)c.crank * T + tid : tid, GS = team ? (long long)c.csize * T : T;
    auto sync = [&]() {
      if (team) team_sync(c);
      else __syncthreads();
    };
    const int n_iso = p.n_iso, n_gp = p.n_gp;
    const long long n_u = (long long)n_iso * n_gp;
    const long long NB = xs_buckets(p);
    const int nbn = xs_nbn(n_gp);
    const Affine *jt = (const Affine *)(ens_smem(c) + S.jmp);
    double *recs = (double *)(c.arena + L.recs);
    uint32_t *ids = (uint32_t *)(c.arena + L.keys);  // record ids, sorted by (energy, id)
    const bool sm_bkt = xs_smem_nb(p) != 0;
    uint32_t *bkt = sm_bkt ? (uint32_t *)(ens_smem(c) + S.ubkt) : (uint32_t *)(c.arena + L.bkt);
    int *ig = (int *)(c.arena + L.index);
    const Affine J6T = lcg_pow(6ULL * (uint64_t)GS);

    for (long long b = g0; b < NB; b += GS) bkt[b] = 0;
    sync();
    // (G) count
    {
      uint64_t s = lcg_pow(6ULL * (uint64_t)g0)(p.gseed);
      for (long long r = g0; r < n_u; r += GS, s = J6T(s)) {
        uint64_t t = s;
        atomicAdd(&bkt[bucket_of(lcg_double(t), r, n_gp, true, NB, nbn)], 1u);
      }
    }
    sync();
    XS_STOP(1);
    // (S) bucket offsets
    if (!team || c.crank == 0) global_exclusive_scan(bkt, NB, ens_sh(c));
    if (team) team_sync(c);
    XS_STOP(2);
    // (P) scatter, energies re-drawn, kQ independent atomics in flight (the
    // returned cursor is an L2 round trip)
    {
      constexpr int kQ = 8;
      const Affine JQT = lcg_pow(6ULL * kQ * (uint64_t)GS);
      uint64_t s = lcg_pow(6ULL * (uint64_t)g0)(p.gseed);
      for (long long r0 = g0; r0 < n_u; r0 += (long long)kQ * GS, s = JQT(s)) {
        unsigned long long eb[kQ];
        uint32_t pos[kQ];
        uint64_t sq = s;
#pragma unroll
        for (int q = 0; q < kQ; q++, sq = J6T(sq)) {
          uint64_t t = sq;
          eb[q] = dbits(lcg_double(t));
        }
#pragma unroll
        for (int q = 0; q < kQ; q++) {
          const long long r = r0 + (long long)q * GS;
          if (r < n_u)
            pos[q] = atomicAdd(&bkt[bucket_of(__longlong_as_double((long long)eb[q]), r, n_gp, true, NB, nbn)], 1u);
        }
#pragma unroll
        for (int q = 0; q < kQ; q++) {
          const long long r = r0 + (long long)q * GS;
          if (r < n_u) {
            ids[pos[q]] = (uint32_t)r;
          }
        }
      }
    }
    sync();
    XS_STOP(3);
    // (B) sort each bucket by (energy, record id); bkt[b] = end of bucket b
    for (long long b = g0; b < NB; b += GS)
      sort_bucket(ids, b ? (long long)bkt[b - 1] : 0, (long long)bkt[b], jt, p.gseed);
    sync();
    XS_STOP(4);

    // (U) ids[] in order is the union (XS-5); owner = record id / n_gp
    uint64_t *uA = (uint64_t *)(c.arena + L.uenergy);
    uint32_t *chist = sm_bkt ? bkt : (uint32_t *)(c.arena + L.chist);  // the sort's counters are dead
    const long long nch = (n_u + kXsSweepRows - 1) / kXsSweepRows;
    uint32_t *uf = (uint32_t *)(c.arena + L.ufind);
    const long long UB = xs_ubins(p);
    for (long long x = g0; x < nch * n_iso; x += GS) chist[x] = 0;
    sync();
    XS_STOP(5);
    // first bin b with u <= b / UB (UB a power of two: exact)
    auto bfirst = [&](unsigned long long bits) {
      const double x = __longlong_as_double((long long)bits) * (double)UB;
      long long bk = (long long)x;
      if ((double)bk < x) bk++;
      return bk < UB ? bk : UB;
    };
    // union energies, chunk owner counts, search table: ufind[b] = #{k >= 1 :
    // u_k <= b / UB} = e on [b_e, b_e+1) (b_0 := 0, b_n_u := UB).  The warp's
    // lanes hold consecutive e: u_{e+1} comes from the next lane (lane 31
    // re-draws it)
    const int lane = tid & 31;
    for (long long w0 = g0 - lane; w0 < n_u; w0 += GS) {
      const long long e = w0 + lane;
      uint32_t id = 0;
      unsigned long long key = 0;
      if (e < n_u) {
        id = ids[e];
        key = dbits(rec_energy(jt, id, p.gseed));
      }
      unsigned long long knext = __shfl_down_sync(0xffffffffu, key, 1);
      if (lane == 31 && e + 1 < n_u) knext = dbits(rec_energy(jt, ids[e + 1], p.gseed));
      if (e < n_u) {
        uA[e] = key;
        atomicAdd(&chist[(e / kXsSweepRows) * n_iso + id / n_gp], 1u);
        const long long lo = e == 0 ? 0 : bfirst(key);
        const long long hi = e + 1 < n_u ? bfirst(knext) : UB;
        for (long long b = lo; b < hi; b++) uf[b] = (uint32_t)e;
      }
    }
    sync();
    for (long long i = g0; i < n_iso; i += GS) {  // exclusive scan over chunks per owner, kU loads in
      constexpr int kU = 16;                      // flight (one at a time: an L2 round trip per chunk)
      uint32_t run = 0;
      long long ch = 0;
      for (; ch + kU <= nch; ch += kU) {
        uint32_t v[kU];
#pragma unroll
        for (int u = 0; u < kU; u++) v[u] = chist[(ch + u) * n_iso + i];
#pragma unroll
        for (int u = 0; u < kU; u++) {
          chist[(ch + u) * n_iso + i] = run;
          run += v[u];
        }
      }
      for (; ch < nch; ch++) {
        const uint32_t v = chist[ch * n_iso + i];
        chist[ch * n_iso + i] = run;
        run += v;
      }
    }
    sync();
    XS_STOP(6);
    // (W) sweep: a warp per chunk, lanes own nuclides; row e of the index grid
    // is clip(#{k>=1: E_i[k] <= u_e}, 0, n_gp-2) = clip(cnt_i(e) - 1, ...),
    // and the owner's new count is the sorted position of that record (XS-4).
    uint32_t *inv = (uint32_t *)(c.arena + L.inv);
    sweep(ids, inv, chist, ig, (int *)(ens_smem(c) + S.nbkt), n_u, n_iso, n_gp, nch, team ? (int)c.crank : 0,
          team ? (int)c.csize : 1);
    sync();
    XS_STOP(7);
    // (R) records in sorted order (coalesced 48-B writes): sorted position s
    // holds record inv[s], its energy re-drawn with the other five
    for (long long s0 = g0; s0 < n_u; s0 += 2LL * GS) {
      unsigned r[2];
#pragma unroll
      for (int q = 0; q < 2; q++)
        if (s0 + q * GS < n_u) r[q] = inv[s0 + q * GS];
#pragma unroll
      for (int q = 0; q < 2; q++)
        if (s0 + q * GS < n_u) {
          double x[6];  // draws 6r+1..6r+6: energy, five cross sections
          lcg_doubles6(jump6(jt, r[q], p.gseed), x);
          const double e = x[0], x1 = x[1], x2 = x[2], x3 = x[3], x4 = x[4], x5 = x[5];
          double2 *d = reinterpret_cast<double2 *>(recs + 6 * (size_t)(s0 + q * GS));
          __stcs(d, make_double2(e, x1));  // evict-first: the tables stream past L2
          __stcs(d + 1, make_double2(x2, x3));
          __stcs(d + 2, make_double2(x4, x5));
        }
    }
    sync();
    phase_mark_if(trc, c, 8);
  }

  // ---- XS-3/4/5, unionized grid, warp path (n_gp <= kXsWarpGp) -----------
  // (N) a warp per nuclide, in its own shared memory: energies (draw 6r+1 of
  // record r = i*n_gp + j, XS-3) are bucket-sorted by (energy, j) (XS-4),
  // each record is written once at its sorted position (coalesced; its five
  // cross sections re-drawn through the jump tables), the sorted energies go
  // to `ecmp` and ustart[i][ch] = #{k: chunk(E_i[k]) < ch} marks where each
  // union value chunk begins in the nuclide's run.  (U) a warp per chunk
  // gathers the chunk's energies from the n_iso runs, sorts them by (energy,
  // nuclide) — the union order of the block-wide sort (reading Q13) — and
  // writes the union energies, the chunk's search-table bins and the chunk's
  // index rows (the nuclides' counts start at ustart[.][ch] and one count
  // steps per row: lanes hold the counts of four nuclides each in registers
  // and store a row as 16-B vectors).  Returns false if a chunk held more
  // than kXsChunkCap energies (the caller then runs the block-wide path).
  __device__ static __forceinline__ int nuc_bkt(double e) {
    const int b = (int)(e * (double)kXsNucBkt);
    return b < kXsNucBkt - 1 ? b : kXsNucBkt - 1;
  }
  __device__ static __forceinline__ long long uchunk(double e, long long NC) {
    const long long ch = (long long)(e * (double)NC);
    return ch < NC - 1 ? ch : NC - 1;
  }
  __device__ static __forceinline__ int chunk_fb(double e, long long ch, long long NC) {
    const int b = (int)((e * (double)NC - (double)ch) * (double)kXsChunkFb);
    return b < 0 ? 0 : (b < kXsChunkFb - 1 ? b : kXsChunkFb - 1);
  }
  // exclusive prefix sum of cnt[0..N) (shared), by one warp, N = 32 * V
  template <int V>
  __device__ static __forceinline__ void warp_scan_smem(uint32_t *cnt, int lane) {
    uint32_t v[V], sum = 0;
#pragma unroll
    for (int q = 0; q < V; q++) {
      v[q] = cnt[lane * V + q];
      sum += v[q];
    }
    uint32_t inc = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += t;
    }
    uint32_t run = inc - sum;
#pragma unroll
    for (int q = 0; q < V; q++) {
      cnt[lane * V + q] = run;
      run += v[q];
    }
  }
  // insertion sort of (E bits, tag) pairs in [lo, hi) (shared memory)
  __device__ static __forceinline__ void isort_pairs(unsigned long long *E, uint16_t *t, int lo, int hi) {
    for (int x = lo + 1; x < hi; x++) {
      const unsigned long long ve = E[x];
      const uint16_t vt = t[x];
      int y = x - 1;
      while (y >= lo && (E[y] > ve || (E[y] == ve && t[y] > vt))) {
        E[y + 1] = E[y];
        t[y + 1] = t[y];
        y--;
      }
      E[y + 1] = ve;
      t[y + 1] = vt;
    }
  }
  // 16-B store to global memory, evict-first (the index grid streams past L2,
  // which keeps the init's scratch — sorted energies, ustart — resident)
  __device__ static __forceinline__ void st_v4(int *p, int x, int y, int z, int w) {
    asm volatile("st.global.cs.v4.s32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(x), "r"(y), "r"(z), "r"(w) : "memory");
  }
  __device__ static __forceinline__ int clip0(int v, int hi) { return v < 0 ? 0 : (v > hi ? hi : v); }
  // one index row: step the lane's counts by the row's owner, store them
  template <int Q, bool CLIP>
  __device__ static __forceinline__ void row_step(int own, const int (&qb)[Q], int4 (&c)[Q], int *row, int hi) {
#pragma unroll
    for (int k = 0; k < Q; k++) {
      // c[k].{x,y,z,w} += (own == qb[k] + {0,1,2,3}): predicated adds (no branch)
      asm("{ .reg .pred p0, p1, p2, p3; .reg .s32 d;\n\t"
          "sub.s32 d, %4, %5;\n\t"
          "setp.eq.s32 p0, d, 0; setp.eq.s32 p1, d, 1; setp.eq.s32 p2, d, 2; setp.eq.s32 p3, d, 3;\n\t"
          "@p0 add.s32 %0, %0, 1; @p1 add.s32 %1, %1, 1; @p2 add.s32 %2, %2, 1; @p3 add.s32 %3, %3, 1; }"
          : "+r"(c[k].x), "+r"(c[k].y), "+r"(c[k].z), "+r"(c[k].w)
          : "r"(own), "r"(qb[k]));
      if (CLIP) st_v4(row + qb[k], clip0(c[k].x, hi), clip0(c[k].y, hi), clip0(c[k].z, hi), clip0(c[k].w, hi));
      else st_v4(row + qb[k], c[k].x, c[k].y, c[k].z, c[k].w);
    }
  }
  // index rows e0 .. e0+m-1 of one union chunk.  Lane holds, for k < Q, the
  // counts of the four nuclides of quad (lane + 32k) mod ip/4 (quads past
  // the row are duplicates: every lane stores, duplicates store equal data),
  // minus one; row r steps the count of its owner Ou[r] and is stored as
  // ip/4 16-B vectors.  ua / ub = the chunk's and the next chunk's rows of
  // ustart: when no count of the chunk can leave [1, n_gp-1], the row
  // values need no clipping (almost every chunk).
  template <int Q, bool CLIP>
  __device__ static __forceinline__ void chunk_rows(const uint16_t *Ou, int m, int *row, int ip, int hi,
                                                    const int (&qb)[Q], int4 (&c)[Q]) {
    int r = 0;
    for (; r + 4 <= m; r += 4) {
      const uint2 o4 = *reinterpret_cast<const uint2 *>(Ou + r);
      row_step<Q, CLIP>((int)(o4.x & 0xffffu), qb, c, row, hi);
      row_step<Q, CLIP>((int)(o4.x >> 16), qb, c, row + ip, hi);
      row_step<Q, CLIP>((int)(o4.y & 0xffffu), qb, c, row + 2 * ip, hi);
      row_step<Q, CLIP>((int)(o4.y >> 16), qb, c, row + 3 * ip, hi);
      row += 4 * ip;
    }
    for (; r < m; r++, row += ip) row_step<Q, CLIP>((int)Ou[r], qb, c, row, hi);
  }
  // the lane's ustart quads of a chunk (rows ch and ch+1), loaded ahead of
  // the chunk's sort so that their latency is hidden
  template <int Q>
  __device__ static __forceinline__ void sweep_quads(const int *ua, int ip, int lane, int4 (&v)[Q], int4 (&w)[Q]) {
    const int ng4 = ip >> 2;
#pragma unroll
    for (int k = 0; k < Q; k++) {
      const int qb = 4 * ((lane + 32 * k) % ng4);
      v[k] = ld_(reinterpret_cast<const int4 *>(ua + qb));
      w[k] = ld_(reinterpret_cast<const int4 *>(ua + ip + qb));
    }
  }
  template <int Q>
  __device__ static __forceinline__ void chunk_sweep(const uint16_t *Ou, int m, int *ig, long long e0, int ip,
                                                     int n_gp, int lane, const int4 (&vq)[Q], const int4 (&wq)[Q]) {
    const int ng4 = ip >> 2;
    int qb[Q];
    int4 c[Q];
    bool inner = true;
#pragma unroll
    for (int k = 0; k < Q; k++) {
      qb[k] = 4 * ((lane + 32 * k) % ng4);
      const int4 v = vq[k], w = wq[k];
      c[k] = make_int4(v.x - 1, v.y - 1, v.z - 1, v.w - 1);
      inner = inner && v.x >= 1 && v.y >= 1 && v.z >= 1 && v.w >= 1 && w.x <= n_gp - 1 && w.y <= n_gp - 1 &&
              w.z <= n_gp - 1 && w.w <= n_gp - 1;
    }
    int *row = ig + (size_t)e0 * ip;
    if (__all_sync(0xffffffffu, inner)) chunk_rows<Q, false>(Ou, m, row, ip, n_gp - 2, qb, c);
    else chunk_rows<Q, true>(Ou, m, row, ip, n_gp - 2, qb, c);
  }
  // energy draw (6r+1) of record r and its 32-bit sort key (the LCG state's
  // top bits: monotone in the energy)
  __device__ static __forceinline__ double rec_energy(const Affine *jt, uint32_t r, uint64_t gseed) {
    uint64_t t = jump6(jt, r, gseed);
    return lcg_double(t);
  }
  // insertion sort of (key, j) in [lo, hi) by (energy, j): keys order the
  // energies except on equal keys, where the energies are re-drawn
  __device__ static __forceinline__ void isort_keys(uint32_t *K, uint16_t *J, int lo, int hi, const Affine *jt,
                                                    uint32_t r0, uint64_t gseed) {
    for (int x = lo + 1; x < hi; x++) {
      const uint32_t vk = K[x];
      const uint16_t vj = J[x];
      int y = x - 1;
      for (; y >= lo; y--) {
        const uint32_t yk = K[y];
        bool after;  // element y sorts after the inserted one
        if (yk != vk) after = yk > vk;
        else {
          const double ey = rec_energy(jt, r0 + J[y], gseed), ev = rec_energy(jt, r0 + vj, gseed);
          after = ey > ev || (ey == ev && J[y] > vj);
        }
        if (!after) break;
        K[y + 1] = yk;
        J[y + 1] = J[y];
      }
      K[y + 1] = vk;
      J[y + 1] = vj;
    }
  }

  // (U) of init_warp: warp per union chunk.  NI = nuclide slots per lane
  // (lane + 32z), Q = index-row quads per lane.  Each chunk's ustart rows are
  // loaded one chunk ahead (registers) so their latency overlaps the
  // previous chunk's rows.  Returns 1 if a chunk exceeded kXsChunkCap.
  template <int NI, int Q>
  __device__ static __noinline__ unsigned union_chunks(Ctx &c, const XsParams &p, const XsLayout &L,
                                                       const XsSmem &S) {
    const bool trc = tracing(c);  // tracing (ENS_F_PHASES) thread, cached
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = xs_warp_scr_warps((int)blockDim.x);
    const int n_iso = p.n_iso, n_gp = p.n_gp, ip = xs_iso_pad(n_iso);
    const int NC = (int)xs_uchunks(p);
    if (warp >= nw) return 0;
    const long long UB = xs_ubins(p), BPC = UB / NC;
    const unsigned long long *ecmp = (const unsigned long long *)(c.arena + L.keys);
    const int *ust = (const int *)(c.arena + L.ustart);
    uint64_t *uA = (uint64_t *)(c.arena + L.uenergy);
    uint32_t *uf = (uint32_t *)(c.arena + L.ufind);
    int *ig = (int *)(c.arena + L.index);
    char *scr = ens_smem(c) + S.nbkt + (size_t)warp * kXsUniScr;
    unsigned long long *Eu = (unsigned long long *)scr;          // sorted chunk
    unsigned long long *Eg0 = Eu + kXsChunkCap;                  // gathered, unsorted (2 buffers)
    uint16_t *Ou = (uint16_t *)(scr + kXsChunkCap * 24);
    uint16_t *Og0 = Ou + kXsChunkCap;
    uint32_t *fc = (uint32_t *)(scr + kXsChunkCap * 30);
    unsigned ovf = 0;
    int an[NI], bn[NI];
    auto load = [&](int ch) {
#pragma unroll
      for (int z = 0; z < NI; z++) {
        const int i = lane + 32 * z;
        an[z] = i < n_iso ? ld_(ust + (size_t)ch * ip + i) : 0;
        bn[z] = i < n_iso ? ld_(ust + (size_t)(ch + 1) * ip + i) : 0;
      }
    };
    // stage a chunk: its runs ecmp[i][an .. bn) copied asynchronously
    // (cp.async) to gather buffer `buf` at their prefix offsets; sets the
    // chunk's size and first union row
    int m_n = 0;
    long long e0_n = 0;
    auto stage = [&](int buf) {
      int e0l = 0, tot = 0;
      unsigned long long *Eg = Eg0 + buf * kXsChunkCap;
      uint16_t *Og = Og0 + buf * kXsChunkCap;
      int o[NI];
#pragma unroll
      for (int z = 0; z < NI; z++) {
        const int len = bn[z] - an[z];
        int inc = len;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const int t = __shfl_up_sync(0xffffffffu, inc, d);
          if (lane >= d) inc += t;
        }
        o[z] = tot + inc - len;
        tot += __shfl_sync(0xffffffffu, inc, 31);
        e0l += an[z];
      }
      e0_n = (long long)warp_sum_u64((unsigned long long)e0l);
      m_n = tot;
      if (tot <= kXsChunkCap) {
#pragma unroll
        for (int z = 0; z < NI; z++) {
          const int i = lane + 32 * z;
          const unsigned long long *src = ecmp + (size_t)i * n_gp + an[z];
          for (int x = 0; x < bn[z] - an[z]; x++) {
            const uint32_t dst = (uint32_t)__cvta_generic_to_shared(Eg + o[z] + x);
            asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(dst), "l"(src + x) : "memory");
            Og[o[z] + x] = (uint16_t)i;
          }
        }
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
    };
    int buf = 0;
    const int gw = warp + (int)c.crank * nw, gn = nw * (int)c.csize;  // chunks striped over the team's warps
    if (gw < NC) {
      load(gw);
      stage(0);
    }
    for (int ch = gw; ch < NC; ch += gn, buf ^= 1) {
      const int m = m_n;
      const long long e0 = e0_n;
      if (ch + gn < NC) load(ch + gn);
      asm volatile("cp.async.wait_all;" ::: "memory");
      __syncwarp();
      if (m > kXsChunkCap) {
        ovf = 1;
        if (ch + gn < NC) stage(buf ^ 1);
        continue;
      }
      const unsigned long long *Eg = Eg0 + buf * kXsChunkCap;
      const uint16_t *Og = Og0 + buf * kXsChunkCap;
      int4 vq[Q], wq[Q];  // this chunk's ustart quads, in flight during the sort
      sweep_quads<Q>(ust + (size_t)ch * ip, ip, lane, vq, wq);
      for (int b = lane; b < kXsChunkFb; b += 32) fc[b] = 0;
      __syncwarp();
      phase_mark_if(trc, c, 12);
      for (int x = lane; x < m; x += 32) atomicAdd(&fc[chunk_fb(__longlong_as_double((long long)Eg[x]), ch, NC)], 1u);
      __syncwarp();
      warp_scan_smem<kXsChunkFb / 32>(fc, lane);
      __syncwarp();
      for (int x = lane; x < m; x += 32) {
        const unsigned long long eb = Eg[x];
        const uint32_t pos = atomicAdd(&fc[chunk_fb(__longlong_as_double((long long)eb), ch, NC)], 1u);
        Eu[pos] = eb;
        Ou[pos] = Og[x];
      }
      __syncwarp();
      phase_mark_if(trc, c, 13);
      for (int b = lane; b < kXsChunkFb; b += 32) isort_pairs(Eu, Ou, b ? (int)fc[b - 1] : 0, (int)fc[b]);
      __syncwarp();
      phase_mark_if(trc, c, 14);
      for (int r = lane; r < m; r += 32) uA[e0 + r] = Eu[r];
      // search table: uf[b] = #{k >= 1: u_k <= b / UB}, b in this chunk's bins
      const double inv_ub = 1.0 / (double)UB;  // UB a power of two: b * inv_ub == b / UB exactly
      for (long long b = ch * BPC + lane; b < (ch + 1) * BPC; b += 32) {
        const unsigned long long vb = dbits((double)b * inv_ub);
        int lo = 0, hi = m;  // first r with Eu[r] > vb
        while (lo < hi) {
          const int mid = (lo + hi) >> 1;
          if (Eu[mid] <= vb) lo = mid + 1;
          else hi = mid;
        }
        const long long v = e0 + lo - 1;
        uf[b] = (uint32_t)(v > 0 ? v : 0);
      }
      phase_mark_if(trc, c, 15);
      if (ch + gn < NC) stage(buf ^ 1);  // the next chunk's gather overlaps this chunk's rows
      chunk_sweep<Q>(Ou, m, ig, e0, ip, n_gp, lane, vq, wq);
      __syncwarp();
      phase_mark_if(trc, c, 9);
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
    return ovf;
  }

  __device__ static __noinline__ bool init_warp(Ctx &c, const XsParams &p, const XsLayout &L, const XsSmem &S) {
    const bool trc = tracing(c);  // tracing (ENS_F_PHASES) thread, cached
    const int tid = threadIdx.x, T = blockDim.x, lane = tid & 31, warp = tid >> 5, nw = xs_warp_scr_warps(T);
    const int n_iso = p.n_iso, n_gp = p.n_gp, ip = xs_iso_pad(n_iso);
    const int NC = (int)xs_uchunks(p);
    const Affine *jt = (const Affine *)(ens_smem(c) + S.jmp);
    double *recs = (double *)(c.arena + L.recs);
    unsigned long long *ecmp = (unsigned long long *)(c.arena + L.keys);  // [n_iso][n_gp] sorted energies
    int *ust = (int *)(c.arena + L.ustart);                                 // [NC+1][ip]
    const Affine J32 = lcg_pow(6ULL * 32ULL);
    const uint64_t gseed = p.gseed;

    // (N) nuclides, a warp each (striped over the team's CTAs)
    for (int x = tid + (int)c.crank * T; x < (NC + 1) * (ip - n_iso); x += T * (int)c.csize)
      ust[(x / (ip - n_iso)) * ip + n_iso + x % (ip - n_iso)] = 0;  // pad columns
    {
      char *scr = ens_smem(c) + S.nbkt + (size_t)warp * kXsNucScr;
      uint32_t *K = (uint32_t *)scr;
      uint16_t *J = (uint16_t *)(scr + kXsWarpGp * 4);
      uint32_t *cnt = (uint32_t *)(scr + kXsWarpGp * 6);
      for (int i = warp + (int)c.crank * nw; i < n_iso && warp < nw; i += nw * (int)c.csize) {
        const uint32_t r0 = (uint32_t)i * (uint32_t)n_gp;
        for (int b = lane; b < kXsNucBkt; b += 32) cnt[b] = 0;
        __syncwarp();
        {
          uint64_t s = jump6(jt, r0 + (uint32_t)lane, gseed);
          for (int j = lane; j < n_gp; j += 32, s = J32(s)) atomicAdd(&cnt[(uint32_t)(lcg_next(s) >> 31) >> (32 - kXsNucBktBits)], 1u);
        }
        __syncwarp();
        phase_mark_if(trc, c, 1);
        warp_scan_smem<kXsNucBkt / 32>(cnt, lane);
        __syncwarp();
        {
          uint64_t s = jump6(jt, r0 + (uint32_t)lane, gseed);
          for (int j = lane; j < n_gp; j += 32, s = J32(s)) {
            const uint32_t key = (uint32_t)(lcg_next(s) >> 31);
            const uint32_t pos = atomicAdd(&cnt[key >> (32 - kXsNucBktBits)], 1u);
            K[pos] = key;
            J[pos] = (uint16_t)j;
          }
        }
        __syncwarp();
        phase_mark_if(trc, c, 2);
        for (int b = lane; b < kXsNucBkt; b += 32) isort_keys(K, J, b ? (int)cnt[b - 1] : 0, (int)cnt[b], jt, r0, gseed);
        __syncwarp();
        phase_mark_if(trc, c, 3);
        // records at their sorted positions (coalesced), sorted energies, and
        // ustart[ch][i] = k for the chunks ch in (chunk(E[k-1]), chunk(E[k])]
        double *rec_i = recs + (size_t)r0 * 6;
        int carry = -1;
#pragma unroll 2
        for (int k0 = 0; k0 < n_gp; k0 += 32) {
          const int k = k0 + lane;
          int chk = NC;
          if (k < n_gp) {
            double x[6];  // draws 6r+1..6r+6: energy, five cross sections
            lcg_doubles6(jump6(jt, r0 + J[k], gseed), x);
            const double e = x[0], x1 = x[1], x2 = x[2], x3 = x[3], x4 = x[4], x5 = x[5];
            double2 *d = reinterpret_cast<double2 *>(rec_i + 6 * (size_t)k);
            __stcs(d, make_double2(e, x1));  // evict-first, like the index rows
            __stcs(d + 1, make_double2(x2, x3));
            __stcs(d + 2, make_double2(x4, x5));
            ecmp[(size_t)r0 + k] = dbits(e);
            chk = (int)uchunk(e, NC);
          }
          int prev = __shfl_up_sync(0xffffffffu, chk, 1);
          if (lane == 0) prev = carry;
          if (k < n_gp)
            for (int ch = prev + 1; ch <= chk; ch++) ust[ch * ip + i] = k;
          if (k == n_gp - 1)
            for (int ch = chk + 1; ch <= NC; ch++) ust[ch * ip + i] = n_gp;
          carry = __shfl_sync(0xffffffffu, chk, 31);
        }
        __syncwarp();
        phase_mark_if(trc, c, 5);
      }
    }
    team_sync(c);  // every nuclide's sorted run and ustart column, team-wide
    phase_mark_if(trc, c, 6);

    // (U) union chunks, a warp each (striped over the team's CTAs)
    const unsigned ovf = ip <= 128 ? union_chunks<3, 1>(c, p, L, S) : union_chunks<12, 3>(c, p, L, S);
    const bool bad = team_any(c, (int)ovf);
    phase_mark_if(trc, c, 8);
    return !bad;
  }

  // XS-8, XS-9 for one nuclide: interpolate the pair (a = low, b = high
  // record: {E, total, elastic, absorption, fission, nu_fission}) at pe and
  // add conc * micro to the five channels, in the oracle's operation order
  __device__ static __forceinline__ void accumulate(double pe, double conc, const double2 &a0, const double2 &a1,
                                                    const double2 &a2, const double2 &b0, const double2 &b1,
                                                    const double2 &b2, double &m0, double &m1, double &m2,
                                                    double &m3, double &m4) {
    const double f = (b0.x - pe) / (b0.x - a0.x);
    m0 += (b0.y - f * (b0.y - a0.y)) * conc;
    m1 += (b1.x - f * (b1.x - a1.x)) * conc;
    m2 += (b1.y - f * (b1.y - a1.y)) * conc;
    m3 += (b2.x - f * (b2.x - a2.x)) * conc;
    m4 += (b2.y - f * (b2.y - a2.y)) * conc;
  }

  // XS-7..XS-9 for one lookup (energy pe, material mat, union row / hash bin
  // idx): the macroscopic XS m[0..4], nuclides summed in list order.  Each
  // grid type is software-pipelined without holding future data in
  // registers: index data a few nuclides ahead is prefetched into L1, the
  // next nuclide's record pair is prefetched into L1 while this one's is
  // gathered (a line's first touch goes to HBM).
  template <int GRID>
  __device__ static __forceinline__ void macro_lookup(const XsParams &p, const double *recs, const int *ig,
                                                      const int *nn, const double *concs, const uint16_t *mats,
                                                      double pe, int mat, int idx, double *m) {
    const int n_iso = p.n_iso, n_gp = p.n_gp, mx = xs_max_nucs(n_iso);
    const int nm = nn[mat];
    const uint16_t *mrow = mats + mat * mx;
    const double *crow = concs + mat * mx;
    double m0 = 0.0, m1 = 0.0, m2 = 0.0, m3 = 0.0, m4 = 0.0;
    auto pf_pair = [&](int j, int lo) {
      const double *q = recs + ((uint32_t)mrow[j] * (uint32_t)n_gp + (uint32_t)lo) * 6u;  // < 2^32 (n_u <= 355 * 16384)
      prefetch_l1(q);
      prefetch_l1(q + 11);
    };
    if constexpr (GRID == XS_HASH) {
      // bracket guess from the entry's quantized energies (XsHashEnt): a
      // lower bound on upstream's bracket, exact unless two energies share a
      // 2^-16 bin quantum; verified on the gathered pair, walked / searched
      // with upstream's logic otherwise
      const int pq = (int)((pe * (double)p.bins - (double)idx) * 65536.0);
        const XsHashEnt *hc = (const XsHashEnt *)ig + idx;
      const uint32_t hs32 = (uint32_t)p.bins + 1u;  // entry index < 355 * (10^7 + 1) < 2^32
      auto ent = [&](int j) { return reinterpret_cast<const uint4 *>(hc + (uint32_t)mrow[j] * hs32); };
      // #{k: pq15 > q_k} over the six 15-bit quanta by a SWAR compare: per
      // halfword 0x8000 + pq15 - q - 1 keeps bit 15 iff pq15 > q (no borrow
      // or carry crosses halves), one popcount for all six
      const uint32_t pq15 = (uint32_t)(pq < 0 ? 0 : (pq >> 1 > 32767 ? 32767 : pq >> 1));
      const uint32_t P = (pq15 | (pq15 << 16) | 0x80008000u) - 0x00010001u;
      auto guess = [&](const uint4 &h) {
        const uint32_t m = 0x80008000u;
        const uint32_t x = ((P - h.y) & m) | (((P - h.z) & m) >> 1) | (((P - h.w) & m) >> 2);
        return (int)(h.x & 0xffffu) + __popc(x);
      };
      // nuclide j's record pair at the guessed bracket
      auto gather = [&](int j, const uint4 &h, double2 &a0, double2 &a1, double2 &a2, double2 &b0, double2 &b1,
                        double2 &b2) {
        const int uh = (int)(h.x >> 16);
        int lo = guess(h);
        lo = lo < uh - 1 ? lo : uh - 1;
        const double2 *r2 = reinterpret_cast<const double2 *>(recs + ((uint32_t)mrow[j] * (uint32_t)n_gp + (uint32_t)lo) * 6u);
        a0 = ld_(r2 + 0); a1 = ld_(r2 + 1); a2 = ld_(r2 + 2);
        b0 = ld_(r2 + 3); b1 = ld_(r2 + 4); b2 = ld_(r2 + 5);
        return 0;
      };
      // lo is upstream's bracket (grid_search on [u_low, u_high], edge cases
      // excluded) iff E[lo] < pe < E[lo+1] and lo+1 <= u_high; walk forward
      // while pe is past the pair (a quantum collision), else upstream logic
      auto gather_fix = [&](int j, const uint4 &h, double2 &a0, double2 &a1, double2 &a2, double2 &b0,
                            double2 &b1, double2 &b2) {
        const double *E = recs + (uint32_t)mrow[j] * (uint32_t)n_gp * 6u;
        const int u_low = (int)(h.x & 0xffffu), uh = (int)(h.x >> 16);
        int lo = guess(h);
        lo = lo < uh - 1 ? lo : uh - 1;
        while (pe >= b0.x && a0.x < pe && lo + 2 <= uh) {
          lo++;
          const double2 *w2 = reinterpret_cast<const double2 *>(E + 6 * (size_t)lo);
          a0 = b0; a1 = b1; a2 = b2;
          b0 = ld_(w2 + 3); b1 = ld_(w2 + 4); b2 = ld_(w2 + 5);
        }
        if (!(a0.x < pe && pe < b0.x && lo + 1 <= uh)) {
          const double e_low = ld_(E + 6 * (size_t)u_low);
          const double e_high = ld_(E + 6 * (size_t)uh);
          int lower;
          if (pe <= e_low) lower = 0;
          else if (pe >= e_high) lower = n_gp - 1;
          else lower = gs_recs(E, pe, u_low, uh);
          const int l2 = lower == n_gp - 1 ? lower - 1 : lower;
          const double2 *w2 = reinterpret_cast<const double2 *>(E + 6 * (size_t)l2);
          a0 = ld_(w2 + 0); a1 = ld_(w2 + 1); a2 = ld_(w2 + 2);
          b0 = ld_(w2 + 3); b1 = ld_(w2 + 4); b2 = ld_(w2 + 5);
        }
        return 0;
      };
      // kXsStep nuclides per step (independent gathers and divisions in
      // flight), accumulated in list order
      constexpr int U = kXsStep;
      const uint4 z = make_uint4(0, 0, 0, 0);
      uint4 cur[U], nxt[U];
#pragma unroll
      for (int u = 0; u < U; u++) {
        cur[u] = u < nm ? ld_(ent(u)) : z;
        nxt[u] = U + u < nm ? ld_(ent(U + u)) : z;
      }
      for (int k = 2 * U; k < 4 * U && k < nm; k++) prefetch_l1(ent(k));
#pragma unroll
      for (int u = 0; u < U; u++)
        if (u < nm) pf_pair(u, guess(cur[u]));
      int j = 0;
      for (; j + U <= nm; j += U) {
        uint4 h[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
          h[u] = cur[u];
          cur[u] = nxt[u];
          if (j + 2 * U + u < nm) nxt[u] = ld_(ent(j + 2 * U + u));
          if (j + 4 * U + u < nm) prefetch_l1(ent(j + 4 * U + u));
          if (j + U + u < nm) pf_pair(j + U + u, guess(cur[u]));
        }
        double2 A[U][6];
#pragma unroll
        for (int u = 0; u < U; u++) {
          auto fix = gather(j + u, h[u], A[u][0], A[u][1], A[u][2], A[u][3], A[u][4], A[u][5]);
          (void)fix;
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
          auto fix = gather_fix(j + u, h[u], A[u][0], A[u][1], A[u][2], A[u][3], A[u][4], A[u][5]);
          (void)fix;
        }
#pragma unroll
        for (int u = 0; u < U; u++)
          accumulate(pe, crow[j + u], A[u][0], A[u][1], A[u][2], A[u][3], A[u][4], A[u][5], m0, m1, m2, m3, m4);
      }
#pragma unroll
      for (int u = 0; u < U - 1; u++) {  // tail
        if (j + u < nm) {
          double2 a0, a1, a2, b0, b1, b2;
          gather(j + u, cur[u], a0, a1, a2, b0, b1, b2);
          gather_fix(j + u, cur[u], a0, a1, a2, b0, b1, b2);
          accumulate(pe, crow[j + u], a0, a1, a2, b0, b1, b2, m0, m1, m2, m3, m4);
        }
      }
    } else if constexpr (GRID == XS_UNIONIZED) {
      // the union row idx holds every nuclide's bracket (XS-7)
      const int *row = ig + (size_t)idx * xs_iso_pad(n_iso);
      auto bracket = [&](int k) { return k == n_gp - 1 ? k - 1 : k; };
      // two nuclides per step (both pairs' loads in flight before either is
      // used), accumulated in list order; index entries two steps ahead,
      // pair prefetches one step ahead
      auto pair = [&](int j, int k) {
        return reinterpret_cast<const double2 *>(recs + ((uint32_t)mrow[j] * (uint32_t)n_gp + (uint32_t)k) * 6u);
      };
      int ia = nm > 0 ? ld_(row + mrow[0]) : 0, ib = nm > 1 ? ld_(row + mrow[1]) : 0;
      int na = nm > 2 ? ld_(row + mrow[2]) : 0, nb = nm > 3 ? ld_(row + mrow[3]) : 0;
      if (nm > 0) pf_pair(0, bracket(ia));
      if (nm > 1) pf_pair(1, bracket(ib));
      int j = 0;
      for (; j + 2 <= nm; j += 2) {
        const int ka = bracket(ia), kb = bracket(ib);
        ia = na;
        ib = nb;
        if (j + 4 < nm) na = ld_(row + mrow[j + 4]);
        if (j + 5 < nm) nb = ld_(row + mrow[j + 5]);
        if (j + 2 < nm) pf_pair(j + 2, bracket(ia));
        if (j + 3 < nm) pf_pair(j + 3, bracket(ib));
        const double2 *ra = pair(j, ka), *rb = pair(j + 1, kb);
        const double2 a0 = ld_(ra + 0), a1 = ld_(ra + 1), a2 = ld_(ra + 2);
        const double2 b0 = ld_(ra + 3), b1 = ld_(ra + 4), b2 = ld_(ra + 5);
        const double2 c0 = ld_(rb + 0), c1 = ld_(rb + 1), c2 = ld_(rb + 2);
        const double2 d0 = ld_(rb + 3), d1 = ld_(rb + 4), d2 = ld_(rb + 5);
        accumulate(pe, crow[j], a0, a1, a2, b0, b1, b2, m0, m1, m2, m3, m4);
        accumulate(pe, crow[j + 1], c0, c1, c2, d0, d1, d2, m0, m1, m2, m3, m4);
      }
      if (j < nm) {
        const double2 *ra = pair(j, bracket(ia));
        const double2 a0 = ld_(ra + 0), a1 = ld_(ra + 1), a2 = ld_(ra + 2);
        const double2 b0 = ld_(ra + 3), b1 = ld_(ra + 4), b2 = ld_(ra + 5);
        accumulate(pe, crow[j], a0, a1, a2, b0, b1, b2, m0, m1, m2, m3, m4);
      }
    } else {
      // nuclide grid: binary search of each nuclide's energies (XS-7)
      for (int j = 0; j < nm; j++) {
        const double *E = recs + (size_t)mrow[j] * n_gp * 6;
        const int k = gs_recs(E, pe, 0, n_gp - 1);
        const double2 *r2 = reinterpret_cast<const double2 *>(E + 6 * (size_t)(k == n_gp - 1 ? k - 1 : k));
        const double2 a0 = ld_(r2 + 0), a1 = ld_(r2 + 1), a2 = ld_(r2 + 2);
        const double2 b0 = ld_(r2 + 3), b1 = ld_(r2 + 4), b2 = ld_(r2 + 5);
        accumulate(pe, crow[j], a0, a1, a2, b0, b1, b2, m0, m1, m2, m3, m4);
      }
    }
    m[0] = m0;
    m[1] = m1;
    m[2] = m2;
    m[3] = m3;
    m[4] = m4;
  }

  // union position of energy pe == grid_search(u, pe, 0, n_u-1) (XS-7), via
  // the search table: ufind[floor(pe*UB)] then a short forward scan
  __device__ static __forceinline__ int union_idx(const uint32_t *uf, const uint64_t *uA, long long UB, long long n_u,
                                                  double pe) {
    long long b = (long long)(pe * (double)UB);
    if (b > UB - 1) b = UB - 1;
    long long cc = ld_(uf + b);
    while (cc < n_u - 1 && __longlong_as_double((long long)ld_(uA + cc + 1)) <= pe) cc++;
    return (int)(cc < n_u - 2 ? cc : n_u - 2);
  }

  // ---- history mode: thread per particle --------
  // Particle q's stream starts at ff(seed, q * L * 10); its L lookups are a
  // dependent chain (after each, skip one draw per macro channel > 1.0, then
  // sample the next energy and material), so particles run in parallel.
  template <int GRID>
  __device__ static __noinline__ void lookups_history(Ctx &c, const XsParams &p, const XsLayout &L,
                                                      const double *thr, const int *nn, const double *concs,
                                                      const uint16_t *mats, Result &R) {
    const int tid = threadIdx.x, T = blockDim.x;
    const long long n_u = (long long)p.n_iso * p.n_gp, nL = p.lookups;
    const double *recs = (const double *)(c.arena + L.recs);
    const int *ig = (const int *)(c.arena + L.index);
    const uint64_t *uA = (const uint64_t *)(c.arena + L.uenergy);
    const uint32_t *uf = (const uint32_t *)(c.arena + L.ufind);
    const long long UB = xs_ubins(p);
    const double du = 1.0 / p.bins;
    const long long g0 = (long long)c.crank * T + tid, gs = (long long)c.csize * T;
    Affine fwd[6];  // skip 0..5 draws
#pragma unroll
    for (int k = 0; k < 6; k++) fwd[k] = lcg_pow((uint64_t)k);
    const Affine J = lcg_pow((uint64_t)gs * (uint64_t)nL * 10ULL);
    uint64_t s0 = lcg_pow((uint64_t)g0 * (uint64_t)nL * 10ULL)(p.seed);
    unsigned long long ver = 0, bsum = 0;
    double fsum = 0.0, fabs_ = 0.0;
    for (long long q = g0; q < p.particles; q += gs, s0 = J(s0)) {
      uint64_t s = s0;
      double pe = lcg_double(s);
      int mat = pick_mat_thr(thr, lcg_double(s));
      for (long long i = 0; i < nL; i++) {
        int idx = 0;
        if (GRID == XS_UNIONIZED) idx = union_idx(uf, uA, UB, n_u, pe);
        else if (GRID == XS_HASH) {
          const long long bb = (long long)(pe / du);
          idx = bb > p.bins - 1 ? p.bins - 1 : (int)bb;  // reading Q14
        }
        double m[5];
        macro_lookup<GRID>(p, recs, ig, nn, concs, mats, pe, mat, idx, m);
        double mxv = -1.0;
        int am = 0;
        int n_forward = 0;
#pragma unroll
        for (int x = 0; x < 5; x++) {
          if (m[x] > mxv) {
            mxv = m[x];
            am = x;
          }
          n_forward += m[x] > 1.0 ? 1 : 0;
          bsum += dbits(m[x]);
          fsum += m[x];
          fabs_ += fabs(m[x]);
        }
        ver += (unsigned long long)(am + 1);
        atomicAdd(&ens_sh(c)->tallies[am], 1u);
        atomicAdd(&ens_sh(c)->tallies[5 + mat], 1u);
        s = fwd[n_forward](s);
        pe = lcg_double(s);
        mat = pick_mat_thr(thr, lcg_double(s));
      }
    }
    ver = team_sum_u64(c, ver);
    bsum = team_sum_u64(c, bsum);
    fsum = team_sum_f64(c, fsum);
    fabs_ = team_sum_f64(c, fabs_);
    R.vhash = ver % 999983ULL;
    R.bitsum = bsum;
    R.fsum = fsum;
    R.fabs = fabs_;
    R.work = (uint64_t)p.particles * (uint64_t)nL;
  }

  // (A)-(C) of the event-mode lookups for the chunk of lookups [c0, c0+nc):
  // lk_pe = their energies sorted into (material, energy) buckets, material
  // m's slots start at mcnt[16+m] (mcnt[28] = nc); material tallies counted
  __device__ static __forceinline__ void lookup_sort(Ctx &c, const XsParams &p, const XsLayout &L, const double *thr,
                                                     uint32_t *mcnt, long long c0, long long nc) {
    const int tid = threadIdx.x, T = blockDim.x;
    double *lk_pe = (double *)(c.arena + L.lk_pe);
    uint32_t *hist = (uint32_t *)(c.arena + L.lk_hist);
    const long long LC = xs_lk_chunk(p);
    const int kb = xs_lk_bits(LC);
    const long long NB = 12LL << kb;
    const double bscale = (double)(1LL << kb);
    const long long g0 = (long long)c.crank * T + tid, gs = (long long)c.csize * T;
    const Affine JG = lcg_pow(2ULL * (uint64_t)gs);
    for (long long b = g0; b <= NB; b += gs) hist[b] = 0u;
    team_sync(c);
    // (A) count
    {
      uint64_t s = lcg_pow(2ULL * (uint64_t)(c0 + g0))(p.seed);
      for (long long li = g0; li < nc; li += gs, s = JG(s)) {
        uint64_t t = s;
        const double pe = lcg_double(t);
        const int mat = pick_mat_thr(thr, lcg_double(t));
        long long eb = (long long)(pe * bscale);
        eb = eb > (1LL << kb) - 1 ? (1LL << kb) - 1 : eb;
        atomicAdd(&hist[((long long)mat << kb) + eb], 1u);
      }
    }
    team_sync(c);
    // (B) bucket offsets (one CTA), material starts to every CTA's smem
    if (c.crank == 0) global_exclusive_scan(hist, NB + 1, ens_sh(c));
    team_sync(c);
    if (tid < 12) mcnt[16 + tid] = ld_(hist + ((long long)tid << kb));
    if (tid == 12) mcnt[28] = (uint32_t)nc;
    team_sync(c);  // every CTA has its offsets before (C) moves the cursors
    if (c.crank == 0 && tid < 12) ens_sh(c)->tallies[5 + tid] += mcnt[17 + tid] - mcnt[16 + tid];  // per material
    // (C) scatter energies to their buckets (hist becomes bucket ends)
    {
      uint64_t s = lcg_pow(2ULL * (uint64_t)(c0 + g0))(p.seed);
      for (long long li = g0; li < nc; li += gs, s = JG(s)) {
        uint64_t t = s;
        const double pe = lcg_double(t);
        const int mat = pick_mat_thr(thr, lcg_double(t));
        long long eb = (long long)(pe * bscale);
        eb = eb > (1LL << kb) - 1 ? (1LL << kb) - 1 : eb;
        lk_pe[atomicAdd(&hist[((long long)mat << kb) + eb], 1u)] = pe;
      }
    }
    team_sync(c);
  }

  // ---- split phases, phase 1b: the lookup sort in items on any CTAs -------
  // The instance's one chunk (xs_split_ok: lookups <= kXsLkChunk) is sorted
  // into lookup_sort's (material, energy-bucket) order — the same buckets
  // (kb energy bits per material); only the order within a bucket (atomic
  // in either) may differ — in three kinds of items, all counting in shared
  // memory: (A) count item ch samples lookups [ch*kXsSortChunk, ...) (XS-6:
  // lookup li draws 2li+1, 2li+2) and writes its coarse histogram — coarse
  // bucket ck = (material, top cb energy bits) — as column ch of CH[ck][NC];
  // the CTA finishing the last count item scans CH (B: in (ck, ch) order
  // that gives each chunk's cursor into each coarse bucket) and writes the
  // descriptor; (C) scatter item ch re-samples its lookups and moves each
  // energy to its coarse bucket in lk_tmp; (D) fine item g sorts coarse
  // buckets [g*G, (g+1)*G) by the remaining kb - cb energy bits into lk_pe,
  // a warp per coarse bucket.  pick_mat: the first i >= 1 with roll <
  // thr[i] is 1 + #{i >= 1: thr[i] <= roll} (thr increasing), 0 past thr[11].
  struct LkKey {
    int kb, cb, fb, nck, nc;  // energy bits, coarse bits, fine bits, coarse buckets, chunks
  };
  __device__ static LkKey lk_key(const XsParams &p) {
    LkKey k;
    k.kb = xs_lk_bits(xs_lk_chunk(p));
    k.cb = xs_lk_cbits(k.kb);
    k.fb = k.kb - k.cb;
    k.nck = 12 << k.cb;
    k.nc = xs_sort_items(p);
    return k;
  }
  // lookups [l0, l1) of the chunk: fn(energy, coarse bucket) for each
  template <class F>
  __device__ static __forceinline__ void lk_sample(const XsParams &p, const LkKey &K, const double *thr, long long l0,
                                                   long long l1, const Affine &JT, F fn) {
    const int T = blockDim.x;
    const double bscale = (double)(1LL << K.kb);
    const long long emax = (1LL << K.kb) - 1;
    double th[11];
#pragma unroll
    for (int m = 0; m < 11; m++) th[m] = thr[m + 1];
    constexpr int U = 4;
    uint64_t s = lcg_pow(2ULL * (uint64_t)(l0 + threadIdx.x))(p.seed);
    for (long long li0 = l0 + threadIdx.x; li0 < l1; li0 += (long long)U * T) {
      double pe[U];
      uint32_t ck[U];
#pragma unroll
      for (int u = 0; u < U; u++) {
        uint64_t t = s;
        pe[u] = lcg_double(t);
        const double roll = lcg_double(t);
        int n = 0;
#pragma unroll
        for (int m = 0; m < 11; m++) n += roll >= th[m] ? 1 : 0;
        const int mat = n == 11 ? 0 : n + 1;
        long long eb = (long long)(pe[u] * bscale);
        eb = eb > emax ? emax : eb;
        ck[u] = ((uint32_t)mat << K.cb) + (uint32_t)(eb >> K.fb);
        s = JT(s);
      }
#pragma unroll
      for (int u = 0; u < U; u++)
        if (li0 + (long long)u * T < l1) fn(pe[u], ck[u]);
    }
  }
  // (A)
  __device__ static void lk_count(const Ctx &c, const XsParams &p, const XsLayout &L, const double *thr, int ch,
                                  const Affine &JT, uint32_t *sc) {
    const LkKey K = lk_key(p);
    const long long nc = xs_lk_chunk(p), l0 = (long long)ch * kXsSortChunk;
    const long long l1 = l0 + kXsSortChunk < nc ? l0 + kXsSortChunk : nc;
    for (int x = threadIdx.x; x < K.nck; x += blockDim.x) sc[x] = 0u;
    __syncthreads();
    lk_sample(p, K, thr, l0, l1, JT, [&](double, uint32_t ck) {
      ENS_CHECK(ck < (uint32_t)K.nck);
      atomicAdd(&sc[ck], 1u);
    });
    __syncthreads();
    uint32_t *CH = (uint32_t *)(c.arena + L.lk_hist);
    for (int x = threadIdx.x; x < K.nck; x += blockDim.x) CH[(size_t)x * K.nc + ch] = sc[x];
  }
  // (B): coarse-bucket cursors and the material starts mcnt[16..28] (one CTA)
  __device__ static void lk_scan(const Ctx &c, const XsParams &p, const XsLayout &L, uint32_t *mcnt) {
    const int tid = threadIdx.x;
    const LkKey K = lk_key(p);
    uint32_t *CH = (uint32_t *)(c.arena + L.lk_hist);
    global_exclusive_scan(CH, (long long)K.nck * K.nc, ens_sh(c));
    __syncthreads();
    // the last cursor plus the last chunk's last count is the chunk size (every lookup counted once)
    ENS_CHECK(ld_(CH + (size_t)K.nck * K.nc - 1) <= (uint32_t)xs_lk_chunk(p));
    if (tid < 12) mcnt[16 + tid] = ld_(CH + ((size_t)tid << K.cb) * K.nc);
    if (tid == 12) mcnt[28] = (uint32_t)xs_lk_chunk(p);
    __syncthreads();
  }
  // (C)
  __device__ static void lk_scatter(const Ctx &c, const XsParams &p, const XsLayout &L, const double *thr, int ch,
                                    const Affine &JT, uint32_t *sc) {
    const LkKey K = lk_key(p);
    const long long nc = xs_lk_chunk(p), l0 = (long long)ch * kXsSortChunk;
    const long long l1 = l0 + kXsSortChunk < nc ? l0 + kXsSortChunk : nc;
    const uint32_t *CH = (const uint32_t *)(c.arena + L.lk_hist);
    for (int x = threadIdx.x; x < K.nck; x += blockDim.x) sc[x] = __ldcg(CH + (size_t)x * K.nc + ch);
    __syncthreads();
    double *tmp = (double *)(c.arena + L.lk_tmp);
    lk_sample(p, K, thr, l0, l1, JT, [&](double pe, uint32_t ck) {
      const uint32_t pos = atomicAdd(&sc[ck], 1u);
      ENS_CHECK(ck < (uint32_t)K.nck && pos < (uint32_t)nc);
      tmp[pos] = pe;
    });
  }
  // (D)
  __device__ static void lk_fine(const Ctx &c, const XsParams &p, const XsLayout &L, int g, uint32_t *sc) {
    const LkKey K = lk_key(p);
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int nf = 1 << K.fb;
    uint32_t *cnt = sc + (size_t)w * nf;
    const uint32_t *CH = (const uint32_t *)(c.arena + L.lk_hist);
    const double *tmp = (const double *)(c.arena + L.lk_tmp);
    double *lk_pe = (double *)(c.arena + L.lk_pe);
    const long long n = xs_lk_chunk(p);
    const double bscale = (double)(1LL << K.kb);
    const long long emax = (1LL << K.kb) - 1;
    auto fine = [&](double pe) {
      long long eb = (long long)(pe * bscale);
      eb = eb > emax ? emax : eb;
      return (int)(eb & (nf - 1));
    };
    const int ck1 = (g + 1) * kXsFineGroup < K.nck ? (g + 1) * kXsFineGroup : K.nck;
    for (int ck = g * kXsFineGroup + w; ck < ck1; ck += nw) {
      const long long s0 = __ldcg(CH + (size_t)ck * K.nc);  // other CTAs' stores: L2
      const long long s1 = ck + 1 < K.nck ? (long long)__ldcg(CH + (size_t)(ck + 1) * K.nc) : n;
      ENS_CHECK(s0 <= s1 && s1 <= n);
      for (int f = lane; f < nf; f += 32) cnt[f] = 0u;
      __syncwarp();
      // buckets of <= 32 * kR energies (~325 on average at C2's size) are
      // loaded once, all loads in flight, and kept in registers; larger ones
      // (the frequent materials' buckets) are re-read in batches of 32 * kR
      constexpr int kR = 16;
      const bool inreg = s1 - s0 <= 32 * kR;
      double v[kR];
#pragma unroll
      for (int r = 0; r < kR; r++) {
        const long long i = s0 + lane + 32 * r;
        v[r] = inreg && i < s1 ? __ldcg(tmp + i) : 0.0;
      }
      if (inreg) {
#pragma unroll
        for (int r = 0; r < kR; r++)
          if (s0 + lane + 32 * r < s1) atomicAdd(&cnt[fine(v[r])], 1u);
      } else {
        for (long long b = s0; b < s1; b += 32 * kR) {
          double w[kR];
#pragma unroll
          for (int r = 0; r < kR; r++) {
            const long long i = b + lane + 32 * r;
            w[r] = i < s1 ? __ldcg(tmp + i) : 0.0;
          }
#pragma unroll
          for (int r = 0; r < kR; r++)
            if (b + lane + 32 * r < s1) atomicAdd(&cnt[fine(w[r])], 1u);
        }
      }
      __syncwarp();
      {  // exclusive scan of cnt[0, nf): lane l owns entries [l*per, (l+1)*per)
        const int per = nf >= 32 ? nf / 32 : 1;
        uint32_t loc = 0;
        for (int q = 0; q < per; q++) {
          const int f = lane * per + q;
          if (f < nf) loc += cnt[f];
        }
        uint32_t inc = loc;
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t t = __shfl_up_sync(0xffffffffu, inc, o);
          if (lane >= o) inc += t;
        }
        uint32_t run = inc - loc;
        for (int q = 0; q < per; q++) {
          const int f = lane * per + q;
          if (f < nf) {
            const uint32_t v = cnt[f];
            cnt[f] = run;
            run += v;
          }
        }
      }
      __syncwarp();
      if (inreg) {
#pragma unroll
        for (int r = 0; r < kR; r++)
          if (s0 + lane + 32 * r < s1) {
            const long long pos = s0 + atomicAdd(&cnt[fine(v[r])], 1u);
            ENS_CHECK(pos < s1);
            lk_pe[pos] = v[r];
          }
      } else {
        for (long long b = s0; b < s1; b += 32 * kR) {
          double w[kR];
#pragma unroll
          for (int r = 0; r < kR; r++) {
            const long long i = b + lane + 32 * r;
            w[r] = i < s1 ? __ldcg(tmp + i) : 0.0;
          }
#pragma unroll
          for (int r = 0; r < kR; r++)
            if (b + lane + 32 * r < s1) lk_pe[s0 + atomicAdd(&cnt[fine(w[r])], 1u)] = w[r];
        }
      }
      __syncwarp();
    }
  }

  // ---- XS-6..XS-10: lookups ----------------------------------------------
  // Per chunk of at most 2^22 lookups (XsLayout.lk_*): (A) every lookup is
  // sampled (XS-6, lookup li draws 2li+1, 2li+2) and counted into its
  // (material, energy) bucket; (B) one scan gives bucket offsets — material
  // m starts at bucket m << kb; (C) lookups are re-sampled and their
  // energies scattered to their bucket; (D) thread-per-slot over the sorted
  // chunk: a warp's lanes share a material (same nuclide list, no
  // divergence) and neighbouring energies (the same hash entries / record
  // pairs, so one L1 line serves many lanes), and each lane sums its
  // lookup's nuclides in list order (XS-9's order, bit-exact).  The order of
  // lookups within a bucket (atomic) only permutes the fsum / fabs terms.
  template <int GRID>
  __device__ static __forceinline__ void lookups(Ctx &c, const XsParams &p, const XsLayout &L, const double *thr,
                                              const int *nn, const double *concs, const uint16_t *mats,
                                              Result &R) {
    const bool trc = tracing(c);  // tracing (ENS_F_PHASES) thread, cached
    const int tid = threadIdx.x, T = blockDim.x;
    const int n_iso = p.n_iso;
    const long long n_u = (long long)n_iso * p.n_gp, nL = p.lookups;
    const double *recs = (const double *)(c.arena + L.recs);
    const int *ig = (const int *)(c.arena + L.index);
    const uint64_t *uA = (const uint64_t *)(c.arena + L.uenergy);
    const uint32_t *uf = (const uint32_t *)(c.arena + L.ufind);
    double *lk_pe = (double *)(c.arena + L.lk_pe);
    const long long UB = xs_ubins(p);
    const XsSmem S = xs_smem(p, T);
    uint32_t *mcnt = (uint32_t *)(ens_smem(c) + S.mcnt);  // [16..28] material offsets of the chunk
    const double du = 1.0 / p.bins;
    const long long LC = xs_lk_chunk(p);
    const long long g0 = (long long)c.crank * T + tid, gs = (long long)c.csize * T;
    unsigned long long ver = 0, bsum = 0;
    double fsum = 0.0, fabs_ = 0.0;
    for (long long c0 = 0; c0 < nL; c0 += LC) {
      const long long nc = nL - c0 < LC ? nL - c0 : LC;
      lookup_sort(c, p, L, thr, mcnt, c0, nc);
      phase_mark_if(trc, c, 10);
      // (D) thread-per-lookup over the sorted chunk
      double *const dmp = c.dump;
      const uint32_t drows = c.dump_rows;
      for (long long sl = g0; sl < nc; sl += gs) {
        int mat = 0;
#pragma unroll
        for (int m = 1; m < 12; m++) mat += (sl >= (long long)mcnt[16 + m]) ? 1 : 0;
        const double pe = ld_(lk_pe + sl);
        int idx = 0;
        if (GRID == XS_UNIONIZED) idx = union_idx(uf, uA, UB, n_u, pe);
        else if (GRID == XS_HASH) {
          const long long bb = (long long)(pe / du);
          idx = bb > p.bins - 1 ? p.bins - 1 : (int)bb;  // reading Q14
        }
        double mv[5];
        macro_lookup<GRID>(p, recs, ig, nn, concs, mats, pe, mat, idx, mv);
        const double m0 = mv[0], m1 = mv[1], m2 = mv[2], m3 = mv[3], m4 = mv[4];
        // XS-10
        double mxv = -1.0;
        int am = 0;
        if (m0 > mxv) { mxv = m0; am = 0; }
        if (m1 > mxv) { mxv = m1; am = 1; }
        if (m2 > mxv) { mxv = m2; am = 2; }
        if (m3 > mxv) { mxv = m3; am = 3; }
        if (m4 > mxv) { mxv = m4; am = 4; }
        ver += (unsigned long long)(am + 1);
        atomicAdd(&ens_sh(c)->tallies[am], 1u);
        if (dmp) dump_row(dmp, drows, c0 + sl, pe, mat, mv, 5, am);
        bsum += dbits(m0) + dbits(m1) + dbits(m2) + dbits(m3) + dbits(m4);
        fsum += m0; fsum += m1; fsum += m2; fsum += m3; fsum += m4;
        fabs_ += fabs(m0); fabs_ += fabs(m1); fabs_ += fabs(m2); fabs_ += fabs(m3); fabs_ += fabs(m4);
      }
      team_sync(c);  // lk_pe / hist reused by the next chunk
      phase_mark_if(trc, c, 11);
    }
    ver = team_sum_u64(c, ver);
    bsum = team_sum_u64(c, bsum);
    fsum = team_sum_f64(c, fsum);
    fabs_ = team_sum_f64(c, fabs_);
    R.vhash = ver % 999983ULL;
    R.bitsum = bsum;
    R.fsum = fsum;
    R.fabs = fabs_;
    R.work = (uint64_t)p.lookups;
  }

  // the hash lookups out of line: their register allocation is then their
  // own (measured: C2 45.5 -> 45.1 ms with TSTAR at 8.71 ms; making both out of line
  // costs TSTAR 2 %)
  __device__ static __noinline__ void lookups_hash(Ctx &c, const XsParams &p, const XsLayout &L, const double *thr,
                                                   const int *nn, const double *concs, const uint16_t *mats,
                                                   Result &R) {
    lookups<XS_HASH>(c, p, L, thr, nn, concs, mats, R);
  }

  __host__ static bool size(int argc, const char *const *argv, int T, int cs, uint64_t *arena, uint32_t *smem) {
    XsParams p;
    if (xs_parse(argc, argv, p) >= 0) {
      *arena = 0;
      *smem = 0;
      return false;
    }
    *arena = xs_layout(p, cs).total;
    *smem = xs_smem(p, T).total;
    return true;
  }
};

}  // namespace ens
