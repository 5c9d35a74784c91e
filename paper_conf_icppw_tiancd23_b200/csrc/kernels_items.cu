// csrc/kernels_items.cu — the split-phase item kernels: phase 1b (XS
// per-nuclide tables and lookup sorts) and phase 2 (XS and RS lookup items of
// every instance of an ensemble, on every SM).
//
// Phase 1 (the ensemble kernel, kernels.cu: one team per instance, the
// paper's mapping) builds each instance's tables and its (material,
// energy)-sorted lookup chunk in a per-instance arena slot and leaves an
// XsDesc.  This persistent kernel then pulls items — kXsItemLookups
// consecutive sorted slots of one instance — from one atomic queue, so the
// lookups of all instances are spread over all SMs whatever the instance
// count (C2: 64 instances on 148 SMs), and it runs with its own register
// budget (the lookups alone, not the init code: more resident warps to hide
// the dependent gathers).  Each lookup is XS-7..XS-10 exactly as the fused
// body computes it (XsApp::macro_lookup, bit-identical); an item's integer
// sums and argmax counts and its fsum / fabs partials go to its own
// XsItemPart, and the CTA that finishes an instance's last item sums the
// parts in item order, writes the record, the tallies and the
// stdout lines (XS-11), exactly what the fused body writes.
#include <cuda_runtime.h>

// phase 2's hash lookups gather one nuclide per step: with the register
// budget of 3 CTAs/SM that beats two (measured: C2 38.8 vs 39.9 ms)
#ifndef ENS_XS_STEP
#define ENS_XS_STEP 1
#endif
#include "apps/rsbench.cuh"
#include "apps/xsbench.cuh"
#include "kparams.h"

namespace ens {

#ifndef ENS_XS2_T
#define ENS_XS2_T 256
#endif
// resident CTAs per SM (register budget 65536 / (T * minB)) per grid type:
// one kernel per grid type, so each carries only its own lookup's registers
#ifndef ENS_XS2_MINB_HASH
#define ENS_XS2_MINB_HASH 3
#endif
#ifndef ENS_XS2_MINB_UNI
#define ENS_XS2_MINB_UNI 2
#endif
#ifndef ENS_XS2_MINB_NUC
#define ENS_XS2_MINB_NUC 2
#endif
// threads per CTA of the XS lookup-item kernel per grid type (ENS_XS2_T_HASH: hash grids)
#ifndef ENS_XS2_T_HASH
#define ENS_XS2_T_HASH 256
#endif
template <int GRID>
struct Xs2T {
  static constexpr int v = GRID == XS_HASH ? ENS_XS2_T_HASH : ENS_XS2_T;
};
template <int GRID>
struct Xs2Minb {
  static constexpr int v = GRID == XS_HASH ? ENS_XS2_MINB_HASH : GRID == XS_UNIONIZED ? ENS_XS2_MINB_UNI : ENS_XS2_MINB_NUC;
};
constexpr int kXs2T = ENS_XS2_T;
constexpr uint32_t kXs2Sh = (sizeof(Shared) + 15) / 16 * 16;
// dynamic shared memory: Shared | XsDesc | thr[12] | nn[16] | concs | mats | scratch
constexpr uint32_t kXs2Desc = kXs2Sh;
constexpr uint32_t kXs2Thr = kXs2Desc + (sizeof(XsDesc) + 15) / 16 * 16;
constexpr uint32_t kXs2Nn = kXs2Thr + 12 * 8;
// hash grids: material rows padded by kXs2RowPad copies of their first
// nuclide, so the lookup's look-ahead loads need no bounds tests
constexpr int kXs2RowPad = 4;
constexpr uint32_t kXs2Concs = kXs2Nn + 16 * 4;
constexpr uint32_t kXs2Mats = kXs2Concs + 12 * (321 + kXs2RowPad) * 8;
constexpr uint32_t kXs2Misc = kXs2Mats + (12 * (321 + kXs2RowPad) * 2 + 15) / 16 * 16;  // u32: item, last, am[5], pos(2)
constexpr uint32_t kXs2Smem = kXs2Misc + 16 * 4;

// 32-bit shared-window loads (the material row's address is computed once
// per lookup; each step's loads then take immediate offsets)
__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
  unsigned short v;
  asm("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ double lds_f64(uint32_t a) {
  double v;
  asm("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
  return v;
}

// Phase 2's hash-grid lookup: XS-7..XS-9 for one lookup, bit-identical to
// XsApp::macro_lookup<XS_HASH> (the same bracket guess, verification, walk /
// upstream fallback and accumulate(), nuclides summed in list order), one
// nuclide per step: entry j+2 loaded and entry j+4 prefetched into L1,
// nuclide j+1's guess and pair address computed and its pair prefetched,
// nuclide j's pair gathered, verified and accumulated.  The material row
// (mrow_s / crow_s: shared-window addresses) has kXs2RowPad padding entries
// (valid nuclides), so the look-ahead needs no bounds tests; entry and
// record indices are 32-bit sums (n_iso * (bins + 1) and n_iso * n_gp * 6
// stay below 2^32).  A nuclide's entry is consumed when its guess is made
// (its u_low / u_high travel with the pair).  The tables were written by an
// earlier kernel: read-only loads (ldro).
// Block shape and register budget (C2's phase 2, measured): 256 threads x 3
// CTAs at 80 registers (24 warps) 19.5 ms; 352 x 2 at 88 (22 warps, no
// spills) 21.4; 320 x 2 (20 warps) 24.2; 192 x 4 21.1; 256 x 4 at 64
// (spills) 21.8; 128 x 6 22.2; the pair's last 64 bytes loaded only when
// needed (fewer registers) 22.1 (x3) / 21.5 (x4): latency exposed.
// L1 prefetches (measured on C2's phase 2: all on 19.5 ms; no entry
// prefetch 21.9, one pair line 20.5, no pair prefetch 22.1; pairs prefetched
// two steps ahead instead of one 19.9)
#ifndef ENS_XS2_PF_ENT
#define ENS_XS2_PF_ENT 1
#endif
#ifndef ENS_XS2_PF_PAIR
#define ENS_XS2_PF_PAIR 2
#endif
struct Xs2Pair {
  const double2 *q;  // the guessed pair
  int lo;            // its lower index
  uint32_t rb;       // the nuclide's first record
  uint32_t hx;       // its entry's u_low | u_high << 16
};
__device__ __forceinline__ void xs2_hash_lookup(uint32_t mrow_s, uint32_t crow_s, int nm, const double *recs,
                                                const XsHashEnt *ig, int bins, int n_gp, double pe, int idx,
                                                double *m) {
  const uint32_t hs32 = (uint32_t)bins + 1u;
  auto ent = [&](int j) {
    return reinterpret_cast<const uint4 *>(ig + ((uint32_t)idx + lds_u16(mrow_s + 2u * (uint32_t)j) * hs32));
  };
  const int pq = (int)((pe * (double)bins - (double)idx) * 65536.0);
  const uint32_t pq15 = (uint32_t)(pq < 0 ? 0 : (pq >> 1 > 32767 ? 32767 : pq >> 1));
  const uint32_t P = (pq15 | (pq15 << 16) | 0x80008000u) - 0x00010001u;
  auto guess = [&](const uint4 &h) {  // #{k: pq15 > q_k} over the six 15-bit quanta (XsApp::macro_lookup)
    const uint32_t mk = 0x80008000u;
    const uint32_t x = ((P - h.y) & mk) | (((P - h.z) & mk) >> 1) | (((P - h.w) & mk) >> 2);
    const int lo = (int)(h.x & 0xffffu) + __popc(x);
    const int uh = (int)(h.x >> 16);
    return lo < uh - 1 ? lo : uh - 1;
  };
  auto pair_of = [&](int j, const uint4 &h, Xs2Pair &o) {
    o.rb = lds_u16(mrow_s + 2u * (uint32_t)j) * (uint32_t)n_gp;
    o.lo = guess(h);
    ENS_CHECK(o.lo >= 0 && o.lo + 1 < n_gp);
    o.hx = h.x;
    o.q = reinterpret_cast<const double2 *>(recs + (o.rb + (uint32_t)o.lo) * 6u);
  };
  double m0 = 0.0, m1 = 0.0, m2 = 0.0, m3 = 0.0, m4 = 0.0;
  // nuclide j: gather its guessed pair pA, verify it (walk / search
  // otherwise) and accumulate
  auto gather_acc = [&](int j, const Xs2Pair &pA) {
    double2 a0 = ldro(pA.q + 0), a1 = ldro(pA.q + 1), a2 = ldro(pA.q + 2);
    double2 b0 = ldro(pA.q + 3), b1 = ldro(pA.q + 4), b2 = ldro(pA.q + 5);
    const int uh = (int)(pA.hx >> 16);
    // the guessed pair is upstream's bracket iff E[lo] < pe < E[lo+1] and
    // lo+1 <= u_high; else walk / search (macro_lookup's gather_fix; the
    // walk's own test fails at once on a valid bracket, so skipping both is
    // the same logic)
    if (!(a0.x < pe && pe < b0.x && pA.lo + 1 <= uh)) {
      const double *E = recs + pA.rb * 6u;  // the nuclide's records
      const int u_low = (int)(pA.hx & 0xffffu);
      int lo = pA.lo;
      while (pe >= b0.x && a0.x < pe && lo + 2 <= uh) {
        lo++;
        const double2 *w2 = reinterpret_cast<const double2 *>(E + 6 * (size_t)lo);
        a0 = b0; a1 = b1; a2 = b2;
        b0 = ldro(w2 + 3); b1 = ldro(w2 + 4); b2 = ldro(w2 + 5);
      }
      if (!(a0.x < pe && pe < b0.x && lo + 1 <= uh)) {
        const double e_low = ldro(E + 6 * (size_t)u_low);
        const double e_high = ldro(E + 6 * (size_t)uh);
        int lower;
        if (pe <= e_low) lower = 0;
        else if (pe >= e_high) lower = n_gp - 1;
        else lower = gs_recs(E, pe, u_low, uh);
        const int l2 = lower == n_gp - 1 ? lower - 1 : lower;
        const double2 *w2 = reinterpret_cast<const double2 *>(E + 6 * (size_t)l2);
        a0 = ldro(w2 + 0); a1 = ldro(w2 + 1); a2 = ldro(w2 + 2);
        b0 = ldro(w2 + 3); b1 = ldro(w2 + 4); b2 = ldro(w2 + 5);
      }
    }
    XsApp::accumulate(pe, lds_f64(crow_s + 8u * (uint32_t)j), a0, a1, a2, b0, b1, b2, m0, m1, m2, m3, m4);
  };
  // step j: hB = entry j+1, hC <- entry j+2; pA = nuclide j's pair, pB <- nuclide j+1's
  auto step = [&](int j, const uint4 &hB, uint4 &hC, const Xs2Pair &pA, Xs2Pair &pB) {
    hC = ldro(ent(j + 2));
    if (ENS_XS2_PF_ENT) prefetch_l1(ent(j + 4));
    pair_of(j + 1, hB, pB);
    if (ENS_XS2_PF_PAIR >= 1) prefetch_l1(pB.q);
    if (ENS_XS2_PF_PAIR >= 2) prefetch_l1(reinterpret_cast<const double *>(pB.q) + 11);
    gather_acc(j, pA);
  };
  uint4 h0 = ldro(ent(0)), h1 = ldro(ent(1));
  prefetch_l1(ent(2));
  prefetch_l1(ent(3));
  Xs2Pair p0, p1;
  pair_of(0, h0, p0);  // entry 0 consumed: h0 is free
  int j = 0;
  for (; j < nm; j++) {  // (unrolled by two without copies: spills at 80 registers, 21.8 vs 19.5 ms)
    step(j, h1, h0, p0, p1);
    h1 = h0;
    p0 = p1;
  }
  m[0] = m0;
  m[1] = m1;
  m[2] = m2;
  m[3] = m3;
  m[4] = m4;
}

template <int GRID>
__device__ __forceinline__ void xs2_item(const XsDesc &d, const XsParams &p, long long s0, long long s1,
                                         const int *nn, const double *concs, const uint16_t *mats, uint32_t *am,
                                         double *dmp, uint32_t drows, unsigned long long &ver,
                                         unsigned long long &bsum, double &fsum, double &fabs_) {
  const double *recs = (const double *)d.recs;
  const int *ig = (const int *)d.index;
  const uint64_t *uA = (const uint64_t *)d.uenergy;
  const uint32_t *uf = (const uint32_t *)d.ufind;
  const double *lk_pe = (const double *)d.lk_pe;
  const long long n_u = (long long)p.n_iso * p.n_gp, UB = d.ubins;
  const double du = 1.0 / p.bins;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(ens_dsmem);  // the shared window base, once
  for (long long sl = s0 + threadIdx.x; sl < s1; sl += Xs2T<GRID>::v) {
    int mat = 0;
#pragma unroll
    for (int m = 1; m < 12; m++) mat += (sl >= (long long)d.mcnt[m]) ? 1 : 0;
    const double pe = ldro(lk_pe + sl);  // read-only here: phase 1 wrote it
    int idx = 0;
    if (GRID == XS_UNIONIZED) idx = XsApp::union_idx(uf, uA, UB, n_u, pe);
    else if (GRID == XS_HASH) {
      const long long bb = (long long)(pe / du);
      idx = bb > p.bins - 1 ? p.bins - 1 : (int)bb;  // reading Q14
    }
    double mv[5];
    if (GRID == XS_HASH) {
      const int rw = xs_max_nucs(p.n_iso) + kXs2RowPad;
      xs2_hash_lookup(sbase + kXs2Mats + 2u * (uint32_t)(mat * rw), sbase + kXs2Concs + 8u * (uint32_t)(mat * rw),
                      nn[mat], recs,
                      reinterpret_cast<const XsHashEnt *>(ig), p.bins, p.n_gp, pe, idx, mv);
    } else {
      XsApp::macro_lookup<GRID>(p, recs, ig, nn, concs, mats, pe, mat, idx, mv);
    }
    const double m0 = mv[0], m1 = mv[1], m2 = mv[2], m3 = mv[3], m4 = mv[4];
    double mxv = -1.0;  // XS-10
    int a = 0;
    if (m0 > mxv) { mxv = m0; a = 0; }
    if (m1 > mxv) { mxv = m1; a = 1; }
    if (m2 > mxv) { mxv = m2; a = 2; }
    if (m3 > mxv) { mxv = m3; a = 3; }
    if (m4 > mxv) { mxv = m4; a = 4; }
    ver += (unsigned long long)(a + 1);
    atomicAdd(&am[a], 1u);
    if (dmp) dump_row(dmp, drows, sl, pe, mat, mv, 5, a);
    bsum += dbits(m0) + dbits(m1) + dbits(m2) + dbits(m3) + dbits(m4);
    fsum += m0; fsum += m1; fsum += m2; fsum += m3; fsum += m4;
    fabs_ += fabs(m0); fabs_ += fabs(m1); fabs_ += fabs(m2); fabs_ += fabs(m3); fabs_ += fabs(m4);
  }
}

__device__ __forceinline__ unsigned long long xs2_gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// the CTA that finished an instance's last item: XS-10's sums over its items
// (in item order: deterministic), XS-11's stdout, the record and the tallies;
// out of line (once per instance) so the lookup loop keeps its registers
__device__ __noinline__ void xs2_finish(const KParams &p, Ctx &c, const XsDesc *d, uint32_t *misc) {
  const int tid = threadIdx.x;
  Shared *sh = ens_sh(c);
  const uint32_t k = d->k;
  c.out = p.stdout_base + (size_t)k * p.stdout_cap;
  if (tid == 0) {
    __threadfence();
    unsigned long long tv = 0, tb = 0;
    double tf = 0.0, ta = 0.0;
    uint32_t tam[5] = {0, 0, 0, 0, 0};
    for (uint32_t it = d->item0; it < d->item0 + d->n_items; it++) {
      const XsItemPart *ip = reinterpret_cast<const XsItemPart *>(p.ipart + (size_t)it * kPartBytes);
      tv += __ldcg(&ip->ver);
      tb += __ldcg(&ip->bsum);
      tf += __ldcg(&ip->fsum);
      ta += __ldcg(&ip->fabs);
      for (int a = 0; a < 5; a++) tam[a] += __ldcg(&ip->am[a]);
    }
    sh->out_len = 0;
    sh->flags = 0;
    const int n_iso = d->n_iso;
    const long long lookups = (long long)d->lookups;
    const unsigned long long vhash = tv % 999983ULL;
    const char *grid = d->grid == XS_UNIONIZED ? "unionized" : d->grid == XS_NUCLIDE ? "nuclide" : "hash";
    ens_printf(c, FMT_XS_HDR, n_iso == 68 ? "small" : "large", n_iso, (long long)d->n_gp, grid, lookups,
               (unsigned long long)d->seed);
    ens_printf(c, FMT_VERIFY, vhash);
    uint32_t *tal = p.tallies + (size_t)k * ENS_TALLIES;
    for (int t = 0; t < ENS_TALLIES; t++)
      tal[t] = t < 5 ? tam[t] : (t < 17 ? d->mcnt[t - 4] - d->mcnt[t - 5] : 0u);
    ens_record rec;
    rec.instance = d->line;
    rec.exit_code = 0;
    rec.app = APP_XSBENCH;
    rec.flags = sh->flags | ENS_RF_DONE;
    rec.vhash = vhash;
    rec.bitsum = tb;
    rec.fsum = tf;
    rec.fabs = ta;
    rec.work = (uint64_t)lookups;
    rec.stdout_len = sh->out_len;
    uint32_t sm = 0;
    if (p.flags & ENS_F_TIMESTAMPS) asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    rec.smid = sm;
    rec.t_start_ns = d->t_start;
    rec.t_end_ns = (p.flags & ENS_F_TIMESTAMPS) ? xs2_gtimer() : 0ull;
    p.recs[k] = rec;
    const unsigned long long pos = atomicAdd(p.stdout_total, (unsigned long long)sh->out_len);
    p.stdout_pos[k] = pos;
    reinterpret_cast<unsigned long long *>(misc + 8)[0] = pos;
  }
  __syncthreads();
  // compact the instance's stdout (whole 8-B words)
  const unsigned long long pos = reinterpret_cast<const unsigned long long *>(misc + 8)[0];
  const unsigned long long *src = reinterpret_cast<const unsigned long long *>(c.out);
  unsigned long long *dst = reinterpret_cast<unsigned long long *>(p.stdout_cmp + pos);
  for (uint32_t w = tid; w < sh->out_len / 8; w += blockDim.x) dst[w] = src[w];
}


// items [p.item_base, p.item_base + p.n_items) of the group's queue, all of grid type GRID
template <int GRID>
__global__ void __launch_bounds__(Xs2T<GRID>::v, Xs2Minb<GRID>::v) xs_items_kernel(const KParams p) {
  constexpr int T = Xs2T<GRID>::v;
  const int tid = threadIdx.x;
  Ctx c{};
  c.sh_off = 0;
  c.smem_off = kXs2Desc;
  c.csize = 1;
  c.flags = p.flags;
  c.out_cap = p.stdout_cap;
  Shared *sh = ens_sh(c);
  XsDesc *d = reinterpret_cast<XsDesc *>(ens_dsmem + kXs2Desc);
  double *thr = reinterpret_cast<double *>(ens_dsmem + kXs2Thr);
  int *nn = reinterpret_cast<int *>(ens_dsmem + kXs2Nn);
  double *concs = reinterpret_cast<double *>(ens_dsmem + kXs2Concs);
  uint16_t *mats = reinterpret_cast<uint16_t *>(ens_dsmem + kXs2Mats);
  uint32_t *misc = reinterpret_cast<uint32_t *>(ens_dsmem + kXs2Misc);
  uint32_t *am = misc + 2;
  int cached = 0;  // n_iso of the material tables in shared memory
  for (;;) {
    if (tid == 0) misc[0] = atomicAdd(p.counter2, 1u);
    if (tid < 5) am[tid] = 0u;
    __syncthreads();
    if (misc[0] >= p.n_items) break;
    const uint32_t item = p.item_base + misc[0];
    const uint32_t j = p.items[item];
    {  // the instance's descriptor (phase 1's stores, an earlier kernel)
      const unsigned long long *src = reinterpret_cast<const unsigned long long *>(p.xs_desc + (size_t)j * kDescBytes);
      unsigned long long *dst = reinterpret_cast<unsigned long long *>(d);
      for (int w = tid; w < (int)(sizeof(XsDesc) / 8); w += T) dst[w] = src[w];
    }
    __syncthreads();
    const int n_iso = d->n_iso, mx = xs_max_nucs(n_iso);
    if (n_iso != cached) {  // XS-2 tables (constant per n_iso: CONC_SEED is fixed)
      if (GRID == XS_HASH) {  // rows of mx + kXs2RowPad, the padding = the row's first nuclide
        const int rw = mx + kXs2RowPad;
        if (tid < 12) {
          nn[tid] = hm_num_nucs(n_iso, tid);
          thr[tid] = hm_threshold(tid);
        }
        for (int x = tid; x < 12 * rw; x += T) {
          const int m = x / rw, jj = x % rw, nm = hm_num_nucs(n_iso, m);
          const int jn = jj < nm ? jj : 0;
          mats[x] = (uint16_t)hm_nuc(m, jn);
          uint64_t s = lcg_pow((uint64_t)hm_draw(n_iso, m, jn))(1070ULL * 1070ULL);  // hm_concs' draw
          concs[x] = lcg_double(s);
        }
      } else {
        hm_tables(n_iso, mx, thr, nn, concs, mats);
        __syncthreads();
        hm_concs(n_iso, mx, concs, 1070ULL * 1070ULL);
      }
      cached = n_iso;
      __syncthreads();
    }
    XsParams xp;
    xp.n_iso = n_iso;
    xp.n_gp = d->n_gp;
    xp.grid = d->grid;
    xp.bins = d->bins;
    xp.lookups = (long long)d->lookups;
    const long long s0 = (long long)(item - d->item0) * kXsItemLookups;
    const long long s1 = s0 + kXsItemLookups < xp.lookups ? s0 + kXsItemLookups : xp.lookups;
    double *dmp = p.dump ? p.dump + (size_t)d->k * p.dump_rows * 8 : nullptr;
    unsigned long long ver = 0, bsum = 0;
    double fsum = 0.0, fabs_ = 0.0;
    xs2_item<GRID>(*d, xp, s0, s1, nn, concs, mats, am, dmp, p.dump_rows, ver, bsum, fsum, fabs_);
    ver = block_sum_u64(sh, ver);
    bsum = block_sum_u64(sh, bsum);
    fsum = block_sum_f64(sh, fsum);
    fabs_ = block_sum_f64(sh, fabs_);
    if (tid == 0) {
      XsItemPart *ip = reinterpret_cast<XsItemPart *>(p.ipart + (size_t)item * kPartBytes);
      ip->ver = ver;
      ip->bsum = bsum;
      ip->fsum = fsum;
      ip->fabs = fabs_;
      for (int a = 0; a < 5; a++) ip->am[a] = am[a];
      __threadfence();
      misc[1] = atomicAdd(&p.idone[j], 1u) == d->n_items - 1 ? 1u : 0u;
    }
    __syncthreads();
    if (misc[1]) xs2_finish(p, c, d, misc);
    __syncthreads();  // misc, desc, am reused by the next item
  }
}

// ---- split phases, phase 1b: the per-nuclide tables of hash / nuclide
// instances (XS-3..XS-5: sort, records, hash column), one (instance,
// nuclide) item at a time, on every SM, beside the ensemble kernel (which
// meanwhile samples and sorts each instance's lookups).  Each item re-reads
// its instance's command line (the same XsParams the instance parses) and
// runs XsApp::init_nuc_range for that one nuclide with this CTA's scratch.
constexpr uint32_t kXsInitArgv = kXs2Sh;                                  // char *argv[ENS_MAX_ARGC + 1]
constexpr uint32_t kXsInitMisc = kXsInitArgv + (ENS_MAX_ARGC + 2) * 8;    // u32 item
constexpr uint32_t kXsInitApp = kXsInitMisc + 64;                          // the app's shared memory

// Per instance: count items, the scan (by the CTA finishing the last count
// item, which also writes the descriptor), scatter items, fine items
// (XsApp::lk_count / lk_scan / lk_scatter / lk_fine: the lookup sort in
// items); per (instance, nuclide) a nuclide item building that nuclide's
// sorted records and hash / nuclide grid column.  The host orders the queue
// count items, a share of the nuclide items, scatter items, another share,
// fine items, the rest: an item that waits (scatter on the scan, fine on
// every scatter item of its instance) only waits for items pulled before
// it, by running CTAs (no deadlock), and in practice finds them done.  Two
// CTAs of 256 threads per SM (compact shared memory: no material tables), so
// one CTA's barrier-separated phases overlap the other's.
struct XsInitSync {            // per instance, zeroed before the launch
  uint32_t fdone;              // scatter items finished
  uint32_t cdone;              // count items finished
  uint32_t sdone;              // coarse histogram scanned, descriptor written
  uint32_t pstate;             // parsed command line: 0 none, 1 being written, 2 ready
  uint32_t pad[4];
  XsParams p;                  // the instance's parsed command line (pstate == 2)
};
static_assert(sizeof(XsInitSync) <= kInitSyncBytes, "XsInitSync");

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t *f) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(f) : "memory");
  return v;
}
// the whole CTA waits until *f >= v (thread 0 acquires, the barrier orders the rest)
__device__ __forceinline__ void cta_wait_flag(const uint32_t *f, uint32_t v = 1u) {
  if (threadIdx.x == 0)
    while (ld_acquire_u32(f) < v) __nanosleep(256);
  __syncthreads();
}
// after a __syncthreads(): publish the CTA's global writes and set *f = v
__device__ __forceinline__ void cta_set_flag(uint32_t *f, uint32_t v) {
  if (threadIdx.x == 0) {
    __threadfence();
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(f), "r"(v) : "memory");
  }
}

__global__ void __launch_bounds__(kXsInitThreads, 2) xs_init_items_kernel(const KParams p) {
  const int tid = threadIdx.x, T = blockDim.x;
  Ctx c{};
  c.sh_off = 0;
  c.smem_off = kXsInitApp;
  c.csize = 1;
  c.flags = p.flags;
  c.phases = p.phases;  // tracing (ENS_F_PHASES): 1..9 init_nuc_t's phases; sort items: 12 count, 13 scan,
                        // 14 scatter, 11 fine, 15 waiting
  char **argv = reinterpret_cast<char **>(ens_dsmem + kXsInitArgv);
  uint32_t *misc = reinterpret_cast<uint32_t *>(ens_dsmem + kXsInitMisc);
  char *scr = p.init_scr + (size_t)blockIdx.x * p.init_scr_bytes;
  bool jt_ok = false;   // the LCG jump tables (seed- and layout-independent: S.jmp is fixed)
  bool thr_ok = false;  // pick_mat thresholds (constant)
  const Affine JT = lcg_pow(2ULL * (uint64_t)T);  // T lookups' draws
  uint32_t cached_j = 0xffffffffu;  // the instance whose command line xp holds (and its layouts)
  XsParams xp;
  XsSmem xS{};
  XsLayout xL{};
  for (;;) {
    if (tid == 0) misc[0] = atomicAdd(p.counter3, 1u);
    __syncthreads();
    const uint32_t it = misc[0];
    if (it >= p.n_init_items) break;
    const uint32_t j = p.init_items[2 * it], i = p.init_items[2 * it + 1];
    phase_mark(c, -1);
    const uint32_t k = p.kmap[j], line = p.line_of_k[k];
    XsInitSync *sy = reinterpret_cast<XsInitSync *>(p.init_sync + (size_t)j * kInitSyncBytes);
    if (j != cached_j) {  // the command line: parsed once per instance, by whichever CTA comes first
      if (tid == 0) misc[1] = ld_acquire_u32(&sy->pstate);
      __syncthreads();
      if (misc[1] == 2u) {
        xp = sy->p;
      } else {
        const uint32_t t0 = p.line_tok[line];
        const int argc = (int)(p.line_tok[line + 1] - t0);
        for (int a = tid; a < argc; a += T) argv[a] = const_cast<char *>(p.blob) + p.tok_off[t0 + a];
        if (tid == 0) argv[argc] = nullptr;
        __syncthreads();
        xp = XsParams();
        xs_parse(argc, argv, xp);  // a valid line: the host made items only for those
        if (tid == 0 && atomicCAS(&sy->pstate, 0u, 1u) == 0u) {
          sy->p = xp;
          __threadfence();
          asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(&sy->pstate), "r"(2u) : "memory");
        }
      }
      cached_j = j;
      xS = xs_init_smem(xp);
      xL = xs_layout(xp, (int)p.team_ctas);  // the instance's arena, as phase 1 lays it out
    }
    phase_mark(c, 0);
    const XsSmem &S = xS;
    const XsLayout &L = xL;
    c.arena = p.arena_base + (size_t)j * p.arena_bytes;
    if (i >= kXsFineItem) {  // the lookup sort's items
      double *thr = reinterpret_cast<double *>(ens_smem(c) + S.thr);
      uint32_t *sc = reinterpret_cast<uint32_t *>(ens_smem(c) + S.nkey);  // kXsLkSortSmem bytes
      if (!thr_ok) {
        if (tid < 12) thr[tid] = hm_threshold(tid);
        thr_ok = true;
        __syncthreads();
      }
      const int q = (int)(i & 0x1fffffffu);
      if (i & kXsCountItem) {
        XsApp::lk_count(c, xp, L, thr, q, JT, sc);
        __syncthreads();
        phase_mark(c, 12);
        if (tid == 0) {
          __threadfence();
          misc[1] = atomicAdd(&sy->cdone, 1u) == (uint32_t)xs_sort_items(xp) - 1u ? 1u : 0u;
          __threadfence();
        }
        __syncthreads();
        if (misc[1]) {  // the last count item: (B) and the descriptor
          uint32_t *mcnt = reinterpret_cast<uint32_t *>(ens_smem(c) + S.mcnt);
          XsApp::lk_scan(c, xp, L, mcnt);
          if (tid == 0) {
            c.desc = p.xs_desc + (size_t)j * kDescBytes;
            c.k = k;
            c.id = line;
            c.t_start = 0;
            XsApp::write_desc(c, xp, L, mcnt);
          }
          __syncthreads();
          cta_set_flag(&sy->sdone, 1u);
          phase_mark(c, 13);
        }
      } else if (i & kXsScatterItem) {
        cta_wait_flag(&sy->sdone);
        phase_mark(c, 15);
        XsApp::lk_scatter(c, xp, L, thr, q, JT, sc);
        __syncthreads();
        if (tid == 0) {
          __threadfence();
          atomicAdd(&sy->fdone, 1u);
        }
        phase_mark(c, 14);
      } else {
        cta_wait_flag(&sy->fdone, (uint32_t)xs_sort_items(xp));
        phase_mark(c, 15);
        XsApp::lk_fine(c, xp, L, q, sc);
        phase_mark(c, 11);
      }
    } else {
      if (!jt_ok) {
        Affine *jt = reinterpret_cast<Affine *>(ens_smem(c) + S.jmp);
        for (int x = tid; x < 320; x += T) jt[x] = lcg_pow((6ULL * (uint64_t)(x & 63)) << (6 * (x >> 6)));
        jt_ok = true;
        __syncthreads();
      }
      const uint64_t e8 = align_up((uint64_t)xp.n_gp * 8, 256), c4 = align_up((uint64_t)(xp.bins + 1) * 4, 256);
      XsApp::init_nuc_range(c, xp, L, S, (int)i, (int)i + 1, 1, scr, scr + e8, scr + e8 + c4);
    }
    __syncthreads();  // argv, misc, scratch reused by the next item
  }
}

uint32_t xs_init_smem_off() { return kXsInitApp; }

cudaError_t xs_init_items_occupancy(int threads, size_t smem, int *ctas) {
  const void *fn = (const void *)xs_init_items_kernel;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int per_sm = 0, dev = 0, sms = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, threads, smem);
  if (e == cudaSuccess) e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  *ctas = per_sm * sms;
  return e;
}

cudaError_t launch_xs_init_items(int ctas, int threads, size_t smem, const KParams &p, cudaStream_t st) {
  const void *fn = (const void *)xs_init_items_kernel;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  void *args[] = {const_cast<KParams *>(&p)};
  return cudaLaunchKernel(fn, dim3((unsigned)ctas), dim3((unsigned)threads), args, smem, st);
}


// TMA bulk copy global -> this CTA's shared memory, completing on mbarrier
// `mbar` (16-B aligned addresses, size a multiple of 16; one thread)
__device__ __forceinline__ void bulk_g2s(void *sdst, const void *gsrc, uint32_t bytes, uint32_t mbar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          (uint32_t)__cvta_generic_to_shared(sdst)),
      "l"(gsrc), "r"(bytes), "r"(mbar)
      : "memory");
}
// every thread waits for the mbarrier's phase `parity` to complete
__device__ __forceinline__ void mbar_wait(uint32_t mbar, uint32_t parity) {
  uint32_t done = 0;
  while (!done)
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                 : "=r"(done)
                 : "r"(mbar), "r"(parity)
                 : "memory");
}

// ---- split phases, phase 2 of RSBench-style instances (kind 3) ----------
constexpr int kRs2T = 256;  // threads per CTA
// Items of kRsItemLookups sorted lookups of one instance; per item the
// instance's pole / window offsets and concentrations (phase 1 copied them
// to its arena) are staged in shared memory and every lookup is RsApp::lookup
// (RS-3, bit-identical to the fused body).  The last item's CTA writes the
// record, tallies (argmax, materials, pole-term counters) and stdout.
// (Measured and reverted: warp-granular items — each warp pulling its own
// 64 / 256 / 1024 lookups, no CTA barrier per item, offsets and
// concentrations read from the arena — C3 phase 2 14.1 / 17.3 / 36.6 ms
// against 14.0 ms with CTA items of 512.)
constexpr uint32_t kRsDesc = kXs2Sh;
constexpr uint32_t kRsThr = kRsDesc + (kDescBytes + 15) / 16 * 16;
constexpr uint32_t kRsNn = kRsThr + 12 * 8;
constexpr uint32_t kRsConcs = kRsNn + 16 * 4;
constexpr uint32_t kRsMats = kRsConcs + 12 * 321 * 8;
constexpr uint32_t kRsOff = kRsMats + (12 * 321 * 2 + 15) / 16 * 16;  // poff, woff: 2 x [356] int
constexpr uint32_t kRsMisc = kRsOff + 2 * 356 * 4;
constexpr uint32_t kRsSmem = kRsMisc + 16 * 4;
#ifndef ENS_RS2_MINB
#define ENS_RS2_MINB 2
#endif

__device__ __noinline__ void rs2_finish(const KParams &p, Ctx &c, const RsDesc *d, uint32_t *misc) {
  const int tid = threadIdx.x;
  Shared *sh = ens_sh(c);
  const uint32_t k = d->k;
  c.out = p.stdout_base + (size_t)k * p.stdout_cap;
  if (tid == 0) {
    __threadfence();
    unsigned long long tv = 0, tb = 0, tt = 0, tn = 0;
    double tf = 0.0, ta = 0.0;
    uint32_t tam[4] = {0, 0, 0, 0};
    for (uint32_t it = d->item0; it < d->item0 + d->n_items; it++) {
      const RsItemPart *ip = reinterpret_cast<const RsItemPart *>(p.ipart + (size_t)it * kPartBytes);
      tv += __ldcg(&ip->ver);
      tb += __ldcg(&ip->bsum);
      tt += __ldcg(&ip->terms);
      tn += __ldcg(&ip->near);
      tf += __ldcg(&ip->fsum);
      ta += __ldcg(&ip->fabs);
      for (int a = 0; a < 4; a++) tam[a] += __ldcg(&ip->am[a]);
    }
    sh->out_len = 0;
    sh->flags = 0;
    const unsigned long long vhash = tv % 999983ULL;
    const long long lookups = (long long)d->lookups;
    ens_printf(c, FMT_RS_HDR, d->n_nuc == 68 ? "small" : "large", d->n_nuc, d->avg_poles, d->avg_windows, d->doppler,
               lookups, (unsigned long long)d->seed);
    ens_printf(c, FMT_VERIFY, vhash);
    uint32_t *tal = p.tallies + (size_t)k * ENS_TALLIES;
    for (int t = 0; t < ENS_TALLIES; t++) {
      uint32_t v = 0;
      if (t < 4) v = tam[t];
      else if (t >= 5 && t < 17) v = d->mcnt[t - 4] - d->mcnt[t - 5];
      else if (t == 24) v = (uint32_t)tt;
      else if (t == 25) v = (uint32_t)(tt >> 32);
      else if (t == 26) v = (uint32_t)tn;
      tal[t] = v;
    }
    ens_record rec;
    rec.instance = d->line;
    rec.exit_code = 0;
    rec.app = APP_RSBENCH;
    rec.flags = sh->flags | ENS_RF_DONE;
    rec.vhash = vhash;
    rec.bitsum = tb;
    rec.fsum = tf;
    rec.fabs = ta;
    rec.work = (uint64_t)lookups;
    rec.stdout_len = sh->out_len;
    uint32_t sm = 0;
    if (p.flags & ENS_F_TIMESTAMPS) asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    rec.smid = sm;
    rec.t_start_ns = d->t_start;
    rec.t_end_ns = (p.flags & ENS_F_TIMESTAMPS) ? xs2_gtimer() : 0ull;
    p.recs[k] = rec;
    const unsigned long long pos = atomicAdd(p.stdout_total, (unsigned long long)sh->out_len);
    p.stdout_pos[k] = pos;
    reinterpret_cast<unsigned long long *>(misc + 8)[0] = pos;
  }
  __syncthreads();
  const unsigned long long pos = reinterpret_cast<const unsigned long long *>(misc + 8)[0];
  const unsigned long long *src = reinterpret_cast<const unsigned long long *>(c.out);
  unsigned long long *dst = reinterpret_cast<unsigned long long *>(p.stdout_cmp + pos);
  for (uint32_t w = tid; w < sh->out_len / 8; w += kRs2T) dst[w] = src[w];
}

__global__ void __launch_bounds__(kRs2T, ENS_RS2_MINB) rs_items_kernel(const KParams p) {
  const int tid = threadIdx.x;
  Ctx c{};
  c.sh_off = 0;
  c.smem_off = kRsDesc;
  c.csize = 1;
  c.flags = p.flags;
  c.out_cap = p.stdout_cap;
  Shared *sh = ens_sh(c);
  RsDesc *d = reinterpret_cast<RsDesc *>(ens_dsmem + kRsDesc);
  double *thr = reinterpret_cast<double *>(ens_dsmem + kRsThr);
  int *nn = reinterpret_cast<int *>(ens_dsmem + kRsNn);
  double *concs = reinterpret_cast<double *>(ens_dsmem + kRsConcs);
  uint16_t *mats = reinterpret_cast<uint16_t *>(ens_dsmem + kRsMats);
  int *poff = reinterpret_cast<int *>(ens_dsmem + kRsOff);
  int *woff = poff + 356;
  uint32_t *misc = reinterpret_cast<uint32_t *>(ens_dsmem + kRsMisc);
  uint32_t *am = misc + 2;
  int cached = 0;  // n_nuc of the material lists in shared memory
  uint32_t cached_j = 0xffffffffu;
  // the staging mbarrier (misc[12..13]) and its phase parity
  const uint32_t mbar = (uint32_t)__cvta_generic_to_shared(misc + 12);
  uint32_t mphase = 0;
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mbar) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  for (;;) {
    if (tid == 0) misc[0] = atomicAdd(p.counter2, 1u);
    if (tid < 4) am[tid] = 0u;
    __syncthreads();
    if (misc[0] >= p.n_items) break;
    const uint32_t item = p.item_base + misc[0];
    const uint32_t j = p.items[item];
    if (j != cached_j) {  // a new instance: its descriptor and shared tables
      const unsigned long long *src = reinterpret_cast<const unsigned long long *>(p.xs_desc + (size_t)j * kDescBytes);
      unsigned long long *dst = reinterpret_cast<unsigned long long *>(d);
      for (int w = tid; w < (int)(sizeof(RsDesc) / 8); w += kRs2T) dst[w] = src[w];
      __syncthreads();
      const int n_nuc = d->n_nuc, mx = xs_max_nucs(n_nuc);
      if (n_nuc != cached) {
        hm_tables(n_nuc, mx, thr, nn, concs, mats);
        cached = n_nuc;
      }
      __syncthreads();
      // the instance's pole / window offsets and concentrations (phase 1's arena copies,
      // 256-B aligned regions) staged by the TMA engine: three bulk global->shared copies
      // completing on one mbarrier, while the threads wait on its phase
      if (tid == 0) {
        const uint32_t bo = ((uint32_t)(n_nuc + 1) * 4u + 15u) & ~15u, bc = 12u * (uint32_t)mx * 8u;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // earlier generic reads of the buffers
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mbar), "r"(2u * bo + bc)
                     : "memory");
        bulk_g2s(poff, reinterpret_cast<const void *>(d->poff), bo, mbar);
        bulk_g2s(woff, reinterpret_cast<const void *>(d->woff), bo, mbar);
        bulk_g2s(concs, reinterpret_cast<const void *>(d->concs), bc, mbar);
      }
      mbar_wait(mbar, mphase);
      mphase ^= 1u;
      cached_j = j;
      __syncthreads();
    }
    const int n_nuc = d->n_nuc, mx = xs_max_nucs(n_nuc);
    const long long L = (long long)d->lookups;
    const long long s0 = (long long)(item - d->item0) * kRsItemLookups;
    const long long s1 = s0 + kRsItemLookups < L ? s0 + kRsItemLookups : L;
    const double *poles = reinterpret_cast<const double *>(d->poles);
    const uint8_t *pl = reinterpret_cast<const uint8_t *>(d->pole_l);
    const double *wins = reinterpret_cast<const double *>(d->windows);
    const double *k0 = reinterpret_cast<const double *>(d->k0rs);
    const double *lk_e = reinterpret_cast<const double *>(d->lk_e);
    double *dmp = p.dump ? p.dump + (size_t)d->k * p.dump_rows * 8 : nullptr;
    unsigned long long ver = 0, bsum = 0, terms = 0, near = 0;
    double fsum = 0.0, fabs_ = 0.0;
    for (long long sl = s0 + tid; sl < s1; sl += kRs2T) {
      int mat = 0;
#pragma unroll
      for (int m = 1; m < 12; m++) mat += (sl >= (long long)d->mcnt[m]) ? 1 : 0;
      const double E = ldro(lk_e + sl);
      double macro[4];
      RsApp::lookup<true>(d->doppler, E, mat, nn, mats, mx, concs, poff, woff, poles, pl, wins, k0, macro, terms, near);
      double mxv = -DBL_MAX;
      int a = 0;
#pragma unroll
      for (int q = 0; q < 4; q++)
        if (macro[q] > mxv) {
          mxv = macro[q];
          a = q;
        }
      ver += (unsigned long long)(a + 1);
      atomicAdd(&am[a], 1u);
      if (dmp) dump_row(dmp, p.dump_rows, sl, E, mat, macro, 4, a);
#pragma unroll
      for (int q = 0; q < 4; q++) {
        bsum += dbits(macro[q]);
        fsum += macro[q];
        fabs_ += fabs(macro[q]);
      }
    }
    ver = block_sum_u64(sh, ver);
    bsum = block_sum_u64(sh, bsum);
    terms = block_sum_u64(sh, terms);
    near = block_sum_u64(sh, near);
    fsum = block_sum_f64(sh, fsum);
    fabs_ = block_sum_f64(sh, fabs_);
    if (tid == 0) {
      RsItemPart *ip = reinterpret_cast<RsItemPart *>(p.ipart + (size_t)item * kPartBytes);
      ip->ver = ver;
      ip->bsum = bsum;
      ip->terms = terms;
      ip->near = near;
      ip->fsum = fsum;
      ip->fabs = fabs_;
      for (int a = 0; a < 4; a++) ip->am[a] = am[a];
      __threadfence();
      misc[1] = atomicAdd(&p.idone[j], 1u) == d->n_items - 1 ? 1u : 0u;
    }
    __syncthreads();
    if (misc[1]) rs2_finish(p, c, d, misc);
    __syncthreads();  // misc, am reused by the next item
  }
}

// threads per CTA of the phase-2 kernel of an item kind: XS grid types 0..2, RS 3
int xs_items_threads(int kind) {
  switch (kind) {
    case XS_HASH: return Xs2T<XS_HASH>::v;
    case XS_UNIONIZED: return Xs2T<XS_UNIONIZED>::v;
    case XS_NUCLIDE: return Xs2T<XS_NUCLIDE>::v;
  }
  return kRs2T;
}

// phase-2 kernel of an item kind: XS grid types 0..2, RS 3
static const void *xs_items_fn(int grid) {
  switch (grid) {
    case XS_HASH: return (const void *)xs_items_kernel<XS_HASH>;
    case XS_UNIONIZED: return (const void *)xs_items_kernel<XS_UNIONIZED>;
    case XS_NUCLIDE: return (const void *)xs_items_kernel<XS_NUCLIDE>;
    case 3: return (const void *)rs_items_kernel;
  }
  return nullptr;
}
static uint32_t items_smem(int kind) { return kind == 3 ? kRsSmem : kXs2Smem; }

cudaError_t xs_items_occupancy(int grid, int *ctas) {
  const void *fn = xs_items_fn(grid);
  if (!fn) return cudaErrorInvalidValue;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)items_smem(grid));
  if (e != cudaSuccess) return e;
  int per_sm = 0, dev = 0, sms = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, xs_items_threads(grid), items_smem(grid));
  if (e == cudaSuccess) e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  *ctas = per_sm * sms;
  return e;
}

cudaError_t launch_xs_items(int grid_type, int ctas, const KParams &p, cudaStream_t st) {
  const void *fn = xs_items_fn(grid_type);
  if (!fn) return cudaErrorInvalidValue;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)items_smem(grid_type));
  if (e != cudaSuccess) return e;
  void *args[] = {const_cast<KParams *>(&p)};
  return cudaLaunchKernel(fn, dim3((unsigned)ctas), dim3((unsigned)xs_items_threads(grid_type)), args,
                          items_smem(grid_type), st);
}

}  // namespace ens
