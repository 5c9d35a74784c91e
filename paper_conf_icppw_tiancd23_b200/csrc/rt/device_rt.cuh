// csrc/rt/device_rt.cuh — N0, the per-instance device runtime.
//
// Everything an instance owns (§3.3: instances must not share
// mutable globals) lives in its Ctx: its argv (shared memory), its heap
// arena (a slot of the workspace, bump-allocated through a host-computed
// layout), its stdout buffer, its tallies and its exit code.  No mutable
// __device__ globals exist anywhere in the instance bodies.
#pragma once
#include <cooperative_groups.h>

#include <cstdint>

#include "fmt_ids.h"
#include "../../../include/ens.h"

namespace ens {

#define ENS_HD __host__ __device__ __forceinline__

// ---------------------------------------------------------------------------
// LCG (SURVEY.md §8(c) "Shared primitives"): s <- (a*s + 1) mod 2^63, held
// as an affine map so that n steps are one multiply-add (jump constants).
// ---------------------------------------------------------------------------
constexpr uint64_t kLcgA = 2806196910506780709ULL;
constexpr uint64_t kMask63 = 0x7FFFFFFFFFFFFFFFULL;

struct Affine {
  uint64_t a, c;  // s -> a*s + c  (mod 2^64; reduced mod 2^63 on apply)
  ENS_HD uint64_t operator()(uint64_t s) const { return (a * s + c) & kMask63; }
  // this ∘ then: apply `first` then this
  ENS_HD Affine after(const Affine &first) const { return {a * first.a, a * first.c + c}; }
};

// the map of n LCG steps, by repeated squaring
ENS_HD Affine lcg_pow(uint64_t n) {
  Affine r{1ULL, 0ULL};
  Affine b{kLcgA, 1ULL};
  n &= kMask63;
  while (n) {
    if (n & 1ULL) r = b.after(r);
    b = b.after(b);
    n >>= 1;
  }
  return r;
}

ENS_HD uint64_t lcg_next(uint64_t s) { return (kLcgA * s + 1ULL) & kMask63; }

// advance, then scale by 2^-63 (exact: the conversion rounds, the scale is a
// power of two)
__device__ __forceinline__ double lcg_double(uint64_t &s) {
  s = lcg_next(s);
  return __ull2double_rn(s) * 0x1p-63;
}
// the six draws after state s (a record's draws 6r+1..6r+6) as six
// independent maps s -> A^k s + C_k (k = 1..6): the same states as six
// lcg_double calls, without their k-step dependency chain
__host__ __device__ constexpr uint64_t lcg_pow_a(int k) { uint64_t a = 1ULL; for (int i = 0; i < k; i++) a *= kLcgA; return a; }
__host__ __device__ constexpr uint64_t lcg_pow_c(int k) { uint64_t c = 0ULL; for (int i = 0; i < k; i++) c = kLcgA * c + 1ULL; return c; }
__device__ __forceinline__ void lcg_doubles6(uint64_t s, double (&x)[6]) {
  constexpr uint64_t A[6] = {lcg_pow_a(1), lcg_pow_a(2), lcg_pow_a(3), lcg_pow_a(4), lcg_pow_a(5), lcg_pow_a(6)};
  constexpr uint64_t C[6] = {lcg_pow_c(1), lcg_pow_c(2), lcg_pow_c(3), lcg_pow_c(4), lcg_pow_c(5), lcg_pow_c(6)};
#pragma unroll
  for (int k = 0; k < 6; k++) x[k] = __ull2double_rn((A[k] * s + C[k]) & kMask63) * 0x1p-63;
}
__device__ __forceinline__ uint64_t lcg_int(uint64_t &s) {
  s = lcg_next(s);
  return s;
}

// ---------------------------------------------------------------------------
// strings / integer flags (reading R-int: optional sign, 1..18 digits)
// ---------------------------------------------------------------------------
ENS_HD bool str_eq(const char *a, const char *b) {
  while (*a && *a == *b) {
    a++;
    b++;
  }
  return *a == *b;
}
ENS_HD uint32_t str_len(const char *a) {
  uint32_t n = 0;
  while (a[n]) n++;
  return n;
}
ENS_HD bool parse_i64(const char *s, long long *v) {
  bool neg = false;
  if (*s == '+' || *s == '-') {
    neg = *s == '-';
    s++;
  }
  long long x = 0;
  int nd = 0;
  for (; *s; s++, nd++) {
    if (*s < '0' || *s > '9' || nd >= 18) return false;
    x = x * 10 + (*s - '0');
  }
  if (nd == 0) return false;
  *v = neg ? -x : x;
  return true;
}

ENS_HD uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

// ---------------------------------------------------------------------------
// per-instance context (identical copy in every thread of the block)
// ---------------------------------------------------------------------------
#ifndef ENS_MAX_TEAM
#define ENS_MAX_TEAM 16
#endif
constexpr int kMaxTeamCtas = ENS_MAX_TEAM;  // thread-block-cluster size (8 portable; 16 non-portable)
constexpr int kMaxSubTeams = 8;  // M instances per CTA (named barriers 1..8)

// Barrier of the threads running this instance.  With M instances per CTA
// (the paper's (N/M, M, 1) block) the
// instance is the row threadIdx.y of the block and uses hardware barrier y;
// otherwise it is the whole CTA.  The row variant is compiled separately
// (ENS_SUB=1, kernels_sub.cu): ptxas reserves every barrier id a kernel
// names, and the SM's barrier pool then caps resident CTAs (16 ids -> 4
// CTAs/SM measured), so the M = 1 kernels only ever use barrier 0, and the
// row kernels use the immediate ids 0..7 (8 ids, never a register id).
#ifndef ENS_SUB
#define ENS_SUB 0
#endif
__device__ __forceinline__ void sub_sync() {
#if ENS_SUB
  const uint32_t n = blockDim.x;
  switch (threadIdx.y) {
    case 0: asm volatile("bar.sync 0, %0;" ::"r"(n) : "memory"); break;
    case 1: asm volatile("bar.sync 1, %0;" ::"r"(n) : "memory"); break;
    case 2: asm volatile("bar.sync 2, %0;" ::"r"(n) : "memory"); break;
    case 3: asm volatile("bar.sync 3, %0;" ::"r"(n) : "memory"); break;
    case 4: asm volatile("bar.sync 4, %0;" ::"r"(n) : "memory"); break;
    case 5: asm volatile("bar.sync 5, %0;" ::"r"(n) : "memory"); break;
    case 6: asm volatile("bar.sync 6, %0;" ::"r"(n) : "memory"); break;
    default: asm volatile("bar.sync 7, %0;" ::"r"(n) : "memory"); break;
  }
#else
  __syncthreads();
#endif
}

struct Shared {             // static shared memory of the scheduler
  uint32_t tallies[32];     // per-instance tallies (smem atomics)
  uint32_t out_len;         // stdout bytes used (thread 0 only)
  uint32_t flags;           // record flags (thread 0 only)
  unsigned long long red_u[32];  // block reduction scratch
  double red_d[32];
  unsigned long long team_u[kMaxTeamCtas];  // cross-CTA partials (rank 0's copy)
  double team_d[kMaxTeamCtas];
};

struct Result {  // meaningful in thread 0 after the body returns
  int exit_code;
  uint64_t vhash, bitsum;
  double fsum, fabs;
  uint64_t work;
  int deferred;  // set by EVERY thread: the record is written by a later phase (split phases)
};

// The team running one instance: one CTA (the paper's team = thread block,
// P:313-318), or on B200 a thread-block cluster of csize CTAs with a hardware
// barrier and distributed shared memory — for ensembles with fewer instances
// than SMs (team-aware bodies only; others run on rank 0 alone).
struct Ctx {
  uint32_t k, id;      // record slot, instance id (line)
  char *arena;         // this team's slot
  uint64_t arena_cap;
  char *out;           // this instance's raw stdout buffer
  uint32_t out_cap;
  uint32_t sh_off;     // scheduler state (Shared) and the app's dynamic
  uint32_t smem_off;   // shared memory: byte offsets in the dynamic smem
  uint32_t crank, csize;  // CTA rank in the team, team CTAs
  uint32_t flags;              // launch flags (ENS_F_*)
  unsigned long long *phases;  // tracing: ns per phase, or null
  unsigned long long t_mark;   // tracing: last mark (team thread 0)
  double *dump;                // element-wise dump rows of this instance (testing), or null
  uint32_t dump_rows;
  char *desc;                  // split phases: this instance's phase-2 descriptor, or null
  unsigned long long t_start;  // ENS_F_TIMESTAMPS: %globaltimer at the instance's start (thread 0)
};
// element-wise dump (ens_launch_cfg.dump_rows): row `slot` = {key, mat,
// v[0..nv), argmax}, zero-padded to 8 doubles
__device__ __forceinline__ void dump_row(double *dump, uint32_t rows, long long slot, double key, int mat,
                                         const double *v, int nv, int argmax) {
  if (!dump || slot < 0 || slot >= (long long)rows) return;
  double *d = dump + (size_t)slot * 8;
  d[0] = key;
  d[1] = (double)mat;
#pragma unroll
  for (int q = 0; q < 5; q++) d[2 + q] = q < nv ? v[q] : 0.0;
  d[7] = (double)argmax;
}

// The instance's shared memory, addressed from the dynamic shared-memory
// symbol: pointers derived from it stay in the shared window after a Ctx
// crosses a call, so accesses compile to LDS/STS/ATOMS, not generic LD/ST.
extern __shared__ __align__(16) char ens_dsmem[];
__device__ __forceinline__ char *ens_smem(const Ctx &c) { return ens_dsmem + c.smem_off; }
__device__ __forceinline__ Shared *ens_sh(const Ctx &c) { return reinterpret_cast<Shared *>(ens_dsmem + c.sh_off); }

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// bounds / invariant checks of the cross-CTA paths (compute-sanitizer is not
// available on the GPU pool): built with -DENS_CHECKS=1 a failed check traps
// (the launch fails with an illegal-instruction error); off in the product
#ifndef ENS_CHECKS
#define ENS_CHECKS 0
#endif
#define ENS_CHECK(cond)                  \
  do {                                   \
    if (ENS_CHECKS && !(cond)) __trap(); \
  } while (0)

// tracing: is this the thread that marks phases?  Hot loops test a cached
// copy (phase_mark_if): the Ctx lives in local memory across calls
__device__ __forceinline__ bool tracing(const Ctx &c) { return c.phases && threadIdx.x == 0 && c.crank == 0; }
// tracing: charge the time since the last mark to phase k (team thread 0)
__device__ __forceinline__ void phase_mark(Ctx &c, int k) {
  if (c.phases && threadIdx.x == 0 && c.crank == 0) {
    const unsigned long long now = gtimer();
    if (k >= 0) atomicAdd(&c.phases[k], now - c.t_mark);
    c.t_mark = now;
  }
}
__device__ __forceinline__ void phase_mark_if(bool on, Ctx &c, int k) {
  if (on) phase_mark(c, k);
}

// barrier of the whole team (cluster barrier: release/acquire at cluster
// scope, so global and shared writes before it are visible after it)
__device__ __forceinline__ void team_sync(const Ctx &c) {
  if (c.csize > 1) cooperative_groups::this_cluster().sync();
  else sub_sync();
}
// `p` (a shared variable of this CTA) in the shared memory of team CTA `rank`
template <class X>
__device__ __forceinline__ X *cta_shared(X *p, uint32_t rank) {
  return cooperative_groups::this_cluster().map_shared_rank(p, rank);
}

// ---- stdout: {u32 fmt, u32 payload bytes, 8-B slots}; strings = len slot +
// bytes padded to 8.  Called by thread 0 only.
struct OutArg {
  int kind;  // 0 int64, 1 uint64, 2 double, 3 string
  union {
    long long i;
    unsigned long long u;
    double d;
    const char *s;
  };
};
__device__ __forceinline__ OutArg oa(int v) { OutArg a; a.kind = 0; a.i = v; return a; }
__device__ __forceinline__ OutArg oa(long long v) { OutArg a; a.kind = 0; a.i = v; return a; }
__device__ __forceinline__ OutArg oa(unsigned long long v) { OutArg a; a.kind = 1; a.u = v; return a; }
__device__ __forceinline__ OutArg oa(double v) { OutArg a; a.kind = 2; a.d = v; return a; }
__device__ __forceinline__ OutArg oa(const char *v) { OutArg a; a.kind = 3; a.s = v; return a; }

__device__ inline void out_write(Ctx &c, unsigned fmt, const OutArg *args, int n) {
  uint32_t payload = 0;
  for (int i = 0; i < n; i++) payload += args[i].kind == 3 ? 8u + (uint32_t)align_up(str_len(args[i].s), 8) : 8u;
  uint32_t need = 8u + payload;
  uint32_t len = ens_sh(c)->out_len;
  if (len + need > c.out_cap) {
    ens_sh(c)->flags |= 1u;  // ENS_RF_STDOUT_TRUNC
    return;
  }
  unsigned long long *w = reinterpret_cast<unsigned long long *>(c.out + len);
  *w++ = (unsigned long long)fmt | ((unsigned long long)payload << 32);
  for (int i = 0; i < n; i++) {
    if (args[i].kind == 3) {
      uint32_t L = str_len(args[i].s);
      *w++ = L;
      for (uint32_t b = 0; b < L; b += 8) {
        unsigned long long v = 0;
        for (uint32_t q = 0; q < 8 && b + q < L; q++) v |= (unsigned long long)(unsigned char)args[i].s[b + q] << (8 * q);
        *w++ = v;
      }
    } else {
      *w++ = args[i].u;
    }
  }
  ens_sh(c)->out_len = len + need;
}

template <class... A>
__device__ __forceinline__ void ens_printf(Ctx &c, unsigned fmt, A... a) {
  if (threadIdx.x != 0 || c.crank != 0) return;
  OutArg args[sizeof...(A) > 0 ? sizeof...(A) : 1] = {oa(a)...};
  out_write(c, fmt, args, (int)sizeof...(A));
}

// ---------------------------------------------------------------------------
// block reductions (result valid in every thread)
// ---------------------------------------------------------------------------
__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v) {
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ double warp_sum_f64(double v) {
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ double warp_max_f64(double v) {  // NaN never wins
  for (int o = 16; o; o >>= 1) {
    double w = __shfl_xor_sync(0xffffffffu, v, o);
    v = (w > v) ? w : v;
  }
  return v;
}

__device__ inline unsigned long long block_sum_u64(Shared *sh, unsigned long long v) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  v = warp_sum_u64(v);
  sub_sync();
  if (lane == 0) sh->red_u[w] = v;
  sub_sync();
  v = lane < nw ? sh->red_u[lane] : 0ULL;
  return warp_sum_u64(v);
}
__device__ inline double block_sum_f64(Shared *sh, double v) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  v = warp_sum_f64(v);
  sub_sync();
  if (lane == 0) sh->red_d[w] = v;
  sub_sync();
  v = lane < nw ? sh->red_d[lane] : 0.0;
  return warp_sum_f64(v);
}
__device__ inline double block_max_f64(Shared *sh, double v) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  v = warp_max_f64(v);
  sub_sync();
  if (lane == 0) sh->red_d[w] = v;
  sub_sync();
  v = lane < nw ? sh->red_d[lane] : v;
  return warp_max_f64(v);
}

// Arena data is written and re-read inside the same persistent launch (and a
// slot is reused by the block's next instance), so it must NOT go through the
// non-coherent read-only path (ld.global.nc / __ldg): plain coherent loads.
template <class T>
__device__ __forceinline__ T ld_(const T *p) { return *p; }

// Read-only global load (ld.global.nc): only for data no thread writes during
// the kernel — split phases' phase 2 reads tables an earlier kernel wrote.
template <class T>
__device__ __forceinline__ T ldro(const T *p) { return __ldg(p); }

// bring the line holding p into L1 without holding registers
__device__ __forceinline__ void prefetch_l1(const void *p) { asm volatile("prefetch.global.L1 [%0];" ::"l"(p)); }

__device__ __forceinline__ uint64_t dbits(double d) { return (uint64_t)__double_as_longlong(d); }

// team reductions: block reduction, then CTA partials gathered in rank 0's
// shared memory and summed in rank order (deterministic); result valid in
// rank 0 (in every thread of it).
__device__ inline unsigned long long team_sum_u64(Ctx &c, unsigned long long v) {
  v = block_sum_u64(ens_sh(c), v);
  if (c.csize == 1) return v;
  if (threadIdx.x == 0) *cta_shared(&ens_sh(c)->team_u[c.crank], 0) = v;
  team_sync(c);
  unsigned long long t = 0;
  if (c.crank == 0)
    for (uint32_t r = 0; r < c.csize; r++) t += ens_sh(c)->team_u[r];
  team_sync(c);
  return t;
}
// whether any thread of the team has v != 0 (valid in every thread of every CTA)
__device__ inline bool team_any(Ctx &c, int v) {
  v = __syncthreads_or(v);
  if (c.csize == 1) return v != 0;
  if (threadIdx.x == 0) *cta_shared(&ens_sh(c)->team_u[c.crank], 0) = (unsigned long long)(v != 0);
  team_sync(c);
  unsigned long long t = 0;
  for (uint32_t r = 0; r < c.csize; r++) t |= *cta_shared(&ens_sh(c)->team_u[r], 0);
  team_sync(c);  // team_u is reused
  return t != 0;
}
__device__ inline double team_sum_f64(Ctx &c, double v) {
  v = block_sum_f64(ens_sh(c), v);
  if (c.csize == 1) return v;
  if (threadIdx.x == 0) *cta_shared(&ens_sh(c)->team_d[c.crank], 0) = v;
  team_sync(c);
  double t = 0.0;
  if (c.crank == 0)
    for (uint32_t r = 0; r < c.csize; r++) t += ens_sh(c)->team_d[r];
  team_sync(c);
  return t;
}

}  // namespace ens
