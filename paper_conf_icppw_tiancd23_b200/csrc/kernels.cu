// csrc/kernels.cu — N2, the ensemble scheduler kernel, and its instances.
//
// The paper maps NI instances onto N teams with `target teams distribute
// num_teams(N) thread_limit(T)` (Fig. 4), one team = one CUDA
// thread block (§2.3), with N = NI in its evaluation.
// Here the grid is persistent: min(NI, occupancy x 148) teams pull instance
// slots from an atomic counter (reading Q5), so NI may exceed the teams that
// fit at once, and each team's heap arena is a fixed slot of the workspace
// (memory = resident teams x arena, not NI x arena).
// A team is one CTA, or (team-aware bodies, ensembles with fewer instances
// than SMs) a thread-block cluster of up to 8 CTAs (see rt/device_rt.cuh).
//
// This file is compiled twice: as kernels.cu (ENS_SUB=0: one instance per
// CTA row = the whole CTA, every host-side entry point) and as
// kernels_sub.cu (ENS_SUB=1: the row kernels of the (N/M, M, 1) mapping for
// the bodies built for it, see sub_sync in rt/device_rt.cuh).
#include <cuda_runtime.h>

#ifndef ENS_SUB
#define ENS_SUB 0
#endif
#include "apps/amgmk.cuh"
#include "apps/echo.cuh"
#include "apps/pagerank.cuh"
#if !ENS_SUB
#include "apps/rsbench.cuh"
#include "apps/xsbench.cuh"
#endif
#include "kparams.h"

namespace ens {
#if ENS_SUB
namespace subk {  // row kernels: distinct symbols from the M = 1 kernels
#endif

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint32_t smid() {
  uint32_t s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  return s;
}

// register budget: min blocks per SM = ENS_MINB_NUM / T (512: 128 registers)
#ifndef ENS_MINB_NUM
#define ENS_MINB_NUM 512
#endif

// Per-instance scheduler state, in dynamic shared memory: one copy per
// instance running in the CTA (M = blockDim.y instances per CTA), followed
// by that instance's app shared memory.
struct SubShared {
  Shared sh;
  char *argv[ENS_MAX_ARGC + 1];
  unsigned long long pos;
  uint32_t j;
  uint32_t clc_phase;          // ENS_F_CLC: the mbarrier's phase parity
  alignas(16) uint4 clc_res;   // ENS_F_CLC: the try_cancel response
  unsigned long long clc_mbar;
};

#if !ENS_SUB
// ENS_F_CLC (SURVEY.md §8(a) S3 ablation): cluster launch control.  The grid
// has one CTA per instance (the paper's N teams); a CTA that finished its
// instance cancels a CTA of the grid the hardware has not launched yet and
// runs that one's instance instead (clusterlaunchcontrol.try_cancel: the
// response arrives in shared memory through an mbarrier transaction).
// Returns false when every CTA has been launched.  One thread.
__device__ __forceinline__ bool clc_steal(SubShared *ss, uint32_t *x) {
  const uint32_t mbar = (uint32_t)__cvta_generic_to_shared(&ss->clc_mbar);
  const uint32_t res = (uint32_t)__cvta_generic_to_shared(&ss->clc_res);
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], 16;" ::"r"(mbar) : "memory");
  asm volatile("clusterlaunchcontrol.try_cancel.async.shared::cta.mbarrier::complete_tx::bytes.b128 [%0], [%1];" ::"r"(res),
               "r"(mbar)
               : "memory");
  uint32_t done = 0;
  while (!done)
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                 : "=r"(done)
                 : "r"(mbar), "r"(ss->clc_phase)
                 : "memory");
  ss->clc_phase ^= 1u;
  uint32_t ok = 0, v = 0;
  asm volatile("{ .reg .pred p; .reg .b128 r; ld.shared.b128 r, [%2];\n\t"
               "clusterlaunchcontrol.query_cancel.is_canceled.pred.b128 p, r;\n\t"
               "selp.u32 %0, 1, 0, p;\n\t"
               "@p clusterlaunchcontrol.query_cancel.get_first_ctaid::x.b32.b128 %1, r; }"
               : "=r"(ok), "=r"(v)
               : "r"(res)
               : "memory");
  *x = v;
  return ok != 0;
}
// ENS_F_CLC: arena slots are not CTA ids (the grid has N CTAs) but a pool as
// large as the resident CTAs: a CTA claims a free bit of the pool bitmap on
// arrival and returns it on exit (memory = resident CTAs x arena, as with the
// persistent grid)
__device__ __forceinline__ uint32_t slot_claim(uint32_t *bm, uint32_t n_slots) {
  for (uint32_t i = blockIdx.x % n_slots;; i = i + 1 == n_slots ? 0 : i + 1) {
    const uint32_t bit = 1u << (i & 31);
    if (!(atomicOr(&bm[i >> 5], bit) & bit)) return i;
  }
}
#endif
constexpr uint32_t kSubSharedBytes = (sizeof(SubShared) + 15) / 16 * 16;

// T = threads per CTA (the launch bound); the instance runs on the CTA's row
// threadIdx.y of blockDim.x threads (all of it when M = 1).
template <class App, int T>
__global__ void __launch_bounds__(T, (ENS_MINB_NUM / T) > 0 ? (ENS_MINB_NUM / T) : 1) ens_kernel(const KParams p) {
  extern __shared__ __align__(16) char dsmem[];
  const int tid = threadIdx.x, B = blockDim.x, y = threadIdx.y, M = blockDim.y;
  SubShared *ss = reinterpret_cast<SubShared *>(dsmem + (size_t)y * p.sub_stride);
  Shared &sh = ss->sh;
  char **s_argv = ss->argv;
  const uint32_t cs = p.team_ctas;  // cluster dims (cs, 1, 1); M > 1 only with cs == 1
  const uint32_t cr = cs > 1 ? cooperative_groups::this_cluster().block_rank() : 0u;
#if ENS_SUB
  const bool clc = false;
  (void)clc;
#else
  const bool clc = p.clc != 0;  // M == 1 and cs == 1 (host-enforced)
#endif
  uint32_t slot = (blockIdx.x / cs) * M + y;
#if !ENS_SUB
  if (clc && !p.split) {
    if (tid == 0) ss->j = slot_claim(p.slot_bm, p.n_slots);
    __syncthreads();
    slot = ss->j;
  }
  if (clc && tid == 0) {
    ss->clc_phase = 0;
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&ss->clc_mbar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
#endif
  char *const arena = p.arena_base + (size_t)slot * p.arena_bytes;
  Ctx c;
  c.arena = arena;
  c.arena_cap = p.arena_bytes;
  c.out_cap = p.stdout_cap;
  c.sh_off = (uint32_t)((size_t)y * p.sub_stride);  // ss: &ss->sh == ss
  c.smem_off = c.sh_off + kSubSharedBytes;
  c.crank = cr;
  c.csize = cs;
  bool first = true;
  for (;;) {
#if ENS_SUB
    if (tid == 0 && cr == 0) ss->j = atomicAdd(p.counter, 1u);
#else
    if (tid == 0 && cr == 0) {
      if (!clc) ss->j = atomicAdd(p.counter, 1u);
      else if (first) ss->j = blockIdx.x;  // this CTA's own instance
      else {
        uint32_t x = 0;
        ss->j = clc_steal(ss, &x) ? x : 0xffffffffu;  // an unlaunched CTA's instance, or done
      }
    }
    first = false;
#endif
    team_sync(c);
    const uint32_t j = cr == 0 ? ss->j : *cta_shared(&ss->j, 0);
    if (cs > 1) team_sync(c);  // every rank has read s_j before rank 0 may exit
    if (j >= p.n) break;       // team-uniform
    const uint32_t k = p.kmap[j];
    const uint32_t line = p.line_of_k[k];
    const uint32_t t0 = p.line_tok[line];
    const int argc = (int)(p.line_tok[line + 1] - t0);
    for (int i = tid; i < argc; i += B) s_argv[i] = const_cast<char *>(p.blob) + p.tok_off[t0 + i];
    if (tid == 0) s_argv[argc] = nullptr;
    if (tid < 32) sh.tallies[tid] = 0;
    if (tid == 0) {
      sh.out_len = 0;
      sh.flags = 0;
    }
    uint64_t t_start = 0;
    if ((p.flags & ENS_F_TIMESTAMPS) && tid == 0) t_start = globaltimer();
    sub_sync();

    c.k = k;
    c.id = line;
    c.t_start = t_start;
    c.out = p.stdout_base + (size_t)k * p.stdout_cap;
    c.phases = p.phases;
    c.flags = p.flags;
    c.dump = p.dump ? p.dump + (size_t)k * p.dump_rows * 8 : nullptr;
    c.dump_rows = p.dump_rows;
    // split phases: one arena slot per instance (phase 2 reads the tables)
    c.arena = p.split ? p.arena_base + (size_t)j * p.arena_bytes : arena;
    c.desc = p.split ? p.xs_desc + (size_t)j * kDescBytes : nullptr;
    phase_mark(c, -1);
    Result r{};
    if (App::kTeam || cr == 0) r = App::run(c, argc, s_argv);
    team_sync(c);
    if (r.deferred) {  // split phases: phase 2 writes this instance's record
      continue;        // (the loop head's team_sync orders the scheduler state)
    }
    if (cs > 1 && cr != 0 && tid < ENS_TALLIES && sh.tallies[tid])  // combine tallies into rank 0
      atomicAdd(cta_shared(&sh.tallies[tid], 0), sh.tallies[tid]);
    team_sync(c);

    if (cr == 0) {
      if (tid < ENS_TALLIES) p.tallies[(size_t)k * ENS_TALLIES + tid] = sh.tallies[tid];
      if (tid == 0) {
        ens_record rec;
        rec.instance = line;
        rec.exit_code = r.exit_code;
        rec.app = App::kId == APP_NOTFOUND ? 0u : App::kId;
        rec.flags = sh.flags | ENS_RF_DONE;
        rec.vhash = r.vhash;
        rec.bitsum = r.bitsum;
        rec.fsum = r.fsum;
        rec.fabs = r.fabs;
        rec.work = r.work;
        rec.stdout_len = sh.out_len;
        rec.smid = (p.flags & ENS_F_TIMESTAMPS) ? smid() : 0u;
        rec.t_start_ns = t_start;
        rec.t_end_ns = (p.flags & ENS_F_TIMESTAMPS) ? globaltimer() : 0ull;
        p.recs[k] = rec;
        ss->pos = atomicAdd(p.stdout_total, (unsigned long long)sh.out_len);
        p.stdout_pos[k] = ss->pos;
      }
      sub_sync();
      {  // compact this instance's stdout (whole 8-B words)
        const unsigned long long *src = reinterpret_cast<const unsigned long long *>(c.out);
        unsigned long long *dst = reinterpret_cast<unsigned long long *>(p.stdout_cmp + ss->pos);
        for (uint32_t w = tid; w < sh.out_len / 8; w += B) dst[w] = src[w];
      }
    }
    team_sync(c);  // j, pos, argv, sh reused by the next instance
  }
#if !ENS_SUB
  if (clc && !p.split && tid == 0) {  // the arena slot back to the pool (its writes first)
    __threadfence();
    atomicAnd(&p.slot_bm[slot >> 5], ~(1u << (slot & 31)));
  }
#endif
  (void)first;
}

template <class App, int T>
static const void *kernel_if() {
  if constexpr (T <= App::kMaxT) return (const void *)ens_kernel<App, T>;
  return nullptr;
}
template <class App>
static const void *kernel_for(int T) {
  switch (T) {
    case 32: return kernel_if<App, 32>();
    case 64: return kernel_if<App, 64>();
    case 128: return kernel_if<App, 128>();
    case 256: return kernel_if<App, 256>();
    case 512: return kernel_if<App, 512>();
    case 1024: return kernel_if<App, 1024>();
  }
  return nullptr;
}

#if ENS_SUB
}  // namespace subk

const void *kernel_ptr_sub(uint32_t app, int T) {
  switch (app) {
    case APP_ECHO: return subk::kernel_for<EchoApp>(T);
    case APP_AMGMK: return subk::kernel_for<AmgApp>(T);
    case APP_PAGERANK: return subk::kernel_for<PrApp>(T);
    case APP_NOTFOUND: return subk::kernel_for<NotFoundApp>(T);
  }
  return nullptr;
}
#else
// the largest block size an app's kernel is built for (the thread limit is an
// upper bound)
int app_max_threads(uint32_t app) {
  switch (app) {
    case APP_ECHO: return EchoApp::kMaxT;
    case APP_XSBENCH: return XsApp::kMaxT;
    case APP_RSBENCH: return RsApp::kMaxT;
    case APP_AMGMK: return AmgApp::kMaxT;
    case APP_PAGERANK: return PrApp::kMaxT;
    case APP_NOTFOUND: return NotFoundApp::kMaxT;
  }
  return 32;
}
// whether the body splits its work over a multi-CTA team
bool app_team_aware(uint32_t app) {
  return app == APP_XSBENCH ? XsApp::kTeam : app == APP_RSBENCH ? RsApp::kTeam : false;
}
// host-side work estimate of one instance (relative units: dependent loads /
// pole terms / row or edge updates), for the schedule only: the instance
// queue is ordered longest-first and the team size covers the heaviest
// instance.  Results never depend on it (reading Q5).
double app_cost(uint32_t app, int argc, const char *const *argv) {
  switch (app) {
    case APP_XSBENCH: {
      XsParams p;
      if (xs_parse(argc, argv, p) >= 0) return 1.0;
      const double nucs = p.n_iso == 68 ? 15.49 : 55.38, n_u = (double)p.n_iso * p.n_gp;
      const double lk = p.history ? (double)p.particles * (double)p.lookups : (double)p.lookups;
      return lk * nucs + n_u * (p.grid == XS_UNIONIZED ? p.n_iso / 8.0 : 2.0);
    }
    case APP_RSBENCH: {
      RsParams p;
      if (rs_parse(argc, argv, p) >= 0) return 1.0;
      const double ppw = (double)p.avg_poles / p.avg_windows, per_term = p.doppler ? 1.0 : 0.6;
      return (double)p.lookups * 15.49 * (4.0 + (ppw > 1.0 ? ppw - 1.0 : 0.0) * per_term) +
             (double)p.avg_poles * p.n_nuc;
    }
    case APP_AMGMK: {
      AmgParams p;
      if (amg_parse(argc, argv, p) >= 0) return 1.0;
      const double n = (double)p.nx * p.ny * p.nz;
      return 7.0 * n * (p.iters + 1);
    }
    case APP_PAGERANK: {
      PrParams p;
      if (pr_parse(argc, argv, p) >= 0) return 1.0;
      return (double)p.n * (p.avg + 1) * (p.iters + 1);
    }
  }
  return 1.0;
}
// split phases: phase-2 items of one instance (0 = the instance runs fused)
// (*kind = the phase-2 kernel: the XS grid type)
uint32_t app_items(uint32_t app, int argc, const char *const *argv, int *kind) {
  *kind = 0;
  if (app == APP_RSBENCH) {  // kind 3: the RS lookup-item kernel
    RsParams q;
    if (rs_parse(argc, argv, q) >= 0) return 0;
    *kind = 3;
    return (uint32_t)rs_items(q);
  }
  if (app != APP_XSBENCH) return 0;
  XsParams p;
  if (xs_parse(argc, argv, p) >= 0) return 0;
  *kind = p.grid;
  return (uint32_t)xs_items(p);
}
// split phases: per-CTA scratch of the init-item kernel for one instance and
// its number of init items (hash / nuclide grids: one per nuclide; 0 = none)
uint64_t app_init_scratch(uint32_t app, int argc, const char *const *argv, int *n_items, int *n_sort, int *n_fine,
                          uint32_t *smem) {
  *n_items = 0;
  *n_sort = 0;
  *n_fine = 0;
  *smem = 0;
  if (app != APP_XSBENCH) return 0;
  XsParams p;
  if (xs_parse(argc, argv, p) >= 0 || !xs_split_ok(p) || p.grid == XS_UNIONIZED) return 0;
  *n_items = p.n_iso;
  *n_sort = xs_sort_items(p);
  *n_fine = xs_sort_fine_items(p);
  *smem = xs_init_smem(p).total;
  return XsApp::nuc_scratch_bytes(p);
}
// whether the body can run as one of M instances per CTA (NEXT 1)
bool app_sub_aware(uint32_t app) {
  switch (app) {
    case APP_ECHO: return EchoApp::kSub;
    case APP_AMGMK: return AmgApp::kSub;
    case APP_PAGERANK: return PrApp::kSub;
    case APP_NOTFOUND: return NotFoundApp::kSub;
  }
  return false;
}
uint32_t sub_shared_bytes() { return kSubSharedBytes; }

const void *kernel_ptr(uint32_t app, int T) {
  switch (app) {
    case APP_ECHO: return kernel_for<EchoApp>(T);
    case APP_XSBENCH: return kernel_for<XsApp>(T);
    case APP_RSBENCH: return kernel_for<RsApp>(T);
    case APP_AMGMK: return kernel_for<AmgApp>(T);
    case APP_PAGERANK: return kernel_for<PrApp>(T);
    case APP_NOTFOUND: return kernel_for<NotFoundApp>(T);
  }
  return nullptr;
}

// host-side sizing from the same parse/layout code the instance runs
bool app_size(uint32_t app, int argc, const char *const *argv, int T, int cs, uint64_t *arena, uint32_t *smem) {
  switch (app) {
    case APP_ECHO: return EchoApp::size(argc, argv, T, cs, arena, smem);
    case APP_XSBENCH: return XsApp::size(argc, argv, T, cs, arena, smem);
    case APP_RSBENCH: return RsApp::size(argc, argv, T, cs, arena, smem);
    case APP_AMGMK: return AmgApp::size(argc, argv, T, cs, arena, smem);
    case APP_PAGERANK: return PrApp::size(argc, argv, T, cs, arena, smem);
    case APP_NOTFOUND: return NotFoundApp::size(argc, argv, T, cs, arena, smem);
  }
  *arena = 0;
  *smem = 0;
  return false;
}

static cudaError_t set_smem(const void *fn, size_t smem) {
  if (kMaxTeamCtas > 8) {  // clusters of up to 16 CTAs (non-portable size)
    const cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
  }
  if (smem == 0) return cudaSuccess;
  return cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
}

// T = threads per CTA; m = instances per CTA: the block is (T/m, m, 1)
cudaError_t launch_group(uint32_t app, int T, int m, int grid, int cs, size_t smem, const KParams &p,
                         cudaStream_t st) {
  const void *fn = m > 1 ? kernel_ptr_sub(app, T) : kernel_ptr(app, T);
  if (!fn) return cudaErrorInvalidValue;
  cudaError_t e = set_smem(fn, smem);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3((unsigned)(T / m), (unsigned)m, 1u);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)cs;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  void *args[] = {const_cast<KParams *>(&p)};
  return cudaLaunchKernelExC(&cfg, fn, args);
}

// resident teams (clusters of cs CTAs; CTAs when m > 1) on the whole device
cudaError_t group_occupancy(uint32_t app, int T, int m, int cs, size_t smem, int *teams) {
  const void *fn = m > 1 ? kernel_ptr_sub(app, T) : kernel_ptr(app, T);
  if (!fn) return cudaErrorInvalidValue;
  cudaError_t e = set_smem(fn, smem);
  if (e != cudaSuccess) return e;
  if (cs <= 1) {
    int per_sm = 0, dev = 0, sms = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, T, smem);
    if (e == cudaSuccess) e = cudaGetDevice(&dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    *teams = per_sm * sms;
    return e;
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((unsigned)(cs * 64));
  cfg.blockDim = dim3((unsigned)T);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)cs;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaOccupancyMaxActiveClusters(teams, fn, &cfg);
}
#endif  // !ENS_SUB

}  // namespace ens
