// csrc/host/api.cpp — N3, the C ABI of libens.so (declared in include/ens.h).
//
// S1  ens_load_args / ens_parse_args: the enhanced loader of §3.2
//      / Fig. 4 — one instance per line, argv[0]
//     first.  The paper's StringCache keeps c_str() pointers into a growing
//     vector<string> (dangling after reallocation for short strings); here
//     every token lives once in an immutable packed blob with offsets.
// S2  ens_launch: one pinned host->device copy of blob + offsets + instance
//     map, then one persistent launch per app present (kernels.cu).
// S10 ens_collect: records, tallies and the compacted stdout back to the
//     host (P:380 `map(from: Ret[:NI])`), stdout formatted here.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "../../../include/ens.h"
#include "../apps/params.cuh"
#include "../kparams.h"

namespace ens {
long format_raw(const void *raw, size_t raw_len, std::string &out);
int expand_args(const char *text, size_t len, std::string &out, long *bad_line);
}

using namespace ens;

// ---------------------------------------------------------------------------
// errors
// ---------------------------------------------------------------------------
static thread_local std::string g_err;
static int fail(int code, const std::string &msg) {
  g_err = msg;
  return code;
}
static int cuda_fail(cudaError_t e, const char *what) {
  g_err = std::string(what) + ": " + cudaGetErrorString(e);
  return ENS_ECUDA;
}
#define CU(call)                                   \
  do {                                             \
    cudaError_t e_ = (call);                       \
    if (e_ != cudaSuccess) return cuda_fail(e_, #call); \
  } while (0)

// ---------------------------------------------------------------------------
// S1: args
// ---------------------------------------------------------------------------
struct ens_args {
  bool has_argv0 = false;
  std::vector<char> blob;            // NUL-terminated tokens
  std::vector<uint32_t> tok_off;     // argv entries of all lines, in order
  std::vector<uint32_t> line_tok;    // [n+1]
  std::vector<const char *> hptr;    // host argv arrays, NULL after each line
  std::vector<uint32_t> hfirst;      // [n] start of line i in hptr
};

static uint32_t blob_add(ens_args *a, const char *s, size_t n) {
  const uint32_t off = (uint32_t)a->blob.size();
  a->blob.insert(a->blob.end(), s, s + n);
  a->blob.push_back('\0');
  return off;
}

extern "C" int ens_parse_args(const char *text, size_t len, const char *argv0, ens_args **out) {
  if (!out || (!text && len)) return fail(ENS_EINVAL, "ens_parse_args: NULL argument");
  *out = nullptr;
  if (len && std::memchr(text, '\0', len)) return fail(ENS_EPARSE, "ens_parse_args: embedded NUL byte");
  // "@repeat N <template>" lines (the args-file script language)
  std::string expanded;
  if ((len && text[0] == '@') || (len && std::strstr(std::string(text, len).c_str(), "\n@"))) {
    long bad = -1;
    if (expand_args(text, len, expanded, &bad))
      return fail(ENS_EPARSE, "ens_parse_args: malformed @repeat template on line " + std::to_string(bad + 1));
    text = expanded.data();
    len = expanded.size();
  }
  ens_args *a = new ens_args();
  uint32_t a0 = 0;
  if (argv0) {
    a->has_argv0 = true;
    a0 = blob_add(a, argv0, std::strlen(argv0));
  }
  a->line_tok.push_back(0);
  size_t pos = 0;
  while (pos < len) {
    const char *nl = (const char *)std::memchr(text + pos, '\n', len - pos);
    size_t end = nl ? (size_t)(nl - text) : len;
    size_t e = end;
    if (e > pos && text[e - 1] == '\r') e--;  // reading Q1
    if (end - pos > ENS_MAX_LINE) {
      delete a;
      return fail(ENS_EINVAL, "ens_parse_args: line longer than ENS_MAX_LINE");
    }
    int argc = 0;
    if (argv0) {
      a->tok_off.push_back(a0);
      argc++;
    }
    size_t i = pos;
    while (i < e) {
      while (i < e && (text[i] == ' ' || text[i] == '\t')) i++;
      const size_t s = i;
      while (i < e && text[i] != ' ' && text[i] != '\t') i++;
      if (i > s) {
        a->tok_off.push_back(blob_add(a, text + s, i - s));
        argc++;
      }
    }
    if (argc > ENS_MAX_ARGC) {
      delete a;
      return fail(ENS_EINVAL, "ens_parse_args: more than ENS_MAX_ARGC argv entries on a line");
    }
    a->line_tok.push_back((uint32_t)a->tok_off.size());
    if (!nl) break;
    pos = end + 1;
  }
  if (a->blob.size() > 0xFFFFFFF0u) {
    delete a;
    return fail(ENS_EINVAL, "ens_parse_args: args larger than 4 GiB");
  }
  const size_t n = a->line_tok.size() - 1;
  for (size_t l = 0; l < n; l++) {
    a->hfirst.push_back((uint32_t)a->hptr.size());
    for (uint32_t t = a->line_tok[l]; t < a->line_tok[l + 1]; t++) a->hptr.push_back(a->blob.data() + a->tok_off[t]);
    a->hptr.push_back(nullptr);
  }
  *out = a;
  return ENS_OK;
}

extern "C" int ens_load_args(const char *path, const char *argv0, ens_args **out) {
  if (!path || !out) return fail(ENS_EINVAL, "ens_load_args: NULL argument");
  FILE *f = std::fopen(path, "rb");
  if (!f) return fail(ENS_ENOENT, std::string("ens_load_args: cannot open ") + path);
  std::string s;
  char buf[1 << 16];
  size_t k;
  while ((k = std::fread(buf, 1, sizeof buf, f)) > 0) s.append(buf, k);
  std::fclose(f);
  return ens_parse_args(s.data(), s.size(), argv0, out);
}

extern "C" int ens_args_count(const ens_args *a) {
  if (!a) return fail(ENS_EINVAL, "ens_args_count: NULL");
  return (int)(a->line_tok.size() - 1);
}

extern "C" int ens_args_get(const ens_args *a, int i, int *argc, const char *const **argv) {
  if (!a || !argc || !argv) return fail(ENS_EINVAL, "ens_args_get: NULL");
  if (i < 0 || i >= ens_args_count(a)) return fail(ENS_ERANGE, "ens_args_get: index out of range");
  *argc = (int)(a->line_tok[i + 1] - a->line_tok[i]);
  *argv = a->hptr.data() + a->hfirst[i];
  return ENS_OK;
}

extern "C" void ens_args_free(ens_args *a) { delete a; }

// ---------------------------------------------------------------------------
// S2..S9: launch
// ---------------------------------------------------------------------------
struct Group {
  uint32_t app = 0;
  int T = 0, grid = 0;  // grid = teams (arena slots); CTAs launched = grid * cs / m
  int cs = 1;           // CTAs per team (cluster size)
  int m = 1;            // instances per CTA (block (T/m, m, 1)); m > 1 only with cs == 1
  uint32_t smem = 0;    // app shared memory of one instance
  uint32_t sub = 0;     // dynamic smem per instance row: scheduler state + app smem
  size_t dyn() const { return (size_t)m * sub; }
  bool clc = false;     // ENS_F_CLC: one CTA per instance launched; grid = arena slots
  size_t slot_bm_off = 0;
  int ctas() const { return clc ? (int)kmap.size() : grid * cs / m; }
  uint64_t arena = 0;
  std::vector<uint32_t> kmap;
  std::vector<double> cost;  // app_cost per kmap entry (schedule only)
  size_t kmap_off = 0;
  size_t arena_off = 0;  // this group's arena region (offset from o_arena)
  // split phases (XS): phase 1 = the ensemble kernel with one arena slot per
  // instance (slots = kmap.size()), phase 2 = the lookup-item kernel
  bool split = false;
  std::vector<uint32_t> item_count;  // per kmap entry
  std::vector<int> item_kind;        // per kmap entry: phase-2 kernel (XS grid type)
  std::vector<uint32_t> items;       // group-local instance of each item, by kind
  std::vector<uint32_t> item0;       // per kmap entry: its first item
  uint32_t kind_base[4] = {0, 0, 0, 0}, kind_n[4] = {0, 0, 0, 0};  // kinds: XS grid types 0..2, RS 3
  int grid2[4] = {0, 0, 0, 0};       // phase-2 CTAs per kind
  // phase 1b (hash / nuclide split instances): (instance, nuclide) init items
  std::vector<uint32_t> init_items;  // pairs
  uint64_t init_scr_bytes = 0;       // per init CTA
  int grid3 = 0;
  size_t smem3 = 0;
  size_t init_off = 0, ctr3_off = 0, init_scr_off = 0, isync_off = 0;
  size_t items_off = 0, desc_off = 0, ipart_off = 0, idone_off = 0, ctr2_off = 0;
  size_t slots() const { return split ? kmap.size() : (size_t)grid; }
};

// kernels one launch of group g enqueues: the ensemble kernel, the init items,
// one lookup-item kernel per XS grid type present
static int kernels_of(const Group &g) {
  if (!g.split) return 1;
  return 1 + (g.init_items.empty() ? 0 : 1) + (g.kind_n[0] > 0) + (g.kind_n[1] > 0) + (g.kind_n[2] > 0) +
         (g.kind_n[3] > 0);
}

struct Plan {  // workspace layout (byte offsets) and groups
  int n = 0;
  uint32_t stdout_cap = 4096;
  uint64_t arena_bytes = 0;
  int slots = 0;
  bool concurrent = false;  // groups on forked streams, each with its own arena region
  std::vector<Group> groups;
  std::vector<uint32_t> line_of_k;
  // staged (H2D) part
  size_t o_blob = 0, o_tok = 0, o_line = 0, o_lok = 0, o_kmap = 0, staged = 0;
  // zeroed part: counters (n_groups + 1 u64 stdout total), recs, pos
  size_t o_ctr = 0, o_recs = 0, o_pos = 0, o_phase = 0, o_dump = 0, zeroed_end = 0;
  uint32_t dump_rows = 0;
  size_t o_tal = 0, o_out = 0, o_cmp = 0, o_arena = 0, total = 0;
};

struct ens_run {
  Plan P;
  const ens_args *args_copy_src = nullptr;
  char *ws = nullptr;
  size_t ws_bytes = 0;
  bool owns_ws = false;
  cudaStream_t stream = nullptr;
  char *h_stage = nullptr;
  size_t h_stage_cap = 0;
  // S10 result of this launch, formatted once (ens_collect is called twice by
  // callers that size their stdout buffer first); cleared by enqueue
  bool collected = false, have_tal = false;
  int bad = 0;
  std::vector<ens_record> c_recs;
  std::vector<uint32_t> c_tal;
  std::vector<uint64_t> c_off;
  std::string c_text;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  std::vector<cudaEvent_t> ev_join;  // concurrent groups: one per forked group
  std::vector<cudaEvent_t> ev_fork, ev_fork_join;  // per group: phase 1b fork / join
  struct KTime {                     // one kernel of a launch, bracketed by two events on its stream
    ens_kernel_time info;
    cudaEvent_t a = nullptr, b = nullptr;
  };
  std::vector<KTime> kt;
  uint32_t flags = 0;
  bool launched = false;
  uint64_t d2h = 0;
};

static size_t al(size_t x) { return (x + 255) / 256 * 256; }

// Pinned staging buffers are pooled for the process: cudaHostAlloc /
// cudaFreeHost cost milliseconds each (page pinning and unmapping), which a
// per-launch buffer would pay on every ens_launch.  A buffer returns to the
// pool in ens_run_free, after the stream (and so its H2D copy) is done.
namespace {
std::mutex g_pin_mu;
std::vector<std::pair<size_t, char *>> g_pin_free;
constexpr size_t kPinPoolMax = 8;

cudaError_t pin_get(size_t bytes, char **p, size_t *cap) {
  {
    std::lock_guard<std::mutex> lk(g_pin_mu);
    size_t best = g_pin_free.size();
    for (size_t i = 0; i < g_pin_free.size(); i++)
      if (g_pin_free[i].first >= bytes && (best == g_pin_free.size() || g_pin_free[i].first < g_pin_free[best].first))
        best = i;
    if (best < g_pin_free.size()) {
      *cap = g_pin_free[best].first;
      *p = g_pin_free[best].second;
      g_pin_free.erase(g_pin_free.begin() + (long)best);
      return cudaSuccess;
    }
  }
  size_t c = 64 << 10;
  while (c < bytes) c *= 2;
  cudaError_t e = cudaHostAlloc((void **)p, c, cudaHostAllocDefault);
  *cap = e == cudaSuccess ? c : 0;
  return e;
}

// Device->host result copies go through a non-blocking stream of their own
// (one per device), after the run's end event: a run is collected without
// waiting for work queued behind it on the launch stream (e.g. the next
// launch, or the legacy default stream's implicit synchronisation).
cudaError_t d2h_copy(void *dst, const void *src, size_t bytes) {
  static std::mutex mu;
  static cudaStream_t streams[64] = {};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaMemcpy(dst, src, bytes, cudaMemcpyDeviceToHost);
  cudaStream_t st;
  {
    std::lock_guard<std::mutex> lk(mu);
    if (!streams[dev]) {
      e = cudaStreamCreateWithFlags(&streams[dev], cudaStreamNonBlocking);
      if (e != cudaSuccess) return e;
    }
    st = streams[dev];
  }
  e = cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, st);
  if (e != cudaSuccess) return e;
  return cudaStreamSynchronize(st);
}

// Forked launch streams for concurrent groups: (device, index) -> a
// non-blocking stream, created once per process.
cudaError_t aux_stream(size_t i, cudaStream_t *out) {
  static std::mutex mu;
  static cudaStream_t streams[64][ENS_N_APPS + 1] = {};  // [ENS_N_APPS]: phase 1b
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64 || i > (size_t)ENS_N_APPS) return cudaErrorInvalidValue;
  std::lock_guard<std::mutex> lk(mu);
  if (!streams[dev][i]) {
    e = cudaStreamCreateWithFlags(&streams[dev][i], cudaStreamNonBlocking);
    if (e != cudaSuccess) return e;
  }
  *out = streams[dev][i];
  return cudaSuccess;
}

void pin_put(char *p, size_t cap) {
  if (!p) return;
  {
    std::lock_guard<std::mutex> lk(g_pin_mu);
    if (g_pin_free.size() < kPinPoolMax) {
      g_pin_free.emplace_back(cap, p);
      return;
    }
  }
  cudaFreeHost(p);
}
}  // namespace

static uint32_t app_of_argv0(const char *a0) {
  const char *b = std::strrchr(a0, '/');
  b = b ? b + 1 : a0;
  if (!std::strcmp(b, "echo")) return APP_ECHO;
  if (!std::strcmp(b, "xsbench")) return APP_XSBENCH;
  if (!std::strcmp(b, "rsbench")) return APP_RSBENCH;
  if (!std::strcmp(b, "amgmk")) return APP_AMGMK;
  if (!std::strcmp(b, "pagerank")) return APP_PAGERANK;
  return APP_NOTFOUND;
}

static int threads_for(int32_t t) {
  if (t <= 0) t = 256;
  int T = 32;
  while (T * 2 <= t && T < 1024) T *= 2;
  return T;
}

// Build the plan: groups, geometry, layout.  mem_cap: bytes available for
// the whole workspace (0 = unlimited).
static int make_plan(ens_app app, const ens_args *a, const ens_launch_cfg *c, size_t mem_cap, Plan &P) {
  if (!a || !c) return fail(ENS_EINVAL, "ens_launch: NULL args or cfg");
  if ((uint32_t)app >= ENS_N_APPS) return fail(ENS_EINVAL, "ens_launch: unknown app");
  const int count = ens_args_count(a);
  const int64_t n = c->n_instances, first = c->first, stride = c->stride <= 0 ? 1 : c->stride;
  if (n < 0 || first < 0) return fail(ENS_EINVAL, "ens_launch: negative first / n_instances");
  if (n > 0 && first + (n - 1) * stride >= count)
    return fail(ENS_ERANGE, "ens_launch: instance id beyond the args file (reading Q4)");
  if (c->grid_blocks < 0) return fail(ENS_EINVAL, "ens_launch: negative grid_blocks");
  P.n = (int)n;
  P.stdout_cap = c->stdout_bytes ? (c->stdout_bytes + 7u) / 8u * 8u : 4096u;
  const int T = threads_for(c->block_threads);
  if (c->instances_per_cta < 0) return fail(ENS_EINVAL, "ens_launch: negative instances_per_cta");
  // M instances per CTA: power of two <= 8, >= 32 threads each
  auto m_for = [&](uint32_t ap) {
    const int Ta = std::min(T, app_max_threads(ap));
    int m = 1;
    if (app_sub_aware(ap))
      while (m * 2 <= c->instances_per_cta && m < kMaxSubTeams && Ta / (m * 2) >= 32) m *= 2;
    return m;
  };
  int dev = 0, sms = 148;
  cudaError_t e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceGetAttribute");

  // group instances by app; shared memory per group (independent of team size)
  Group g_by_app[kApps];
  P.line_of_k.resize((size_t)n);
  for (int64_t k = 0; k < n; k++) {
    const uint32_t line = (uint32_t)(first + k * stride);
    P.line_of_k[(size_t)k] = line;
    int argc;
    const char *const *argv;
    ens_args_get(a, (int)line, &argc, &argv);
    uint32_t ap = (uint32_t)app;
    if (app == ENS_APP_BY_ARGV0) ap = argc > 0 ? app_of_argv0(argv[0]) : (uint32_t)APP_NOTFOUND;
    uint64_t ar = 0;
    uint32_t sm = 0;
    app_size(ap, argc, argv, std::min(T, app_max_threads(ap)) / m_for(ap), 1, &ar, &sm);
    Group &g = g_by_app[ap];
    g.app = ap;
    g.smem = std::max(g.smem, sm);
    g.kmap.push_back((uint32_t)k);
    g.cost.push_back(app_cost(ap, argc, argv));
    int kind = 0;
    g.item_count.push_back(app_items(ap, argc, argv, &kind));
    g.item_kind.push_back(kind);
  }
  // longest-first instance queue (LPT): teams pull the heavy instances first
  // and the light ones fill the tail (results are schedule-independent, Q5)
  for (Group &g : g_by_app) {
    if (g.kmap.size() < 2) continue;
    std::vector<uint32_t> ord(g.kmap.size());
    for (size_t x = 0; x < ord.size(); x++) ord[x] = (uint32_t)x;
    std::stable_sort(ord.begin(), ord.end(), [&](uint32_t u, uint32_t v) { return g.cost[u] > g.cost[v]; });
    std::vector<uint32_t> km(ord.size()), ic(ord.size());
    std::vector<int> ik(ord.size());
    std::vector<double> co(ord.size());
    for (size_t x = 0; x < ord.size(); x++)
      km[x] = g.kmap[ord[x]], co[x] = g.cost[ord[x]], ic[x] = g.item_count[ord[x]], ik[x] = g.item_kind[ord[x]];
    g.kmap.swap(km);
    g.cost.swap(co);
    g.item_count.swap(ic);
    g.item_kind.swap(ik);
  }
  // team size: team-aware bodies get a cluster of cs CTAs when the group has
  // fewer instances than resident CTAs (the largest power of two <= 8 with
  // n_group * cs <= resident CTAs), or the cfg's team_ctas
  uint64_t need_arena = 0;
  for (uint32_t ap : {(uint32_t)APP_XSBENCH, (uint32_t)APP_RSBENCH, (uint32_t)APP_AMGMK, (uint32_t)APP_PAGERANK,
                      (uint32_t)APP_ECHO, (uint32_t)APP_NOTFOUND}) {
    Group &g = g_by_app[ap];
    if (g.kmap.empty()) continue;
    g.T = std::min(T, app_max_threads(ap));
    g.m = m_for(ap);
    g.sub = sub_shared_bytes() + (g.smem + 15u) / 16u * 16u;
    int ctas = 0;
    e = group_occupancy(ap, g.T, g.m, 1, g.dyn(), &ctas);
    if (e != cudaSuccess) return cuda_fail(e, "cudaOccupancyMaxActiveBlocksPerMultiprocessor");
    if (ctas <= 0) return fail(ENS_EINVAL, "ens_launch: an instance needs more shared memory than one SM has");
    int cs = 1;
    if (g.m > 1) {  // teams are CTA rows: m slots per resident CTA, grid a multiple of m
      int grid = c->grid_blocks ? c->grid_blocks * g.m : ctas * g.m;
      const int64_t nn = (int64_t)g.kmap.size();
      if (grid > nn) grid = (int)((nn + g.m - 1) / g.m * g.m);
      g.grid = std::max(grid, g.m);
    } else if (app_team_aware(ap) && !(c->flags & ENS_F_CLC)) {
      if (c->team_ctas > 0) {
        cs = (int)std::min<uint32_t>(c->team_ctas, (uint32_t)kMaxTeamCtas);  // any cluster size up to the cap
      } else if (!c->grid_blocks) {
        while (cs < kMaxTeamCtas && (int64_t)g.kmap.size() * cs * 2 <= ctas) cs *= 2;
        // uneven ensembles: a team large enough that the heaviest instance
        // ends within one CTA's fair share of the total work
        double tot = 0.0, mx = 0.0;
        for (double w : g.cost) tot += w, mx = std::max(mx, w);
        const double fair = tot / (double)std::min<int64_t>((int64_t)ctas, (int64_t)g.kmap.size());
        while (cs < kMaxTeamCtas && mx > 1.5 * fair * cs) cs *= 2;
      }
    }
    if (g.m == 1) {
      int teams = ctas;
      if (cs > 1) {
        e = group_occupancy(ap, g.T, 1, cs, g.dyn(), &teams);
        if (e != cudaSuccess) return cuda_fail(e, "cudaOccupancyMaxActiveClusters");
        if (teams <= 0) cs = 1, teams = ctas;
        // an automatic team size whose clusters cannot all be resident at once (a GPC holds only
        // so many 16- or 8-CTA clusters) would run the ensemble in two waves: shrink it (any
        // size, not only powers of two) until every instance has a resident team (XS at N = 8:
        // 0.47 ms on 7 16-CTA teams)
        while (!c->team_ctas && !c->grid_blocks && cs > 1 && (int64_t)teams < (int64_t)g.kmap.size()) {
          cs -= 1;
          teams = ctas;
          if (cs > 1) {
            e = group_occupancy(ap, g.T, 1, cs, g.dyn(), &teams);
            if (e != cudaSuccess) return cuda_fail(e, "cudaOccupancyMaxActiveClusters");
            if (teams <= 0) cs = 1, teams = ctas;
          }
        }
      }
      int grid = c->grid_blocks ? std::max(1, c->grid_blocks / cs) : teams;
      grid = (int)std::min<int64_t>(grid, (int64_t)g.kmap.size());
      g.grid = std::max(grid, 1);
    }
    g.cs = cs;
    g.clc = (c->flags & ENS_F_CLC) && g.m == 1 && cs == 1;
    for (uint32_t k : g.kmap) {  // arena of this team size
      int argc;
      const char *const *argv;
      ens_args_get(a, (int)P.line_of_k[k], &argc, &argv);
      uint64_t ar = 0;
      uint32_t sm = 0;
      app_size(ap, argc, argv, g.T / g.m, cs, &ar, &sm);
      g.arena = std::max(g.arena, ar);
    }
    need_arena = std::max(need_arena, g.arena);
    // split phases when some instance has lookup items (and arenas are host-sized:
    // a caller's smaller arena_bytes could make an instance exit NOMEM in phase 1)
    if (!(c->flags & ENS_F_FUSED) && !c->arena_bytes) {
      // items grouped by kind (one phase-2 kernel each), instances in queue order within a kind
      g.item0.assign(g.kmap.size(), 0);
      for (int kd = 0; kd < 4; kd++) {
        g.kind_base[kd] = (uint32_t)g.items.size();
        for (size_t x = 0; x < g.kmap.size(); x++) {
          if (g.item_kind[x] != kd || !g.item_count[x]) continue;
          g.item0[x] = (uint32_t)g.items.size();
          for (uint32_t b = 0; b < g.item_count[x]; b++) g.items.push_back((uint32_t)x);
        }
        g.kind_n[kd] = (uint32_t)g.items.size() - g.kind_base[kd];
        if (g.kind_n[kd]) {
          e = xs_items_occupancy(kd, &g.grid2[kd]);
          if (e != cudaSuccess) return cuda_fail(e, "cudaOccupancyMaxActiveBlocksPerMultiprocessor (phase 2)");
        }
      }
      // split when it pays (measured): fewer instances than
      // resident CTAs (phase 1 alone would leave SMs idle) and enough items to
      // fill every phase-2 CTA.  C2 45.1 -> 38.2 ms, C2u 66.2 -> 62.9 ms;
      // TSTAR (1024 instances) and C1 (12 items) stay fused.
      int fill = 0;
      for (int kd = 0; kd < 4; kd++) fill = std::max(fill, g.grid2[kd]);
      // RS groups, and XS groups with per-nuclide table items (hash / nuclide grids) whose
      // instances are not small, split at any instance count: the item kernels' read-only
      // loads, register budgets and all-SM table builds beat the fused body (C5's 1024 RS lines:
      // 26.1 -> 23.7 ms; 300 C2 lines: 240 -> 128 ms; 600 small 11303-point lines with 200k
      // lookups: 42.6 -> 29.9 ms) — but 1024 small 1000-point lines with 10k lookups run fused
      // faster (6.8 vs 7.3 ms): XS groups below an average app_cost of 2^20 stay fused;
      // unionized XS groups split only below the resident CTAs (T*: 8.94 split vs 8.92 fused)
      double mean_cost = 0.0;
      for (double w : g.cost) mean_cost += w;
      mean_cost /= std::max<size_t>(1, g.cost.size());
      bool any_init = false;
      if (ap == APP_XSBENCH && mean_cost >= 1048576.0)
        for (size_t x = 0; x < g.kmap.size() && !any_init; x++) {
          int argc;
          const char *const *argv;
          ens_args_get(a, (int)P.line_of_k[g.kmap[x]], &argc, &argv);
          int ni = 0, ns = 0, nf = 0;
          uint32_t sm3 = 0;
          app_init_scratch(ap, argc, argv, &ni, &ns, &nf, &sm3);
          any_init = ni > 0;
        }
      g.split = !g.items.empty() && (((c->flags & ENS_F_SPLIT_PHASES) != 0) ||
                                     (((int64_t)g.kmap.size() < (int64_t)ctas || ap == APP_RSBENCH || any_init) &&
                                      (int64_t)g.items.size() >= fill));
      if (!g.split) {
        g.items.clear();
        for (int kd = 0; kd < 4; kd++) g.kind_n[kd] = 0;
      }
      if (g.split) {  // phase 1b: the lookup sorts' items and the (instance, nuclide) table items
        // queue: count items, a share of the nuclide items (the scans finish
        // meanwhile), scatter items, another share, fine items, the rest
        std::vector<uint32_t> count_items, scatter_items, fine_items, nuc_items;
        uint32_t smem_need = 0;
        auto pair = [](std::vector<uint32_t> &v, size_t x, uint32_t i) {
          v.push_back((uint32_t)x);
          v.push_back(i);
        };
        for (size_t x = 0; x < g.kmap.size(); x++) {
          int argc;
          const char *const *argv;
          ens_args_get(a, (int)P.line_of_k[g.kmap[x]], &argc, &argv);
          int ni = 0, ns = 0, nf = 0;
          uint32_t sm3 = 0;
          const uint64_t scr = app_init_scratch(ap, argc, argv, &ni, &ns, &nf, &sm3);
          if (!g.item_count[x] || !ni) continue;
          g.init_scr_bytes = std::max<uint64_t>(g.init_scr_bytes, al(scr));
          smem_need = std::max(smem_need, sm3);
          for (int q = 0; q < ns; q++) pair(count_items, x, kXsCountItem | (uint32_t)q);
          for (int q = 0; q < ns; q++) pair(scatter_items, x, kXsScatterItem | (uint32_t)q);
          for (int q = 0; q < nf; q++) pair(fine_items, x, kXsFineItem | (uint32_t)q);
          for (int i = 0; i < ni; i++) pair(nuc_items, x, (uint32_t)i);
        }
        const size_t share = (size_t)2 * 2 * (size_t)std::max(1, (int)ctas);  // pairs: 2 x ctas items
        const size_t f1 = std::min(nuc_items.size(), share), f2 = std::min(nuc_items.size(), 2 * share);
        g.init_items = count_items;
        g.init_items.insert(g.init_items.end(), nuc_items.begin(), nuc_items.begin() + f1);
        g.init_items.insert(g.init_items.end(), scatter_items.begin(), scatter_items.end());
        g.init_items.insert(g.init_items.end(), nuc_items.begin() + f1, nuc_items.begin() + f2);
        g.init_items.insert(g.init_items.end(), fine_items.begin(), fine_items.end());
        g.init_items.insert(g.init_items.end(), nuc_items.begin() + f2, nuc_items.end());
        if (!g.init_items.empty()) {
          g.smem3 = xs_init_smem_off() + (smem_need + 15u) / 16u * 16u;
          e = xs_init_items_occupancy(kXsInitThreads, g.smem3, &g.grid3);
          if (e != cudaSuccess) return cuda_fail(e, "cudaOccupancyMaxActiveBlocksPerMultiprocessor (phase 1b)");
          if (g.grid3 <= 0) return fail(ENS_EINVAL, "ens_launch: init items need more shared memory than an SM has");
          g.grid3 = std::max(1, std::min<int>(g.grid3, (int)(g.init_items.size() / 2)));
        }
      }
    }
    P.groups.push_back(g);
  }
  P.arena_bytes = c->arena_bytes ? al(c->arena_bytes) : al(need_arena);
  size_t o = 0;
  auto layout = [&]() {
  o = 0;
  // staged part
  P.o_blob = o; o = al(o + a->blob.size());
  P.o_tok = o; o = al(o + a->tok_off.size() * 4);
  P.o_line = o; o = al(o + a->line_tok.size() * 4);
  P.o_lok = o; o = al(o + (size_t)n * 4);
  P.o_kmap = o;
  for (Group &g : P.groups) {
    g.kmap_off = o;
    o += g.kmap.size() * 4;
  }
  o = al(o);
  for (Group &g : P.groups) {  // split phases: item table, descriptors (item0 / n_items pre-filled)
    if (!g.split) continue;
    g.items_off = o; o = al(o + g.items.size() * 4);
    g.desc_off = o; o = al(o + g.kmap.size() * kDescBytes);
    g.init_off = o; o = al(o + g.init_items.size() * 4);
  }
  P.staged = o;
  // zeroed part
  P.o_ctr = o; o = al(o + (P.groups.size() + 1) * 8);
  for (Group &g : P.groups) {  // ENS_F_CLC: arena-slot pool bitmaps
    if (!g.clc) continue;
    g.slot_bm_off = o; o = al(o + ((size_t)g.grid + 31) / 32 * 4);
  }
  for (Group &g : P.groups) {
    if (!g.split) continue;
    g.ctr2_off = o; o = al(o + 4 * 8);
    g.ctr3_off = o; o = al(o + 8);
    g.idone_off = o; o = al(o + g.kmap.size() * 4);
    if (!g.init_items.empty()) g.isync_off = o, o = al(o + g.kmap.size() * kInitSyncBytes);
  }
  P.o_recs = o; o = al(o + (size_t)n * sizeof(ens_record));
  P.o_pos = o; o = al(o + (size_t)n * 8);
  P.o_phase = o; o = al(o + ENS_PHASES * 8);
  P.dump_rows = c->dump_rows;
  P.o_dump = o; o = al(o + (size_t)n * c->dump_rows * 64);  // unwritten rows read as zero
  P.zeroed_end = o;
  P.o_tal = o; o = al(o + (size_t)n * ENS_TALLIES * 4);
  P.o_out = o; o = al(o + (size_t)n * P.stdout_cap);
  P.o_cmp = o; o = al(o + (size_t)n * P.stdout_cap);
  for (Group &g : P.groups) {
    if (!g.split) continue;
    g.ipart_off = o; o = al(o + g.items.size() * kPartBytes);
    g.init_scr_off = o; o = al(o + (size_t)g.grid3 * g.init_scr_bytes);
  }
  P.o_arena = o;
  };
  layout();
  // split groups keep one arena slot per instance: only when that fits
  if (mem_cap) {
    size_t need = o;
    for (const Group &g : P.groups) need += g.slots() * (size_t)P.arena_bytes;
    if (need > mem_cap) {
      for (Group &g : P.groups) g.split = false;
      layout();
    }
  }
  int want = 0;
  for (const Group &g : P.groups) want = std::max(want, (int)g.slots());
  if (P.arena_bytes && mem_cap) {
    if (mem_cap < o + P.arena_bytes) return fail(ENS_ENOMEM, "ens_launch: workspace cannot hold one arena slot");
    const uint64_t fit = (mem_cap - o) / P.arena_bytes;
    if ((uint64_t)want > fit) {
      if (c->grid_blocks) return fail(ENS_ENOMEM, "ens_launch: grid_blocks x arena does not fit the workspace");
      want = (int)fit;
      for (Group &g : P.groups) {
        if (g.split) return fail(ENS_ENOMEM, "ens_launch: split-phase arena slots do not fit the workspace");
        g.grid = std::min(g.grid, want / g.m * g.m);  // whole CTAs of m slots
        if (g.grid <= 0)
          return fail(ENS_ENOMEM, "ens_launch: workspace cannot hold one CTA of instances_per_cta arena slots");
      }
    }
  }
  P.slots = want;
  P.total = o + (size_t)want * P.arena_bytes;
  // several groups: give each its own arena region (slots x arena_bytes) so
  // their kernels may run concurrently, when that fits the workspace cap
  if (P.groups.size() > 1 && !(c->flags & ENS_F_SERIAL)) {
    size_t off = 0;
    for (const Group &g : P.groups) off += g.slots() * P.arena_bytes;
    if (!mem_cap || o + off <= mem_cap) {
      off = 0;
      for (Group &g : P.groups) {
        g.arena_off = off;
        off += g.slots() * P.arena_bytes;
      }
      P.concurrent = true;
      P.total = o + off;
    }
  }
  return ENS_OK;
}

static size_t free_device_bytes() {
  size_t fr = 0, tot = 0;
  if (cudaMemGetInfo(&fr, &tot) != cudaSuccess) return 0;
  return fr > (512u << 20) ? fr - (512u << 20) : fr / 2;  // leave headroom
}

extern "C" int ens_workspace_bytes(ens_app app, const ens_args *a, const ens_launch_cfg *c, size_t *bytes) {
  if (!bytes) return fail(ENS_EINVAL, "ens_workspace_bytes: NULL");
  Plan P;
  int rc = make_plan(app, a, c, c && c->grid_blocks ? 0 : free_device_bytes(), P);
  if (rc) return rc;
  *bytes = P.total;
  return ENS_OK;
}

static int enqueue(ens_run *r) {
  const Plan &P = r->P;
  r->collected = r->have_tal = false;
  CU(cudaMemsetAsync(r->ws + P.o_ctr, 0, P.zeroed_end - P.o_ctr, r->stream));
  CU(cudaEventRecord(r->ev0, r->stream));
  for (size_t gi = 0; gi < P.groups.size(); gi++) {
    const Group &g = P.groups[gi];
    KParams k{};
    k.blob = r->ws + P.o_blob;
    k.tok_off = (const uint32_t *)(r->ws + P.o_tok);
    k.line_tok = (const uint32_t *)(r->ws + P.o_line);
    k.kmap = (const uint32_t *)(r->ws + g.kmap_off);
    k.line_of_k = (const uint32_t *)(r->ws + P.o_lok);
    k.n = (uint32_t)g.kmap.size();
    k.flags = r->flags;
    k.counter = (uint32_t *)(r->ws + P.o_ctr + 8 * gi);
    k.stdout_total = (unsigned long long *)(r->ws + P.o_ctr + 8 * P.groups.size());
    k.recs = (ens_record *)(r->ws + P.o_recs);
    k.stdout_pos = (unsigned long long *)(r->ws + P.o_pos);
    k.tallies = (uint32_t *)(r->ws + P.o_tal);
    k.stdout_base = r->ws + P.o_out;
    k.stdout_cmp = r->ws + P.o_cmp;
    k.stdout_cap = P.stdout_cap;
    k.arena_bytes = P.arena_bytes;
    k.team_ctas = (uint32_t)g.cs;
    k.phases = (r->flags & ENS_F_PHASES) ? (unsigned long long *)(r->ws + P.o_phase) : nullptr;
    k.sub_stride = g.sub;
    k.arena_base = r->ws + P.o_arena + g.arena_off;
    k.dump = P.dump_rows ? (double *)(r->ws + P.o_dump) : nullptr;
    k.dump_rows = P.dump_rows;
    k.split = g.split ? 1u : 0u;
    k.clc = g.clc ? 1u : 0u;
    k.slot_bm = g.clc ? (uint32_t *)(r->ws + g.slot_bm_off) : nullptr;
    k.n_slots = (uint32_t)g.grid;
    if (g.split) {
      k.xs_desc = r->ws + g.desc_off;
      k.items = (const uint32_t *)(r->ws + g.items_off);
      k.n_items = (uint32_t)g.items.size();
      k.ipart = r->ws + g.ipart_off;
      k.idone = (uint32_t *)(r->ws + g.idone_off);
      k.counter2 = (uint32_t *)(r->ws + g.ctr2_off);
      k.init_items = (const uint32_t *)(r->ws + g.init_off);
      k.n_init_items = (uint32_t)(g.init_items.size() / 2);
      k.counter3 = (uint32_t *)(r->ws + g.ctr3_off);
      k.init_scr = r->ws + g.init_scr_off;
      k.init_scr_bytes = g.init_scr_bytes;
      k.init_smem_off = xs_init_smem_off();
      k.init_sync = g.init_items.empty() ? nullptr : r->ws + g.isync_off;
    }
    cudaStream_t st = r->stream;
    if (P.concurrent && gi > 0) {  // fork: group gi on an aux stream after ev0
      CU(aux_stream(gi - 1, &st));
      CU(cudaStreamWaitEvent(st, r->ev0, 0));
    }
    size_t nk = 0;  // kernels of this launch so far (r->kt grows on the first enqueue)
    for (size_t q = 0; q < gi; q++) nk += kernels_of(P.groups[q]);
    auto kt_begin = [&](int phase, int kind, int grid, int block) -> int {
      if (r->kt.size() <= nk) {
        ens_run::KTime t;
        if (cudaEventCreate(&t.a) != cudaSuccess || cudaEventCreate(&t.b) != cudaSuccess) return -1;
        r->kt.push_back(t);
      }
      ens_kernel_time &i = r->kt[nk].info;
      i.app = (int32_t)(g.app == APP_NOTFOUND ? 0u : g.app);
      i.phase = phase;
      i.kind = kind;
      i.grid_ctas = grid;
      i.block_threads = block;
      i.ms = 0.f;
      return cudaEventRecord(r->kt[nk].a, st) == cudaSuccess ? 0 : -1;
    };
    auto kt_end = [&]() -> int { return cudaEventRecord(r->kt[nk++].b, st) == cudaSuccess ? 0 : -1; };
    cudaStream_t st3 = nullptr;
    if (g.split && !g.init_items.empty()) {  // phase 1b beside phase 1: fork after this group's start
      CU(aux_stream(ENS_N_APPS, &st3));
      CU(cudaEventRecord(r->ev_fork[gi], st));
      CU(cudaStreamWaitEvent(st3, r->ev_fork[gi], 0));
      std::swap(st, st3);
      if (kt_begin(3, -1, g.grid3, kXsInitThreads)) return fail(ENS_ECUDA, "ens_launch: kernel timing events");
      cudaError_t e3 = launch_xs_init_items(g.grid3, kXsInitThreads, g.smem3, k, st);
      if (e3 != cudaSuccess) return cuda_fail(e3, "xs_init_items_kernel launch");
      if (kt_end()) return fail(ENS_ECUDA, "ens_launch: kernel timing events");
      CU(cudaEventRecord(r->ev_fork_join[gi], st));
      std::swap(st, st3);
    }
    if (kt_begin(1, -1, g.ctas(), g.T)) return fail(ENS_ECUDA, "ens_launch: kernel timing events");
    cudaError_t e = launch_group(g.app, g.T, g.m, g.ctas(), g.cs, g.dyn(), k, st);
    if (e != cudaSuccess) return cuda_fail(e, "ens_kernel launch");
    if (kt_end()) return fail(ENS_ECUDA, "ens_launch: kernel timing events");
    if (st3) CU(cudaStreamWaitEvent(st, r->ev_fork_join[gi], 0));  // phase 2 after both
    for (int kd = 0; g.split && kd < 4; kd++) {  // phase 2: every instance's lookup items, on every SM
      if (!g.kind_n[kd]) continue;
      const int ctas2 = std::max(1, std::min<int>(g.grid2[kd], (int)g.kind_n[kd]));
      KParams k2 = k;
      k2.item_base = g.kind_base[kd];
      k2.n_items = g.kind_n[kd];
      k2.counter2 = (uint32_t *)(r->ws + g.ctr2_off + 8 * kd);
      if (kt_begin(2, kd, ctas2, xs_items_threads(kd))) return fail(ENS_ECUDA, "ens_launch: kernel timing events");
      e = launch_xs_items(kd, ctas2, k2, st);
      if (e != cudaSuccess) return cuda_fail(e, "xs_items_kernel launch");
      if (kt_end()) return fail(ENS_ECUDA, "ens_launch: kernel timing events");
    }
    if (P.concurrent && gi > 0) {  // join back into the launch stream
      CU(cudaEventRecord(r->ev_join[gi - 1], st));
      CU(cudaStreamWaitEvent(r->stream, r->ev_join[gi - 1], 0));
    }
  }
  CU(cudaEventRecord(r->ev1, r->stream));
  r->launched = true;
  return ENS_OK;
}

extern "C" int ens_launch(ens_app app, const ens_args *a, const ens_launch_cfg *c, void *d_workspace, size_t ws_bytes,
                          void *cuda_stream, ens_run **out) {
  if (!out) return fail(ENS_EINVAL, "ens_launch: NULL out");
  *out = nullptr;
  ens_run *r = new ens_run();
  r->stream = (cudaStream_t)cuda_stream;
  r->flags = c ? c->flags : 0;
  const size_t cap = d_workspace ? ws_bytes : (c && c->grid_blocks ? 0 : free_device_bytes());
  int rc = make_plan(app, a, c, cap, r->P);
  if (rc) {
    delete r;
    return rc;
  }
  Plan &P = r->P;
  if (d_workspace) {
    if (ws_bytes < P.total) {
      delete r;
      return fail(ENS_ENOMEM, "ens_launch: ws_bytes < ens_workspace_bytes");
    }
    r->ws = (char *)d_workspace;
    r->ws_bytes = ws_bytes;
  } else if (P.n > 0) {
    cudaError_t e = cudaMalloc(&r->ws, P.total);
    if (e != cudaSuccess) {
      delete r;
      return fail(ENS_ENOMEM, std::string("ens_launch: cudaMalloc: ") + cudaGetErrorString(e));
    }
    r->owns_ws = true;
    r->ws_bytes = P.total;
  }
  cudaError_t e = cudaEventCreate(&r->ev0);
  if (e == cudaSuccess) e = cudaEventCreate(&r->ev1);
  if (P.concurrent)
    for (size_t gi = 1; gi < P.groups.size() && e == cudaSuccess; gi++) {
      cudaEvent_t ej = nullptr;
      e = cudaEventCreateWithFlags(&ej, cudaEventDisableTiming);
      if (e == cudaSuccess) r->ev_join.push_back(ej);
    }
  for (size_t gi = 0; gi < P.groups.size() && e == cudaSuccess; gi++) {
    cudaEvent_t a = nullptr, b = nullptr;
    e = cudaEventCreateWithFlags(&a, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&b, cudaEventDisableTiming);
    r->ev_fork.push_back(a);
    r->ev_fork_join.push_back(b);
  }
  if (e != cudaSuccess) {
    ens_run_free(r);
    return cuda_fail(e, "cudaEventCreate");
  }
  *out = r;
  if (P.n == 0) return ENS_OK;
  // one pinned staging buffer, one H2D copy
  e = pin_get(P.staged, &r->h_stage, &r->h_stage_cap);
  if (e != cudaSuccess) {
    *out = nullptr;
    ens_run_free(r);
    return cuda_fail(e, "cudaHostAlloc");
  }
  std::memset(r->h_stage, 0, P.staged);
  std::memcpy(r->h_stage + P.o_blob, a->blob.data(), a->blob.size());
  std::memcpy(r->h_stage + P.o_tok, a->tok_off.data(), a->tok_off.size() * 4);
  std::memcpy(r->h_stage + P.o_line, a->line_tok.data(), a->line_tok.size() * 4);
  std::memcpy(r->h_stage + P.o_lok, P.line_of_k.data(), P.line_of_k.size() * 4);
  for (const Group &g : P.groups) std::memcpy(r->h_stage + g.kmap_off, g.kmap.data(), g.kmap.size() * 4);
  for (const Group &g : P.groups) {
    if (!g.split) continue;
    std::memcpy(r->h_stage + g.items_off, g.items.data(), g.items.size() * 4);
    if (!g.init_items.empty()) std::memcpy(r->h_stage + g.init_off, g.init_items.data(), g.init_items.size() * 4);
    for (size_t x = 0; x < g.kmap.size(); x++) {  // phase 1 fills the rest of each descriptor
      char *dp = r->h_stage + g.desc_off + x * kDescBytes;
      if (g.app == APP_RSBENCH) {
        reinterpret_cast<RsDesc *>(dp)->item0 = g.item0[x];
        reinterpret_cast<RsDesc *>(dp)->n_items = g.item_count[x];
      } else {
        reinterpret_cast<XsDesc *>(dp)->item0 = g.item0[x];
        reinterpret_cast<XsDesc *>(dp)->n_items = g.item_count[x];
      }
    }
  }
  e = cudaMemcpyAsync(r->ws, r->h_stage, P.staged, cudaMemcpyHostToDevice, r->stream);
  if (e != cudaSuccess) {
    *out = nullptr;
    ens_run_free(r);
    return cuda_fail(e, "cudaMemcpyAsync H2D");
  }
  rc = enqueue(r);
  if (rc) {
    *out = nullptr;
    ens_run_free(r);
  }
  return rc;
}

extern "C" int ens_run_relaunch(ens_run *r, void *cuda_stream) {
  if (!r) return fail(ENS_EINVAL, "ens_run_relaunch: NULL");
  if (cuda_stream) r->stream = (cudaStream_t)cuda_stream;
  if (r->P.n == 0) return ENS_OK;
  return enqueue(r);
}

// ---------------------------------------------------------------------------
// S10: collect
// ---------------------------------------------------------------------------
extern "C" int ens_collect(ens_run *r, ens_record *recs, uint32_t *tallies, char *stdout_buf, size_t cap,
                           uint64_t *stdout_off) {
  if (!r) return fail(ENS_EINVAL, "ens_collect: NULL run");
  const Plan &P = r->P;
  const int n = P.n;
  if (n == 0) {
    if (stdout_off) stdout_off[0] = 0;
    return ENS_OK;
  }
  if (!r->collected) {
    CU(cudaEventSynchronize(r->ev1));
    CU(cudaGetLastError());
    r->d2h = 0;
    // counters | records | stdout positions | tallies (contiguous: o_tal ==
    // zeroed_end): one copy into a pooled pinned buffer, then the compacted
    // raw stdout: a second copy
    const size_t head = P.o_tal + (size_t)n * ENS_TALLIES * 4 - P.o_ctr;
    char *hb = nullptr;
    size_t hb_cap = 0;
    CU(pin_get(head, &hb, &hb_cap));
    cudaError_t ce = d2h_copy(hb, r->ws + P.o_ctr, head);
    if (ce != cudaSuccess) {
      pin_put(hb, hb_cap);
      return cuda_fail(ce, "ens_collect: D2H");
    }
    r->d2h += head;
    const uint64_t total = *(const uint64_t *)(hb + 8 * P.groups.size());
    std::vector<ens_record> &R = r->c_recs;
    R.resize((size_t)n);
    std::memcpy(R.data(), hb + (P.o_recs - P.o_ctr), (size_t)n * sizeof(ens_record));
    std::vector<uint64_t> posv((size_t)n);
    std::memcpy(posv.data(), hb + (P.o_pos - P.o_ctr), (size_t)n * 8);
    const uint64_t *pos = posv.data();
    r->c_tal.resize((size_t)n * ENS_TALLIES);
    std::memcpy(r->c_tal.data(), hb + (P.o_tal - P.o_ctr), (size_t)n * ENS_TALLIES * 4);
    r->have_tal = true;
    const char *cmp = hb;
    if (total > hb_cap) {
      pin_put(hb, hb_cap);
      hb = nullptr;
      ce = pin_get(total, &hb, &hb_cap);
      if (ce != cudaSuccess) return cuda_fail(ce, "ens_collect: cudaHostAlloc");
      cmp = hb;
    }
    if (total) ce = d2h_copy(hb, r->ws + P.o_cmp, (size_t)total);
    if (ce != cudaSuccess) {
      pin_put(hb, hb_cap);
      return cuda_fail(ce, "ens_collect: D2H stdout");
    }
    r->d2h += total;
    std::string &text = r->c_text;
    text.clear();
    std::vector<uint64_t> &off = r->c_off;
    off.assign((size_t)n + 1, 0);
    int bad = 0;
    for (int k = 0; k < n; k++) {
      ens_record &x = R[(size_t)k];
      if (!(x.flags & ENS_RF_DONE)) {  // never completed
        std::memset(&x, 0, sizeof x);
        x.instance = P.line_of_k[(size_t)k];
        x.flags = ENS_RF_NOT_RUN;
      } else if (x.stdout_len) {
        const size_t before = text.size();
        if (pos[k] + x.stdout_len > total || format_raw(cmp + pos[k], x.stdout_len, text) < 0) {
          bad++;
          text.resize(before);
        }
        x.stdout_len = (uint32_t)(text.size() - before);
      }
      off[(size_t)k + 1] = text.size();
    }
    pin_put(hb, hb_cap);
    r->bad = bad;
    r->collected = true;
  }
  if (tallies && !r->have_tal) {
    r->c_tal.resize((size_t)n * ENS_TALLIES);
    CU(d2h_copy(r->c_tal.data(), r->ws + P.o_tal, (size_t)n * ENS_TALLIES * 4));
    r->d2h += (size_t)n * ENS_TALLIES * 4;
    r->have_tal = true;
  }
  if (tallies) std::memcpy(tallies, r->c_tal.data(), r->c_tal.size() * 4);
  const std::vector<ens_record> &R = r->c_recs;
  const std::vector<uint64_t> &off = r->c_off;
  const std::string &text = r->c_text;
  const int bad = r->bad;
  if (recs) std::memcpy(recs, R.data(), R.size() * sizeof(ens_record));
  if (stdout_off) std::memcpy(stdout_off, off.data(), off.size() * 8);
  if (bad) return fail(ENS_ECUDA, "ens_collect: malformed device stdout records");
  if (stdout_buf) {
    if (cap < text.size()) return fail(ENS_ERANGE, "ens_collect: stdout buffer too small");
    std::memcpy(stdout_buf, text.data(), text.size());
  }
  return ENS_OK;
}

extern "C" int ens_collect_dump(ens_run *r, double *out, size_t cap) {
  if (!r || (!out && cap)) return fail(ENS_EINVAL, "ens_collect_dump: NULL");
  const Plan &P = r->P;
  if (!P.dump_rows) return fail(ENS_EINVAL, "ens_collect_dump: launched with dump_rows = 0");
  const size_t want = (size_t)P.n * P.dump_rows * 8;
  if (cap < want) return fail(ENS_ERANGE, "ens_collect_dump: cap < n x dump_rows x 8");
  if (P.n == 0 || !r->launched) return ENS_OK;
  CU(cudaEventSynchronize(r->ev1));
  CU(d2h_copy(out, r->ws + P.o_dump, want * 8));
  return ENS_OK;
}

extern "C" int ens_run_phases(ens_run *r, uint64_t ns[ENS_PHASES]) {
  if (!r || !ns) return fail(ENS_EINVAL, "ens_run_phases: NULL");
  std::memset(ns, 0, sizeof(uint64_t) * ENS_PHASES);
  if (r->P.n == 0 || !r->launched) return ENS_OK;
  if (!(r->flags & ENS_F_PHASES)) return fail(ENS_EINVAL, "ens_run_phases: launched without ENS_F_PHASES");
  CU(cudaStreamSynchronize(r->stream));
  CU(cudaMemcpy(ns, r->ws + r->P.o_phase, sizeof(uint64_t) * ENS_PHASES, cudaMemcpyDeviceToHost));
  return ENS_OK;
}

extern "C" int ens_run_elapsed_ms(ens_run *r, float *ms) {
  if (!r || !ms) return fail(ENS_EINVAL, "ens_run_elapsed_ms: NULL");
  if (!r->launched) {
    *ms = 0.f;
    return ENS_OK;
  }
  cudaError_t e = cudaEventQuery(r->ev1);
  if (e == cudaErrorNotReady) return fail(ENS_EBUSY, "ens_run_elapsed_ms: not finished");
  CU(cudaEventElapsedTime(ms, r->ev0, r->ev1));
  return ENS_OK;
}

extern "C" int ens_run_kernel_times(ens_run *r, ens_kernel_time *out, int cap) {
  if (!r || (!out && cap)) return fail(ENS_EINVAL, "ens_run_kernel_times: NULL");
  if (!r->launched || r->P.n == 0) return 0;
  CU(cudaEventSynchronize(r->ev1));
  int n = 0;
  for (int q = 0; q < (int)r->P.groups.size(); q++) {
    const Group &g = r->P.groups[q];
    n += kernels_of(g);
  }
  if (cap < n) return fail(ENS_ERANGE, "ens_run_kernel_times: cap smaller than the kernel count");
  for (int q = 0; q < n; q++) {
    ens_kernel_time t = r->kt[(size_t)q].info;
    CU(cudaEventElapsedTime(&t.ms, r->kt[(size_t)q].a, r->kt[(size_t)q].b));
    out[q] = t;
  }
  return n;
}

extern "C" int ens_run_get_info(const ens_run *r, ens_run_info *info) {
  if (!r || !info) return fail(ENS_EINVAL, "ens_run_get_info: NULL");
  std::memset(info, 0, sizeof *info);
  const Plan &P = r->P;
  info->n_instances = P.n;
  info->n_groups = (int32_t)P.groups.size();
  for (const Group &g : P.groups) {
    const uint32_t ap = g.app == APP_NOTFOUND ? 0u : g.app;
    info->grid_blocks[ap] = g.ctas();
    info->team_ctas[ap] = g.cs;
    info->instances_per_cta[ap] = g.m;
    info->block_threads[ap] = g.T;
  }
  info->kernel_launches = (int32_t)P.groups.size();
  info->kernel_launches = 0;
  for (const Group &g : P.groups) info->kernel_launches += kernels_of(g);
  info->arena_bytes = P.arena_bytes;
  info->ws_bytes = r->ws_bytes;
  info->records_offset = P.o_recs;
  info->tallies_offset = P.o_tal;
  info->stdout_offset = P.o_out;
  info->stdout_bytes = P.stdout_cap;
  info->h2d_bytes = P.n ? P.staged : 0;
  info->d2h_bytes = r->d2h;
  return ENS_OK;
}

extern "C" long ens_format_stdout(uint32_t app, const void *raw, size_t raw_len, char *out, size_t cap) {
  (void)app;
  std::string s;
  long k = format_raw(raw, raw_len, s);
  if (k < 0) return fail(ENS_EINVAL, "ens_format_stdout: malformed records");
  if (out) std::memcpy(out, s.data(), std::min(cap, s.size()));
  return (long)s.size();
}

extern "C" void ens_run_free(ens_run *r) {
  if (!r) return;
  if (r->launched)
    cudaEventSynchronize(r->ev1);  // the run's own work (H2D, kernels) is done
  else if (r->h_stage)
    cudaStreamSynchronize(r->stream);  // a failed enqueue may leave the H2D in flight
  if (r->owns_ws && r->ws) cudaFree(r->ws);
  pin_put(r->h_stage, r->h_stage_cap);
  if (r->ev0) cudaEventDestroy(r->ev0);
  if (r->ev1) cudaEventDestroy(r->ev1);
  for (cudaEvent_t ej : r->ev_join) cudaEventDestroy(ej);
  for (cudaEvent_t ej : r->ev_fork) if (ej) cudaEventDestroy(ej);
  for (cudaEvent_t ej : r->ev_fork_join) if (ej) cudaEventDestroy(ej);
  for (auto &t : r->kt) {
    cudaEventDestroy(t.a);
    cudaEventDestroy(t.b);
  }
  delete r;
}

extern "C" const char *ens_strerror(int err) {
  switch (err) {
    case ENS_OK: return "ok";
    case ENS_EINVAL: return "invalid argument";
    case ENS_ENOENT: return "args file not found";
    case ENS_ENOMEM: return "out of memory";
    case ENS_ECUDA: return "CUDA error";
    case ENS_ERANGE: return "out of range";
    case ENS_EBUSY: return "busy";
    case ENS_EPARSE: return "parse error";
  }
  return "unknown error";
}

extern "C" const char *ens_last_error(void) { return g_err.c_str(); }
extern "C" const char *ens_version(void) { return "ens 0.1.0 (sm_100a)"; }
