// csrc/apps/params.cuh — S5 (instance CLI parse) and the arena / shared-
// memory layout of every app, compiled for BOTH host and device: the host
// sizes the slot arenas and the dynamic shared memory from exactly the code
// the instance runs, so a valid line can never run out of arena.
//
// Flag grammars follow SURVEY.md §8(c) XS-1 / RS-1 / AMG-1; an unknown flag,
// a missing value or a bad value makes the instance print the usage text and
// exit 1 (the paper's loader passes each line to the app's own main,
// Fig. 4).
#pragma once
#include "../rt/device_rt.cuh"

namespace ens {

enum AppId : uint32_t { APP_BY_ARGV0 = 0, APP_ECHO = 1, APP_XSBENCH = 2, APP_RSBENCH = 3, APP_AMGMK = 4,
                        APP_PAGERANK = 5, APP_NOTFOUND = 6 /* internal: argv[0] names no app */ };
constexpr int kApps = 7;

// ============================ Page-Rank-style ==============================
struct PrParams {
  long long n = 100000;
  int avg = 8;
  int iters = 10;
  unsigned long long gseed = 42;
};
ENS_HD int pr_parse(int argc, const char *const *argv, PrParams &p) {
  for (int i = 1; i < argc; i++) {
    const char *f = argv[i];
    if (i + 1 >= argc) return i;
    const char *v = argv[i + 1];
    long long x;
    if (str_eq(f, "-n")) {
      if (!parse_i64(v, &x) || x < 1 || x > (1LL << 24)) return i + 1;
      p.n = x;
    } else if (str_eq(f, "-e")) {
      if (!parse_i64(v, &x) || x < 1 || x > 1024) return i + 1;
      p.avg = (int)x;
    } else if (str_eq(f, "-i")) {
      if (!parse_i64(v, &x) || x < 0 || x > 100000) return i + 1;
      p.iters = (int)x;
    } else if (str_eq(f, "-R")) {
      if (!parse_i64(v, &x) || x < 0) return i + 1;
      p.gseed = (unsigned long long)x;
    } else {
      return i;
    }
    i++;
  }
  if (p.n * (2LL * p.avg - 1) > (1LL << 28)) return 0;  // edge-count cap (reading R-pr-range)
  return -1;
}
struct PrLayout {
  uint64_t deg, dstart, src_of_edge, tgt, in_ptr, cursor, in_e, r, r2, total;
};
ENS_HD PrLayout pr_layout(const PrParams &p) {
  PrLayout L{};
  const uint64_t n = (uint64_t)p.n, emax = (uint64_t)p.n * (uint64_t)(2 * p.avg - 1);
  uint64_t o = 0;
  auto take = [&](uint64_t bytes) {
    const uint64_t at = o;
    o = (o + bytes + 255) / 256 * 256;
    return at;
  };
  L.deg = take(n * 4);
  L.dstart = take((n + 8) * 4);
  L.src_of_edge = take(emax * 4);
  L.tgt = take(emax * 4);
  L.in_ptr = take((n + 8) * 4);
  L.cursor = take(n * 4);
  L.in_e = take(emax * 4);
  L.r = take(n * 8);
  L.r2 = take(n * 8);
  L.total = o;
  return L;
}

// ============================ XSBench-style ================================
enum { XS_UNIONIZED = 0, XS_NUCLIDE = 1, XS_HASH = 2 };
// -g range (reading R-xs-range): 2 <= n_gp <= 2^16, the oracle's bound since
// its first commit; every per-nuclide grid index then fits 16 bits
constexpr int kXsMaxGp = 65536;
// hash / nuclide init: one nuclide's sort keys (6 B each) and bucket counters
// sit in shared memory up to this n_gp, in per-CTA arena scratch above it
constexpr int kXsSmemGp = 16384;

struct XsParams {
  int n_iso = 355;
  int n_gp = 11303;
  long long lookups = 17000000;  // event: total; history: per particle (default 34)
  int grid = XS_UNIONIZED;
  int bins = 10000;
  unsigned long long seed = 1070, gseed = 42;
  bool history = false;          // -m history
  long long particles = 500000;  // -p
  bool lookups_set = false;
};

// returns the offending argv index, or -1
ENS_HD int xs_parse(int argc, const char *const *argv, XsParams &p) {
  for (int i = 1; i < argc; i++) {
    const char *f = argv[i];
    if (i + 1 >= argc) return i;
    const char *v = argv[i + 1];
    long long x;
    if (str_eq(f, "-s")) {
      if (str_eq(v, "small")) p.n_iso = 68;
      else if (str_eq(v, "large")) p.n_iso = 355;
      else return i + 1;
    } else if (str_eq(f, "-g")) {
      if (!parse_i64(v, &x) || x < 2 || x > kXsMaxGp) return i + 1;
      p.n_gp = (int)x;
    } else if (str_eq(f, "-l")) {
      if (!parse_i64(v, &x) || x < 0 || x > (1LL << 40)) return i + 1;
      p.lookups = x;
      p.lookups_set = true;
    } else if (str_eq(f, "-G")) {
      if (str_eq(v, "unionized")) p.grid = XS_UNIONIZED;
      else if (str_eq(v, "nuclide")) p.grid = XS_NUCLIDE;
      else if (str_eq(v, "hash")) p.grid = XS_HASH;
      else return i + 1;
    } else if (str_eq(f, "-h")) {
      if (!parse_i64(v, &x) || x < 1 || x > 10000000) return i + 1;
      p.bins = (int)x;
    } else if (str_eq(f, "-m")) {
      if (str_eq(v, "event")) p.history = false;
      else if (str_eq(v, "history")) p.history = true;
      else return i + 1;
    } else if (str_eq(f, "-p")) {
      if (!parse_i64(v, &x) || x < 0 || x > (1LL << 32)) return i + 1;
      p.particles = x;
    } else if (str_eq(f, "-r")) {
      if (!parse_i64(v, &x) || x < 0) return i + 1;
      p.seed = (unsigned long long)x;
    } else if (str_eq(f, "-R")) {
      if (!parse_i64(v, &x) || x < 0) return i + 1;
      p.gseed = (unsigned long long)x;
    } else {
      return i;
    }
    i++;
  }
  if (p.history && !p.lookups_set) p.lookups = 34;
  return -1;
}

ENS_HD int xs_max_nucs(int n_iso) { return n_iso == 68 ? 34 : 321; }
// unionized index grid row stride: n_iso padded to 4 ints, so that a row is
// written as 16-B vectors (the padding is never read)
ENS_HD int xs_iso_pad(int n_iso) { return (n_iso + 3) & ~3; }
ENS_HD int pow2_ceil(int n) {
  int p = 1;
  while (p < n) p <<= 1;
  return p;
}

// Init sort = one bucket sort of all n_u records (energies are uniform in
// [0,1)): unionized by energy alone (the union order; each nuclide's order
// is its subsequence), otherwise by (nuclide, energy).  Power-of-two bucket
// counts keep floor(E * nb) exact.
// Small unionized problems keep the sort's bucket counters (and after the
// sort, the sweep's chunk owner counts) in shared memory: kXsSmemBkt u32,
// ~2 keys per bucket.  0 = counters in the arena.
constexpr int kXsSmemBkt = 32768;
ENS_HD bool xs_warp_union(const XsParams &p);
ENS_HD long long xs_smem_nb(const XsParams &p) {
  // the warp path's problems keep the block-wide fallback's counters in the
  // arena: its shared memory then fits two CTAs per SM at T <= 256
  if (p.grid != XS_UNIONIZED || xs_warp_union(p)) return 0;
  const long long n_u = (long long)p.n_iso * p.n_gp;
  const long long nch = (n_u + 511) / 512;  // kXsSweepRows
  if (n_u > 4LL * kXsSmemBkt || nch * p.n_iso > kXsSmemBkt) return 0;
  long long nb = 1;
  while (nb * 2 <= n_u / 2 && nb < kXsSmemBkt) nb *= 2;
  return nb;
}
#ifndef ENS_XS_UBKT_DIV
#define ENS_XS_UBKT_DIV 4
#endif
ENS_HD long long xs_buckets(const XsParams &p) {
  const long long n_u = (long long)p.n_iso * p.n_gp;
  if (xs_smem_nb(p)) return xs_smem_nb(p);
  if (p.grid == XS_UNIONIZED) return pow2_ceil((int)((n_u + ENS_XS_UBKT_DIV - 1) / ENS_XS_UBKT_DIV));
  return (long long)p.n_iso * (pow2_ceil(p.n_gp) / 2 > 0 ? pow2_ceil(p.n_gp) / 2 : 1);
}
// per-nuclide sort buckets of the hash / nuclide init (~ENS_XS_NBN_DIV / 2 keys each)
#ifndef ENS_XS_NBN_DIV
#define ENS_XS_NBN_DIV 2
#endif
ENS_HD int xs_nbn(int n_gp) {
  return pow2_ceil(n_gp) / ENS_XS_NBN_DIV > 0 ? pow2_ceil(n_gp) / ENS_XS_NBN_DIV : 1;
}
// hash / nuclide grids: the per-nuclide sort runs in shared memory
ENS_HD bool xs_nuc_smem(const XsParams &p) { return p.n_gp <= kXsSmemGp; }
// bytes of per-CTA arena scratch of the per-nuclide sort when it does not fit
// shared memory: [nbn] u32 counters | [n_gp] u32 keys | [n_gp] u16 record ids
ENS_HD uint64_t xs_nscr_bytes(const XsParams &p) {
  if (p.grid == XS_UNIONIZED || xs_nuc_smem(p)) return 0;
  return align_up((uint64_t)xs_nbn(p.n_gp) * 4, 256) + align_up((uint64_t)p.n_gp * 4, 256) +
         align_up((uint64_t)p.n_gp * 2, 256);
}
// bins of the union search table: ufind[b] = #{k >= 1 : u_k <= b / ubins}
// (power of two, ~1 union energy per bin), so the union position of energy
// p is ufind[floor(p * ubins)] plus a short forward scan — the same index as
// XS-7's binary search, in two dependent loads instead of ~17
#ifndef ENS_XS_UB_MUL
#define ENS_XS_UB_MUL 1
#endif
ENS_HD long long xs_ubins(const XsParams &p) {
  return (long long)pow2_ceil((int)(((long long)p.n_iso * p.n_gp + 1) / 2)) * ENS_XS_UB_MUL;
}
// union-sweep chunks (rows per chunk) for the index grid
constexpr int kXsSweepRows = 512;

// Unionized init, warp path (n_gp <= kXsWarpGp): a warp sorts one nuclide at
// a time in its own shared memory and writes the nuclide's records, its
// sorted energies and, per union value chunk, how many of its energies lie
// below the chunk; then a warp per value chunk [ch/NC, (ch+1)/NC) gathers the
// chunk's energies from the sorted runs, sorts them in shared memory and
// writes the union energies, the search table and the index rows of the
// chunk.  NC = ubins / kXsBinsPerChunk (powers of two: chunk and bin bounds
// are exact), so a chunk holds 64..128 union energies on average; one that
// exceeds kXsChunkCap (never seen: ~10 sigma) sends the instance to the
// block-wide path.
constexpr int kXsWarpGp = 1024;
#ifndef ENS_XS_NUC_BKT_BITS
#define ENS_XS_NUC_BKT_BITS 9
#endif
constexpr int kXsNucBktBits = ENS_XS_NUC_BKT_BITS;
constexpr int kXsNucBkt = 1 << kXsNucBktBits;  // per-nuclide sort buckets (top bits of the 32-bit key)
constexpr uint32_t kXsNucScr = kXsWarpGp * 6 + kXsNucBkt * 4;  // bytes per warp: u32 keys, u16 j, counters
constexpr int kXsBinsPerChunk = 64 * ENS_XS_UB_MUL;   // search-table bins per union chunk
constexpr int kXsChunkCap = 256;      // union energies a warp sorts at once
#ifndef ENS_XS_CHUNK_FB
#define ENS_XS_CHUNK_FB 32
#endif
constexpr int kXsChunkFb = ENS_XS_CHUNK_FB;  // fine sort buckets per union chunk
constexpr uint32_t kXsUniScr = kXsChunkCap * 30 + kXsChunkFb * 4;  // bytes per chunk warp (2 gather buffers)
ENS_HD bool xs_warp_union(const XsParams &p) { return p.grid == XS_UNIONIZED && p.n_gp <= kXsWarpGp; }
// warps of a CTA with warp-path scratch (larger blocks leave the rest idle in the init)
ENS_HD int xs_warp_scr_warps(int T) { return T / 32 < 16 ? T / 32 : 16; }
ENS_HD long long xs_uchunks(const XsParams &p) {
  const long long ub = xs_ubins(p);
  return ub > kXsBinsPerChunk ? ub / kXsBinsPerChunk : 1;
}

// arena layout (byte offsets, 256-B aligned)
struct XsLayout {
  uint64_t recs;      // [n_iso][n_gp] x 48 B records, sorted per nuclide
  uint64_t keys;      // unionized: [n_u] u32 record ids sorted by energy (block path) or [n_iso][n_gp] u64 sorted energies (warp path); hash / nuclide: [cs][n_gp] u64 sorted energies
  uint64_t bkt;       // [xs_buckets] u32 bucket counts -> offsets
  uint64_t uenergy;   // unionized: [n_u] sorted union energies (u64 bits)
  uint64_t ufind;     // unionized: [xs_ubins] u32 union search table (private accelerator)
  uint64_t chist;     // unionized: [n_chunks][n_iso] u32 owner counts per sweep chunk
  uint64_t ustart;    // unionized, warp path: [NC+1][iso_pad] i32 #{k: E_i[k] < ch/NC}
  uint64_t inv;       // unionized: [n_u] u32 record id at each sorted position (block path)
  uint64_t index;     // unionized [n_u][xs_iso_pad] int32 / hash [n_iso][bins+1] XsHashEnt
  uint64_t hcol;      // hash: [cs][bins+1] int32 column being built
  uint64_t nscr;      // hash / nuclide, n_gp > kXsSmemGp: [cs] x xs_nscr_bytes per-nuclide sort scratch
  uint64_t lk_pe;     // event mode: [chunk] lookup energies sorted by (material, energy)
  uint64_t lk_hist;   // event mode: [(12 << kb) + 1] u32 (material, energy) bucket counts -> cursors
                      // (split phases, phase 1b: [12 << cb][chunks] coarse counts -> offsets)
  uint64_t lk_tmp;    // split phases, phase 1b: [chunk] energies in coarse-bucket order
  uint64_t total;
};
// Event-mode lookups are sampled, then bucket-sorted by (material, energy)
// in chunks of at most 2^22 (upstream XSBench's GPU versions offer the same
// material / energy sort; results per lookup are unchanged): a warp's lanes
// then take neighbouring energies of one material, so they gather the same
// index entries and record pairs.  kb = energy-bucket bits per material
// (~8 lookups per bucket).
constexpr long long kXsLkChunk = 1LL << 22;
ENS_HD long long xs_lk_chunk(const XsParams &p) { return p.lookups < kXsLkChunk ? p.lookups : kXsLkChunk; }
#ifndef ENS_XS_LK_KB_MAX
#define ENS_XS_LK_KB_MAX 18
#endif
#ifndef ENS_XS_LK_PER_BKT
#define ENS_XS_LK_PER_BKT 8
#endif
ENS_HD int xs_lk_bits(long long n_c) {
  int kb = 0;
  while (kb < ENS_XS_LK_KB_MAX && (12LL << kb) * ENS_XS_LK_PER_BKT < n_c) kb++;
  return kb;
}
// hash index entry (a private accelerator; results are unchanged): the
// upstream index u_low = ig[b][i], u_high = ig[b+1][i] + 1 (n_gp <= 65536:
// u_high <= n_gp - 1 fits 16 bits) and the energies E[u_low+1..u_low+6] quantized within bin b,
// q = floor((E*bins - b) * 2^16) clamped to [0, 65535] (65535 also past the
// grid), stored as q >> 1 (15 bits: the lookup compares six at once, SWAR).
// q is monotone in E, so #{k: q(pe) > q_k} never exceeds the number of those
// energies below pe: one 16-B load gives a bracket guess that is exact
// unless two energies share a quantum, and it is always verified.
struct XsHashEnt {
  uint16_t u_low, u_high, q[6];
};
// cs = CTAs in the team: hash / nuclide grids give each CTA its own
// per-nuclide scratch
ENS_HD int xs_lk_cbits(int kb);
ENS_HD int xs_sort_items(const XsParams &p);
ENS_HD bool xs_split_ok(const XsParams &p);
ENS_HD XsLayout xs_layout(const XsParams &p, int cs = 1) {
  XsLayout L{};
  const uint64_t n_u = (uint64_t)p.n_iso * p.n_gp;
  uint64_t o = 0;
  // unionized: one sort of all n_u records; otherwise one nuclide at a time
  const uint64_t n_s = p.grid == XS_UNIONIZED ? n_u : (uint64_t)p.n_gp * (uint64_t)cs;
  L.recs = o; o = align_up(o + n_u * 48, 256);
  L.keys = o; o = align_up(o + n_s * 8, 256);  // u32 ids (unionized, block path) or u64 energies
  L.bkt = o;
  if (p.grid == XS_UNIONIZED) o = align_up(o + (uint64_t)xs_buckets(p) * 4, 256);
  if (p.grid == XS_UNIONIZED) {
    const uint64_t nch = (n_u + kXsSweepRows - 1) / kXsSweepRows;
    L.uenergy = o; o = align_up(o + n_u * 8, 256);
    L.ufind = o; o = align_up(o + (uint64_t)xs_ubins(p) * 4, 256);
    L.chist = o; o = align_up(o + nch * (uint64_t)p.n_iso * 4, 256);
    if (xs_warp_union(p)) { L.ustart = o; o = align_up(o + (uint64_t)xs_iso_pad(p.n_iso) * (xs_uchunks(p) + 1) * 4, 256); }
    L.inv = o; o = align_up(o + n_u * 4, 256);  // the block path (also under ENS_F_GENERIC)
    L.index = o; o = align_up(o + n_u * (uint64_t)xs_iso_pad(p.n_iso) * 4, 256);
  } else if (p.grid == XS_HASH) {
    L.index = o; o = align_up(o + (uint64_t)p.n_iso * (p.bins + 1) * 16, 256);
    L.hcol = o; o = align_up(o + (uint64_t)cs * (p.bins + 1) * 4, 256);
  }
  if (p.grid != XS_UNIONIZED) { L.nscr = o; o = align_up(o + (uint64_t)cs * xs_nscr_bytes(p), 256); }
  if (!p.history) {
    const long long n_c = xs_lk_chunk(p);
    const int kb = xs_lk_bits(n_c);
    const uint64_t coarse = (12ULL << xs_lk_cbits(kb)) * (uint64_t)xs_sort_items(p) + 1;
    L.lk_pe = o; o = align_up(o + (uint64_t)n_c * 8, 256);
    L.lk_hist = o; o = align_up(o + (((12ULL << kb) + 1) > coarse ? ((12ULL << kb) + 1) : coarse) * 4, 256);
    L.lk_tmp = o;
    if (xs_split_ok(p) && p.grid != XS_UNIONIZED) o = align_up(o + (uint64_t)n_c * 8, 256);
  }
  L.total = o;
  return L;
}

// ---- split phases (ENS_F_FUSED off): XS event-mode instances whose lookups
// fit one sorted chunk run as two kernels.  The ensemble kernel (phase 1:
// one team per instance, as always) builds the tables and the sorted lookup
// chunk in a per-INSTANCE arena and writes an XsDesc; phase 2 is a
// persistent kernel over every SM whose CTAs pull lookup batches ("items":
// kXsItemLookups consecutive sorted slots of one instance; 1024 measured best
// over 4096 / 2048: C2 35.6 / 35.0 / 34.9 ms) from one queue,
// so all instances' lookups share every SM; the CTA finishing an instance's
// last item writes its record and stdout.  Per-lookup results are unchanged.
#ifndef ENS_XS_ITEM
#define ENS_XS_ITEM 1024
#endif
constexpr long long kXsItemLookups = ENS_XS_ITEM;
// split phases, phase 1b: lookups per count / scatter item of the lookup sort
#ifndef ENS_XS_SORT_ITEM
#define ENS_XS_SORT_ITEM 65536
#endif
constexpr long long kXsSortChunk = ENS_XS_SORT_ITEM;
ENS_HD int xs_sort_items(const XsParams &p) { return (int)((xs_lk_chunk(p) + kXsSortChunk - 1) / kXsSortChunk); }
// ... the sort's (material, energy) bucket key (kb energy bits) splits into a
// coarse bucket (material, top cb bits: counted and scattered in shared
// memory per chunk) and a fine sub-bucket (the other kb - cb bits: sorted per
// coarse bucket by a warp); fine items take kXsFineGroup coarse buckets
ENS_HD int xs_lk_cbits(int kb) { return kb < 8 ? kb : 8; }
constexpr int kXsFineGroup = 64;
ENS_HD int xs_sort_fine_items(const XsParams &p) {
  const int kb = xs_lk_bits(xs_lk_chunk(p));
  return ((12 << xs_lk_cbits(kb)) + kXsFineGroup - 1) / kXsFineGroup;
}
// shared memory of the sort items: the coarse counters (12 << 8 u32) or up to
// 16 warps' fine counters (1 << (18 - 8) u32 each)
constexpr uint32_t kXsLkSortSmem = 16u * 1024u * 4u;
ENS_HD bool xs_split_ok(const XsParams &p) { return !p.history && p.lookups > 0 && p.lookups <= kXsLkChunk; }
ENS_HD long long xs_items(const XsParams &p) {
  return xs_split_ok(p) ? (p.lookups + kXsItemLookups - 1) / kXsItemLookups : 0;
}
struct XsDesc {            // written by phase 1 (team rank 0, thread 0), read by phase 2
  uint64_t recs, index, uenergy, ufind, lk_pe;  // device addresses in the instance's arena
  uint64_t lookups, seed, t_start;
  long long ubins;
  uint32_t mcnt[13];       // material starts in the sorted chunk, mcnt[12] = lookups
  int32_t n_iso, n_gp, grid, bins;
  uint32_t k, line;        // record slot, instance id
  uint32_t item0, n_items; // this instance's items in the phase-2 queue
  uint32_t pad[2];
};
struct XsItemPart {        // one phase-2 item's partial results (summed in item order)
  unsigned long long ver, bsum;
  double fsum, fabs;
  uint32_t am[5], pad[3];
};

// hash lookups: nuclides gathered per step (independent loads and divisions
// in flight per lane)
#ifndef ENS_XS_STEP
#define ENS_XS_STEP 2
#endif
constexpr int kXsStep = ENS_XS_STEP;
// dynamic shared memory layout: material tables + the sort's bucket counters
constexpr int kXsMaxT = 512;  // XsApp::kMaxT
struct XsSmem {
  uint32_t thr, nn, mats, concs, mcnt, jmp, nbkt, ubkt, nkey, njdx, njdx2, total;
};
// per-nuclide sort buckets when the sort runs in shared memory (~4 keys each:
// the rank pass, init_nuc_t, wants few buckets and two index arrays)
#ifndef ENS_XS_NBN_SMEM_DIV
#define ENS_XS_NBN_SMEM_DIV 4
#endif
ENS_HD int xs_nbn_smem(int n_gp) {
  return pow2_ceil(n_gp) / ENS_XS_NBN_SMEM_DIV > 0 ? pow2_ceil(n_gp) / ENS_XS_NBN_SMEM_DIV : 1;
}
// hash / nuclide grids, per-nuclide sort in shared memory: [nkey] u32 sort
// keys (after the sort: the hash column's per-record codes, init_nuc_t) |
// [nbkt] u32 bucket counters | [njdx] u16 record indices in bucket order |
// [njdx2] u16 record indices sorted; the hash column (bins+1 u32) reuses
// [nbkt, end) once the records are written, the region grown by up to 16 KB
// so that it fits (else it goes to arena scratch)
ENS_HD uint32_t xs_nuc_smem_block(const XsParams &p, uint32_t o, XsSmem &S) {
  S.nkey = o; o += (uint32_t)align_up((uint64_t)p.n_gp * 4, 16);
  S.nbkt = o; o += (uint32_t)align_up((uint64_t)xs_nbn_smem(p.n_gp) * 4, 16);
  S.njdx = o; o += (uint32_t)align_up((uint64_t)p.n_gp * 2, 16);
  S.njdx2 = o; o += (uint32_t)align_up((uint64_t)p.n_gp * 2, 16);
  if (p.grid == XS_HASH) {
    const uint64_t need = align_up((uint64_t)(p.bins + 1) * 4, 16), have = o - S.nbkt;
    if (need > have && need - have <= 16384) o = S.nbkt + (uint32_t)need;
  }
  return o;
}
// T = the block size the instance runs with
ENS_HD XsSmem xs_smem(const XsParams &p, int T) {
  XsSmem S{};
  const uint32_t mx = (uint32_t)xs_max_nucs(p.n_iso);
  uint32_t o = 0;
  S.thr = o; o += 12 * 8;                 // pick_mat thresholds
  S.nn = o; o += 16 * 4;                  // num_nucs
  S.concs = o; o += 12 * mx * 8;          // concentrations
  S.mats = o; o += (uint32_t)align_up(12 * mx * 2, 16);  // nuclide ids (u16)
  S.mcnt = o; o += 32 * 4;                // material counts / offsets of a lookup chunk
  S.jmp = o; o += 5 * 64 * 16;            // LCG jump tables: A^(6 d 64^l), l < 5, d < 64
  if (p.grid != XS_UNIONIZED) {  // hash / nuclide grids: one nuclide's sort (xs_nuc_smem_block)
    if (xs_nuc_smem(p)) o = xs_nuc_smem_block(p, o, S);
    else S.nkey = S.nbkt = S.njdx = S.njdx2 = o;
    S.ubkt = o;
  } else {
    S.nbkt = o;  // unionized: per-warp sweep rows
    o += (uint32_t)(T / 32) * 2u * (uint32_t)xs_iso_pad(p.n_iso) * 4u;
    S.ubkt = o;  // unionized, small: bucket counters, then chunk owner counts
    if (xs_smem_nb(p)) o += (uint32_t)kXsSmemBkt * 4u;
    S.nkey = S.njdx = S.njdx2 = o;
  }
  // unionized warp path: kXsWarpScr per warp, overlaying nbkt / ubkt
  if (xs_warp_union(p)) {
    const uint32_t need = (uint32_t)xs_warp_scr_warps(T) * (kXsNucScr > kXsUniScr ? kXsNucScr : kXsUniScr);
    if (S.nbkt + need > o) o = S.nbkt + need;
  }
  S.total = o;
  return S;
}

// split phases, phase 1b (the init-item kernel): a compact layout without the
// material tables — pick_mat thresholds, the lookup sort's material offsets,
// the LCG jump tables, then the per-nuclide sort's counters and keys exactly
// as xs_smem places them (so init_nuc_t's hash-column reuse test is the same)
ENS_HD XsSmem xs_init_smem(const XsParams &p) {
  XsSmem S{};
  uint32_t o = 0;
  S.thr = o; o += 12 * 8;
  S.nn = o; o += 16 * 4;
  S.concs = o;
  S.mats = o;
  S.mcnt = o; o += 32 * 4;
  S.jmp = o; o += 5 * 64 * 16;
  if (p.grid != XS_UNIONIZED && xs_nuc_smem(p)) o = xs_nuc_smem_block(p, o, S);
  else S.nkey = S.nbkt = S.njdx = S.njdx2 = o;
  S.ubkt = o;
  if (o < S.nkey + kXsLkSortSmem) o = S.nkey + kXsLkSortSmem;  // the lookup sort's items use [nkey, ...)
  S.total = o;
  return S;
}

// ============================ RSBench-style ================================
struct RsParams {
  int n_nuc = 355;
  long long lookups = 10000000;
  int avg_poles = 1000;
  int avg_windows = 100;
  int doppler = 1;
  unsigned long long seed = 1070, iseed = 42;
};

ENS_HD int rs_parse(int argc, const char *const *argv, RsParams &p) {
  for (int i = 1; i < argc; i++) {
    const char *f = argv[i];
    if (str_eq(f, "-d")) {
      p.doppler = 0;
      continue;
    }
    if (i + 1 >= argc) return i;
    const char *v = argv[i + 1];
    long long x;
    if (str_eq(f, "-s")) {
      if (str_eq(v, "small")) p.n_nuc = 68;
      else if (str_eq(v, "large")) p.n_nuc = 355;
      else return i + 1;
    } else if (str_eq(f, "-l")) {
      if (!parse_i64(v, &x) || x < 0 || x > (1LL << 40)) return i + 1;
      p.lookups = x;
    } else if (str_eq(f, "-p")) {
      if (!parse_i64(v, &x) || x < 1 || x > 100000) return i + 1;
      p.avg_poles = (int)x;
    } else if (str_eq(f, "-w")) {
      if (!parse_i64(v, &x) || x < 1 || x > 100000) return i + 1;
      p.avg_windows = (int)x;
    } else if (str_eq(f, "-r")) {
      if (!parse_i64(v, &x) || x < 0) return i + 1;
      p.seed = (unsigned long long)x;
    } else if (str_eq(f, "-R")) {
      if (!parse_i64(v, &x) || x < 0) return i + 1;
      p.iseed = (unsigned long long)x;
    } else {
      return i;
    }
    i++;
  }
  return -1;
}

struct RsLayout {
  uint64_t poff_g, woff_g, concs_g;  // split phases: global copies of the shared-memory pole /
                                     // window offsets and concentrations, for phase 2
  uint64_t pole_off;   // [n_nuc+1] int32 prefix of n_poles
  uint64_t win_off;    // [n_nuc+1] int32 prefix of n_windows
  uint64_t poles;      // [total_poles] x 64 B {EA, RT, RA, RF} complex
  uint64_t pole_l;     // [total_poles] u8 l_value
  uint64_t windows;    // [total_windows] x 32 B {T, A, F, (start,end)}
  uint64_t k0rs;       // [n_nuc][4] double
  uint64_t lk_e;       // [chunk] lookup energies sorted by (material, energy)
  uint64_t lk_hist;    // [(12 << kb) + 1] u32 (material, energy) bucket counts -> cursors
  uint64_t total;
};
// RS-3 lookups run in chunks sorted by (material, energy) (a private
// schedule: every lookup's result is unchanged), ~8 lookups per bucket
constexpr long long kRsLkChunk = 1LL << 20;
ENS_HD long long rs_lk_chunk(const RsParams &p) { return p.lookups < kRsLkChunk ? p.lookups : kRsLkChunk; }
ENS_HD int rs_lk_bits(long long n_c) {
  int kb = 0;
  while (kb < 16 && (12LL << kb) * 8 < n_c) kb++;
  return kb;
}
ENS_HD RsLayout rs_layout(const RsParams &p) {
  RsLayout L{};
  const uint64_t tp = (uint64_t)p.avg_poles * p.n_nuc, tw = (uint64_t)p.avg_windows * p.n_nuc;
  uint64_t o = 0;
  L.poff_g = o; o = align_up(o + (p.n_nuc + 1) * 4ULL, 256);
  L.woff_g = o; o = align_up(o + (p.n_nuc + 1) * 4ULL, 256);
  L.concs_g = o; o = align_up(o + 12ULL * xs_max_nucs(p.n_nuc) * 8, 256);
  L.pole_off = o; o = align_up(o + (p.n_nuc + 1) * 4ULL, 256);
  L.win_off = o; o = align_up(o + (p.n_nuc + 1) * 4ULL, 256);
  L.poles = o; o = align_up(o + tp * 64, 256);
  L.pole_l = o; o = align_up(o + tp, 256);
  L.windows = o; o = align_up(o + tw * 32, 256);
  L.k0rs = o; o = align_up(o + p.n_nuc * 32ULL, 256);
  const long long n_c = rs_lk_chunk(p);
  L.lk_e = o; o = align_up(o + (uint64_t)n_c * 8, 256);
  L.lk_hist = o; o = align_up(o + ((12ULL << rs_lk_bits(n_c)) + 1) * 4, 256);
  L.total = o;
  return L;
}
// split phases (see XsDesc): RS instances whose lookups fit one sorted chunk;
// items of 512 lookups (C3: 2048 / 1024 / 512 / 256 -> 16.3 / 15.9 / 15.6 / 15.8 ms)
#ifndef ENS_RS_ITEM
#define ENS_RS_ITEM 512
#endif
constexpr long long kRsItemLookups = ENS_RS_ITEM;
ENS_HD bool rs_split_ok(const RsParams &p) { return p.lookups > 0 && p.lookups <= kRsLkChunk; }
ENS_HD long long rs_items(const RsParams &p) {
  return rs_split_ok(p) ? (p.lookups + kRsItemLookups - 1) / kRsItemLookups : 0;
}
struct RsDesc {            // written by phase 1, read by phase 2
  uint64_t poles, pole_l, windows, k0rs, lk_e, poff, woff, concs;  // device addresses in the arena
  uint64_t lookups, seed, t_start;
  uint32_t mcnt[13];
  int32_t n_nuc, doppler, avg_poles, avg_windows;
  uint32_t k, line;
  uint32_t item0, n_items; // this instance's items in the phase-2 queue (host-staged)
};
struct RsItemPart {
  unsigned long long ver, bsum, terms, near;
  double fsum, fabs;
  uint32_t am[4];
};
// one descriptor / item-part stride for every split app
constexpr uint32_t kDescBytes = ((sizeof(XsDesc) > sizeof(RsDesc) ? sizeof(XsDesc) : sizeof(RsDesc)) + 15) / 16 * 16;
constexpr uint32_t kPartBytes =
    ((sizeof(XsItemPart) > sizeof(RsItemPart) ? sizeof(XsItemPart) : sizeof(RsItemPart)) + 15) / 16 * 16;

struct RsSmem {
  uint32_t thr, nn, concs, mats, npol, nwin, mcnt, total;
};
ENS_HD RsSmem rs_smem(const RsParams &p) {
  RsSmem S{};
  const uint32_t mx = (uint32_t)xs_max_nucs(p.n_nuc);
  uint32_t o = 0;
  S.thr = o; o += 12 * 8;
  S.nn = o; o += 16 * 4;
  S.concs = o; o += 12 * mx * 8;
  S.mats = o; o += (uint32_t)align_up(12 * mx * 2, 16);
  S.npol = o; o += (uint32_t)align_up((p.n_nuc + 1) * 4, 16);   // pole counts -> offsets
  S.nwin = o; o += (uint32_t)align_up((p.n_nuc + 1) * 4, 16);   // window counts -> offsets
  S.mcnt = o; o += 64;                                            // sorted chunk: material starts [13]
  S.total = o;
  return S;
}

// ============================ AMGmk-style ==================================
struct AmgParams {
  int nx = 50, ny = 50, nz = 50;
  int iters = 100;
  int kind = 0;  // 0 relax, 1 matvec, 2 both
  unsigned long long seed = 0;
};
ENS_HD int amg_parse(int argc, const char *const *argv, AmgParams &p) {
  for (int i = 1; i < argc; i++) {
    const char *f = argv[i];
    if (i + 1 >= argc) return i;
    const char *v = argv[i + 1];
    long long x;
    if (str_eq(f, "-x") || str_eq(f, "-y") || str_eq(f, "-z")) {
      if (!parse_i64(v, &x) || x < 1 || x > 1024) return i + 1;
      (str_eq(f, "-x") ? p.nx : str_eq(f, "-y") ? p.ny : p.nz) = (int)x;
    } else if (str_eq(f, "-i")) {
      if (!parse_i64(v, &x) || x < 0 || x > 1000000) return i + 1;
      p.iters = (int)x;
    } else if (str_eq(f, "-k")) {
      if (str_eq(v, "relax")) p.kind = 0;
      else if (str_eq(v, "matvec")) p.kind = 1;
      else if (str_eq(v, "both")) p.kind = 2;
      else return i + 1;
    } else if (str_eq(f, "-r")) {
      if (!parse_i64(v, &x) || x < 0) return i + 1;
      p.seed = (unsigned long long)x;
    } else {
      return i;
    }
    i++;
  }
  if ((long long)p.nx * p.ny * p.nz > (1LL << 24)) return 0;  // reading R-amg-range
  return -1;
}

// SELL-32 layout: rows in slices of 32; within a slice entries are stored
// column-major by entry position (entry e of the slice's 32 rows are
// contiguous), padded to 7 entries per row; padding entries have col = -1.
struct AmgLayout {
  long long n, nnz, n_slices;
  uint64_t col;    // [n_slices][7][32] int32
  uint64_t val;    // [n_slices][7][32] double
  uint64_t rlen;   // [n] u8 entries per row
  uint64_t f, u, u2, y;  // [n] double
  uint64_t total;
};
ENS_HD AmgLayout amg_layout(const AmgParams &p) {
  AmgLayout L{};
  L.n = (long long)p.nx * p.ny * p.nz;
  L.nnz = 7 * L.n - 2 * ((long long)p.nx * p.ny + (long long)p.ny * p.nz + (long long)p.nx * p.nz);
  L.n_slices = (L.n + 31) / 32;
  const uint64_t ent = (uint64_t)L.n_slices * 7 * 32;
  uint64_t o = 0;
  L.col = o; o = align_up(o + ent * 4, 256);
  L.val = o; o = align_up(o + ent * 8, 256);
  L.rlen = o; o = align_up(o + (uint64_t)L.n, 256);
  L.f = o; o = align_up(o + (uint64_t)L.n * 8, 256);
  L.u = o; o = align_up(o + (uint64_t)L.n * 8, 256);
  L.u2 = o; o = align_up(o + (uint64_t)L.n * 8, 256);
  L.y = o; o = align_up(o + (uint64_t)L.n * 8, 256);
  L.total = o;
  return L;
}

}  // namespace ens
