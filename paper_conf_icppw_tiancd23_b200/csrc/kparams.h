// csrc/kparams.h — kernel parameters of one app group launch and the
// host <-> kernel-file interface (internal to libens).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/ens.h"

namespace ens {

struct KParams {
  const char *blob;           // NUL-terminated tokens (argv0 once + all lines)
  const uint32_t *tok_off;    // byte offset of each argv entry in blob
  const uint32_t *line_tok;   // [n_lines+1] first argv entry of each line
  const uint32_t *kmap;       // [n] group-local index -> record slot k
  const uint32_t *line_of_k;  // [n_instances] record slot -> line
  uint32_t n;                 // instances in this group
  uint32_t flags;             // ENS_F_*
  uint32_t *counter;          // scheduler counter (zeroed before launch)
  unsigned long long *stdout_total;  // compacted stdout bytes (zeroed)
  ens_record *recs;           // [n_instances]
  unsigned long long *stdout_pos;    // [n_instances] offset in stdout_cmp
  uint32_t *tallies;          // [n_instances][ENS_TALLIES]
  char *stdout_base;          // [n_instances][stdout_cap] raw, per instance
  char *stdout_cmp;           // compacted raw stdout (for a small D2H)
  uint32_t stdout_cap;
  char *arena_base;           // [teams][arena_bytes]
  uint64_t arena_bytes;
  uint32_t team_ctas;         // CTAs per team (thread-block cluster size)
  unsigned long long *phases; // [ENS_PHASES] ns per phase (ENS_F_PHASES) or null
  uint32_t sub_stride;        // dynamic smem bytes per instance slot of the CTA
  double *dump;               // [n_instances][dump_rows][8] element-wise results, or null
  uint32_t dump_rows;
  // split phases (XS): phase 1 = this kernel with one arena slot per instance
  // (slot = group-local queue index) and a descriptor per instance; phase 2 =
  // the lookup kernel over the item queue
  uint32_t split;
  char *xs_desc;              // [n] XsDesc
  const uint32_t *items;      // [all items] group-local instance of each item (batch = item - its item0)
  uint32_t item_base, n_items; // phase 2: this launch's items (one grid type)
  char *ipart;                // [n_items] XsItemPart
  uint32_t *idone;            // [n] items finished per instance (zeroed)
  uint32_t *counter2;         // phase-2 item counter (zeroed)
  // split phases, hash / nuclide tables: (group-local instance, nuclide) init
  // items, run by the init-item kernel beside the ensemble kernel
  const uint32_t *init_items; // [n_init_items][2]
  uint32_t n_init_items;
  uint32_t *counter3;         // init-item counter (zeroed)
  char *init_scr;             // [grid][init_scr_bytes] per-CTA scratch
  uint64_t init_scr_bytes;
  uint32_t init_smem_off;     // dynamic smem offset of the app's shared memory
  char *init_sync;            // [n] x kInitSyncBytes per-instance phase-1b state (zeroed)
  // ENS_F_CLC: one CTA per instance, cluster launch control for the rest,
  // arena slots from a bitmap pool of n_slots
  uint32_t clc;
  uint32_t *slot_bm;          // [ceil(n_slots / 32)] (zeroed)
  uint32_t n_slots;
};

const void *kernel_ptr(uint32_t app, int T);
const void *kernel_ptr_sub(uint32_t app, int T);  // row kernels (m > 1), kernels_sub.cu
int app_max_threads(uint32_t app);
bool app_team_aware(uint32_t app);
double app_cost(uint32_t app, int argc, const char *const *argv);
bool app_sub_aware(uint32_t app);
uint32_t app_items(uint32_t app, int argc, const char *const *argv, int *kind);
uint32_t sub_shared_bytes();
bool app_size(uint32_t app, int argc, const char *const *argv, int T, int cs, uint64_t *arena, uint32_t *smem);
cudaError_t launch_group(uint32_t app, int T, int m, int grid, int cs, size_t smem, const KParams &p,
                         cudaStream_t st);
cudaError_t group_occupancy(uint32_t app, int T, int m, int cs, size_t smem, int *teams);
// split phases, phase 2 (kernels_items.cu): the XS lookup-item kernel
cudaError_t launch_xs_items(int grid_type, int ctas, const KParams &p, cudaStream_t st);
cudaError_t xs_items_occupancy(int grid_type, int *ctas);
int xs_items_threads(int kind);
cudaError_t launch_xs_init_items(int ctas, int threads, size_t smem, const KParams &p, cudaStream_t st);
cudaError_t xs_init_items_occupancy(int threads, size_t smem, int *ctas);
uint32_t xs_init_smem_off();
uint64_t app_init_scratch(uint32_t app, int argc, const char *const *argv, int *n_items, int *n_sort, int *n_fine,
                          uint32_t *smem);
constexpr uint32_t kInitSyncBytes = 128;  // XsInitSync (kernels_items.cu)
// phase-1b item codes (the second word of an init item; nuclide items are < 2^16)
constexpr uint32_t kXsCountItem = 0x80000000u;    // | chunk: count lookups
constexpr uint32_t kXsScatterItem = 0x40000000u;  // | chunk: scatter lookups
constexpr uint32_t kXsFineItem = 0x20000000u;     // | group: sort coarse buckets
#ifndef ENS_XS_INIT_T
#define ENS_XS_INIT_T 256
#endif
constexpr int kXsInitThreads = ENS_XS_INIT_T;  // init-item kernel block (launch bounds: 2 CTAs/SM; C2's 1b:
                                               // 256 8.07 ms, 320 8.27, 384 8.45 at 80 registers)

}  // namespace ens
