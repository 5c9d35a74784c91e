/* include/ens.h — C ABI of libens.so, the B200-native ensemble-execution
 * runtime (Tian, Chapman, Doerfert, ICPP-W 2023; PAPER.md cited "P:a-b").
 *
 * Ensemble execution (§3): N independent invocations of a CPU-style
 * application, each with its own command line, run as N teams (CUDA thread
 * blocks) of ONE kernel launch.  Each instance gets its own argc/argv, a
 * bump-allocated heap arena, an RNG stream, a stdout buffer and an exit code.
 *
 * Conventions
 *  - Every int-returning function returns ENS_OK (0) or a negative ENS_E*
 *    code; none aborts or throws.  ens_last_error() gives a thread-local
 *    detail string for the last failure on the calling thread.
 *  - Instance failures are NOT API errors: they are exit codes in the
 *    per-instance records (0 ok, 1 usage, ENS_EXIT_NOMEM, 127 unknown app,
 *    anything else = the app's own return value).
 *  - The caller owns every handle and every buffer it passes; the library
 *    never keeps a caller host pointer after a call returns.  ens_args is
 *    immutable after load and may be shared across threads and ranks; an
 *    ens_run is used by one thread at a time.
 *  - Device pointers are plain CUDA device addresses (e.g. a torch uint8
 *    tensor's data_ptr()); streams are cudaStream_t passed as void*.
 */
#ifndef ENS_H
#define ENS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- error codes ---------------------------------------------------------- */
enum {
  ENS_OK = 0,
  ENS_EINVAL = -1,  /* bad argument (NULL handle, bad cfg, line too long, ...)   */
  ENS_ENOENT = -2,  /* args file cannot be opened                                 */
  ENS_ENOMEM = -3,  /* host or device allocation failed / workspace too small     */
  ENS_ECUDA = -4,   /* a CUDA call failed (sticky launch faults included)         */
  ENS_ERANGE = -5,  /* instance range outside the args, output buffer too small   */
  ENS_EBUSY = -6,   /* run not finished (ens_run_elapsed_ms before completion)    */
  ENS_EPARSE = -7   /* args text not parseable (embedded NUL)                     */
};

/* instance exit codes the runtime itself produces */
enum { ENS_EXIT_USAGE = 1, ENS_EXIT_NOMEM = 12, ENS_EXIT_NOTFOUND = 127 };

/* ens_record.flags */
enum {
  ENS_RF_STDOUT_TRUNC = 1u << 0, /* a stdout record did not fit the buffer     */
  ENS_RF_NOMEM = 1u << 1,        /* the arena was exhausted                     */
  ENS_RF_NOT_RUN = 1u << 2,      /* never completed (launch-level fault)        */
  ENS_RF_DONE = 1u << 3          /* the instance ran to completion              */
};

/* ens_launch_cfg.flags */
enum {
  ENS_F_TIMESTAMPS = 1u << 0, /* fill smid / t_start_ns / t_end_ns in records  */
  ENS_F_PHASES = 1u << 1,     /* accumulate per-phase device time (tracing)    */
  ENS_F_GENERIC = 1u << 2,    /* bodies take their general paths only (no fast
                                 paths such as XS's warp-per-nuclide unionized
                                 init): results are identical — for testing   */
  ENS_F_SERIAL = 1u << 3,     /* mixed-app ensembles: launch the per-app kernels
                                 one after another on one shared arena (the
                                 default gives each its own arena region, when
                                 they fit, and runs them concurrently on forked
                                 streams so one's tail overlaps the next)      */
  ENS_F_FUSED = 1u << 4,      /* run every instance start to finish inside the
                                 one ensemble kernel (the paper's mapping)     */
  ENS_F_CLC = 1u << 6,        /* scheduler ablation (Blackwell cluster launch
                                 control): the ensemble kernel is launched with
                                 one CTA per instance (the paper's N teams); a
                                 CTA that finished its instance cancels a CTA
                                 the hardware has not launched yet
                                 (clusterlaunchcontrol.try_cancel) and runs its
                                 instance, instead of persistent CTAs pulling ids
                                 from an atomic counter.  Arena slots come from
                                 a pool as large as the resident CTAs.  Teams of
                                 one CTA, M = 1.  Results are identical.       */
  ENS_F_SPLIT_PHASES = 1u << 5 /* run XSBench-style event-mode instances whose
                                 lookups fit one sorted chunk (<= 2^22) in
                                 SPLIT PHASES: the ensemble kernel builds every
                                 instance's tables and sorted lookups in an
                                 arena slot of its own, then a second
                                 persistent kernel spreads all instances'
                                 lookup batches over every SM and writes their
                                 records.  Default (neither flag): split when
                                 the group has fewer instances than resident
                                 CTAs and enough lookup batches to fill every
                                 SM, and one slot per instance fits the
                                 workspace.  Results are identical either way. */
};
#define ENS_PHASES 16

typedef enum {
  ENS_APP_BY_ARGV0 = 0, /* basename of argv[0] selects the app per instance */
  ENS_APP_ECHO = 1,
  ENS_APP_XSBENCH = 2,
  ENS_APP_RSBENCH = 3,
  ENS_APP_AMGMK = 4,
  ENS_APP_PAGERANK = 5
} ens_app;
#define ENS_N_APPS 6

typedef struct ens_args ens_args;
typedef struct ens_run ens_run;

/* ---- S1: args file (Fig. 4; §3.2 -f) -----------------
 * One instance per line.  argv of instance I = [argv0] + the line's tokens
 * (Fig. 4: the loader's own argv[0] first, then Line.split(' ')).
 * Readings: tokens are maximal runs of non-blank bytes (blank =
 * ' ' or '\t'), one trailing '\r' stripped, no quoting (Q1); every
 * '\n'-terminated line is an instance, an empty line has argc = 1, a final
 * newline adds no instance (Q2); argv0 == NULL means the first token of each
 * line is argv[0] (mixed-app files, Q3).  A line may hold at most
 * ENS_MAX_ARGC argv entries and ENS_MAX_LINE bytes, else ENS_EINVAL.
 * ens_load_args: ENS_ENOENT if the file cannot be read.  *out is owned by the
 * caller (ens_args_free).                                                       */
#define ENS_MAX_ARGC 128
#define ENS_MAX_LINE 65536
int ens_load_args(const char *path, const char *argv0, ens_args **out);
int ens_parse_args(const char *text, size_t len, const char *argv0, ens_args **out);
/* Args-file script language (the paper's planned extension, §3.2):
 * a line "@repeat N <template>" stands for N lines, i = 0..N-1, where
 * "{expr}" is an integer expression in i (+ - * / % parentheses literals)
 * and "{a|b|c}" the (i mod 3)-th alternative; other lines are unchanged.
 * ens_load_args / ens_parse_args expand such lines (ENS_EPARSE if malformed).
 * ens_expand_args writes the expanded text (at most cap bytes) and returns
 * its full length, or <0.                                                      */
long ens_expand_args(const char *text, size_t len, char *out, size_t cap);
int ens_args_count(const ens_args *a); /* number of instances (lines), or <0 */
/* host view of instance i: *argv borrowed from a, valid until ens_args_free */
int ens_args_get(const ens_args *a, int i, int *argc, const char *const **argv);
void ens_args_free(ens_args *a);

/* ---- S2..S9: launch (Fig. 4; §3.2 -n / -t) ----------
 * Instance ids are first + k*stride for k in [0, n_instances) (sharding by
 * instance id across ranks); records are indexed by k.
 * n_instances == 0 is valid (nothing is launched); an id outside the args is
 * ENS_ERANGE (reading Q4: no wrap-around).
 * grid_blocks ("num_teams"): 0 = auto = min(n, occupancy x SMs, slots that fit
 *   the workspace); persistent blocks pull instance ids from an atomic counter
 *   so n may exceed the co-resident blocks (reading Q5).
 * block_threads (-t, the thread limit, an upper bound per P:431-435): the
 *   kernel runs with the largest power of two in [32, 1024] not above it
 *   (0 = 256); results never depend on it (reading Q6).
 * arena_bytes: per-slot heap; 0 = the exact maximum the launch's instances
 *   need (computed on the host from their flags).
 * stdout_bytes: per-instance raw stdout buffer; 0 = 4096.                       */
typedef struct {
  int32_t first, n_instances, stride;
  int32_t grid_blocks;
  int32_t block_threads;
  uint64_t arena_bytes;
  uint32_t stdout_bytes;
  uint32_t flags;
  int32_t team_ctas;  /* CTAs per team for team-aware bodies (XSBench, RSBench):
                         1..16 (a thread-block cluster with distributed shared
                         memory; above 8 a non-portable cluster size; larger
                         values are capped at 16); 0 = auto (the largest power
                         of two <= 16 with n x team_ctas <= resident CTAs, then
                         shrunk until every instance's cluster is resident, or
                         sized for the heaviest instance of an uneven ensemble),
                         ignored by other apps */
  int32_t instances_per_cta; /* M, the paper's (N/M, M, 1) block mapping
                         (P:393-404): M instances share one CTA, each on the
                         row threadIdx.y of block_threads/M threads with its
                         own arena slot and scheduler state.  1, 2, 4 or 8
                         (rounded down to a power of two, and so that each
                         instance keeps >= 32 threads); 0 = 1.  Applies to the
                         bodies built for it (AMGmk, Page-Rank, echo, unknown
                         programs) with team_ctas == 1; ignored by others.    */
  uint32_t dump_rows; /* element-wise result dump (testing): 0 = off; else each
                         instance writes up to dump_rows result rows of 8
                         doubles {key, material, v[0..4], argmax} into the
                         workspace, read back with ens_collect_dump.  XS / RS
                         event lookups: one row per lookup (key = its energy,
                         v = the macroscopic cross sections of XS-9 / RS-3,
                         argmax of XS-10 / RS-3), in the kernel's (sorted)
                         lookup order, the first dump_rows slots; AMG: rows
                         0..dump_rows-1 of the reported vector (key = row
                         index, v[0] = value, argmax = -1).  Unwritten rows
                         are all zero.  Results never depend on it.           */
} ens_launch_cfg;

/* Device bytes ens_launch needs for (app, a, c).  With c->grid_blocks == 0
 * the auto grid is additionally capped so the workspace fits the free device
 * memory of the current device.                                               */
int ens_workspace_bytes(ens_app app, const ens_args *a, const ens_launch_cfg *c, size_t *bytes);

/* Enqueue one ensemble on cuda_stream (NULL = legacy default stream) and
 * return.  d_workspace: caller-owned device memory of ws_bytes bytes
 * (>= ens_workspace_bytes); NULL = the library allocates (and frees in
 * ens_run_free).  All argument marshalling (one pinned H2D copy) happens
 * inside.  *out is owned by the caller.                                        */
int ens_launch(ens_app app, const ens_args *a, const ens_launch_cfg *c, void *d_workspace, size_t ws_bytes,
               void *cuda_stream, ens_run **out);

/* Re-enqueue the same ensemble on the same workspace with the arguments
 * already resident on the device (no host->device copy): resets the
 * scheduler counters and records, then launches.  For repeated timing.       */
int ens_run_relaunch(ens_run *r, void *cuda_stream);

/* ---- S10: collect (P:380 map(from: Ret[:NI])) -----------------------------
 * Fixed 80-byte little-endian record per instance, identical in layout to
 * the oracle's output.                                                          */
typedef struct {
  uint32_t instance;   /* instance id (line index)                              */
  int32_t exit_code;   /* Ret[I]                                          */
  uint32_t app;        /* ens_app that ran                                        */
  uint32_t flags;      /* ENS_RF_*                                                */
  uint64_t vhash;      /* app verification hash                       exact      */
  uint64_t bitsum;     /* wrapping sum of result bit patterns         exact(XS,AMG) */
  double fsum, fabs;   /* sum of results, sum of |results|            1e-12 rel  */
  uint64_t work;       /* lookups / row updates                       exact      */
  uint32_t stdout_len; /* formatted stdout bytes                      exact      */
  uint32_t smid;       /* diagnostic                                             */
  uint64_t t_start_ns, t_end_ns; /* %globaltimer, diagnostic                     */
} ens_record;

#define ENS_TALLIES 32

/* Wait for the run, copy results to the host.  recs: n records (may be NULL);
 * tallies: n*ENS_TALLIES uint32 (may be NULL); stdout: every instance's stdout
 * formatted on the host and concatenated in instance order into stdout_buf
 * (cap bytes) with stdout_off[k]..stdout_off[k+1] the bytes of instance k
 * (stdout_off has n+1 entries).  stdout_buf == NULL: only stdout_off is
 * filled (to size a buffer); cap too small: ENS_ERANGE with stdout_off
 * filled.  Blocks until this run's kernels are done (its end event, not the
 * whole stream: a launch queued behind it keeps running while this one is
 * collected; copies use a non-blocking stream).  The first call after a (re)launch copies
 * and formats; later calls for the same launch return the same result from
 * the run's host copy (tallies are copied on the first call that asks).      */
int ens_collect(ens_run *r, ens_record *recs, uint32_t *tallies, char *stdout_buf, size_t cap,
                uint64_t *stdout_off);

/* Element-wise dump of the last (re)launch (cfg.dump_rows > 0): copies
 * n x dump_rows x 8 doubles (row layout: see ens_launch_cfg.dump_rows), for
 * record slot k at out + k*dump_rows*8.  cap = doubles available at out;
 * ENS_ERANGE if smaller, ENS_EINVAL if the run was launched without a dump.
 * Blocks until the run's kernels are done.                                   */
int ens_collect_dump(ens_run *r, double *out, size_t cap);

/* CUDA-event time of the last (re)launch's kernels, in ms.                   */
int ens_run_elapsed_ms(ens_run *r, float *ms);

/* Device time of each kernel of the last (re)launch, in launch order: per
 * app group its ensemble kernel (phase 1), then, for split XS groups, one
 * lookup-item kernel per XS grid type present (phase 2; kind = 0 unionized,
 * 1 nuclide, 2 hash).  Each is bracketed by CUDA events on the stream it
 * runs on.  Returns the number of kernels (<= cap) or <0 (ENS_ERANGE if cap
 * is too small).  Blocks until the run is done.                              */
typedef struct {
  int32_t app, phase, kind;  /* ens_app; 1 or 2; XS grid type of phase 2, else -1 */
  int32_t grid_ctas, block_threads;
  float ms;
} ens_kernel_time;
int ens_run_kernel_times(ens_run *r, ens_kernel_time *out, int cap);

/* Tracing (launched with ENS_F_PHASES): ns[p] = sum over instances of the
 * %globaltimer time team thread 0 spent in phase p of the last (re)launch
 * (XS: 0 materials, 1 generate, 2 bucket scan, 3 scatter, 4 bucket sort,
 * 5 clear tables, 6 union tables, 7 index sweep, 8 record permute, 9 hash
 * column, 10 lookup sampling + sort, 11 lookup gathers).  Blocks on the
 * stream.                                                                    */
int ens_run_phases(ens_run *r, uint64_t ns[ENS_PHASES]);

/* Launch geometry actually used, and where the device-side results live
 * inside the workspace (for an in-place NCCL all-gather of the records).     */
typedef struct {
  int32_t n_instances;
  int32_t n_groups;        /* kernel launches (one per app present)            */
  int32_t grid_blocks[ENS_N_APPS];  /* CTAs launched, per ens_app, 0 if absent   */
  int32_t block_threads[ENS_N_APPS];
  int32_t kernel_launches; /* kernels per (re)launch                             */
  uint64_t arena_bytes;    /* per slot (max over groups)                         */
  uint64_t ws_bytes;
  uint64_t records_offset; /* byte offset of ens_record[n] in the workspace       */
  uint64_t tallies_offset; /* byte offset of uint32[n][ENS_TALLIES]               */
  uint64_t stdout_offset;  /* byte offset of the raw stdout buffers              */
  uint32_t stdout_bytes;   /* raw stdout bytes per instance                      */
  uint64_t h2d_bytes;      /* bytes copied host->device by ens_launch            */
  uint64_t d2h_bytes;      /* bytes copied device->host collecting the last launch */
  int32_t team_ctas[ENS_N_APPS];  /* CTAs per team (cluster size), per ens_app    */
  int32_t instances_per_cta[ENS_N_APPS]; /* M per ens_app (0 if absent)          */
} ens_run_info;
int ens_run_get_info(const ens_run *r, ens_run_info *info);

/* Format raw stdout bytes (as produced on the device, e.g. gathered from
 * another rank) of an instance of `app` into text.  Returns the formatted
 * length (needed size) or <0; writes at most cap bytes.                       */
long ens_format_stdout(uint32_t app, const void *raw, size_t raw_len, char *out, size_t cap);

void ens_run_free(ens_run *r); /* waits for the run's own work, then frees      */
const char *ens_strerror(int err);
const char *ens_last_error(void);
const char *ens_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ENS_H */
