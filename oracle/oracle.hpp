// oracle/oracle.hpp — TEST INFRASTRUCTURE ONLY.
//
// The plain, slow, obviously-correct CPU definition of ensemble execution
// (Tian, Chapman, Doerfert, ICPP-W 2023; reference PAPER.md, cited "P:a-b").
// Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
// --impl reference leg may build, link, call or execute anything here.  It
// shares no code, header, table or constant generator with the CUDA path
// under paper_conf_icppw_tiancd23_b200/ and neither side includes the other.
//
// The ensemble result is defined by the sequential loop of Fig. 4
// (P:378-385): for I in [0, NI): Ret[I] = main(Argc[I], Argv[I]), each
// instance with a fresh heap, RNG state, stdout and exit code.  The instance
// bodies follow SURVEY.md §8(c) (XS-*, RS-*, AMG-*), the normative reading of
// the paper's proxy apps, step by step in upstream order.
#pragma once
#include <cstdint>
#include <cstddef>
#include <string>
#include <vector>

namespace oracle {

// ---- record layout (identical bytes to what ens_collect returns) ----------
struct Record {
  uint32_t instance;
  int32_t exit_code;
  uint32_t app;
  uint32_t flags;
  uint64_t vhash;
  uint64_t bitsum;
  double fsum;
  double fabs;
  uint64_t work;
  uint32_t stdout_len;
  uint32_t smid;
  uint64_t t_start_ns;
  uint64_t t_end_ns;
};
static_assert(sizeof(Record) == 80, "record is 80 bytes");

constexpr int kTallies = 32;
constexpr uint32_t kFlagStdoutTrunc = 1u << 0;
constexpr uint32_t kFlagNomem = 1u << 1;
constexpr uint32_t kFlagNotRun = 1u << 2;
constexpr uint32_t kFlagDone = 1u << 3;

enum App : uint32_t { APP_BY_ARGV0 = 0, APP_ECHO = 1, APP_XSBENCH = 2, APP_RSBENCH = 3, APP_AMGMK = 4,
                      APP_PAGERANK = 5 };

// ---- args file (Fig. 4, Fig. 5; readings Q1-Q4) -------
struct Args {
  std::string argv0;                         // empty => first token is argv[0]
  std::vector<std::vector<std::string>> lines;  // tokens of each line
  // argv of instance i, argv[0] first (Fig. 4)
  std::vector<std::string> argv(size_t i) const;
};
Args parse_args_text(const std::string &text, const char *argv0);

// ---- per-instance output ----------------------------------------------------
struct Instance {
  Record rec{};
  uint32_t tallies[kTallies] = {0};
  std::string out;  // stdout bytes
  // Element-wise results (tests only): the first dump_cap result vectors of
  // the run as rows of 8 doubles {key, material, v[0..4], argmax}: XS / RS
  // lookups in index order (key = the lookup's energy), AMG rows of the
  // reported vector (key = row index).  min_margin = the smallest relative
  // argmax margin (max - runner-up) / |max| over every lookup (XS-10 / RS-3).
  size_t dump_cap = 0;
  std::vector<double> dump;
  double min_margin = 1.0 / 0.0;
};
// append one dump row (if dump_cap allows) and fold the lookup's argmax margin
void note_result(Instance &inst, double key, int mat, const double *v, int nv, int argmax);

// LCG of SURVEY.md §8(c) "Shared primitives" (upstream XSBench/RSBench).
uint64_t lcg_step(uint64_t s);
double lcg_double(uint64_t *s);
uint64_t lcg_int(uint64_t *s);
uint64_t lcg_ff(uint64_t s, uint64_t n);
int pick_mat(uint64_t *s);
long grid_search(const double *A, double q, long lo, long hi);

// app bodies: fill inst (exit code, record fields, tallies, stdout)
void run_echo(const std::vector<std::string> &argv, Instance &inst);
void run_xsbench(const std::vector<std::string> &argv, Instance &inst);
void run_rsbench(const std::vector<std::string> &argv, Instance &inst);
void run_amgmk(const std::vector<std::string> &argv, Instance &inst);
void run_pagerank(const std::vector<std::string> &argv, Instance &inst);

// one isolated run: dispatch on app (BY_ARGV0 → basename of argv[0])
void run_isolated(uint32_t app, const std::vector<std::string> &argv, Instance &inst);

// helpers shared by the oracle's own bodies
void oprintf(std::string &out, const char *fmt, ...);
bool parse_long(const std::string &s, long long *v);
uint64_t dbits(double d);

}  // namespace oracle
