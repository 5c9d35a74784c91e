// oracle/core.cpp — TEST INFRASTRUCTURE ONLY (see oracle.hpp header).
// Args-file loader, shared primitives, echo body, instance dispatch.
#include <cmath>
#include "oracle.hpp"

#include <cstdarg>
#include <cstdio>
#include <cstring>

namespace oracle {

// ---------------------------------------------------------------------------
// Loader.  Fig. 4: for each line of the arguments file, the argv
// of that instance starts with the loader's argv[0], followed by the
// line split on ' '; Argc = number of argv entries.
// Readings: Q1 split on runs of ' '/'\t', drop empty
// tokens, strip one trailing '\r'; Q2 every '\n'-terminated line is one
// instance (an empty line is an instance with argc = 1), a final newline adds
// none, text after the last '\n' is a line; Q3 argv0 == NULL means the first
// token of each line is argv[0] (mixed-app files).
// ---------------------------------------------------------------------------
Args parse_args_text(const std::string &text, const char *argv0) {
  Args a;
  a.argv0 = argv0 ? argv0 : "";
  size_t pos = 0;
  const size_t n = text.size();
  while (pos < n) {
    size_t eol = text.find('\n', pos);
    size_t end = (eol == std::string::npos) ? n : eol;
    std::string line = text.substr(pos, end - pos);
    if (!line.empty() && line.back() == '\r') line.pop_back();
    std::vector<std::string> toks;
    std::string cur;
    for (char c : line) {
      if (c == ' ' || c == '\t') {
        if (!cur.empty()) toks.push_back(cur);
        cur.clear();
      } else {
        cur.push_back(c);
      }
    }
    if (!cur.empty()) toks.push_back(cur);
    a.lines.push_back(toks);
    if (eol == std::string::npos) break;
    pos = eol + 1;
  }
  return a;
}

std::vector<std::string> Args::argv(size_t i) const {
  std::vector<std::string> v;
  if (!argv0.empty()) v.push_back(argv0);  // AV.push_back(argv[0])
  for (const auto &t : lines[i]) v.push_back(t);
  return v;
}

// ---------------------------------------------------------------------------
// LCG (SURVEY.md §8(c) "Shared primitives"): s <- (a*s + 1) mod 2^63.
// ---------------------------------------------------------------------------
static const uint64_t kA = 2806196910506780709ULL;
static const uint64_t kM = 9223372036854775808ULL;  // 2^63

uint64_t lcg_step(uint64_t s) { return (kA * s + 1ULL) % kM; }

double lcg_double(uint64_t *s) {
  *s = lcg_step(*s);
  return (double)(*s) / (double)kM;  // advance first, then scale
}

uint64_t lcg_int(uint64_t *s) {
  *s = lcg_step(*s);
  return *s;
}

// Fast-forward n steps by repeated squaring of the affine map (a, c).
uint64_t lcg_ff(uint64_t s, uint64_t n) {
  uint64_t a = kA, c = 1ULL;
  uint64_t an = 1ULL, cn = 0ULL;
  n = n % kM;
  while (n > 0) {
    if (n & 1ULL) {
      an = an * a;
      cn = cn * a + c;
    }
    c = c * (a + 1ULL);
    a = a * a;
    n >>= 1;
  }
  return (an * s + cn) % kM;
}

// pick_mat: one roll; for i = 0..11, running = sum of
// dist[j] for j = i down to 1 (dist[0] never added: upstream quirk kept);
// return i if roll < running; otherwise 0.
int pick_mat(uint64_t *s) {
  double dist[12];
  dist[0] = 0.140;
  dist[1] = 0.052;
  dist[2] = 0.275;
  dist[3] = 0.134;
  dist[4] = 0.154;
  dist[5] = 0.064;
  dist[6] = 0.066;
  dist[7] = 0.055;
  dist[8] = 0.008;
  dist[9] = 0.015;
  dist[10] = 0.025;
  dist[11] = 0.013;
  double roll = lcg_double(s);
  for (int i = 0; i < 12; i++) {
    double running = 0;
    for (int j = i; j > 0; j--) running += dist[j];
    if (roll < running) return i;
  }
  return 0;
}

// grid_search: bisection on [lo, hi].
long grid_search(const double *A, double q, long lo, long hi) {
  long len = hi - lo;
  while (len > 1) {
    long m = lo + len / 2;
    if (A[m] > q)
      hi = m;
    else
      lo = m;
    len = hi - lo;
  }
  return lo;
}

// ---------------------------------------------------------------------------
// helpers
// ---------------------------------------------------------------------------
void oprintf(std::string &out, const char *fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  int k = vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  if (k > 0) out.append(buf, (size_t)k < sizeof buf ? (size_t)k : sizeof buf - 1);
}

// Integer grammar of every app flag (reading R-int): optional '+'
// or '-', then 1..18 decimal digits, nothing else.
bool parse_long(const std::string &s, long long *v) {
  size_t i = 0;
  bool neg = false;
  if (i < s.size() && (s[i] == '+' || s[i] == '-')) {
    neg = s[i] == '-';
    i++;
  }
  size_t nd = s.size() - i;
  if (nd < 1 || nd > 18) return false;
  long long x = 0;
  for (; i < s.size(); i++) {
    if (s[i] < '0' || s[i] > '9') return false;
    x = x * 10 + (s[i] - '0');
  }
  *v = neg ? -x : x;
  return true;
}

void note_result(Instance &inst, double key, int mat, const double *v, int nv, int argmax) {
  if (argmax >= 0 && nv > 1) {  // argmax margin: v[argmax] minus the largest other channel
    double second = -1.0 / 0.0;
    for (int c = 0; c < nv; c++)
      if (c != argmax && v[c] > second) second = v[c];
    const double m = (v[argmax] - second) / std::fabs(v[argmax]);
    if (m < inst.min_margin) inst.min_margin = m;
  }
  if (inst.dump.size() / 8 >= inst.dump_cap) return;
  double row[8] = {key, (double)mat, 0, 0, 0, 0, 0, (double)argmax};
  for (int c = 0; c < nv && c < 5; c++) row[2 + c] = v[c];
  inst.dump.insert(inst.dump.end(), row, row + 8);
}

uint64_t dbits(double d) {
  uint64_t u;
  std::memcpy(&u, &d, 8);
  return u;
}

// ---------------------------------------------------------------------------
// echo body: prints argc and every argv entry, returns argc.
// ---------------------------------------------------------------------------
void run_echo(const std::vector<std::string> &argv, Instance &inst) {
  int argc = (int)argv.size();
  oprintf(inst.out, "argc=%d\n", argc);
  for (int i = 0; i < argc; i++) oprintf(inst.out, "argv[%d]=%s\n", i, argv[i].c_str());
  inst.rec.exit_code = argc;
  inst.rec.work = (uint64_t)argc;
}

static uint32_t app_of_argv0(const std::string &a0) {
  size_t sl = a0.rfind('/');
  std::string b = (sl == std::string::npos) ? a0 : a0.substr(sl + 1);
  if (b == "echo") return APP_ECHO;
  if (b == "xsbench") return APP_XSBENCH;
  if (b == "rsbench") return APP_RSBENCH;
  if (b == "amgmk") return APP_AMGMK;
  if (b == "pagerank") return APP_PAGERANK;
  return APP_BY_ARGV0;
}

void run_isolated(uint32_t app, const std::vector<std::string> &argv, Instance &inst) {
  const size_t dump_cap = inst.dump_cap;  // the caller's request survives the reset
  inst = Instance();
  inst.dump_cap = dump_cap;
  if (app == APP_BY_ARGV0) {
    app = argv.empty() ? (uint32_t)APP_BY_ARGV0 : app_of_argv0(argv[0]);
    if (app == APP_BY_ARGV0) {
      oprintf(inst.out, "%s: command not found\n", argv.empty() ? "" : argv[0].c_str());
      inst.rec.exit_code = 127;
      inst.rec.flags = kFlagDone;
      inst.rec.stdout_len = (uint32_t)inst.out.size();
      return;
    }
  }
  inst.rec.app = app;
  switch (app) {
    case APP_ECHO: run_echo(argv, inst); break;
    case APP_XSBENCH: run_xsbench(argv, inst); break;
    case APP_RSBENCH: run_rsbench(argv, inst); break;
    case APP_AMGMK: run_amgmk(argv, inst); break;
    case APP_PAGERANK: run_pagerank(argv, inst); break;
    default: inst.rec.exit_code = 127; break;
  }
  inst.rec.flags |= kFlagDone;
  inst.rec.stdout_len = (uint32_t)inst.out.size();
}

}  // namespace oracle
