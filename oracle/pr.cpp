// oracle/pr.cpp — TEST INFRASTRUCTURE ONLY (see oracle.hpp header).
//
// Page-Rank-style instance: the propagation step of the paper's fourth
// benchmark (HeCBench Page-Rank), on a
// synthetic random graph, step by step (readings R-pr-*):
//   PR-1 flags  -n nodes (100000) -e avg out-degree (8) -i iterations (10)
//               -R graph seed (42)
//   PR-2 graph  from one LCG stream s = gseed: first the n out-degrees
//               deg_u = 1 + LCG_int % (2e - 1) (u = 0..n-1), then, source by
//               source in order, deg_u targets v = LCG_int % n
//   PR-3 ranks  r_0 = 1/n; each iteration, for every node v, s = 0.0 and for
//               its in-edges in (source, edge) order s += r[u] / deg_u, then
//               r'[v] = (1 - d)/n + d*s with d = 0.85 (Jacobi: all from r)
//   PR-4 result checksums of r; vhash = bitsum mod 999983; stdout reports
//               the node of maximal rank (first on ties)
#include <cmath>
#include <vector>

#include "oracle.hpp"

namespace oracle {

namespace {

struct PrIn {
  long n = 100000;
  long avg = 8;
  long iters = 10;
  uint64_t gseed = 42;
};

const char *kPrUsage = "usage: %s [-n nodes] [-e avg_degree] [-i iterations] [-R graph_seed]\n";

int parse_pr(const std::vector<std::string> &argv, PrIn &in) {
  int argc = (int)argv.size();
  for (int i = 1; i < argc; i++) {
    const std::string &f = argv[i];
    if (i + 1 >= argc) return i;
    const std::string &v = argv[i + 1];
    long long x;
    if (f == "-n") {
      if (!parse_long(v, &x) || x < 1 || x > (1LL << 24)) return i + 1;
      in.n = (long)x;
    } else if (f == "-e") {
      if (!parse_long(v, &x) || x < 1 || x > 1024) return i + 1;
      in.avg = (long)x;
    } else if (f == "-i") {
      if (!parse_long(v, &x) || x < 0 || x > 100000) return i + 1;
      in.iters = (long)x;
    } else if (f == "-R") {
      if (!parse_long(v, &x) || x < 0) return i + 1;
      in.gseed = (uint64_t)x;
    } else {
      return i;
    }
    i++;
  }
  if (in.n * (2 * in.avg - 1) > (1LL << 28)) return 0;  // edge-count cap (reading R-pr-range)
  return -1;
}

}  // namespace

void run_pagerank(const std::vector<std::string> &argv, Instance &inst) {
  PrIn in;
  const char *a0 = argv.empty() ? "" : argv[0].c_str();
  int bad = parse_pr(argv, in);
  if (bad >= 0) {
    oprintf(inst.out, "%s: invalid argument '%s'\n", a0, argv[(size_t)bad].c_str());
    oprintf(inst.out, kPrUsage, a0);
    inst.rec.exit_code = 1;
    return;
  }
  const long n = in.n;
  // PR-2: graph
  uint64_t s = in.gseed;
  std::vector<long> deg((size_t)n);
  for (long u = 0; u < n; u++) deg[(size_t)u] = 1 + (long)(lcg_int(&s) % (uint64_t)(2 * in.avg - 1));
  std::vector<std::vector<long>> in_src((size_t)n);  // in-edges of v, in (source, edge) order
  long edges = 0;
  for (long u = 0; u < n; u++)
    for (long k = 0; k < deg[(size_t)u]; k++) {
      const long v = (long)(lcg_int(&s) % (uint64_t)n);
      in_src[(size_t)v].push_back(u);
      edges++;
    }
  // PR-3: iterations
  const double d = 0.85;
  const double base = (1.0 - d) / (double)n;
  std::vector<double> r((size_t)n, 1.0 / (double)n), r2((size_t)n);
  for (long it = 0; it < in.iters; it++) {
    for (long v = 0; v < n; v++) {
      double acc = 0.0;
      for (long u : in_src[(size_t)v]) acc += r[(size_t)u] / (double)deg[(size_t)u];
      r2[(size_t)v] = base + d * acc;
    }
    r.swap(r2);
  }
  // PR-4
  uint64_t bitsum = 0;
  long double fsum = 0.0L, fabs_ = 0.0L;
  long top = 0;
  for (long v = 0; v < n; v++) {
    bitsum += dbits(r[(size_t)v]);
    fsum += r[(size_t)v];
    fabs_ += std::fabs(r[(size_t)v]);
    if (r[(size_t)v] > r[(size_t)top]) top = v;
  }
  inst.rec.vhash = bitsum % 999983ULL;
  inst.rec.bitsum = bitsum;
  inst.rec.fsum = (double)fsum;
  inst.rec.fabs = (double)fabs_;
  inst.rec.work = (uint64_t)edges * (uint64_t)in.iters;
  oprintf(inst.out, "PageRank-style n=%ld edges=%ld iters=%ld top=%ld\n", n, edges, in.iters, top);
  inst.rec.exit_code = 0;
}

namespace pr_hooks {
// the graph of PR-2 as (deg, in-edge CSR in (source, edge) order)
void graph(long n, long avg, uint64_t gseed, std::vector<long> &deg, std::vector<long> &ptr, std::vector<long> &src) {
  uint64_t s = gseed;
  deg.assign((size_t)n, 0);
  for (long u = 0; u < n; u++) deg[(size_t)u] = 1 + (long)(lcg_int(&s) % (uint64_t)(2 * avg - 1));
  std::vector<std::vector<long>> in_src((size_t)n);
  for (long u = 0; u < n; u++)
    for (long k = 0; k < deg[(size_t)u]; k++) in_src[(size_t)(lcg_int(&s) % (uint64_t)n)].push_back(u);
  ptr.assign((size_t)n + 1, 0);
  src.clear();
  for (long v = 0; v < n; v++) {
    for (long u : in_src[(size_t)v]) src.push_back(u);
    ptr[(size_t)v + 1] = (long)src.size();
  }
}
}  // namespace pr_hooks

}  // namespace oracle
