// oracle/runner.cpp — TEST INFRASTRUCTURE ONLY (see oracle.hpp header).
//
// The ensemble definition (Fig. 4) as a plain loop: instance I runs
// isolated on argv(I); a thread pool only runs independent instances on
// different cores (each instance itself is sequential).  Exposes a C API
// for the Python tests (ctypes) and the ens_oracle CLI (main.cpp).
#include <atomic>
#include <cstdio>
#include <cstring>
#include <thread>
#include <vector>

#include "oracle.hpp"

namespace oracle {
namespace xs_hooks {
void build(int n_iso, long n_gp, int grid, long bins, uint64_t gseed, std::vector<double> &energies,
           std::vector<double> &uenergy, std::vector<int> &index_grid);
long bracket(int n_iso, long n_gp, int grid, long bins, const std::vector<double> &energies,
             const std::vector<double> &uenergy, const std::vector<int> &ig, int nuc, double p);
void materials(int n_iso, int *num_nucs, std::vector<int> &mats, int *max_num_nucs);
void set_conc_seed(uint64_t s);
}  // namespace xs_hooks
namespace rs_hooks {
void fast_w(double zr, double zi, double *wr, double *wi);
double trig_eval(int kind, double x);
void init_tables(int small, int avg_poles, int avg_windows, uint64_t iseed, std::vector<int> &n_poles,
                 std::vector<int> &n_windows, std::vector<int> &win_start, std::vector<int> &win_end);
void dump_and_micro(int small, int avg_poles, int avg_windows, uint64_t iseed, int doppler, int n,
                    const int *nucs, const double *Es, double *micro, std::vector<double> &poles,
                    std::vector<double> &wins, std::vector<double> &k0rs);
}  // namespace rs_hooks
namespace pr_hooks {
void graph(long n, long avg, uint64_t gseed, std::vector<long> &deg, std::vector<long> &ptr, std::vector<long> &src);
}
namespace amg_hooks {
void laplacian(long nx, long ny, long nz, std::vector<int> &row_ptr, std::vector<int> &col, std::vector<double> &val);
void sweeps(long nx, long ny, long nz, long iters, std::vector<double> &u);
void apply(long nx, long ny, long nz, const std::vector<double> &u, std::vector<double> &y);
}  // namespace amg_hooks

struct Run {
  std::vector<Instance> inst;
};

Run *run_ensemble(const Args &args, uint32_t app, long n, int jobs, size_t dump_cap) {
  Run *r = new Run();
  r->inst.resize((size_t)n);
  for (Instance &I : r->inst) I.dump_cap = dump_cap;
  std::atomic<long> next(0);
  auto worker = [&]() {
    for (;;) {
      long i = next.fetch_add(1);
      if (i >= n) break;
      Instance &I = r->inst[(size_t)i];
      run_isolated(app, args.argv((size_t)i), I);
      I.rec.instance = (uint32_t)i;
    }
  };
  if (jobs < 1) jobs = 1;
  std::vector<std::thread> th;
  for (int j = 1; j < jobs; j++) th.emplace_back(worker);
  worker();
  for (auto &t : th) t.join();
  return r;
}
Run *run_ensemble(const Args &args, uint32_t app, long n, int jobs) { return run_ensemble(args, app, n, jobs, 0); }

}  // namespace oracle

using namespace oracle;

extern "C" {

// ---- ensemble --------------------------------------------------------------
// Runs the first n lines (n < 0: all lines) of `text`; returns NULL if n is
// larger than the number of lines (reading Q4).
void *oracle_run(const char *text, size_t len, const char *argv0, uint32_t app, long n, int jobs) {
  Args a = parse_args_text(std::string(text, len), argv0);
  if (n < 0) n = (long)a.lines.size();
  if (n > (long)a.lines.size()) return nullptr;
  return run_ensemble(a, app, n, jobs);
}
// the same with element-wise dumps of the first dump_cap results per instance
void *oracle_run_dump(const char *text, size_t len, const char *argv0, uint32_t app, long n, int jobs,
                      long dump_cap) {
  Args a = parse_args_text(std::string(text, len), argv0);
  if (n < 0) n = (long)a.lines.size();
  if (n > (long)a.lines.size() || dump_cap < 0) return nullptr;
  return run_ensemble(a, app, n, jobs, (size_t)dump_cap);
}
// dump rows of instance i (8 doubles each) into out (may be NULL); returns the row count
long oracle_dump(void *h, long i, double *out) {
  const std::vector<double> &d = ((Run *)h)->inst[(size_t)i].dump;
  if (out) std::memcpy(out, d.data(), d.size() * 8);
  return (long)(d.size() / 8);
}
double oracle_margin(void *h, long i) { return ((Run *)h)->inst[(size_t)i].min_margin; }
long oracle_count(void *h) { return (long)((Run *)h)->inst.size(); }
void oracle_records(void *h, Record *out) {
  Run *r = (Run *)h;
  for (size_t i = 0; i < r->inst.size(); i++) out[i] = r->inst[i].rec;
}
void oracle_tallies(void *h, uint32_t *out) {
  Run *r = (Run *)h;
  for (size_t i = 0; i < r->inst.size(); i++) std::memcpy(out + i * kTallies, r->inst[i].tallies, sizeof(uint32_t) * kTallies);
}
size_t oracle_stdout_len(void *h, long i) { return ((Run *)h)->inst[(size_t)i].out.size(); }
void oracle_stdout(void *h, long i, char *out) {
  const std::string &s = ((Run *)h)->inst[(size_t)i].out;
  std::memcpy(out, s.data(), s.size());
}
void oracle_free(void *h) { delete (Run *)h; }

// ---- loader hooks ----------------------------------------------------------
long oracle_args_lines(const char *text, size_t len) {
  return (long)parse_args_text(std::string(text, len), "x").lines.size();
}
// argv of line i joined by '\x1f' into out (cap bytes); returns argc or -1
int oracle_args_argv(const char *text, size_t len, const char *argv0, long i, char *out, size_t cap) {
  Args a = parse_args_text(std::string(text, len), argv0);
  if (i < 0 || i >= (long)a.lines.size()) return -1;
  std::vector<std::string> v = a.argv((size_t)i);
  std::string j;
  for (size_t k = 0; k < v.size(); k++) {
    if (k) j.push_back('\x1f');
    j += v[k];
  }
  if (j.size() + 1 > cap) return -1;
  std::memcpy(out, j.c_str(), j.size() + 1);
  return (int)v.size();
}

// ---- primitive hooks ---------------------------------------------------------
uint64_t oracle_lcg_step(uint64_t s) { return lcg_step(s); }
uint64_t oracle_lcg_ff(uint64_t s, uint64_t n) { return lcg_ff(s, n); }
double oracle_lcg_double(uint64_t *s) { return lcg_double(s); }
int oracle_pick_mat(uint64_t *s) { return pick_mat(s); }
long oracle_grid_search(const double *A, double q, long lo, long hi) { return grid_search(A, q, lo, hi); }

// ---- XS hooks ----------------------------------------------------------------
struct XsTiny {
  int n_iso;
  long n_gp, bins;
  int grid;
  std::vector<double> e, u;
  std::vector<int> ig;
};
void *oracle_xs_build(int n_iso, long n_gp, int grid, long bins, uint64_t gseed) {
  XsTiny *t = new XsTiny();
  t->n_iso = n_iso;
  t->n_gp = n_gp;
  t->grid = grid;
  t->bins = bins;
  xs_hooks::build(n_iso, n_gp, grid, bins, gseed, t->e, t->u, t->ig);
  return t;
}
void oracle_xs_energies(void *h, double *out) {
  XsTiny *t = (XsTiny *)h;
  std::memcpy(out, t->e.data(), t->e.size() * 8);
}
void oracle_xs_union(void *h, double *out) {
  XsTiny *t = (XsTiny *)h;
  std::memcpy(out, t->u.data(), t->u.size() * 8);
}
size_t oracle_xs_index_len(void *h) { return ((XsTiny *)h)->ig.size(); }
void oracle_xs_index(void *h, int *out) {
  XsTiny *t = (XsTiny *)h;
  std::memcpy(out, t->ig.data(), t->ig.size() * 4);
}
long oracle_xs_bracket(void *h, int nuc, double p) {
  XsTiny *t = (XsTiny *)h;
  return xs_hooks::bracket(t->n_iso, t->n_gp, t->grid, t->bins, t->e, t->u, t->ig, nuc, p);
}
void oracle_xs_free(void *h) { delete (XsTiny *)h; }
int oracle_xs_materials(int n_iso, int *num_nucs, int *mats_out /*12*max*/, int *max_num_nucs) {
  std::vector<int> m;
  xs_hooks::materials(n_iso, num_nucs, m, max_num_nucs);
  if (mats_out) std::memcpy(mats_out, m.data(), m.size() * 4);
  return (int)m.size();
}
void oracle_xs_set_conc_seed(uint64_t s) { xs_hooks::set_conc_seed(s); }

// ---- RS hooks ----------------------------------------------------------------
void oracle_rs_fast_w(double zr, double zi, double *wr, double *wi) { rs_hooks::fast_w(zr, zi, wr, wi); }
// RS-3's sin (kind 0), cos (1), atan (2) at n points (reading R-rs-trig)
void oracle_rs_trig(int kind, long n, const double *x, double *y) {
  for (long k = 0; k < n; k++) y[k] = rs_hooks::trig_eval(kind, x[k]);
}
// RS-3 micro cross sections at n (nuc, E) points plus the flattened tables
// (9 doubles per pole, 3 per window, 4 K0RS per nuclide); returns 0, or -1
// if a table exceeds its capacity (in doubles)
int oracle_rs_micro(int small, int avg_poles, int avg_windows, uint64_t iseed, int doppler, int n, const int *nucs,
                    const double *Es, double *micro, double *poles, long pcap, double *wins, long wcap,
                    double *k0rs, long kcap) {
  std::vector<double> p, w, k;
  rs_hooks::dump_and_micro(small, avg_poles, avg_windows, iseed, doppler, n, nucs, Es, micro, p, w, k);
  if ((long)p.size() > pcap || (long)w.size() > wcap || (long)k.size() > kcap) return -1;
  std::memcpy(poles, p.data(), p.size() * 8);
  std::memcpy(wins, w.data(), w.size() * 8);
  std::memcpy(k0rs, k.data(), k.size() * 8);
  return 0;
}
// returns total windows; arrays sized n_nuc (n_poles, n_windows) and total windows
int oracle_rs_tables(int small, int avg_poles, int avg_windows, uint64_t iseed, int *n_poles, int *n_windows,
                     int *win_start, int *win_end, int cap) {
  std::vector<int> a, b, c, d;
  rs_hooks::init_tables(small, avg_poles, avg_windows, iseed, a, b, c, d);
  if ((int)c.size() > cap) return -1;
  std::memcpy(n_poles, a.data(), a.size() * 4);
  std::memcpy(n_windows, b.data(), b.size() * 4);
  std::memcpy(win_start, c.data(), c.size() * 4);
  std::memcpy(win_end, d.data(), d.size() * 4);
  return (int)c.size();
}

// ---- AMG hooks ---------------------------------------------------------------
long oracle_amg_nnz(long nx, long ny, long nz) {
  std::vector<int> rp, c;
  std::vector<double> v;
  amg_hooks::laplacian(nx, ny, nz, rp, c, v);
  return (long)c.size();
}
void oracle_amg_csr(long nx, long ny, long nz, int *row_ptr, int *col, double *val) {
  std::vector<int> rp, c;
  std::vector<double> v;
  amg_hooks::laplacian(nx, ny, nz, rp, c, v);
  std::memcpy(row_ptr, rp.data(), rp.size() * 4);
  std::memcpy(col, c.data(), c.size() * 4);
  std::memcpy(val, v.data(), v.size() * 8);
}
void oracle_amg_sweeps(long nx, long ny, long nz, long iters, double *u) {
  long n = nx * ny * nz;
  std::vector<double> v(u, u + n);
  amg_hooks::sweeps(nx, ny, nz, iters, v);
  std::memcpy(u, v.data(), (size_t)n * 8);
}
void oracle_amg_apply(long nx, long ny, long nz, const double *u, double *y) {
  long n = nx * ny * nz;
  std::vector<double> v(u, u + n), w;
  amg_hooks::apply(nx, ny, nz, v, w);
  std::memcpy(y, w.data(), (size_t)n * 8);
}

// ---- PageRank hooks ------------------------------------------------------------
// in-edge CSR of the PR-2 graph; returns the edge count (arrays may be NULL to size)
long oracle_pr_graph(long n, long avg, uint64_t gseed, long *deg, long *ptr, long *src) {
  std::vector<long> d, p, s;
  pr_hooks::graph(n, avg, gseed, d, p, s);
  if (deg) std::memcpy(deg, d.data(), d.size() * sizeof(long));
  if (ptr) std::memcpy(ptr, p.data(), p.size() * sizeof(long));
  if (src) std::memcpy(src, s.data(), s.size() * sizeof(long));
  return (long)s.size();
}

}  // extern "C"
