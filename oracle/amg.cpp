// oracle/amg.cpp — TEST INFRASTRUCTURE ONLY (see oracle.hpp header).
//
// AMGmk-style instance: the relax kernel of AMGmk on a CSR
// matrix, as SURVEY.md §8(c) AMG-1..AMG-4 fixes it.  The relax is pure Jacobi
// (reading Q15), rows and entries in CSR order (reading Q16).
#include <cmath>
#include <vector>

#include "oracle.hpp"

namespace oracle {

namespace {

struct AmgIn {
  long nx = 50, ny = 50, nz = 50;
  long iters = 100;
  int kind = 0;  // 0 relax, 1 matvec, 2 both
  uint64_t seed = 0;
};

const char *kAmgUsage = "usage: %s [-x nx] [-y ny] [-z nz] [-i iters] [-k relax|matvec|both] [-r seed]\n";

int parse_amg(const std::vector<std::string> &argv, AmgIn &in) {
  int argc = (int)argv.size();
  for (int i = 1; i < argc; i++) {
    const std::string &f = argv[i];
    if (i + 1 >= argc) return i;
    const std::string &v = argv[i + 1];
    long long x;
    if (f == "-x" || f == "-y" || f == "-z") {
      if (!parse_long(v, &x) || x < 1 || x > 1024) return i + 1;
      (f == "-x" ? in.nx : f == "-y" ? in.ny : in.nz) = (long)x;
    } else if (f == "-i") {
      if (!parse_long(v, &x) || x < 0 || x > 1000000) return i + 1;
      in.iters = (long)x;
    } else if (f == "-k") {
      if (v == "relax")
        in.kind = 0;
      else if (v == "matvec")
        in.kind = 1;
      else if (v == "both")
        in.kind = 2;
      else
        return i + 1;
    } else if (f == "-r") {
      if (!parse_long(v, &x) || x < 0) return i + 1;
      in.seed = (uint64_t)x;
    } else {
      return i;
    }
    i++;
  }
  // problem size cap: n <= 2^24 rows (reading R-amg-range)
  if (in.nx * in.ny * in.nz > (1L << 24)) return 0;
  return -1;
}

struct Csr {
  long n = 0;
  std::vector<int> row_ptr, col;
  std::vector<double> val;
};

// AMG-2: 7-point Laplacian, rows lexicographic r = ix + nx*(iy + ny*iz),
// entries: diag 6.0; iz>0: r-nx*ny; iy>0: r-nx; ix>0: r-1; ix<nx-1: r+1;
// iy<ny-1: r+nx; iz<nz-1: r+nx*ny; off-diagonals -1.0.
Csr build_laplacian(long nx, long ny, long nz) {
  Csr A;
  A.n = nx * ny * nz;
  A.row_ptr.push_back(0);
  for (long iz = 0; iz < nz; iz++)
    for (long iy = 0; iy < ny; iy++)
      for (long ix = 0; ix < nx; ix++) {
        long r = ix + nx * (iy + ny * iz);
        A.col.push_back((int)r);
        A.val.push_back(6.0);
        if (iz > 0) { A.col.push_back((int)(r - nx * ny)); A.val.push_back(-1.0); }
        if (iy > 0) { A.col.push_back((int)(r - nx)); A.val.push_back(-1.0); }
        if (ix > 0) { A.col.push_back((int)(r - 1)); A.val.push_back(-1.0); }
        if (ix < nx - 1) { A.col.push_back((int)(r + 1)); A.val.push_back(-1.0); }
        if (iy < ny - 1) { A.col.push_back((int)(r + nx)); A.val.push_back(-1.0); }
        if (iz < nz - 1) { A.col.push_back((int)(r + nx * ny)); A.val.push_back(-1.0); }
        A.row_ptr.push_back((int)A.col.size());
      }
  return A;
}

// f = A*1: sequential CSR sum from 0.0
std::vector<double> rhs_ones(const Csr &A) {
  std::vector<double> f((size_t)A.n);
  for (long i = 0; i < A.n; i++) {
    double s = 0.0;
    for (int k = A.row_ptr[(size_t)i]; k < A.row_ptr[(size_t)i + 1]; k++) s += A.val[(size_t)k] * 1.0;
    f[(size_t)i] = s;
  }
  return f;
}

// AMG-3 relax: one Jacobi sweep; res = f_i, then res -= a*u_old[j] for every
// entry after the diagonal (CSR order), u_new = res / a_ii.
void jacobi_sweep(const Csr &A, const std::vector<double> &f, const std::vector<double> &u_old,
                  std::vector<double> &u_new) {
  for (long i = 0; i < A.n; i++) {
    int k0 = A.row_ptr[(size_t)i];
    double res = f[(size_t)i];
    for (int k = k0 + 1; k < A.row_ptr[(size_t)i + 1]; k++) res -= A.val[(size_t)k] * u_old[(size_t)A.col[(size_t)k]];
    u_new[(size_t)i] = res / A.val[(size_t)k0];
  }
}

// AMG-3 matvec: y_i = ((0.0 + a_0 u_0) + a_1 u_1) + ... in CSR order
void matvec(const Csr &A, const std::vector<double> &u, std::vector<double> &y) {
  for (long i = 0; i < A.n; i++) {
    double s = 0.0;
    for (int k = A.row_ptr[(size_t)i]; k < A.row_ptr[(size_t)i + 1]; k++) s += A.val[(size_t)k] * u[(size_t)A.col[(size_t)k]];
    y[(size_t)i] = s;
  }
}

}  // namespace

void run_amgmk(const std::vector<std::string> &argv, Instance &inst) {
  AmgIn in;
  const char *a0 = argv.empty() ? "" : argv[0].c_str();
  int bad = parse_amg(argv, in);
  if (bad >= 0) {
    oprintf(inst.out, "%s: invalid argument '%s'\n", a0, argv[(size_t)bad].c_str());
    oprintf(inst.out, kAmgUsage, a0);
    inst.rec.exit_code = 1;
    return;
  }
  Csr A = build_laplacian(in.nx, in.ny, in.nz);
  std::vector<double> f = rhs_ones(A);
  std::vector<double> u((size_t)A.n), tmp((size_t)A.n);
  for (long i = 0; i < A.n; i++) {
    if (in.seed == 0) {
      u[(size_t)i] = 1.0;
    } else {
      uint64_t s = lcg_ff(in.seed, (uint64_t)i);
      u[(size_t)i] = lcg_double(&s);
    }
  }
  // AMG-3: the reported vector R is u after the sweeps (relax), or y = A u
  // recomputed every iteration from the current u (matvec: u stays u0;
  // both: one sweep then y = A u per iteration) — reading R-amg-kind.
  std::vector<double> y((size_t)A.n, 0.0);
  for (long it = 0; it < in.iters; it++) {
    if (in.kind == 0 || in.kind == 2) {
      jacobi_sweep(A, f, u, tmp);
      u.swap(tmp);
    }
    if (in.kind == 1 || in.kind == 2) matvec(A, u, y);
  }
  const std::vector<double> &R = (in.kind == 0) ? u : y;
  // AMG-4: checksums of R; maxerr = max |R_i - 1| (relax) or |R_i - f_i|
  // (matvec, both); a NaN never raises the max.
  uint64_t bitsum = 0;
  long double fsum = 0.0L, fabs_ = 0.0L;
  double maxerr = 0.0;
  for (long i = 0; i < A.n; i++) {
    bitsum += dbits(R[(size_t)i]);
    fsum += R[(size_t)i];
    fabs_ += std::fabs(R[(size_t)i]);
    double e = std::fabs(R[(size_t)i] - (in.kind == 0 ? 1.0 : f[(size_t)i]));
    if (e > maxerr) maxerr = e;
    if ((size_t)i < inst.dump_cap) note_result(inst, (double)i, 0, &R[(size_t)i], 1, -1);
  }
  inst.rec.vhash = bitsum % 999983ULL;
  inst.rec.bitsum = bitsum;
  inst.rec.fsum = (double)fsum;
  inst.rec.fabs = (double)fabs_;
  inst.rec.work = (uint64_t)A.n * (uint64_t)in.iters * (in.kind == 2 ? 2u : 1u);
  oprintf(inst.out, "AMGmk-style n=%d nnz=%d iters=%d maxerr=%.17g\n", (int)A.n, (int)A.col.size(), (int)in.iters,
          maxerr);
  inst.rec.exit_code = 0;
}

namespace amg_hooks {
void laplacian(long nx, long ny, long nz, std::vector<int> &row_ptr, std::vector<int> &col, std::vector<double> &val) {
  Csr A = build_laplacian(nx, ny, nz);
  row_ptr = A.row_ptr;
  col = A.col;
  val = A.val;
}
// run `iters` sweeps from u (in place), return nothing
void sweeps(long nx, long ny, long nz, long iters, std::vector<double> &u) {
  Csr A = build_laplacian(nx, ny, nz);
  std::vector<double> f = rhs_ones(A), tmp((size_t)A.n);
  for (long it = 0; it < iters; it++) {
    jacobi_sweep(A, f, u, tmp);
    u.swap(tmp);
  }
}
void apply(long nx, long ny, long nz, const std::vector<double> &u, std::vector<double> &y) {
  Csr A = build_laplacian(nx, ny, nz);
  y.assign((size_t)A.n, 0.0);
  matvec(A, u, y);
}
}  // namespace amg_hooks

}  // namespace oracle
