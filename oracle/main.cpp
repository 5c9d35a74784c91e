// oracle/main.cpp — TEST INFRASTRUCTURE ONLY (see oracle.hpp header).
//
// ens_oracle -f <args file> [-n N] [-j jobs] [-a echo|xsbench|rsbench|amgmk|auto]
//            [--argv0 name] [-o out.bin] [-q]
// Mirrors the paper's loader flags -f / -n (§3.2); -t (thread
// limit) has no meaning for a sequential CPU run and is accepted and ignored.
// Prints every instance's stdout in instance order, then a summary on stderr.
// -o writes the binary result: "ENSORC01", u32 n, u32 tallies/instance,
// n x 80-B records, n x tallies u32, (n+1) x u64 stdout offsets, stdout bytes.
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <sstream>
#include <string>
#include <thread>

#include "oracle.hpp"

namespace oracle {
struct Run {
  std::vector<Instance> inst;
};
Run *run_ensemble(const Args &args, uint32_t app, long n, int jobs);
}  // namespace oracle

using namespace oracle;

int main(int argc, char **argv) {
  const char *file = nullptr, *out = nullptr, *argv0 = nullptr;
  long n = -1;
  int jobs = (int)std::thread::hardware_concurrency();
  uint32_t app = APP_BY_ARGV0;
  bool quiet = false;
  for (int i = 1; i < argc; i++) {
    std::string f = argv[i];
    auto need = [&]() -> const char * {
      if (i + 1 >= argc) {
        std::fprintf(stderr, "ens_oracle: %s needs a value\n", f.c_str());
        std::exit(2);
      }
      return argv[++i];
    };
    if (f == "-f") file = need();
    else if (f == "-n") n = std::atol(need());
    else if (f == "-j") jobs = std::atoi(need());
    else if (f == "-t") (void)need();
    else if (f == "-o") out = need();
    else if (f == "--argv0") argv0 = need();
    else if (f == "-q") quiet = true;
    else if (f == "-a") {
      std::string a = need();
      app = a == "echo" ? APP_ECHO : a == "xsbench" ? APP_XSBENCH : a == "rsbench" ? APP_RSBENCH
          : a == "amgmk" ? APP_AMGMK : a == "pagerank" ? APP_PAGERANK : APP_BY_ARGV0;
    } else {
      std::fprintf(stderr, "usage: ens_oracle -f file [-n N] [-j jobs] [-a app] [--argv0 name] [-o out.bin] [-q]\n");
      return 2;
    }
  }
  if (!file) {
    std::fprintf(stderr, "ens_oracle: -f required\n");
    return 2;
  }
  std::ifstream in(file, std::ios::binary);
  if (!in) {
    std::fprintf(stderr, "ens_oracle: cannot open %s\n", file);
    return 2;
  }
  std::stringstream ss;
  ss << in.rdbuf();
  // explicit app without --argv0: the app name is argv[0] (reading Q3)
  static const char *names[] = {"", "echo", "xsbench", "rsbench", "amgmk", "pagerank"};
  if (!argv0 && app != APP_BY_ARGV0) argv0 = names[app];
  Args a = parse_args_text(ss.str(), argv0);
  if (n < 0) n = (long)a.lines.size();
  if (n > (long)a.lines.size()) {
    std::fprintf(stderr, "ens_oracle: -n %ld > %zu lines\n", n, a.lines.size());
    return 2;
  }
  auto t0 = std::chrono::steady_clock::now();
  Run *r = run_ensemble(a, app, n, jobs);
  double sec = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  if (!quiet)
    for (auto &I : r->inst) std::fwrite(I.out.data(), 1, I.out.size(), stdout);
  uint64_t work = 0;
  for (auto &I : r->inst) work += I.rec.work;
  std::fprintf(stderr, "ens_oracle: %ld instances, %d jobs, %.6f s, %.3f instances/s, work %llu\n", n, jobs, sec,
               n / sec, (unsigned long long)work);
  if (out) {
    FILE *fo = std::fopen(out, "wb");
    if (!fo) return 2;
    uint32_t hdr[2] = {(uint32_t)n, (uint32_t)kTallies};
    std::fwrite("ENSORC01", 1, 8, fo);
    std::fwrite(hdr, 4, 2, fo);
    for (auto &I : r->inst) std::fwrite(&I.rec, sizeof(Record), 1, fo);
    for (auto &I : r->inst) std::fwrite(I.tallies, 4, kTallies, fo);
    uint64_t off = 0;
    std::fwrite(&off, 8, 1, fo);
    for (auto &I : r->inst) {
      off += I.out.size();
      std::fwrite(&off, 8, 1, fo);
    }
    for (auto &I : r->inst) std::fwrite(I.out.data(), 1, I.out.size(), fo);
    std::fclose(fo);
  }
  delete r;
  return 0;
}
