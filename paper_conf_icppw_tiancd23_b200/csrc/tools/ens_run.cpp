// csrc/tools/ens_run.cpp — N5, the enhanced loader's command line (§3.2
// P:422-436, Fig. 5c):
//   ens_run -f <args file> [-n <num instances>] [-t <thread limit>]
//           [-a auto|echo|xsbench|rsbench|amgmk|pagerank] [-g grid]
//           [-M instances per CTA] [--argv0 name] [--timestamps] [-q]
// Runs the first n lines as one ensemble on the current GPU, prints every
// instance's stdout in instance order, then one summary line on stderr.
// (Multi-GPU runs go through the Python launcher, python -m
// paper_conf_icppw_tiancd23_b200.run, one process per GPU.)
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "../../../include/ens.h"

static int die(const char *what, int rc) {
  std::fprintf(stderr, "ens_run: %s: %s (%s)\n", what, ens_strerror(rc), ens_last_error());
  return 2;
}

int main(int argc, char **argv) {
  const char *file = nullptr, *argv0 = nullptr;
  int n = -1, t = 0, grid = 0, m = 0;
  bool quiet = false, ts = false;
  ens_app app = ENS_APP_BY_ARGV0;
  for (int i = 1; i < argc; i++) {
    std::string f = argv[i];
    auto val = [&]() -> const char * {
      if (i + 1 >= argc) {
        std::fprintf(stderr, "ens_run: %s needs a value\n", f.c_str());
        std::exit(2);
      }
      return argv[++i];
    };
    if (f == "-f") file = val();
    else if (f == "-n") n = std::atoi(val());
    else if (f == "-t") t = std::atoi(val());
    else if (f == "-g") grid = std::atoi(val());
    else if (f == "-M") m = std::atoi(val());
    else if (f == "--argv0") argv0 = val();
    else if (f == "--timestamps") ts = true;
    else if (f == "-q") quiet = true;
    else if (f == "-a") {
      std::string a = val();
      app = a == "echo" ? ENS_APP_ECHO : a == "xsbench" ? ENS_APP_XSBENCH : a == "rsbench" ? ENS_APP_RSBENCH
          : a == "amgmk" ? ENS_APP_AMGMK : a == "pagerank" ? ENS_APP_PAGERANK : ENS_APP_BY_ARGV0;
    } else {
      std::fprintf(stderr, "usage: ens_run -f file [-n N] [-t T] [-a auto|echo|xsbench|rsbench|amgmk|pagerank] [-g grid] "
                           "[-M instances per CTA] "
                           "[--argv0 name] [--timestamps] [-q]\n");
      return 2;
    }
  }
  if (!file) {
    std::fprintf(stderr, "ens_run: -f is required\n");
    return 2;
  }
  static const char *names[] = {nullptr, "echo", "xsbench", "rsbench", "amgmk", "pagerank"};
  if (!argv0 && app != ENS_APP_BY_ARGV0) argv0 = names[app];
  ens_args *a = nullptr;
  int rc = ens_load_args(file, argv0, &a);
  if (rc) return die("ens_load_args", rc);
  if (n < 0) n = ens_args_count(a);
  ens_launch_cfg cfg{};
  cfg.first = 0;
  cfg.n_instances = n;
  cfg.stride = 1;
  cfg.grid_blocks = grid;
  cfg.block_threads = t;
  cfg.instances_per_cta = m;
  cfg.flags = ts ? ENS_F_TIMESTAMPS : 0;
  ens_run *r = nullptr;
  rc = ens_launch(app, a, &cfg, nullptr, 0, nullptr, &r);
  if (rc) return die("ens_launch", rc);
  std::vector<ens_record> recs((size_t)n);
  std::vector<uint64_t> off((size_t)n + 1);
  rc = ens_collect(r, recs.data(), nullptr, nullptr, 0, off.data());
  if (rc) return die("ens_collect", rc);
  std::vector<char> out((size_t)off[(size_t)n] + 1);
  rc = ens_collect(r, recs.data(), nullptr, out.data(), out.size(), off.data());
  if (rc) return die("ens_collect", rc);
  if (!quiet) std::fwrite(out.data(), 1, (size_t)off[(size_t)n], stdout);
  float ms = 0;
  ens_run_elapsed_ms(r, &ms);
  ens_run_info info;
  ens_run_get_info(r, &info);
  int nonzero = 0;
  for (auto &x : recs) nonzero += x.exit_code != 0;
  std::fprintf(stderr, "ens_run: %d instances, %d kernel launch(es), %.3f ms, %.1f instances/s, %d nonzero exit\n", n,
               info.kernel_launches, ms, ms > 0 ? n / (ms * 1e-3) : 0.0, nonzero);
  ens_run_free(r);
  ens_args_free(a);
  return 0;
}
