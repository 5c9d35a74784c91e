// csrc/tools/ens_run.cpp — N5, the enhanced loader's command line (§3.2
// P:422-436, Fig. 5c; SURVEY.md §8(b) CLI):
//   ens_run -f <args file> [-n <num instances>] [-t <thread limit>]
//           [-a auto|echo|xsbench|rsbench|amgmk|pagerank] [-g grid]
//           [-M instances per CTA] [--gpus G] [--json out.json]
//           [--argv0 name] [--timestamps] [-q]
// Runs the first n lines as one ensemble, prints every instance's stdout in
// instance order, then one summary line on stderr.  --gpus G shards the
// instances by id over the first G GPUs of this process (instance i on GPU
// i mod G: ens_launch with first = g, stride = G, one workspace per GPU, all
// G launches in flight at once) and merges the records and stdout back into
// instance order on the host — no collective is needed inside one process
// (the torch.distributed launcher, python -m paper_conf_icppw_tiancd23_b200.run,
// is the one-process-per-GPU form with its NCCL all-gather).  --json writes
// every instance's record and the run's summary.
#include <cuda_runtime.h>

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

struct Shard {  // one GPU's part of the ensemble
  ens_run *r = nullptr;
  int n = 0;  // its instances: global ids g, g + G, ...
  std::vector<ens_record> recs;
  std::vector<uint64_t> off;
  std::vector<char> out;
  float ms = 0.f;
  int kernels = 0;
};

static void json_str(FILE *f, const char *s, size_t n) {
  std::fputc('"', f);
  for (size_t i = 0; i < n; i++) {
    const unsigned char ch = (unsigned char)s[i];
    if (ch == '"' || ch == '\\') std::fprintf(f, "\\%c", ch);
    else if (ch == '\n') std::fputs("\\n", f);
    else if (ch < 0x20) std::fprintf(f, "\\u%04x", ch);
    else std::fputc(ch, f);
  }
  std::fputc('"', f);
}

int main(int argc, char **argv) {
  const char *file = nullptr, *argv0 = nullptr, *json = nullptr;
  int n = -1, t = 0, grid = 0, m = 0, gpus = 1;
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
    else if (f == "--gpus") gpus = std::atoi(val());
    else if (f == "--json") json = val();
    else if (f == "--argv0") argv0 = val();
    else if (f == "--timestamps") ts = true;
    else if (f == "-q") quiet = true;
    else if (f == "-a") {
      std::string a = val();
      app = a == "echo" ? ENS_APP_ECHO : a == "xsbench" ? ENS_APP_XSBENCH : a == "rsbench" ? ENS_APP_RSBENCH
          : a == "amgmk" ? ENS_APP_AMGMK : a == "pagerank" ? ENS_APP_PAGERANK : ENS_APP_BY_ARGV0;
    } else {
      std::fprintf(stderr, "usage: ens_run -f file [-n N] [-t T] [-a auto|echo|xsbench|rsbench|amgmk|pagerank] [-g grid] "
                           "[-M instances per CTA] [--gpus G] [--json out.json] "
                           "[--argv0 name] [--timestamps] [-q]\n");
      return 2;
    }
  }
  if (!file) {
    std::fprintf(stderr, "ens_run: -f is required\n");
    return 2;
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess) ndev = 0;
  if (gpus < 1 || gpus > ndev) {
    std::fprintf(stderr, "ens_run: --gpus %d, but %d GPU(s) visible\n", gpus, ndev);
    return 2;
  }
  static const char *names[] = {nullptr, "echo", "xsbench", "rsbench", "amgmk", "pagerank"};
  if (!argv0 && app != ENS_APP_BY_ARGV0) argv0 = names[app];
  ens_args *a = nullptr;
  int rc = ens_load_args(file, argv0, &a);
  if (rc) return die("ens_load_args", rc);
  if (n < 0) n = ens_args_count(a);
  if (n > ens_args_count(a)) return die("ens_launch", ENS_ERANGE);  // reading Q4: the first n lines
  // shard g: instances g, g + G, ... (launched on GPU g; every launch in flight before any collect)
  std::vector<Shard> sh((size_t)gpus);
  for (int g = 0; g < gpus; g++) {
    Shard &s = sh[(size_t)g];
    s.n = n > g ? (n - g + gpus - 1) / gpus : 0;
    if (cudaSetDevice(g) != cudaSuccess) return die("cudaSetDevice", ENS_ECUDA);
    ens_launch_cfg cfg{};
    cfg.first = (uint32_t)g;
    cfg.n_instances = (uint32_t)s.n;
    cfg.stride = (uint32_t)gpus;
    cfg.grid_blocks = grid;
    cfg.block_threads = t;
    cfg.instances_per_cta = m;
    cfg.flags = ts ? ENS_F_TIMESTAMPS : 0;
    rc = ens_launch(app, a, &cfg, nullptr, 0, nullptr, &s.r);
    if (rc) return die("ens_launch", rc);
  }
  for (int g = 0; g < gpus; g++) {
    Shard &s = sh[(size_t)g];
    if (cudaSetDevice(g) != cudaSuccess) return die("cudaSetDevice", ENS_ECUDA);
    s.recs.resize((size_t)s.n);
    s.off.resize((size_t)s.n + 1);
    rc = ens_collect(s.r, s.recs.data(), nullptr, nullptr, 0, s.off.data());
    if (rc) return die("ens_collect", rc);
    s.out.resize((size_t)s.off[(size_t)s.n] + 1);
    rc = ens_collect(s.r, s.recs.data(), nullptr, s.out.data(), s.out.size(), s.off.data());
    if (rc) return die("ens_collect", rc);
    ens_run_elapsed_ms(s.r, &s.ms);
    ens_run_info info;
    ens_run_get_info(s.r, &info);
    s.kernels = info.kernel_launches;
  }
  // instance i = shard i mod G, local index i / G
  auto rec_of = [&](int i) -> const ens_record & { return sh[(size_t)(i % gpus)].recs[(size_t)(i / gpus)]; };
  if (!quiet)
    for (int i = 0; i < n; i++) {
      const Shard &s = sh[(size_t)(i % gpus)];
      const size_t k = (size_t)(i / gpus);
      std::fwrite(s.out.data() + s.off[k], 1, (size_t)(s.off[k + 1] - s.off[k]), stdout);
    }
  float ms = 0.f;  // the slowest GPU's launch
  int kernels = 0, nonzero = 0;
  for (const Shard &s : sh) {
    ms = s.ms > ms ? s.ms : ms;
    kernels += s.kernels;
  }
  for (int i = 0; i < n; i++) nonzero += rec_of(i).exit_code != 0;
  std::fprintf(stderr, "ens_run: %d instances on %d GPU(s), %d kernel launch(es), %.3f ms, %.1f instances/s, %d nonzero exit\n",
               n, gpus, kernels, ms, ms > 0 ? n / (ms * 1e-3) : 0.0, nonzero);
  if (json) {
    FILE *f = std::fopen(json, "w");
    if (!f) {
      std::fprintf(stderr, "ens_run: cannot write %s\n", json);
      return 2;
    }
    std::fprintf(f, "{\"instances\": %d, \"gpus\": %d, \"kernel_launches\": %d, \"ms\": %.6f, \"instances_per_s\": %.3f, "
                    "\"nonzero_exit\": %d, \"records\": [\n", n, gpus, kernels, ms, ms > 0 ? n / (ms * 1e-3) : 0.0, nonzero);
    for (int i = 0; i < n; i++) {
      const ens_record &r = rec_of(i);
      const Shard &s = sh[(size_t)(i % gpus)];
      const size_t k = (size_t)(i / gpus);
      std::fprintf(f, "  {\"instance\": %u, \"gpu\": %d, \"exit_code\": %d, \"app\": %u, \"flags\": %u, \"vhash\": %llu, "
                      "\"bitsum\": %llu, \"fsum\": %.17g, \"fabs\": %.17g, \"work\": %llu, \"stdout\": ",
                   r.instance, i % gpus, r.exit_code, r.app, r.flags, (unsigned long long)r.vhash,
                   (unsigned long long)r.bitsum, r.fsum, r.fabs, (unsigned long long)r.work);
      json_str(f, s.out.data() + s.off[k], (size_t)(s.off[k + 1] - s.off[k]));
      std::fprintf(f, "}%s\n", i + 1 < n ? "," : "");
    }
    std::fprintf(f, "]}\n");
    std::fclose(f);
  }
  for (int g = 0; g < gpus; g++) {
    cudaSetDevice(g);
    ens_run_free(sh[(size_t)g].r);
  }
  ens_args_free(a);
  return 0;
}
