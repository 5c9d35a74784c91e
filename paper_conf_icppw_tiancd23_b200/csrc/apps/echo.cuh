// csrc/apps/echo.cuh — N1 instance bodies: `echo` (prints its argc/argv and
// returns argc: the loader's contract of Fig. 4 P:362-385 made visible) and
// the internal `notfound` body (argv[0] names no app under
// ENS_APP_BY_ARGV0: print "<argv0>: command not found", exit 127).
#pragma once
#include "../rt/device_rt.cuh"
#include "params.cuh"

namespace ens {

struct EchoApp {
  static constexpr uint32_t kId = APP_ECHO;
  static constexpr int kMaxT = 1024;
  static constexpr bool kTeam = false;
  static constexpr bool kSub = true;
  __device__ static Result run(Ctx &c, int argc, char **argv) {
    Result R{};
    ens_printf(c, FMT_ECHO_ARGC, argc);
    for (int i = 0; i < argc; i++) ens_printf(c, FMT_ECHO_ARGV, i, (const char *)argv[i]);
    R.exit_code = argc;
    R.work = (uint64_t)argc;
    return R;
  }
  __host__ static bool size(int, const char *const *, int, int, uint64_t *arena, uint32_t *smem) {
    *arena = 0;
    *smem = 0;
    return true;
  }
};

struct NotFoundApp {
  static constexpr uint32_t kId = APP_NOTFOUND;
  static constexpr int kMaxT = 1024;
  static constexpr bool kTeam = false;
  static constexpr bool kSub = true;
  __device__ static Result run(Ctx &c, int argc, char **argv) {
    Result R{};
    ens_printf(c, FMT_NOTFOUND, argc > 0 ? (const char *)argv[0] : "");
    R.exit_code = ENS_EXIT_NOTFOUND;
    return R;
  }
  __host__ static bool size(int, const char *const *, int, int, uint64_t *arena, uint32_t *smem) {
    *arena = 0;
    *smem = 0;
    return true;
  }
};

}  // namespace ens
