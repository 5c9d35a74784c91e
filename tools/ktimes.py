"""Per-kernel CUDA-event times of a bench workload (a probe, not the bench).

    python tools/ktimes.py <C1|C2|C2U|C3|C4|C5|TSTAR> [reps] [--phases] [--split | --fused] [--team CS]

Launches the workload once (cold), relaunches it `reps` times (default 5) and
prints the best launch time and, for that launch, every kernel's time
(ens_run_kernel_times).  With --phases the launch is traced (ENS_F_PHASES)
and the per-phase device time summed over CTAs is printed too.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_icppw_tiancd23_b200 import Args, workloads  # noqa: E402
from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble  # noqa: E402


def main():
    argv = sys.argv[1:]
    phases = "--phases" in argv
    if phases:
        argv.remove("--phases")
    mode = {}
    for flag in ("--split", "--fused"):
        if flag in argv:
            argv.remove(flag)
            mode[flag[2:]] = True
    if "--team" in argv:
        i = argv.index("--team")
        mode["team_ctas"] = int(argv[i + 1])
        del argv[i:i + 2]
    name = argv[0]
    reps = int(argv[1]) if len(argv) > 1 else 5
    lines, _ = bench.workload_lines(name, 1)
    threads = bench.THREADS.get(name, 256)
    e = Ensemble(Args.parse(workloads.text(lines)), app="auto", threads=threads, phases=phases, **mode).launch()
    torch.cuda.synchronize()
    best, kt, ph = None, None, None
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        e.relaunch()
        b.record()
        torch.cuda.synchronize()
        t = a.elapsed_time(b)
        if best is None or t < best:
            best, kt = t, e.run.kernel_times()
            ph = e.run.phases_ns() if phases else None
    r = e.collect(stdout=False)
    ok = bool((r.records["exit_code"] == 0).all())
    print(f"{name}: best {best:.3f} ms of {reps} (exit ok={ok})")
    for app, phase, kind, ctas, thr, ms in kt:
        print(f"  app {app} phase {phase} kind {kind:2d} {ctas:5d} x {thr:4d}: {ms:8.3f} ms")
    if ph:
        for k, v in enumerate(ph):
            if v:
                print(f"  phase {k:2d}: {v / 1e6:10.3f} ms summed over CTAs")
    e.close()


if __name__ == "__main__":
    main()
