"""One warm launch of a bench workload, for profilers (not the bench).

    python tools/prof_workload.py <C1|C2|C2U|C3|C4|C5|TSTAR> [relaunches] [--threads T] [--team K] [--fused | --split]

Launches the workload's ensemble once (cold) and relaunches it `relaunches` times (default 1):
`ncu --launch-skip <kernels per launch> --launch-count 1 -k regex:ens_kernel` then captures a
warm launch.  Prints each relaunch's CUDA-event time.
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
    fused = "--fused" in argv
    if fused:
        argv.remove("--fused")
    split = "--split" in argv
    if split:
        argv.remove("--split")
    opt = {}
    for k in ("--threads", "--team"):
        if k in argv:
            i = argv.index(k)
            opt[k] = int(argv[i + 1])
            del argv[i:i + 2]
    name = argv[0]
    reps = int(argv[1]) if len(argv) > 1 else 1
    lines, desc = bench.workload_lines(name, 1)
    threads = opt.get("--threads", bench.THREADS.get(name, 256))
    e = Ensemble(Args.parse(workloads.text(lines)), app="auto", threads=threads,
                 team_ctas=opt.get("--team", 0), fused=fused, split=split).launch()
    torch.cuda.synchronize()
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        e.relaunch()
        b.record()
        torch.cuda.synchronize()
        print(f"{name}{' fused' if fused else ''}{' split' if split else ''}: {a.elapsed_time(b):.3f} ms", flush=True)
    r = e.collect(stdout=False)
    i = e.info()
    print(f"exit ok={bool((r.records['exit_code'] == 0).all())} kernels/launch={i.kernel_launches} "
          f"grid={list(i.grid_blocks)} T={list(i.block_threads)} team={list(i.team_ctas)}", flush=True)
    e.close()


if __name__ == "__main__":
    main()
