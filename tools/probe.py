"""Time ensembles of arbitrary lines on the GPU (phase probes, not the bench).

    python tools/probe.py "<line template with {i}>" N [threads] [reps] [--phases] [--team K] [--m M]

Prints the best-of-reps CUDA-event time of the ensemble launch; with
--phases also the per-phase device time (ENS_F_PHASES tracing), summed over
instances and divided by the number of concurrently running teams (so the
numbers are comparable to the wall time).
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_icppw_tiancd23_b200 import Args  # noqa: E402
from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble  # noqa: E402

XS_PHASES = [  # phase ids by init path: block-wide unionized / hash+nuclide (init_nuc) / warp path (init_warp)
    "materials", "count", "scan | warp: scan+scatter", "scatter | warp: bucket sort", "bucket sort",
    "clear tables | warp: records+ustart", "union tables | warp: wait for nuclides", "index sweep",
    "record permute | warp: wait for chunks", "hash column | warp: index rows", "lookup sample+sort",
    "lookup gathers", "warp: chunk setup", "warp: chunk gather+count+scatter", "warp: chunk sort",
    "warp: union energies + search table"]


def probe(template, n, threads=512, reps=3, phases=False, team=0, m=0):
    text = "".join(template.format(i=i) + "\n" for i in range(n))
    e = Ensemble(Args.parse(text), app="auto", threads=threads, phases=phases, team_ctas=team,
                 instances_per_cta=m).launch()
    torch.cuda.synchronize()
    ts = []
    ph = None
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        e.relaunch()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
        if phases:
            ph = e.run.phases_ns()
    r = e.collect(stdout=False)
    ok = bool((r.records["exit_code"] == 0).all())
    info = e.info()
    e.close()
    return min(ts), ok, list(info.grid_blocks), list(info.block_threads), list(info.team_ctas), ph


if __name__ == "__main__":
    args = [x for x in sys.argv[1:] if not x.startswith("--")]
    phases = "--phases" in sys.argv
    team = 0
    if "--team" in sys.argv:
        team = int(sys.argv[sys.argv.index("--team") + 1])
        args.remove(str(team))
    if "--l2fetch" in sys.argv:  # cudaLimitMaxL2FetchGranularity experiment
        from cuda.bindings import runtime as rt
        g = int(sys.argv[sys.argv.index("--l2fetch") + 1])
        args.remove(str(g))
        torch.cuda.init()
        torch.zeros(1, device="cuda")
        print("set", rt.cudaDeviceSetLimit(rt.cudaLimit.cudaLimitMaxL2FetchGranularity, g),
              "get", rt.cudaDeviceGetLimit(rt.cudaLimit.cudaLimitMaxL2FetchGranularity), flush=True)
    m = 0
    if "--m" in sys.argv:
        m = int(sys.argv[sys.argv.index("--m") + 1])
        args.remove(str(m))
    t, ok, g, T, cs, ph = probe(args[0], int(args[1]), *(int(x) for x in args[2:]), phases=phases, team=team, m=m)
    print(f"{t:9.3f} ms ok={ok} grid={g} T={T} team={cs} m={m} :: {args[0]} x{args[1]}", flush=True)
    if ph:
        teams = max(max(g) // max(1, max(cs)), 1)
        for k, v in enumerate(ph):
            if v:
                name = XS_PHASES[k] if k < len(XS_PHASES) else str(k)
                print(f"    phase {k:2d} {name:20s} {v / 1e6 / teams:9.3f} ms per team", flush=True)
