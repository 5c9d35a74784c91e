"""SWEEP: the paper's Fig. 6 measurement on B200.

    python tools/sweep.py [--out profiles/sweep_r1.json] [--max-n 1024] [--reps 3] [--auto]

For each app and thread limit T, the ensemble of N instances (distinct seeds)
is launched N = 1, 2, 4, ... and timed with CUDA events on its stream (median
of `reps` relaunches, arguments resident).  The paper's metric is the relative
speedup T1*N/TN, T1 = the same launch at N = 1 with the same T
(one T1 per thread-limit panel, reading Q7); "linear" = N is its upper bound
(P:549-554).  Teams are one CTA (the paper's team = one thread block,
P:313-318), M = 1, every instance start to finish in the one ensemble kernel
(ENS_F_FUSED: the paper's mapping).  Also reported: instances/s and busy SMs (from the
per-instance smid of the records).  With --auto the launches use the product's own mapping
instead (cluster teams, split phases, longest-first queue: the library's defaults), so the
curve shows what the framework delivers at each N next to the paper's mapping.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
from paper_conf_icppw_tiancd23_b200 import Args  # noqa: E402
from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble  # noqa: E402

APPS = {
    "XSBench": "xsbench -s small -g 1000 -l 10000 -G unionized -r {s}",
    "RSBench": "rsbench -s small -l 10000 -p 1000 -w 100 -r {s}",
    "AMGmk": "amgmk -x 32 -y 32 -z 32 -i 20 -k relax -r {s}",
    "Page-Rank": "pagerank -n 100000 -e 8 -i 10 -R {s}",
}


def time_launch(lines, threads, reps, auto=False):
    text = "".join(l + "\n" for l in lines)
    kw = {} if auto else dict(team_ctas=1, fused=True)
    e = Ensemble(Args.parse(text), app="auto", threads=threads, timestamps=True, **kw).launch()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        e.relaunch()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    r = e.collect(tallies=False, stdout=False)
    ok = bool((r.records["exit_code"] == 0).all())
    sms = len(set(int(x) for x in r.records["smid"]))
    info = e.info()
    e.close()
    return statistics.median(ts), ok, sms, int(max(info.block_threads)), int(max(info.grid_blocks))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "sweep_r2.json"))
    ap.add_argument("--max-n", type=int, default=4096)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--threads", default="32,256,1024")
    ap.add_argument("--apps", default=",".join(APPS))
    ap.add_argument("--auto", action="store_true", help="the library's default mapping (not the paper's)")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    ns = []
    n = 1
    while n <= a.max_n:
        ns.append(n)
        n *= 2
    rows = []
    for app in a.apps.split(","):
        tmpl = APPS[app]
        for T in (int(x) for x in a.threads.split(",")):
            t1 = None
            for n in ns:
                lines = [tmpl.format(s=1 + i) for i in range(n)]
                ms, ok, sms, Treal, grid = time_launch(lines, T, a.reps, a.auto)
                if n == 1:
                    t1 = ms
                row = {"app": app, "T_limit": T, "T": Treal, "N": n, "grid": grid, "ms": ms, "ok": ok,
                       "busy_sms": sms, "instances_per_s": n / (ms * 1e-3), "speedup": t1 * n / ms}
                rows.append(row)
                print(f"{app:10s} T={Treal:5d} N={n:5d} grid={grid:5d} {ms:9.3f} ms  speedup {row['speedup']:8.2f}"
                      f"  sms {sms:3d}  ok={ok}", flush=True)
    what = ("T1*N/TN on one B200 (paper Fig. 6 metric, P:540-554); the library's default mapping (cluster teams, "
            "split phases); median of reps" if a.auto else
            "T1*N/TN on one B200 (paper Fig. 6 metric, P:540-554); team = 1 CTA, fused; median of reps")
    out = {"what": what,
           "paper_context": "up to 51x at 64 instances on an A100 40GB (P:44-45, P:639-640)",
           "device": torch.cuda.get_device_name(0), "apps": APPS, "rows": rows}
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
