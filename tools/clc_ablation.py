"""Scheduler ablation: persistent CTAs + atomic counter (default) vs one CTA
per instance + cluster launch control (ENS_F_CLC), fused, teams of one CTA, median of 5 relaunches.

    python tools/clc_ablation.py [out.json]
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_icppw_tiancd23_b200 import Args  # noqa: E402
from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble  # noqa: E402


def t(lines, threads, **kw):
    e = Ensemble(Args.parse(bench.W.text(lines)), app="auto", threads=threads, team_ctas=1, fused=True, **kw).launch()
    torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        e.relaunch()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    r = e.collect(stdout=False)
    e.close()
    return statistics.median(ts), r.records


rows = []
cases = [("C4", None), ("TSTAR", None), ("C5", None), ("C3", None),
         ("echo x4096", ["echo %d" % i for i in range(4096)]),
         ("AMG 8^3 x 20000", ["amgmk -x 8 -y 8 -z 8 -i 20 -r %d" % i for i in range(20000)])]
for name, lines in cases:
    threads = bench.THREADS.get(name, 256)
    if lines is None:
        lines, _ = bench.workload_lines(name, 1)
    a, ra = t(lines, threads)
    b, rb = t(lines, threads, clc=True)
    same = bool((ra[["instance", "exit_code", "vhash", "bitsum"]] == rb[["instance", "exit_code", "vhash", "bitsum"]]).all())
    rows.append({"config": name, "instances": len(lines), "threads": threads, "counter_ms": a, "clc_ms": b,
                 "clc_over_counter": b / a, "records_equal": same})
    print(f"{name:18s} n={len(lines):6d} counter {a:9.3f} ms  clc {b:9.3f} ms  ratio {b / a:6.3f}  equal={same}",
          flush=True)
out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "clc_ablation_r2.json")
json.dump({"what": "persistent CTAs + atomic counter vs one CTA per instance + cluster launch control "
                   "(ENS_F_CLC); fused, one-CTA teams; median of 5 relaunches (CUDA events)", "rows": rows},
          open(out, "w"), indent=1)
