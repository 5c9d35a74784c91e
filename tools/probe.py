"""Time ensembles of arbitrary lines on the GPU (phase probes, not the bench).

    python tools/probe.py "xsbench -s large -g 11303 -G hash -l 0 -r {i}" 64 [threads] [reps]
"""
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_icppw_tiancd23_b200 import Args  # noqa: E402
from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble  # noqa: E402


def probe(template, n, threads=512, reps=3):
    text = "".join(template.format(i=i) + "\n" for i in range(n))
    e = Ensemble(Args.parse(text), app="auto", threads=threads).launch()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        e.relaunch()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    r = e.collect(stdout=False)
    ok = bool((r.records["exit_code"] == 0).all())
    info = e.info()
    e.close()
    return min(ts), ok, list(info.grid_blocks), list(info.block_threads)


if __name__ == "__main__":
    if len(sys.argv) > 2:
        t, ok, g, T = probe(sys.argv[1], int(sys.argv[2]), *(int(x) for x in sys.argv[3:]))
        print(f"{t:9.3f} ms ok={ok} grid={g} T={T} :: {sys.argv[1]} x{sys.argv[2]}")
    else:
        cases = [
            ("xsbench -s large -g 11303 -G hash -h 10000 -l 0 -r {i}", 64, 512),
            ("xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r {i}", 64, 512),
            ("xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r {i}", 1, 512),
            ("xsbench -s small -g 1000 -G unionized -l 0 -r {i}", 1024, 256),
            ("xsbench -s small -g 1000 -G unionized -l 10000 -r {i}", 1024, 256),
            ("xsbench -s small -g 1000 -G unionized -l 10000 -r {i}", 1024, 128),
            ("xsbench -s small -g 1000 -G unionized -l 10000 -r {i}", 1024, 512),
            ("rsbench -s small -l 10000 -p 1000 -w 100 -r {i}", 256, 256),
            ("amgmk -x 32 -y 32 -z 32 -i 20 -k relax -r {i}", 1024, 1024),
        ]
        for tpl, n, T in cases:
            t, ok, g, TT = probe(tpl, n, T)
            print(f"{t:9.3f} ms ok={ok} grid={g} T={TT} :: {tpl} x{n}", flush=True)
