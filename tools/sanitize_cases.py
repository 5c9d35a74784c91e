"""Small ensembles for compute-sanitizer (memcheck / racecheck / synccheck) over the runtime's
isolation-critical paths (instances share nothing): persistent teams with slot reuse
(more instances than slots), a 2-CTA cluster team (DSMEM partials, cluster barriers), M = 4
instances per CTA (named barriers), a concurrent mixed-app ensemble (forked streams, separate
arena regions) and split phases (init items, lookup items, last-item records).

    compute-sanitizer --tool racecheck python tools/sanitize_cases.py [case ...]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
from paper_conf_icppw_tiancd23_b200 import Args  # noqa: E402
from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble  # noqa: E402

XS = "xsbench -s small -g 60 -l 600 -G {g} -h 30 -r {s}"
CASES = {
    # C1-style N = 8 at T = 64 on 2 slots: slot reuse by later instances
    "slots": (["xsbench -s small -g 100 -l 800 -G unionized -r %d" % (1070 + i) for i in range(8)],
              dict(threads=64, grid=2, team_ctas=1)),
    "cluster2": ([XS.format(g="hash", s=i) for i in range(3)] + ["rsbench -s small -l 300 -p 20 -w 4 -r 2"],
                 dict(threads=128, team_ctas=2, fused=True)),
    "sub4": (["amgmk -x 4 -y 4 -z 4 -i 3 -r %d" % i for i in range(9)] + ["echo m4"],
             dict(threads=256, instances_per_cta=4)),
    "mixed": ([XS.format(g="unionized", s=1), "rsbench -s small -l 200 -p 10 -w 3 -r 3",
               "amgmk -x 5 -y 4 -z 3 -i 2 -r 1", "pagerank -n 300 -e 3 -i 2 -R 1", "echo x", "nosuch"],
              dict(threads=128)),
    "split": ([XS.format(g=g, s=i) for i, g in enumerate(["hash", "unionized", "nuclide", "hash"])] +
              ["rsbench -s small -l 2500 -p 20 -w 4 -r 5", "rsbench -s small -l 300 -p 12 -w 3 -d -r 6"],
              dict(threads=128, split=True)),
    # phase 1b's lookup sort over several chunks (count / scan / scatter / fine items
    # and their cross-CTA flags), two hash instances
    "split2": (["xsbench -s small -g 200 -l 140000 -G hash -h 150 -r %d" % (7 + i) for i in range(2)],
               dict(threads=128, split=True)),
}


def main():
    names = sys.argv[1:] or list(CASES)
    torch.cuda.set_device(0)
    for n in names:
        lines, kw = CASES[n]
        e = Ensemble(Args.parse("".join(l + "\n" for l in lines)), app="auto", **kw).launch()
        e.relaunch()
        r = e.collect()
        e.close()
        torch.cuda.synchronize()
        print(n, "exit codes", [int(x) for x in r.records["exit_code"]], flush=True)


if __name__ == "__main__":
    main()
