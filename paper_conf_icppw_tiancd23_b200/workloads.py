"""Seeded synthetic workloads: args files for the configs of SURVEY.md §8(d).

This module only writes command lines (it holds none of the method's
arithmetic); both the CUDA path and the oracle consume its output.  Each line
names its app in argv[0] (the mixed-app form, reading Q3).

  C1     4 x XSBench-style small (68 nuclides, 1000 gridpoints, 10k lookups)
  C2     64 x XSBench-style large (355 nuclides, 11303 gridpoints), hash grid,
         1M lookups — the paper's 64-instance point
  C3     256 x RSBench-style small with varied lookups/poles/windows, 1/4 no-doppler
  C4     1024 x AMGmk-style 32^3 relax, 20 sweeps (T = 1024)
  C5     4096 mixed lines (XS / XS / RS / AMG by i mod 4), sharded by instance id
  TSTAR  1024 x C1-style XSBench instances — the north-star target launch
"""
import numpy as np

C1_LINE = "xsbench -s small -g 1000 -l 10000 -m event -G unionized -r {seed}"
C2_LINE = "xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r {seed}"
C4_LINE = "amgmk -x 32 -y 32 -z 32 -i 20 -k relax -r {seed}"
C5_RS_LINE = "rsbench -s small -l 10000 -p 1000 -w 100 -r {seed}"


def c1(n=4, seed0=1070):
    return [C1_LINE.format(seed=seed0 + i) for i in range(n)]


def c2(n=64, seed0=1070, lookups=1000000):
    return [C2_LINE.format(seed=seed0 + i).replace("-l 1000000", f"-l {lookups}") for i in range(n)]


def c3(n=256, gen_seed=0):
    rng = np.random.default_rng(gen_seed)
    out = []
    for i in range(n):
        L = int(rng.choice([10000, 20000, 40000]))
        P = int(rng.choice([500, 1000, 2000]))
        W = int(rng.choice([50, 100, 200]))
        d = " -d" if rng.random() < 0.25 else ""
        out.append(f"rsbench -s small -l {L} -p {P} -w {W}{d} -r {1 + i}")
    return out


def c4(n=1024):
    return [C4_LINE.format(seed=1 + i) for i in range(n)]


def c5(n=4096):
    out = []
    for i in range(n):
        m = i % 4
        if m in (0, 1):
            out.append(C1_LINE.format(seed=1070 + i))
        elif m == 2:
            out.append(C5_RS_LINE.format(seed=1 + i))
        else:
            out.append(C4_LINE.format(seed=1 + i))
    return out


def tstar(n=1024, seed0=1070):
    return c1(n, seed0)


def pr(n=256):
    """NEXT 3: Page-Rank-style instances (100k nodes, mean out-degree 8, 10 iterations)."""
    return [f"pagerank -n 100000 -e 8 -i 10 -R {i}" for i in range(n)]


def xs_history(n=64, particles=100000):
    """NEXT 2: XSBench-style history mode (small), distinct seeds."""
    return [f"xsbench -s small -m history -p {particles} -G unionized -r {1070 + i}" for i in range(n)]


CONFIGS = {"C1": c1, "C2": c2, "C3": c3, "C4": c4, "C5": c5, "TSTAR": tstar, "PR": pr, "XSHIST": xs_history}


def text(lines):
    return "".join(l + "\n" for l in lines)


def write(path, lines):
    with open(path, "w") as f:
        f.write(text(lines))
    return path
