"""Element-wise parity: every lookup's result vector, not only the per-instance sums.

The launch is made with ens_launch_cfg.dump_rows = L, so each XS / RS instance writes one row
{energy, material, macro[0..4], argmax} per lookup (in the kernel's sorted order) and each AMG
instance the rows of its reported vector; the oracle writes the same rows in lookup order
(oracle.hpp Instance::dump).  Rows are matched by (energy, material): lookup energies are
distinct 63-bit LCG doubles, so the match is one-to-one, and the set of GPU keys must equal the
oracle's (every lookup ran exactly once).

Bar (SURVEY.md §8(c) "FP parity policy"):
  * XS, AMG: every element bit-exact (both sides --fmad=false / -ffp-contract=off, XS-8/9 and
    AMG-3 in the oracle's operation order);
  * RS: bit-exact as well (reading R-rs-trig: RS-3's sin/cos/atan follow one fixed algorithm on
    both sides; every division is IEEE); the test still derives the argmax safety margin: for
    every lookup the oracle's margin (max - runner-up) exceeds the two channels' combined GPU
    error (zero when bit-exact), and each instance's minimum relative margin (logged by the
    oracle over all its lookups) is positive — so vhash equality is not luck.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def run_dump(oracle, lines, rows, threads=256, **kw):
    from paper_conf_icppw_tiancd23_b200.ensemble import run_text
    text = "".join(l + "\n" for l in lines)
    g = run_text(text, app="auto", threads=threads, dump_rows=rows, **kw)
    o = oracle.run_text(text, dump=rows)
    return g, o


def match_rows(gd, od):
    """GPU rows (any order, zero rows unwritten) matched to oracle rows by (key, mat)."""
    gd = gd[gd[:, 1] >= 0]
    written = ~np.all(gd == 0, axis=1)
    gd = gd[written]
    go = np.lexsort((gd[:, 1], gd[:, 0]))
    oo = np.lexsort((od[:, 1], od[:, 0]))
    gs, os_ = gd[go], od[oo]
    assert gs.shape == os_.shape, (gs.shape, os_.shape)
    assert np.array_equal(gs[:, :2], os_[:, :2]), "lookup (energy, material) sets differ"
    return gs, os_


XS_LINES = [
    "xsbench -s small -g 1000 -l 10000 -G unionized -r 1070",
    "xsbench -s small -g 37 -l 3000 -G unionized -r 3",
    "xsbench -s small -g 1500 -l 4000 -G hash -h 1000 -r 11 -R 5",
    "xsbench -s small -g 300 -l 3000 -G nuclide -r 9",
    "xsbench -s large -g 200 -l 3000 -G hash -h 500 -r 6",
    "xsbench -s large -g 60 -l 3000 -G unionized -r 8",
    "xsbench -s small -g 20000 -l 2000 -G hash -h 1000 -r 21",
]


@pytest.mark.parametrize("team", [0, 1])
def test_xs_elementwise_bitexact(oracle, team):
    L = 10000
    g, o = run_dump(oracle, XS_LINES, L, threads=512, team_ctas=team)
    for k, line in enumerate(XS_LINES):
        gs, os_ = match_rows(g.dump[k], o.dumps[k])
        n = int(line.split("-l ")[1].split()[0])
        assert len(gs) == n, (line, len(gs))
        # every macro channel and the argmax, bit for bit
        assert np.array_equal(gs[:, 2:8].view(np.uint64), os_[:, 2:8].view(np.uint64)), line


def _rs_check(g, o, lines):
    worst = 0.0
    for k, line in enumerate(lines):
        gs, os_ = match_rows(g.dump[k], o.dumps[k])
        gv, ov = gs[:, 2:6], os_[:, 2:6]
        err = np.abs(gv - ov)
        rel = err / np.maximum(np.abs(ov), 1e-300)
        assert np.array_equal(gv.view(np.uint64), ov.view(np.uint64)), (line, float(rel.max()))
        assert np.array_equal(gs[:, 7], os_[:, 7]), line  # argmax
        # margin: the oracle's max minus runner-up exceeds the GPU error of those two channels
        am = os_[:, 7].astype(int)
        idx = np.arange(len(ov))
        top = ov[idx, am]
        others = ov.copy()
        others[idx, am] = -np.inf
        ru = others.argmax(axis=1)
        margin = top - ov[idx, ru]
        assert np.all(margin > err[idx, am] + err[idx, ru]), line
        worst = max(worst, float(rel.max()))
        assert o.margins[k] > 2 * float(rel.max()) and o.margins[k] > 0, (line, o.margins[k], float(rel.max()))
    return worst


RS_LINES = [
    "rsbench -s small -l 4000 -p 100 -w 10 -r 1",
    "rsbench -s small -l 3000 -p 1000 -w 100 -d -r 3",
    "rsbench -s small -l 4000 -p 2 -w 2 -r 6",
    "rsbench -s small -l 4000 -p 100 -w 10 -d -r 2",
    "rsbench -s small -l 3000 -p 1000 -w 100 -r 3",
    "rsbench -s large -l 1500 -p 50 -w 7 -r 4 -R 8",
    "rsbench -s small -l 2000 -p 5 -w 9 -r 5",
]


@pytest.mark.parametrize("team", [0, 1])
def test_rs_elementwise(oracle, team):
    g, o = run_dump(oracle, RS_LINES, 4000, threads=256, team_ctas=team)
    worst = _rs_check(g, o, RS_LINES)
    print(f"RS worst relative element error {worst:.3e}; min margins {o.margins.min():.3e}")


AMG_LINES = [
    "amgmk -x 9 -y 9 -z 9 -i 5 -k both -r 4",
    "amgmk -x 33 -y 2 -z 3 -i 6 -k matvec -r 3",
    "amgmk -x 16 -y 16 -z 16 -i 20 -k relax -r 7",
]


def test_amg_elementwise_bitexact(oracle):
    rows = 4096
    g, o = run_dump(oracle, AMG_LINES, rows, threads=1024)
    for k, line in enumerate(AMG_LINES):
        od = o.dumps[k]
        gd = g.dump[k][: len(od)]
        assert np.array_equal(gd[:, 0], od[:, 0]), line
        assert np.array_equal(gd[:, 2].view(np.uint64), od[:, 2].view(np.uint64)), line


def test_dump_off_by_default():
    from paper_conf_icppw_tiancd23_b200.ensemble import run_text
    g = run_text("xsbench -s small -g 50 -l 100 -r 1\n", app="auto", threads=128)
    assert g.dump is None
