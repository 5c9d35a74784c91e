"""Oracle XSBench-style pins.

* upstream XSBench v20's documented default checksum (tests/golden/) pins the
  whole chain: LCG, concentrations, material lists, grid, sort, bracket,
  interpolation, macro sum, argmax/verification;
* the index grids equal their closed forms (numpy, brute force);
* the three grid types and a linear scan give the same bracket;
* verification invariants hold.
"""
import json
import os

import numpy as np
import pytest

GOLD = os.path.join(os.path.dirname(__file__), "golden")


@pytest.mark.slow
def test_upstream_default_checksum_small(oracle):
    gold = json.load(open(os.path.join(GOLD, "xsbench_upstream_checksums.json")))["checksums"]
    r = oracle.run_text("-s small -m event -G hash\n", app=oracle.APP_XSBENCH)
    rec = r.records[0]
    assert rec["exit_code"] == 0
    assert int(rec["vhash"]) == gold["-s small -m event"]
    assert r.stdout[0].endswith(b"Verification checksum: %d\n" % gold["-s small -m event"])


@pytest.mark.slow
def test_upstream_history_checksum_small(oracle):
    """History mode (NEXT 2): 500,000 particles x 34 dependent lookups."""
    gold = json.load(open(os.path.join(GOLD, "xsbench_upstream_checksums.json")))["checksums"]
    r = oracle.run_text("-s small -m history -G hash\n", app=oracle.APP_XSBENCH)
    assert r.records[0]["exit_code"] == 0
    assert int(r.records[0]["vhash"]) == gold["-s small -m history"]
    assert r.records[0]["work"] == 500000 * 34


@pytest.mark.slow
def test_upstream_default_checksum_large(oracle):
    gold = json.load(open(os.path.join(GOLD, "xsbench_upstream_checksums.json")))["checksums"]
    r = oracle.run_text("-s large -m event -G hash\n", app=oracle.APP_XSBENCH)
    assert r.records[0]["exit_code"] == 0
    assert int(r.records[0]["vhash"]) == gold["-s large -m event"]


@pytest.mark.parametrize("n_iso,n_gp,seed", [(3, 2, 1), (4, 5, 2), (7, 16, 3), (12, 9, 4), (5, 33, 5)])
def test_unionized_index_closed_form(oracle, n_iso, n_gp, seed):
    """XS-5: union = sorted energies; ig[e][i] = clip(#{k>=1: E_i[k] <= u_e}, 0, n_gp-2)."""
    t = oracle.XsTiny(n_iso, n_gp, 0, gseed=seed)
    E = t.energies
    assert np.all(np.diff(E, axis=1) > 0)
    u = np.sort(E.ravel())
    assert np.array_equal(t.union, u)
    ig = t.index.reshape(n_iso * n_gp, n_iso)
    for i in range(n_iso):
        exp = np.clip(np.searchsorted(E[i, 1:], u, side="right"), 0, n_gp - 2)
        assert np.array_equal(ig[:, i], exp)


@pytest.mark.parametrize("n_iso,n_gp,bins", [(3, 2, 1), (4, 5, 7), (6, 16, 10), (5, 40, 64)])
def test_hash_index_closed_form(oracle, n_iso, n_gp, bins):
    """XS-5 hash: ig[b][i] = grid_search(E_i, b/bins) = clip(#{k>=1: E_i[k] <= b*du}, 0, n_gp-2)."""
    t = oracle.XsTiny(n_iso, n_gp, 2, bins=bins, gseed=9)
    E = t.energies
    ig = t.index.reshape(bins, n_iso)
    q = np.arange(bins) * (1.0 / bins)
    for i in range(n_iso):
        exp = np.clip(np.searchsorted(E[i, 1:], q, side="right"), 0, n_gp - 2)
        assert np.array_equal(ig[:, i], exp)


@pytest.mark.parametrize("n_gp", [2, 3, 4, 8, 16])
def test_bracket_all_grids_equal_linear_scan(oracle, n_gp):
    """XS-7: unionized == nuclide == hash == linear scan (the bracketing pair [lo, lo+1])."""
    n_iso = 6
    grids = [oracle.XsTiny(n_iso, n_gp, g, bins=b, gseed=11) for g, b in [(0, 1), (1, 1), (2, 5), (2, 37)]]
    E = grids[0].energies
    rng = np.random.default_rng(n_gp)
    ps = list(rng.random(200)) + list(E.ravel()) + [0.0, np.nextafter(1.0, 0)]
    for p in ps:
        for nuc in range(n_iso):
            # linear scan: largest k in [0, n_gp-2] with k == 0 or E[k] <= p
            lo = 0
            for k in range(1, n_gp - 1):
                if E[nuc, k] <= p:
                    lo = k
            got = [g.bracket(nuc, p) for g in grids]
            assert got == [lo] * 4, (p, nuc, got, lo)


def test_materials_tables(oracle):
    """Hoogenboom-Martin lists: counts, ranges, large appends 68..354 to the fuel."""
    num_s, mats_s = oracle.xs_materials(68)
    num_l, mats_l = oracle.xs_materials(355)
    assert list(num_s) == [34, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9]
    assert list(num_l) == [321] + list(num_s[1:])
    assert list(mats_l[0, 34:321]) == list(range(68, 355))
    assert np.array_equal(mats_l[0, :34], mats_s[0, :34])
    for m in range(12):
        row = mats_s[m, :num_s[m]]
        assert len(set(row)) == len(row) and row.max() < 68


@pytest.mark.parametrize("grid", ["unionized", "nuclide", "hash"])
def test_verification_invariants(oracle, grid):
    L = 3000
    text = f"-s small -g 200 -l {L} -G {grid} -h 100 -r 7\n"
    r = oracle.run_text(text, app=oracle.APP_XSBENCH)
    rec, tal = r.records[0], r.tallies[0]
    assert rec["exit_code"] == 0 and rec["work"] == L
    ver = sum((c + 1) * int(tal[c]) for c in range(5))
    assert L <= ver <= 5 * L
    assert int(rec["vhash"]) == ver % 999983
    assert int(tal[5:17].sum()) == L
    assert tal[0:5].sum() == L
    assert rec["fabs"] >= abs(rec["fsum"]) > 0  # extrapolation outside [E0, En-1] may go negative


def test_grid_types_agree_bitwise(oracle):
    """All three grids give identical records (same bracket => same arithmetic)."""
    recs = []
    for g in ["unionized", "nuclide", "hash"]:
        r = oracle.run_text(f"-s small -g 300 -l 2000 -G {g} -h 77 -r 5 -R 9\n", app=oracle.APP_XSBENCH)
        recs.append(r.records[0])
    for k in ["vhash", "bitsum", "fsum", "work"]:
        assert recs[0][k] == recs[1][k] == recs[2][k]


@pytest.mark.parametrize("line", ["-s medium", "-g 1", "-g", "-l -5", "-G sorted", "-m hist", "-q 1",
                                  "-g 12x", "-r -1", "-h 0", "-g 65537"])
def test_usage_errors(oracle, line):
    r = oracle.run_text(line + "\n", app=oracle.APP_XSBENCH)
    assert r.records[0]["exit_code"] == 1
    assert b"invalid argument" in r.stdout[0] and b"usage: xsbench" in r.stdout[0]


def test_gp_range_upper_bound(oracle):
    """Reading R-xs-range: -g up to 2^16 is a valid line (the oracle's bound since its first
    commit); a run at the bound keeps the XS-10 invariants."""
    L = 300
    r = oracle.run_text(f"-s small -g 65536 -l {L} -G hash -h 100 -r 5\n", app=oracle.APP_XSBENCH)
    rec, tal = r.records[0], r.tallies[0]
    assert rec["exit_code"] == 0 and rec["work"] == L
    ver = sum((c + 1) * int(tal[c]) for c in range(5))
    assert L <= ver <= 5 * L and int(rec["vhash"]) == ver % 999983
