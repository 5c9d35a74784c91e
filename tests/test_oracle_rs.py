"""Oracle RSBench-style pins.

* fast_nuclear_W against an accurate Faddeeva function (scipy.special.wofz)
  in the region where the expansions are valid (Im z > 0);
* window partition and pole / window totals (RS-2);
* verification invariants.
Absolute RS values beyond these are "parity unpinned" vs upstream.
"""
import numpy as np
import pytest
from scipy.special import wofz


def test_fast_w_vs_faddeeva(oracle):
    rng = np.random.default_rng(3)
    errs = []
    for _ in range(400):
        r = rng.uniform(0, 12)
        th = rng.uniform(0.05, np.pi - 0.05)
        z = r * np.exp(1j * th)
        if abs(z) < 0.3:
            continue
        w = oracle.rs_fast_w(z)
        errs.append(abs(w - wofz(z)) / max(1.0, abs(wofz(z))))
    assert max(errs) < 2e-4, max(errs)


def test_fast_w_branches(oracle):
    """|z| >= 6 uses the 3-term asymptotic series: accurate to ~1e-6 there."""
    for z in [6.5 + 0.5j, -7 + 2j, 3 + 9j, 20 + 1j]:
        assert abs(oracle.rs_fast_w(z) - wofz(z)) < 1e-5


@pytest.mark.parametrize("small,P,W", [(1, 10, 3), (1, 50, 7), (1, 1000, 100), (0, 20, 20), (1, 5, 9)])
def test_window_partition(oracle, small, P, W):
    npol, nwin, ws, we = oracle.rs_tables(small, P, W)
    n_nuc = 68 if small else 355
    assert npol.min() >= 1 and nwin.min() >= 1
    assert npol.sum() == P * n_nuc and nwin.sum() == W * n_nuc
    off = 0
    for i in range(n_nuc):
        s, e = ws[off:off + nwin[i]], we[off:off + nwin[i]]
        assert s[0] == 0
        # windows tile [0, n_poles) in order: next start = end + 1
        assert np.all(s[1:] == e[:-1] + 1)
        assert e[-1] == npol[i] - 1
        assert int((e - s + 1).sum()) == npol[i]
        off += nwin[i]


@pytest.mark.parametrize("extra", ["", "-d"])
def test_verification_invariants(oracle, extra):
    L = 500
    r = oracle.run_text(f"-s small -l {L} -p 40 -w 8 {extra} -r 3\n", app=oracle.APP_RSBENCH)
    rec, tal = r.records[0], r.tallies[0]
    assert rec["exit_code"] == 0 and rec["work"] == L
    ver = sum((c + 1) * int(tal[c]) for c in range(4))
    assert L <= ver <= 4 * L and int(rec["vhash"]) == ver % 999983
    assert int(tal[5:17].sum()) == L
    assert np.isfinite(rec["fsum"])


@pytest.mark.parametrize("line", ["-s x", "-p 0", "-w", "-l q", "-d 1"])
def test_usage_errors(oracle, line):
    r = oracle.run_text(line + "\n", app=oracle.APP_RSBENCH)
    assert r.records[0]["exit_code"] == 1 and b"usage: rsbench" in r.stdout[0]


@pytest.mark.parametrize("extra", ["", "-d"])
def test_pole_term_counter(oracle, extra):
    """tallies[24..25] = pole terms evaluated (the RS roofline's work unit): recomputed from the
    window table (RS-2.5) and the lookup stream (RS-3: E, mat; window = (int)(E / (1/n_win)),
    poles [start, end)); tallies[26] (Abrarov branch) is 0 without doppler and <= terms with it."""
    L, P, W, seed = 300, 40, 8, 3
    r = oracle.run_text(f"-s small -l {L} -p {P} -w {W} {extra} -r {seed}\n", app=oracle.APP_RSBENCH)
    tal = r.tallies[0]
    npol, nwin, ws, we = oracle.rs_tables(1, P, W)
    woff = np.concatenate([[0], np.cumsum(nwin)])
    num, mats = oracle.xs_materials(68)
    want = 0
    for i in range(L):
        s = oracle.lcg_ff(seed, 2 * i)
        E, s = oracle.lcg_double(s)
        mat, s = oracle.pick_mat(s)
        for j in range(num[mat]):
            nuc = mats[mat, j]
            w = int(E / (1.0 / nwin[nuc]))
            if w == nwin[nuc]:
                w -= 1
            want += int(we[woff[nuc] + w] - ws[woff[nuc] + w])
    got = int(tal[24]) | (int(tal[25]) << 32)
    assert got == want and want > 0
    if extra == "-d":
        assert int(tal[26]) == 0
    else:
        assert 0 <= int(tal[26]) <= got
