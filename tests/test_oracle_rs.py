"""Oracle RSBench-style pins.

* fast_nuclear_W against an accurate Faddeeva function (scipy.special.wofz)
  in the region where the expansions are valid (Im z > 0);
* window partition and pole / window totals (RS-2);
* verification invariants;
* RS-3 micro cross sections against the multipole form evaluated in numpy with
  scipy's Faddeeva function from the oracle's RS-2 tables.
The RS-2 draws themselves are "parity unpinned" vs upstream.
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


@pytest.mark.parametrize("small,P,W,doppler", [(1, 60, 6, 1), (1, 60, 6, 0), (0, 30, 10, 1), (1, 200, 1, 0)])
def test_micro_xs_vs_multipole_form(oracle, small, P, W, doppler):
    """RS-3 micro cross sections against an independent evaluation of the multipole
    form from the oracle's own RS-2 tables: sigma_x(E) = E*x_w + sum_p Re(r_x,p * g_p),
    g_p = wofz(Z_p) with Z_p = (E - EA_p)/2 (doppler; scipy's Faddeeva function in place
    of fast_nuclear_W) or i / ((EA_p - sqrt E) E) (no doppler), the sigT residue turned
    by exp(-2i phi_l) with phi_l the hard-sphere phase shifts of rho = K0RS_l sqrt E
    (reading: upstream's l = 1 sign, phi_1 = rho + atan rho); sigE = sigT - sigA.
    Pole energies lie above the real axis, so every Z is below it: far from 0 the
    expansion fast_nuclear_W sums is that of -W(-Z) (scipy at -Z), near 0 that of W(Z).  The
    sums are done in numpy vector form (not the oracle's loop), so a wrong window,
    pole range, l index, residue channel or sign shows up as an O(1) difference."""
    n_nuc = 68 if small else 355
    rng = np.random.default_rng(11 + doppler)
    nucs = rng.integers(0, n_nuc, 300)
    Es = rng.random(300)
    Es[:4] = [0.0, 1.0 - 2 ** -53, 0.5, 1e-300]
    micro, poles, wins, k0 = oracle.rs_micro(small, P, W, doppler, nucs, Es)
    npol, nwin, ws, we = oracle.rs_tables(small, P, W)
    poff = np.concatenate([[0], np.cumsum(npol)])
    woff = np.concatenate([[0], np.cumsum(nwin)])
    EA = poles[:, 0] + 1j * poles[:, 1]
    R = {"T": poles[:, 2] + 1j * poles[:, 3], "A": poles[:, 4] + 1j * poles[:, 5],
         "F": poles[:, 6] + 1j * poles[:, 7]}
    lv = poles[:, 8].astype(int)
    assert np.all((lv >= 0) & (lv < 4))
    skipped = 0
    for k, (nuc, E) in enumerate(zip(nucs, Es)):
        w = min(int(E * nwin[nuc]), nwin[nuc] - 1)
        assert w == min(int(E / (1.0 / nwin[nuc])), nwin[nuc] - 1)
        sl = slice(poff[nuc] + ws[woff[nuc] + w], poff[nuc] + we[woff[nuc] + w])
        T, A, F = wins[woff[nuc] + w]
        rho = k0[nuc] * np.sqrt(E)
        phi = np.array([rho[0], rho[1] + np.arctan(rho[1]),
                        rho[2] - np.arctan(3 * rho[2] / (3 - rho[2] ** 2)),
                        rho[3] - np.arctan(rho[3] * (15 - rho[3] ** 2) / (15 - 6 * rho[3] ** 2))])
        turn = np.exp(-2j * phi)[lv[sl]]
        near = np.zeros(sl.stop - sl.start, bool)
        if doppler:
            Z = (E - EA[sl]) / 2
            near = np.abs(Z) < 6
            # |Z| >= 6: the asymptotic series is that of W(Z) above the real axis and of
            # -W(-Z) = W(Z) - 2 exp(-Z^2) below it; |Z| < 6: the Abrarov series of W(Z)
            far = np.where(Z.imag >= 0, Z, -Z)
            g = np.where(near, wofz(np.where(near, Z, 1j)), np.where(Z.imag >= 0, 1, -1) * wofz(far))
        else:
            if E < 1e-100:
                continue  # upstream divides by E: inf / nan there, nothing to compare
            g = 1j / ((EA[sl] - np.sqrt(E)) * E)
        want_T = E * T + np.sum((R["T"][sl] * turn * g).real)
        want_A = E * A + np.sum((R["A"][sl] * g).real)
        want_F = E * F + np.sum((R["F"][sl] * g).real)
        scale = E * (abs(T) + abs(A) + abs(F)) + np.sum((np.abs(R["T"][sl]) + np.abs(R["A"][sl])
                                                         + np.abs(R["F"][sl])) * np.abs(g)) + 1e-300
        if near.any():
            # a |Z| < 6 term below the axis: the Abrarov series' denominators
            # (n pi)^2 - (12 Z)^2 come near 0 there (upstream behaviour, no W to
            # compare with); that branch is pinned above the axis by test_fast_w_*
            skipped += 1
            continue
        rtol = 1e-6 if doppler else 1e-12
        slack = 0.0
        got = micro[k]
        for got_x, want_x in zip(got, [want_T, want_A, want_F, want_T - want_A]):
            assert abs(got_x - want_x) <= rtol * scale + slack, (k, nuc, E, got, want_T, want_A, want_F)
    assert skipped <= len(Es) // 5, skipped
