"""Pins of the oracle's RS-2 tables (upstream RSBench init order).

RS-2 draws every table value from ONE LCG stream s = iseed, in this order:
  1. concs (C = sum of num_nucs draws, XS-2's m-major order)
  2. pole-count histogram:   (P-1)*n draws, LCG_int mod n
  3. window-count histogram: (W-1)*n draws
  4. poles, nuclide-major: EA = 152.5*(d1 + i d2), RT = (152.5 d3, d4), RA = (152.5 d5, d6),
     RF = (152.5 d7, d8), l = LCG_int mod 4         (9 draws each, P*n poles)
  5. windows: T, A, F                                  (3 draws each, W*n windows)
  6. K0RS: n*4 draws.
These tests fix the oracle's tables from the mathematics of that stream, not from the oracle:
  * per-field ranges and means (a swapped field, a wrong scale or a missing factor moves a
    range or a mean by many sigma);
  * the draw-count identity: the last K0RS value is draw number D of the stream,
    D = C + (P-1)n + (W-1)n + 9Pn + 3Wn + 4n (a dropped or extra draw anywhere shifts it);
  * random-access spot checks: a pole / window / K0RS field equals its own draw, addressed by
    its index through an O(log k) fast-forward written here in plain Python (affine-map
    squaring: no loop shared with the oracle's sequential generator);
and every mutation of the tables that a plausible bug would cause fails the checker
(test_rs2_checker_kills_mutations), as the RS-3 pin does for the lookup arithmetic.
"""
import numpy as np
import pytest

MASK63 = (1 << 63) - 1
A_LCG, C_LCG = 2806196910506780709, 1
SCALE = 152.5
NUM_NUCS = {68: [34, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9],
            355: [321, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9]}


def ff(s, k):
    """State after k LCG steps: compose the affine map x -> a x + c (mod 2^63) k times by
    squaring (SURVEY.md §8(c) 'LCG')."""
    a, c = A_LCG, C_LCG
    ra, rc = 1, 0
    while k:
        if k & 1:
            ra, rc = (ra * a) & MASK63, (rc * a + c) & MASK63
        a, c = (a * a) & MASK63, (c * a + c) & MASK63
        k >>= 1
    return (ra * s + rc) & MASK63


def draw(iseed, k):
    """Draw number k (1-based) of the stream as LCG_double: state / 2^63."""
    return ff(iseed, k) / 2.0 ** 63


def layout(n, P, W):
    C = sum(NUM_NUCS[n])
    o_pol = C + (P - 1) * n + (W - 1) * n  # draws before the first pole
    o_win = o_pol + 9 * P * n
    o_k0 = o_win + 3 * W * n
    D = o_k0 + 4 * n
    return C, o_pol, o_win, o_k0, D


def check_rs2(n, P, W, iseed, poles, wins, k0, npol, nwin, spots=64, rng_seed=0):
    """Raise AssertionError if the tables are not RS-2's. poles: (Pn, 9) = EA, RT, RA, RF as
    (re, im), l; wins: (Wn, 3) = T, A, F; k0: (n, 4)."""
    C, o_pol, o_win, o_k0, D = layout(n, P, W)
    assert poles.shape == (P * n, 9) and wins.shape == (W * n, 3) and k0.shape == (n, 4)
    assert int(npol.sum()) == P * n and int(nwin.sum()) == W * n
    # ranges: 152.5-scaled fields in [0, 152.5), unit fields in [0, 1), l in {0..3}
    scaled = [0, 1, 2, 4, 6]
    unit = [3, 5, 7]
    for f in scaled:
        assert poles[:, f].min() >= 0 and poles[:, f].max() < SCALE, ("scaled field", f)
    for f in unit:
        assert poles[:, f].min() >= 0 and poles[:, f].max() < 1.0, ("unit field", f)
    assert wins.min() >= 0 and wins.max() < 1.0
    assert k0.min() >= 0 and k0.max() < 1.0
    lv = poles[:, 8]
    assert np.all(lv == np.round(lv)) and lv.min() >= 0 and lv.max() <= 3
    # means within 5 sigma of the uniform law (sigma = range / sqrt(12 m))
    m = P * n
    for f in scaled:
        assert abs(poles[:, f].mean() - SCALE / 2) < 5 * SCALE / np.sqrt(12 * m), ("mean", f)
    for f in unit:
        assert abs(poles[:, f].mean() - 0.5) < 5 / np.sqrt(12 * m), ("mean", f)
    for f in range(3):
        assert abs(wins[:, f].mean() - 0.5) < 5 / np.sqrt(12 * W * n), ("window mean", f)
    assert abs(k0.mean() - 0.5) < 5 / np.sqrt(12 * 4 * n)
    # l uniform on {0..3}: each count within 5 sigma of m/4
    cnt = np.bincount(lv.astype(int), minlength=4)
    assert np.all(np.abs(cnt - m / 4) < 5 * np.sqrt(m * 3 / 16) + 1), cnt
    # draw-count identity: the last K0RS value is draw D
    assert k0[-1, 3] == draw(iseed, D), "draw count"
    assert k0[0, 0] == draw(iseed, o_k0 + 1), "first K0RS draw"
    # random-access spot checks, every field of sampled poles / windows / K0RS
    rng = np.random.default_rng(rng_seed)
    for g in np.concatenate([[0, P * n - 1], rng.integers(0, P * n, spots)]):
        b = o_pol + 9 * int(g)
        want = [SCALE * draw(iseed, b + 1), SCALE * draw(iseed, b + 2),
                draw(iseed, b + 3) * SCALE, draw(iseed, b + 4),
                draw(iseed, b + 5) * SCALE, draw(iseed, b + 6),
                draw(iseed, b + 7) * SCALE, draw(iseed, b + 8),
                float(ff(iseed, b + 9) % 4)]
        assert list(poles[g]) == want, ("pole", int(g))
    for g in np.concatenate([[0, W * n - 1], rng.integers(0, W * n, spots)]):
        b = o_win + 3 * int(g)
        assert list(wins[g]) == [draw(iseed, b + 1), draw(iseed, b + 2), draw(iseed, b + 3)], ("window", int(g))
    for i in np.concatenate([[0, n - 1], rng.integers(0, n, 8)]):
        for l in range(4):
            assert k0[i, l] == draw(iseed, o_k0 + 4 * int(i) + l + 1), ("K0RS", int(i), l)
    # histograms: n_poles[i] = 1 + #{k < (P-1)n : LCG_int(draw C+k+1) mod n == i} (exhaustive
    # for small tables; the stream is stepped here one state at a time)
    if (P + W) * n <= 200000:
        for base, cnt_draws, hist in ((C, (P - 1) * n, npol), (C + (P - 1) * n, (W - 1) * n, nwin)):
            h = np.ones(n, dtype=np.int64)
            s = ff(iseed, base)
            for _ in range(cnt_draws):
                s = (A_LCG * s + C_LCG) & MASK63
                h[s % n] += 1
            assert np.array_equal(h, hist), "count histogram"


CASES = [(1, 40, 8, 42), (1, 7, 3, 5), (0, 12, 4, 42), (1, 1000, 100, 42), (1, 500, 50, 1234)]


@pytest.mark.parametrize("small,P,W,iseed", CASES)
def test_rs2_tables_pinned(oracle, small, P, W, iseed):
    n = 68 if small else 355
    _, poles, wins, k0 = oracle.rs_micro(small, P, W, 1, [0], [0.5], iseed=iseed)
    npol, nwin, _, _ = oracle.rs_tables(small, P, W, iseed=iseed)
    check_rs2(n, P, W, iseed, poles, wins, k0, npol, nwin)


def test_rs2_fast_forward_is_stepping():
    """The test's own ff (affine squaring) equals k single steps (brute force)."""
    s = 42
    for k in range(1, 300):
        s = (A_LCG * s + C_LCG) & MASK63
        assert ff(42, k) == s


def _mutants(poles, wins, k0):
    """Tables as plausible bugs would produce them."""
    out = {}
    p = poles.copy(); p[:, [2, 3]] = p[:, [3, 2]]; out["RT re/im swapped"] = (p, wins, k0)
    p = poles.copy(); p[:, 3] *= SCALE; out["RT.i scaled by 152.5"] = (p, wins, k0)
    p = poles.copy(); p[:, 0] /= SCALE; out["EA.r unscaled"] = (p, wins, k0)
    p = poles.copy(); p[:, [4, 5, 6, 7]] = p[:, [6, 7, 4, 5]]; out["RA/RF swapped"] = (p, wins, k0)
    p = poles.copy(); p[:, [2, 3, 4, 5, 6, 7]] = p[:, [4, 5, 6, 7, 2, 3]]; out["residue order rotated"] = (p, wins, k0)
    p = poles.copy(); p[:, 8] = (p[:, 8] + 1) % 4; out["l shifted"] = (p, wins, k0)
    # one draw too many before the poles: every field takes the next draw
    p = poles.copy(); p[:-1, :8] = np.concatenate([p[:-1, 1:8], p[1:, :1]], axis=1); out["pole draws shifted"] = (p, wins, k0)
    w = wins.copy(); w[:, [0, 1]] = w[:, [1, 0]]; out["T/A swapped"] = (poles, w, k0)
    k = k0.copy(); k[:, :] = k[:, ::-1]; out["K0RS l order reversed"] = (poles, wins, k)
    k = k0.copy(); k[:-1, :] = k[1:, :]; out["K0RS one nuclide early"] = (poles, wins, k)
    return out


def test_rs2_checker_kills_mutations(oracle):
    small, P, W, iseed = 1, 40, 8, 42
    n = 68
    _, poles, wins, k0 = oracle.rs_micro(small, P, W, 1, [0], [0.5], iseed=iseed)
    npol, nwin, _, _ = oracle.rs_tables(small, P, W, iseed=iseed)
    check_rs2(n, P, W, iseed, poles, wins, k0, npol, nwin)
    for name, (p, w, k) in _mutants(poles, wins, k0).items():
        with pytest.raises(AssertionError):
            check_rs2(n, P, W, iseed, p, w, k, npol, nwin)
            print("survived:", name)
    # a wrong histogram (one draw to the wrong nuclide) is caught too
    bad = npol.copy(); bad[0] += 1; bad[1] -= 1
    with pytest.raises(AssertionError):
        check_rs2(n, P, W, iseed, poles, wins, k0, bad, nwin)
