"""Oracle primitive pins: LCG, fast-forward, pick_mat, grid_search.

LCG/pick_mat/grid_search are SURVEY.md §8(c) "Shared primitives".  Pins are
brute force (stepping vs fast-forward), number theory (Hull-Dobell full
period), the distribution they must realise, and numpy's searchsorted.
"""
import numpy as np

A = 2806196910506780709
M = 1 << 63


def test_ff_equals_stepping(oracle):
    rng = np.random.default_rng(0)
    for s in [0, 1, 42, 1070, int(rng.integers(0, M))]:
        x = s
        for n in range(200):
            assert oracle.lcg_ff(s, n) == x
            x = oracle.lcg_step(x)
    for _ in range(20):
        s = int(rng.integers(0, M))
        n = int(rng.integers(0, 3000))
        x = s
        for _ in range(n):
            x = oracle.lcg_step(x)
        assert oracle.lcg_ff(s, n) == x


def test_ff_composition_and_period(oracle):
    """ff(ff(s,a),b) == ff(s,a+b); Hull-Dobell: c odd, a = 1 mod 4 => period 2^63, so ff(s, 2^63) == s."""
    assert A % 4 == 1
    for s in [0, 7, 123456789]:
        for a, b in [(5, 7), (1 << 40, 12345), (M - 3, 2)]:
            assert oracle.lcg_ff(oracle.lcg_ff(s, a), b) == oracle.lcg_ff(s, (a + b) % M)
    assert oracle.lcg_ff(99, M) == 99  # n mod 2^63 == 0
    # the step itself is the affine map mod 2^63 (python big ints)
    assert oracle.lcg_step(12345) == (A * 12345 + 1) % M


def test_lcg_double_scaling(oracle):
    s = 1070
    for _ in range(100):
        d, s2 = oracle.lcg_double(s)
        assert s2 == (A * s + 1) % M
        assert d == float(s2) / float(M)  # exact division by 2^63 after round-to-nearest
        assert 0.0 <= d <= 1.0
        s = s2


def test_pick_mat_distribution(oracle):
    """The effective material distribution: P(0)=1-sum(dist[1:]), P(i)=dist[i] (dist[0] never added)."""
    dist = [.140, .052, .275, .134, .154, .064, .066, .055, .008, .015, .025, .013]
    p = np.array([1 - sum(dist[1:])] + dist[1:])
    assert abs(p.sum() - 1) < 1e-12
    n = 200000
    s = 1
    cnt = np.zeros(12)
    for _ in range(n):
        m, s = oracle.pick_mat(s)
        cnt[m] += 1
    sigma = np.sqrt(n * p * (1 - p))
    assert np.all(np.abs(cnt - n * p) < 5 * sigma), (cnt, n * p)


def test_grid_search_is_clipped_upper_bound(oracle):
    """grid_search(A, q, 0, n-1) == clip(#{k>=1: A[k] <= q}, 0, n-2) for strictly increasing A."""
    rng = np.random.default_rng(1)
    for n in [2, 3, 5, 17, 100]:
        A = np.sort(rng.random(n))
        for q in list(rng.random(50)) + list(A) + [-1.0, 2.0]:
            exp = min(max(int(np.searchsorted(A[1:], q, side="right")), 0), n - 2)
            assert oracle.grid_search(A, q, 0, n - 1) == exp
