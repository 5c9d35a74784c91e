"""Pins of RS-3's sin / cos / atan (reading R-rs-trig; oracle/rs.cpp namespace trig).

The oracle evaluates RS-3's transcendentals with one fixed algorithm (fdlibm's scheme) so that
the RS result is one defined number on every platform.  These tests pin that algorithm to the
mathematics through numpy's libm (an independent implementation): at most 1 ulp from numpy
(which is itself within 1 ulp of the exact value, so within 2 ulp of exact) over RS-3's
argument ranges and far beyond, the exact symmetries, and special values.  A wrong constant,
a swapped quadrant or a dropped polynomial term moves results by many ulp.
"""
import numpy as np
import pytest


def ulps(got, want):
    return np.abs(got - want) / np.spacing(np.maximum(np.abs(want), np.finfo(float).tiny))


@pytest.mark.parametrize("kind,ref", [("sin", np.sin), ("cos", np.cos)])
def test_sincos_accuracy(oracle, kind, ref):
    rng = np.random.default_rng(7)
    # RS-3 arguments: sigT phases 2*phi (|.| < ~10) and 12*Re(Z) with |Z| < 6 (|.| < 72); far beyond too
    x = np.concatenate([rng.uniform(-10, 10, 400000), rng.uniform(-80, 80, 400000),
                        rng.uniform(-1e5, 1e5, 200000), np.exp(rng.uniform(-60, 0, 50000))])
    # near the multiples of pi/2, where the reduction must be accurate
    k = np.arange(-60, 61)
    near = (k * (np.pi / 2))[:, None] + np.array([-1e-9, -1e-13, 0.0, 1e-13, 1e-9])[None, :]
    x = np.concatenate([x, near.ravel(), [0.0, -0.0, np.pi / 4, -np.pi / 4, 0.78125, 0.3, 1e-300]])
    got = oracle.rs_trig(kind, x)
    u = ulps(got, ref(x))
    small = np.abs(x) <= 100
    assert u[small].max() <= 1.0 and u.max() <= 2.0, (u[small].max(), u.max())


def test_atan_accuracy(oracle):
    rng = np.random.default_rng(8)
    x = np.concatenate([rng.uniform(-3, 3, 400000), np.exp(rng.uniform(-50, 50, 400000)),
                        -np.exp(rng.uniform(-50, 50, 100000)),
                        [0.4375, 0.6875, 1.1875, 2.4375, 2.0 ** -29, 2.0 ** 66, 1e300, np.inf, -np.inf, 0.0]])
    got = oracle.rs_trig("atan", x)
    assert ulps(got, np.arctan(x)).max() <= 1.0
    for bp in [0.4375, 0.6875, 1.1875, 2.4375]:  # both sides of every breakpoint
        xs = np.array([np.nextafter(bp, 0), bp, np.nextafter(bp, 4)])
        assert ulps(oracle.rs_trig("atan", xs), np.arctan(xs)).max() <= 1.0


def test_symmetries_and_specials(oracle):
    rng = np.random.default_rng(9)
    x = rng.uniform(0, 100, 100000)
    s, c, a = (oracle.rs_trig(k, x) for k in ("sin", "cos", "atan"))
    assert np.array_equal(oracle.rs_trig("sin", -x), -s)  # odd, exactly
    assert np.array_equal(oracle.rs_trig("cos", -x), c)   # even, exactly
    assert np.array_equal(oracle.rs_trig("atan", -x), -a)
    assert np.all(np.abs(s * s + c * c - 1) < 4e-16)
    assert oracle.rs_trig("sin", np.array([0.0]))[0] == 0.0 and oracle.rs_trig("cos", np.array([0.0]))[0] == 1.0
    assert oracle.rs_trig("atan", np.array([np.inf]))[0] == np.pi / 2
    assert np.isnan(oracle.rs_trig("atan", np.array([np.nan]))[0])
