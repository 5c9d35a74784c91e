"""The RS body's scalar math on the device (csrc/tools/rs_math_check.cu runs the body's own
device functions from apps/rsbench.cuh, built with the product flags):

* dtrig sin / cos / atan (reading R-rs-trig) equal the oracle's, bit for bit, on a million
  points over RS-3's argument ranges and beyond (two independent implementations of one
  algorithm);
* the shared-reciprocal quotient (Markstein correction, c_div_x) equals IEEE division n / den
  bit for bit on random operands over a wide exponent range and on edge values;
* c_abs_lt6 equals sqrt(|A|^2) < 6 around |A| = 6, including the sliver just below 36.
"""
import ctypes
import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def tool(kind, x, n):
    lib = ctypes.CDLL(os.path.join(ROOT, "paper_conf_icppw_tiancd23_b200", "libens_tools.so"))
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.zeros(n)
    rc = lib.ens_tool_rs_math(ctypes.c_int(kind), ctypes.c_long(n), x.ctypes.data_as(ctypes.c_void_p),
                              y.ctypes.data_as(ctypes.c_void_p))
    assert rc == 0, rc
    return y


@pytest.mark.parametrize("kind,name", [(0, "sin"), (1, "cos"), (2, "atan")])
def test_trig_bitexact_vs_oracle(oracle, kind, name):
    rng = np.random.default_rng(20 + kind)
    k = np.arange(-60, 61)
    x = np.concatenate([rng.uniform(-10, 10, 400000), rng.uniform(-80, 80, 400000),
                        rng.uniform(-1e5, 1e5, 100000), np.exp(rng.uniform(-60, 60, 100000)),
                        ((k * (np.pi / 2))[:, None] + np.array([-1e-9, 0.0, 1e-9])[None, :]).ravel(),
                        [0.0, -0.0, 0.3, 0.78125, 0.4375, 0.6875, 1.1875, 2.4375, 2.0 ** 66, 2.0 ** -30]])
    if kind < 2:
        x = x[np.abs(x) <= 2.0 ** 19]
    got = tool(kind, x, x.size)
    want = oracle.rs_trig(name, x)
    assert np.array_equal(got.view(np.uint64), want.view(np.uint64))


def test_quotient_exact():
    rng = np.random.default_rng(5)
    n = 2_000_000
    num = rng.standard_normal(n) * np.exp2(rng.integers(-520, 520, n))
    den = np.abs(rng.standard_normal(n)) * np.exp2(rng.integers(-520, 520, n))
    # significands with all-ones / all-zeros tails, powers of two, exact quotients, edge values
    sp = np.array([1.0, 2.0, 3.0, 1.5, np.nextafter(2.0, 0), np.nextafter(1.0, 2), 2.0 ** -500, 2.0 ** 500,
                   np.nextafter(2.0 ** -500, 0), np.nextafter(2.0 ** 500, np.inf), np.nextafter(2.0 ** 501, 0), 2.0 ** 501,
                   0.0, -0.0, 1e-310, np.inf, np.nan])
    a, b = np.meshgrid(sp, sp)
    num = np.concatenate([num, a.ravel(), rng.integers(1, 2 ** 20, 1000) * 1.0])
    den = np.concatenate([den, b.ravel(), rng.integers(1, 2 ** 10, 1000) * 1.0])
    x = np.empty(2 * num.size)
    x[0::2], x[1::2] = num, den
    got = tool(4, x, num.size)
    with np.errstate(all="ignore"):
        want = num / den
    same = (got.view(np.uint64) == want.view(np.uint64)) | (np.isnan(got) & np.isnan(want))
    assert same.all(), (num[~same][:5], den[~same][:5])


def test_abs_lt6_decision():
    rng = np.random.default_rng(6)
    th = rng.uniform(0, 2 * np.pi, 400000)
    r = 6.0 + rng.uniform(-1e-13, 1e-13, th.size)
    ar, ai = r * np.cos(th), r * np.sin(th)
    # |A|^2 on and just below 36: A = (a, 0) with a^2 rounding into the sliver [36 - 2^-45, 36)
    a = np.nextafter(6.0, 0) - np.arange(0, 64) * np.spacing(6.0)
    ar = np.concatenate([ar, a, -a, [6.0, np.nextafter(6.0, 7)]])
    ai = np.concatenate([ai, np.zeros(2 * a.size + 2)])
    x = np.empty(2 * ar.size)
    x[0::2], x[1::2] = ar, ai
    got = tool(3, x, ar.size) == 1.0
    s = ar * ar + ai * ai
    want = np.sqrt(s) < 6.0
    assert np.array_equal(got, want)
    sliver = (s >= 36.0 - 2.0 ** -45) & (s < 36.0)
    assert sliver.sum() >= 4  # the sliver itself was exercised
