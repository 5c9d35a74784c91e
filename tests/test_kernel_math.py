"""Host-side checks of exactness claims the CUDA bodies rely on (no GPU needed).

rsbench.cuh c_abs_lt6: `sqrt(s) < 6.0` (RS-3's |Z| < 6 branch, c_abs) is decided as
s >= 36 -> False, s < 36 - 2^-45 -> True, else sqrt(s) < 6.0; the two agree for every
double s near 36 (IEEE sqrt is correctly rounded on both sides).
"""
import math

import numpy as np


def _lt6(s):
    if s >= 36.0:
        return False
    if s < 36.0 - 2.0 ** -45:
        return True
    return math.sqrt(s) < 6.0


def test_abs_lt6_decision_matches_sqrt():
    xs = []
    x = 36.0
    for _ in range(20000):  # 20000 doubles below 36 (past the 2^-45 sliver) and 200 above
        x = float(np.nextafter(x, 0.0))
        xs.append(x)
    x = 36.0
    for _ in range(200):
        xs.append(x)
        x = float(np.nextafter(x, 100.0))
    xs += [0.0, 1e-300, 35.0, 35.999999, 36.000001, 1e300, float(np.nextafter(36.0 - 2.0 ** -45, 0.0))]
    for s in xs:
        assert _lt6(s) == (math.sqrt(s) < 6.0), s
