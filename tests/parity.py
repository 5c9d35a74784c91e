"""Parity helpers: compare device records/tallies/stdout with the oracle's.

Bar (SURVEY.md §8(c) "FP parity policy", BASELINE.json north_star):
exit codes, vhash, work, tallies, stdout bytes: bit-exact; bitsum bit-exact
for XS / AMG / echo (every FP value is computed in the oracle's order with
separate IEEE ops); fsum and fabs within 1e-12 relative (|d| <= 1e-12*fabs):
the sum order over lookups / rows differs (parallel tree vs sequential).
RS: bit-exact too since round 2 — both sides evaluate RS-3's sin/cos/atan
with one fixed algorithm (reading R-rs-trig) and every division is IEEE (the
CUDA path's shared-reciprocal quotients are corrected to IEEE's, exactly), so
RS bitsum binds like XS / AMG.
"""
import numpy as np

APP_RS = 3
FSUM_RTOL = 1e-12


def assert_parity(gpu, orc, rs_bitsum=True, check_stdout=True):
    g, o = gpu.records, orc.records
    assert len(g) == len(o)
    for k in range(len(o)):
        a, b = g[k], o[k]
        ctx = f"instance {k} (line {b['instance']})"
        assert a["instance"] == b["instance"], ctx
        assert a["exit_code"] == b["exit_code"], (ctx, a["exit_code"], b["exit_code"], gpu.stdout[k] if gpu.stdout else None)
        assert a["app"] == b["app"], ctx
        assert a["flags"] == b["flags"], (ctx, a["flags"], b["flags"])
        assert a["vhash"] == b["vhash"], (ctx, a["vhash"], b["vhash"])
        assert a["work"] == b["work"], ctx
        if b["app"] != APP_RS or rs_bitsum:
            assert a["bitsum"] == b["bitsum"], (ctx, hex(int(a["bitsum"])), hex(int(b["bitsum"])))
        tol = FSUM_RTOL * max(abs(float(b["fabs"])), 1e-300)
        assert abs(float(a["fsum"]) - float(b["fsum"])) <= tol, (ctx, a["fsum"], b["fsum"])
        assert abs(float(a["fabs"]) - float(b["fabs"])) <= tol, (ctx, a["fabs"], b["fabs"])
        if check_stdout:
            assert gpu.stdout[k] == orc.stdout[k], (ctx, gpu.stdout[k], orc.stdout[k])
            assert a["stdout_len"] == b["stdout_len"], ctx
    if gpu.tallies is not None:
        assert np.array_equal(gpu.tallies, orc.tallies)
