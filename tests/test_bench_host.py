"""bench.py host logic on CPU: algorithmic work accounting, the roofline choice, and the
reference arm's hygiene (it runs the oracle and never loads libens.so)."""
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def test_xs_bytes_formulas():
    p = bench.xs_params("xsbench -s small -g 1000 -l 10000 -G unionized -r 1")
    n_u = 68 * 1000
    assert bench.xs_init_bytes(p) == 48 * n_u + 16 * n_u + 4 * n_u * 68
    q = bench.xs_params("xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r 1")
    assert bench.xs_init_bytes(q) == 48 * 355 * 11303 + 4 * 355 * 10000
    counts = np.zeros(12, dtype=np.int64)
    counts[0], counts[2] = 3, 5
    assert bench.xs_lookup_bytes(68, counts) == 3 * (16 + 100 * 34) + 5 * (16 + 100 * 4)


def test_amg_bytes_formula():
    n, nnz = 32 ** 3, 7 * 32 ** 3 - 2 * 3 * 32 * 32
    assert bench.amg_bytes("amgmk -x 32 -y 32 -z 32 -i 20 -k relax -r 1") == \
        20 * (12 * nnz + 4 * (n + 1) + 24 * n) + 12 * nnz + 32 * n


class _Res:
    def __init__(self, lines):
        self.records = np.zeros(len(lines), dtype=[("exit_code", "<i4"), ("work", "<u8")])
        self.tallies = np.zeros((len(lines), 32), dtype=np.uint32)
        self.tallies[:, 5] = 1000  # every lookup in material 0


def test_roofline_picks_a_bound_that_binds(monkeypatch):
    lines = ["xsbench -s large -g 11303 -G hash -h 10000 -l 1000 -r %d" % i for i in range(4)]
    res = _Res(lines)
    monkeypatch.setattr(bench, "ncu_counters", lambda: {"T": {"kernels": {
        "phase2_kind2": {"dram_bytes": 1e9, "inst_executed": 5e9, "source": "x"}}}})
    # phase 2 dominant: its algorithmic lookup bytes over 1 us exceed the peak (L1/L2-served) and
    # must not bind; the issue candidate (5e9 instructions in 10 ms) does
    kt = [(2, 1, -1, 128, 512, 1.0), (2, 2, 2, 444, 256, 10.0)]
    rl = bench.roofline("T", lines, res, kt, {"sm_mhz": 1965.0}, 6535.4, "measured")
    assert rl["kernel_ms"] == 10.0 and rl["binding"] == "issue"
    assert abs(rl["frac"] - 5e9 / 10e-3 / (148 * 4 * 1965e6)) < 1e-12
    assert all(v["frac"] <= 1.05 for k, v in rl["candidates"].items() if k == rl["binding"])
    # algorithmic bytes over a long enough time do bind when the counters are absent
    monkeypatch.setattr(bench, "ncu_counters", lambda: {})
    kt = [(2, 1, -1, 148, 512, 1e4)]
    rl = bench.roofline("T", lines, res, kt, {"sm_mhz": 1965.0}, 6535.4, "measured")
    assert rl["binding"] == "hbm" and rl["bound"] == "hbm" and rl["frac"] < 1


def test_reference_arm_never_loads_libens():
    code = ("import runpy, sys; sys.argv = ['bench.py', '--impl', 'reference', '--workload', 'C1', '--steps', '1'];"
            "runpy.run_path('bench.py', run_name='__main__');"
            "maps = open('/proc/self/maps').read();"
            "assert 'libens' not in maps, 'libens mapped';"
            "assert not any(m.startswith('paper_conf_icppw_tiancd23_b200') for m in sys.modules)")
    p = subprocess.run([sys.executable, "-c", code], cwd=ROOT, capture_output=True, timeout=600)
    assert p.returncode == 0, p.stderr.decode()[-2000:]
    assert b'"impl": "reference"' in p.stdout
