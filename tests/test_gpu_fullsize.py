"""Full-size configurations (BASELINE.json configs) in the launch
configuration bench.py times, checked on a sample of instances the oracle
runs in seconds, plus properties that hold at any size."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

from parity import assert_parity  # noqa: E402


class Sub:
    def __init__(self, r, idx):
        self.records = r.records[idx]
        self.tallies = r.tallies[idx] if r.tallies is not None else None
        self.stdout = [r.stdout[i] for i in idx]


def run_cfg(lines, threads, **kw):
    from paper_conf_icppw_tiancd23_b200 import ensemble, workloads
    return ensemble.run_text(workloads.text(lines), app="auto", threads=threads, **kw)


def check_sample(oracle, lines, r, idx):
    o = oracle.run_text("".join(lines[i] + "\n" for i in idx))
    o.records["instance"] = np.array(idx, dtype=np.uint32)
    assert_parity(Sub(r, idx), o)


def test_c1_full(oracle):
    from paper_conf_icppw_tiancd23_b200 import workloads
    lines = workloads.c1()
    r = run_cfg(lines, 256)
    check_sample(oracle, lines, r, list(range(4)))


def test_c2_full_sampled(oracle):
    """64 x large hash, 1M lookups: the bench workload; oracle on 2 sampled instances."""
    from paper_conf_icppw_tiancd23_b200 import workloads
    lines = workloads.c2()
    r = run_cfg(lines, 1024)
    assert np.all(r.records["exit_code"] == 0)
    assert np.all(r.records["work"] == 1000000)
    v = r.tallies[:, :5].astype(np.int64)
    ver = (v * np.arange(1, 6)).sum(axis=1)
    assert np.all(ver % 999983 == r.records["vhash"])
    assert np.all(r.tallies[:, 5:17].sum(axis=1) == 1000000)
    check_sample(oracle, lines, r, [0, 63])


def test_tstar_sampled(oracle):
    from paper_conf_icppw_tiancd23_b200 import workloads
    lines = workloads.tstar()
    r = run_cfg(lines, 256)
    assert np.all(r.records["exit_code"] == 0)
    check_sample(oracle, lines, r, [0, 1, 511, 1023])


def test_c3_sampled(oracle):
    from paper_conf_icppw_tiancd23_b200 import workloads
    lines = workloads.c3()
    r = run_cfg(lines, 256)
    assert np.all(r.records["exit_code"] == 0)
    check_sample(oracle, lines, r, [0, 1, 2, 3, 100, 255])


def test_c4_sampled(oracle):
    from paper_conf_icppw_tiancd23_b200 import workloads
    lines = workloads.c4()
    r = run_cfg(lines, 1024)
    assert np.all(r.records["exit_code"] == 0)
    check_sample(oracle, lines, r, [0, 1, 777, 1023])
