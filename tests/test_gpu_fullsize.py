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


def test_c2_full_elementwise_sample(oracle):
    """C2 at bench size and launch config: the first 20000 sorted lookup slots of two instances,
    element by element (bit-exact) against the oracle's per-lookup rows (all 1M, by energy)."""
    from paper_conf_icppw_tiancd23_b200 import workloads
    lines = workloads.c2()
    rows = 20000
    r = run_cfg(lines, 512, dump_rows=rows)
    for i in (0, 63):
        o = oracle.run_text(lines[i] + "\n", dump=1000000)
        od = o.dumps[0]
        gd = r.dump[i]
        gd = gd[~np.all(gd == 0, axis=1)]
        assert len(gd) == rows
        pos = np.searchsorted(od[:, 0], gd[:, 0], sorter=np.argsort(od[:, 0]))
        srt = od[np.argsort(od[:, 0])]
        hit = srt[pos]
        assert np.array_equal(hit[:, 0], gd[:, 0]) and np.array_equal(hit[:, 1], gd[:, 1])
        assert np.array_equal(hit[:, 2:8].view(np.uint64), gd[:, 2:8].view(np.uint64))


def test_c5_full_sampled(oracle):
    """C5: 4096 mixed lines (XS / XS / RS / AMG) at the bench's thread limit, concurrent per-app
    groups on forked streams with separate arena regions; 16 sampled instances spanning the
    three apps, the queue's head and tail, against the oracle."""
    from paper_conf_icppw_tiancd23_b200 import workloads
    lines = workloads.c5()
    r = run_cfg(lines, 1024)
    assert np.all(r.records["exit_code"] == 0)
    assert np.all(r.records["instance"] == np.arange(4096))
    check_sample(oracle, lines, r, [0, 1, 2, 3, 1021, 1022, 1023, 1024, 2046, 2047, 2048, 2049, 4092, 4093, 4094, 4095])


def test_c2u_full_sampled(oracle):
    """C2u: 24 x large unionized (5.92 GB of tables each; 142 GB of slot arenas), 1M lookups,
    the bench launch; the first and last instance against the oracle."""
    from paper_conf_icppw_tiancd23_b200 import workloads
    lines = [l.replace("-G hash -h 10000", "-G unionized") for l in workloads.c2(24)]
    r = run_cfg(lines, 512)
    assert np.all(r.records["exit_code"] == 0)
    check_sample(oracle, lines, r, [0, 23])
