"""ENS_F_CLC (the scheduler ablation of SURVEY.md §8(a) S3): one CTA per instance, cluster
launch control steals not-yet-launched CTAs, arena slots from a pool.  Results must equal the
oracle's and the counter scheduler's exactly."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

from parity import assert_parity  # noqa: E402

LINES = ["xsbench -s small -g 60 -l 500 -G unionized -r %d" % i for i in range(40)] + \
        ["rsbench -s small -l 200 -p 10 -w 3 -r %d" % i for i in range(20)] + \
        ["amgmk -x 6 -y 5 -z 4 -i 3 -r %d" % i for i in range(300)] + \
        ["echo clc %d" % i for i in range(3000)] + ["nosuchapp", "xsbench -g 1"]


def run(lines, **kw):
    from paper_conf_icppw_tiancd23_b200 import Args
    from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble
    e = Ensemble(Args.parse("".join(l + "\n" for l in lines)), app="auto", **kw).launch()
    out = e.collect()
    e.relaunch()
    again = e.collect()
    info = e.info()
    e.close()
    return out, again, info


@pytest.mark.parametrize("threads", [64, 256])
def test_clc_matches_oracle(oracle, threads):
    g, g2, info = run(LINES, threads=threads, clc=True)
    o = oracle.run_text("".join(l + "\n" for l in LINES))
    assert_parity(g, o)
    assert_parity(g2, o)  # a relaunch (slot pool and mbarriers reset) too
    assert max(info.team_ctas) == 1


def test_clc_equals_counter_and_split():
    lines = ["xsbench -s large -g 100 -l 6000 -G hash -h 100 -r %d" % i for i in range(12)]
    a, _, _ = run(lines, threads=256, clc=True)
    b, _, _ = run(lines, threads=256)
    c, _, _ = run(lines, threads=256, clc=True, split=True)
    for f in ("instance", "exit_code", "vhash", "bitsum", "work", "stdout_len"):
        assert np.array_equal(a.records[f], b.records[f]) and np.array_equal(a.records[f], c.records[f]), f
    assert np.array_equal(a.tallies, b.tallies) and a.stdout == b.stdout == c.stdout
