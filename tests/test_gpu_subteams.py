"""The (N/M, M, 1) block mapping: M
instances share one CTA, each on its own row threadIdx.y with its own
scheduler state, arena slot and named barrier.  Results must not depend on M
(reading Q6 extended), nor on how many CTA rows are resident."""
import pytest

pytestmark = pytest.mark.gpu

from parity import assert_parity  # noqa: E402

LINES = [
    "amgmk -x 5 -y 3 -z 7 -i 4 -r 2",
    "amgmk -x 9 -y 9 -z 9 -i 5 -k both -r 4",
    "amgmk -x 33 -y 2 -z 3 -i 6 -k matvec -r 3",
    "amgmk -x 1 -y 1 -z 1 -i 3 -r 1",
    "pagerank -n 1000 -e 8 -i 10 -R 4",
    "pagerank -n 7 -e 2 -i 5 -R 3",
    "pagerank -n 4097 -e 3 -i 7 -R 5",
    "echo a b  c",
    "echo",
    "nosuchapp -x 1",
    "amgmk -k jacobi",
    "pagerank -x 1",
    # bodies not built for sub-teams run with M = 1 in the same ensemble
    "xsbench -s small -g 37 -l 1000 -G hash -h 7 -r 3",
    "rsbench -s small -l 500 -p 5 -w 9 -r 3",
]


def _run(oracle, lines, **kw):
    from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble
    from paper_conf_icppw_tiancd23_b200._ens import Args, APP_IDS
    text = "".join(l + "\n" for l in lines)
    ens = Ensemble(Args.parse(text), app="auto", **kw).launch()
    g = ens.collect()
    info = ens.info()
    ens.close()
    return g, oracle.run_text(text), info, APP_IDS


@pytest.mark.parametrize("threads,m", [(256, 2), (256, 4), (256, 8), (1024, 8), (64, 8), (128, 3)])
def test_sub_team_parity(oracle, threads, m):
    g, o, info, ids = _run(oracle, LINES, threads=threads, instances_per_cta=m)
    assert_parity(g, o)
    # effective M: power of two <= the request, >= 32 threads per instance
    want = 1
    while want * 2 <= m and want < 8 and threads // (want * 2) >= 32:
        want *= 2
    assert info.instances_per_cta[ids["amgmk"]] == want
    assert info.instances_per_cta[ids["pagerank"]] == want
    assert info.instances_per_cta[ids["xsbench"]] == 1
    assert info.instances_per_cta[ids["rsbench"]] == 1


@pytest.mark.parametrize("grid", [1, 2])
def test_sub_team_slot_reuse(oracle, grid):
    """More instances than CTA rows: each row pulls ids from the counter and
    reuses its arena slot (reading Q5) independently of its sibling rows."""
    lines = [f"amgmk -x {3 + i % 5} -y {2 + i % 3} -z 4 -i {2 + i % 4} -k {['relax', 'matvec', 'both'][i % 3]} -r {i}"
             for i in range(13)]
    lines += [f"pagerank -n {50 + 37 * i} -e {1 + i % 6} -i {i % 5} -R {i}" for i in range(11)]
    g, o, info, ids = _run(oracle, lines, threads=256, instances_per_cta=4, grid=grid)
    assert_parity(g, o)
    assert info.grid_blocks[ids["amgmk"]] == grid
    assert info.instances_per_cta[ids["amgmk"]] == 4
