"""GPU parity: the CUDA path (libens.so through its C ABI) vs the oracle.

Small and ragged cases compare every instance element by element; the
full-size configurations compare a sample of instances the oracle can run in
seconds (tests/test_gpu_fullsize.py).
"""
import pytest

pytestmark = pytest.mark.gpu

from parity import assert_parity  # noqa: E402

XS_CASES = [
    # n_gp ragged vs the pow2 sort (37 -> 64), several tiles, one below T
    "xsbench -s small -g 37 -l 1000 -G unionized -r 3",
    "xsbench -s small -g 37 -l 1000 -G nuclide -r 3",
    "xsbench -s small -g 37 -l 1000 -G hash -h 7 -r 3",
    "xsbench -s small -g 1000 -l 10000 -m event -G unionized -r 1070",
    "xsbench -s small -g 1500 -l 3000 -G hash -h 1000 -r 11 -R 5",
    "xsbench -s small -g 2 -l 500 -G unionized -r 2",
    "xsbench -s small -g 2 -l 500 -G hash -h 1 -r 2",
    "xsbench -s small -g 300 -l 0 -r 2",
    "xsbench -s small -g 300 -l 5 -G hash -h 3 -r 9",
    "xsbench -s large -g 40 -l 2000 -G unionized -r 5",
    "xsbench -s large -g 200 -l 2000 -G hash -h 500 -r 6",
    "xsbench -s small -g 16384 -l 2000 -G hash -h 100 -r 4",
    # hash column in shared memory (fits) vs the arena scratch (bins >= 2^16)
    "xsbench -s small -g 11303 -l 3000 -G hash -h 10000 -r 13",
    "xsbench -s small -g 3000 -l 2000 -G hash -h 70000 -r 12",
    # n_gp above the shared-memory per-nuclide sort (kXsSmemGp = 16384): keys and
    # counters in arena scratch; up to the -g bound 65536 (reading R-xs-range)
    "xsbench -s small -g 20000 -l 3000 -G hash -h 1000 -r 21",
    "xsbench -s small -g 20000 -l 3000 -G nuclide -r 22",
    "xsbench -s small -g 20000 -l 3000 -G unionized -r 23",
    "xsbench -s small -g 65536 -l 2000 -G hash -h 5000 -r 24",
    "xsbench -s small -g 65536 -l 2000 -G unionized -r 25",
    "xsbench -s small -g 16385 -l 1000 -m history -p 20 -G hash -h 300 -r 26",
    # r >= 2^24 records (the fifth jump-table level): 355 * 50000 = 17.75 M records
    "xsbench -s large -g 50000 -l 1000 -G hash -h 2000 -r 27",
]

RS_CASES = [
    "rsbench -s small -l 2000 -p 100 -w 10 -r 1",
    "rsbench -s small -l 2000 -p 100 -w 10 -d -r 2",
    "rsbench -s small -l 500 -p 5 -w 9 -r 3",
    "rsbench -s large -l 300 -p 50 -w 7 -r 4 -R 8",
    "rsbench -s small -l 0 -p 20 -w 3",
]

AMG_CASES = [
    "amgmk -x 1 -y 1 -z 1 -i 3 -r 1",
    "amgmk -x 5 -y 3 -z 7 -i 4 -r 2",
    "amgmk -x 33 -y 2 -z 3 -i 6 -k matvec -r 3",
    "amgmk -x 9 -y 9 -z 9 -i 5 -k both -r 4",
    "amgmk -x 16 -y 16 -z 16 -i 20 -k relax -r 0",
    "amgmk -x 32 -y 32 -z 32 -i 3 -k relax -r 7",
]

MISC_CASES = [
    "echo",
    "echo a b  c",
    "nosuchapp -x 1",
    "xsbench -g 1",
    "xsbench -g 65537",
    "xsbench -s tiny",
    "xsbench -l",
    "rsbench -q",
    "amgmk -k jacobi",
    "amgmk -x 2000",
]


def run_both(oracle, lines, threads=256, grid=0, **kw):
    from paper_conf_icppw_tiancd23_b200.ensemble import run_text
    text = "".join(l + "\n" for l in lines)
    g = run_text(text, app="auto", threads=threads, grid=grid, **kw)
    o = oracle.run_text(text)
    return g, o


@pytest.mark.parametrize("line", XS_CASES)
def test_xs_parity(oracle, line):
    g, o = run_both(oracle, [line])
    assert_parity(g, o)


@pytest.mark.parametrize("line", RS_CASES)
def test_rs_parity(oracle, line):
    g, o = run_both(oracle, [line])
    assert_parity(g, o)


@pytest.mark.parametrize("line", AMG_CASES)
def test_amg_parity(oracle, line):
    g, o = run_both(oracle, [line])
    assert_parity(g, o)


def test_misc_parity(oracle):
    g, o = run_both(oracle, MISC_CASES)
    assert_parity(g, o)


@pytest.mark.parametrize("threads", [32, 64, 128, 512, 1024, 100, 5000])
def test_thread_limit_independence(oracle, threads):
    """-t is an upper bound and results never depend on it (reading Q6)."""
    lines = [XS_CASES[0], XS_CASES[2], RS_CASES[0], AMG_CASES[1], AMG_CASES[2], "echo t"]
    g, o = run_both(oracle, lines, threads=threads)
    assert_parity(g, o)


@pytest.mark.parametrize("grid", [1, 2, 3])
def test_more_instances_than_blocks(oracle, grid):
    """Persistent blocks pull ids from the counter; a slot arena is reused (reading Q5)."""
    lines = [f"xsbench -s small -g {50 + 7 * i} -l 700 -G {['unionized', 'nuclide', 'hash'][i % 3]} -h 13 -r {i}"
             for i in range(9)]
    g, o = run_both(oracle, lines, grid=grid)
    assert_parity(g, o)


@pytest.mark.parametrize("team", [2, 3, 4, 6, 8, 13, 16])
def test_cluster_team_parity(oracle, team):
    """A team = a thread-block cluster of `team` CTAs (XS is team-aware): same results."""
    lines = [XS_CASES[0], XS_CASES[1], XS_CASES[2], XS_CASES[4], XS_CASES[10], "xsbench -s small -g 77 -l 999 -G hash -h 5 -r 2",
             RS_CASES[0], AMG_CASES[1], "echo team"]
    g, o = run_both(oracle, lines, threads=128, team_ctas=team)
    assert_parity(g, o)


# unionized init: warp path (n_gp <= 1024) at its edges, the block-wide path
# just past it, large (89 quads per index row) and history mode; each also
# with ENS_F_GENERIC (the block-wide path forced) — both equal the oracle
WARP_UNION_CASES = [
    "xsbench -s small -g 1024 -l 3000 -G unionized -r 21",
    "xsbench -s small -g 1025 -l 3000 -G unionized -r 22",
    "xsbench -s large -g 1000 -l 3000 -G unionized -r 23",
    "xsbench -s small -g 3 -l 1000 -G unionized -r 24",
    "xsbench -s small -g 500 -m history -p 300 -l 20 -G unionized -r 25",
]


@pytest.mark.parametrize("generic", [False, True])
@pytest.mark.parametrize("line", WARP_UNION_CASES)
def test_xs_union_paths(oracle, line, generic):
    g, o = run_both(oracle, [line], generic=generic)
    assert_parity(g, o)


@pytest.mark.parametrize("team", [1, 3, 5, 16])
def test_xs_union_block_arena_team(oracle, team):
    """The block-wide unionized init with its sort counters in the arena (n_u = 355 x 1100 >
    4 x kXsSmemBkt): ~4-record buckets of record ids, their energies re-drawn; the union pass's
    next energy from the neighbouring lane; the sweep's inverse map and the record pass in sorted
    order — on 1..16-CTA teams (non-power-of-two striding), two instances."""
    lines = ["xsbench -s large -g 1100 -l 3000 -G unionized -r 31",
             "xsbench -s large -g 1050 -l 2000 -G unionized -r 32"]
    g, o = run_both(oracle, lines, threads=256, team_ctas=team)
    assert_parity(g, o)


@pytest.mark.parametrize("threads", [32, 64, 128, 512])
def test_xs_warp_union_threads(oracle, threads):
    """The warp path with 1..16 warps per team (T=32 runs every nuclide and chunk on one warp)."""
    lines = ["xsbench -s small -g 300 -l 2000 -G unionized -r 26", "xsbench -s large -g 64 -l 500 -G unionized -r 27"]
    g, o = run_both(oracle, lines, threads=threads)
    assert_parity(g, o)


RS_UNEVEN = [f"rsbench -s small -l {L} -p {P} -w {W}{d} -r {i + 1}"
             for i, (L, P, W, d) in enumerate([(3000, 400, 10, ""), (200, 50, 25, ""), (100, 20, 10, " -d"),
                                               (1500, 100, 50, " -d"), (50, 10, 5, ""), (700, 300, 30, "")])]


@pytest.mark.parametrize("team", [0, 1, 2, 5, 8, 16])
def test_rs_team_parity(oracle, team):
    """RS is team-aware: a cluster of CTAs stripes the pole/window draws and the sorted lookup
    batches; the auto team (0) sizes it for the heaviest instance of an uneven ensemble and the
    queue is longest-first.  Every team size and order gives the oracle's results."""
    g, o = run_both(oracle, RS_CASES + RS_UNEVEN, threads=256, team_ctas=team)
    assert_parity(g, o)


def test_rs_chunk_boundary(oracle):
    """More lookups than one sorted chunk (kRsLkChunk = 2^20): chunks are sampled in order."""
    g, o = run_both(oracle, ["rsbench -s small -l 1100000 -p 10 -w 10 -r 9", RS_CASES[0]])
    assert_parity(g, o)


@pytest.mark.parametrize("team", [1, 2, 3, 8, 16])
def test_xs_blockwide_union_team(oracle, team):
    """The block-wide unionized init (n_gp > 1024, counters in the arena) is striped over the
    team's CTAs (cluster barriers between passes): same union, index grid and records."""
    lines = ["xsbench -s small -g 2000 -l 2000 -G unionized -r 31",
             "xsbench -s large -g 1100 -l 1000 -G unionized -r 32",
             "xsbench -s small -g 1500 -l 1000 -G unionized -r 33"]
    g, o = run_both(oracle, lines, threads=256, team_ctas=team)
    assert_parity(g, o)


@pytest.mark.parametrize("team", [2, 5, 8, 16])
def test_xs_warp_union_team(oracle, team):
    """The unionized warp-path init (n_gp <= 1024) striped over a team's CTAs: nuclides and
    union chunks on every CTA, a cluster barrier between, the chunk-overflow fallback decided
    team-wide; small and large problems, several instances per team in turn."""
    lines = [f"xsbench -s {'small' if i % 3 else 'large'} -g {100 + 83 * i} -l {1500 + 97 * i} -G unionized -r {60 + i}"
             for i in range(7)]
    g, o = run_both(oracle, lines, threads=256, team_ctas=team, grid=2 * team)
    assert_parity(g, o)
