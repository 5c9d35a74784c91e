"""Split phases (ENS_F_SPLIT_PHASES): phase 1 = the ensemble kernel builds each XS instance's
tables and sorted lookups in an arena slot of its own; phase 2 = the lookup-item kernel over
every SM writes the records.  Results must equal the oracle's (and the fused path's) exactly:
records, tallies, stdout, element-wise dumps."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

from parity import assert_parity  # noqa: E402

LINES = [
    "xsbench -s small -g 1000 -l 10000 -G unionized -r 1070",
    "xsbench -s small -g 37 -l 4096 -G unionized -r 3",          # exactly one item
    "xsbench -s small -g 1500 -l 4097 -G hash -h 1000 -r 11",    # one item + 1 lookup
    "xsbench -s small -g 300 -l 9000 -G nuclide -r 9",
    "xsbench -s large -g 200 -l 12000 -G hash -h 500 -r 6",
    "xsbench -s large -g 60 -l 5000 -G unionized -r 8",
    "xsbench -s small -g 20000 -l 3000 -G hash -h 1000 -r 21",   # arena-scratch init
    "xsbench -s small -g 100 -l 0 -r 5",                         # no lookups: fused in phase 1
    "xsbench -s small -g 100 -m history -p 50 -l 4 -r 7",        # history: fused in phase 1
    "xsbench -g 1",                                              # usage error
    "rsbench -s small -l 500 -p 20 -w 4 -r 3",                   # other apps alongside
    "amgmk -x 8 -y 8 -z 8 -i 5 -r 4",
]


def run(lines, **kw):
    from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble
    from paper_conf_icppw_tiancd23_b200 import Args
    e = Ensemble(Args.parse("".join(l + "\n" for l in lines)), app="auto", **kw).launch()
    out = e.collect()
    info = e.info()
    e.close()
    return out, info


@pytest.mark.parametrize("threads,team", [(512, 0), (256, 1), (128, 2)])
def test_split_matches_oracle(oracle, threads, team):
    g, info = run(LINES, threads=threads, team_ctas=team, split=True)
    assert info.kernel_launches > info.n_groups  # phase-2 kernels were launched
    o = oracle.run_text("".join(l + "\n" for l in LINES))
    assert_parity(g, o)


def test_split_elementwise(oracle):
    rows = 12000
    g, _ = run(LINES, threads=512, split=True, dump_rows=rows)
    o = oracle.run_text("".join(l + "\n" for l in LINES), dump=rows)
    for k, line in enumerate(LINES):
        if not line.startswith("xsbench") or "-l 0" in line or "history" in line or "-g 1" == line[-5:]:
            continue
        gd = g.dump[k]
        gd = gd[~np.all(gd == 0, axis=1)]
        od = o.dumps[k]
        if len(od) == 0:
            continue
        gs, os_ = gd[np.lexsort((gd[:, 1], gd[:, 0]))], od[np.lexsort((od[:, 1], od[:, 0]))]
        assert gs.shape == os_.shape, line
        assert np.array_equal(gs.view(np.uint64), os_.view(np.uint64)), line


def test_split_equals_fused_and_relaunch():
    from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble
    from paper_conf_icppw_tiancd23_b200 import Args
    lines = [f"xsbench -s large -g 300 -l 20000 -G hash -h 300 -r {i}" for i in range(6)]
    a, _ = run(lines, threads=512, split=True)
    b, _ = run(lines, threads=512, fused=True)
    for f in ("instance", "exit_code", "vhash", "bitsum", "work", "stdout_len"):
        assert np.array_equal(a.records[f], b.records[f]), f
    assert np.allclose(a.records["fsum"], b.records["fsum"], rtol=1e-12, atol=0)
    assert np.array_equal(a.tallies, b.tallies) and a.stdout == b.stdout
    # relaunch on the same workspace (device-resident args): identical up to fsum / fabs, whose
    # terms the sort's atomic bucket order permutes (as in the fused path)
    e = Ensemble(Args.parse("".join(l + "\n" for l in lines)), app="auto", threads=512, split=True).launch()
    r1 = e.collect()
    e.relaunch()
    r2 = e.collect()
    e.close()
    for f in ("instance", "exit_code", "vhash", "bitsum", "work", "stdout_len"):
        assert np.array_equal(r1.records[f], r2.records[f]), f
    assert np.allclose(r1.records["fsum"], r2.records["fsum"], rtol=1e-12, atol=0)
    assert np.array_equal(r1.tallies, r2.tallies) and r1.stdout == r2.stdout


def test_auto_policy():
    # 64 large hash instances x 1M lookups: fewer instances than SMs -> split; 1024 small: fused
    from paper_conf_icppw_tiancd23_b200 import workloads
    _, info = run(workloads.c2(16, lookups=200000), threads=512)
    assert info.kernel_launches >= 2
    _, info = run(workloads.tstar(300), threads=512)
    assert info.kernel_launches == 1
    # above the resident CTAs: large hash instances split, small ones stay fused; RS splits
    _, info = run(workloads.c2(200, lookups=100000), threads=512)
    assert info.kernel_launches >= 3
    _, info = run([f"xsbench -s small -g 1000 -l 10000 -G hash -h 1000 -r {i}" for i in range(300)], threads=512)
    assert info.kernel_launches == 1
    _, info = run([f"rsbench -s small -l 2000 -p 100 -w 10 -r {i}" for i in range(400)], threads=512)
    assert info.kernel_launches == 2


# phase 1b's lookup sort in items: chunk boundaries (kXsSortChunk = 65536 lookups per count /
# scatter item), several chunks, coarse buckets with and without fine bits, both table kinds
SORT_LINES = [
    "xsbench -s small -g 300 -l 65536 -G hash -h 200 -r 31",    # exactly one chunk
    "xsbench -s small -g 300 -l 65537 -G hash -h 200 -r 32",    # one chunk + 1 lookup
    "xsbench -s large -g 120 -l 140000 -G hash -h 300 -r 33",   # three chunks
    "xsbench -s small -g 250 -l 200003 -G nuclide -r 34",       # four chunks, nuclide grid
    "xsbench -s small -g 90 -l 700 -G hash -h 50 -r 35",        # coarse buckets only (kb <= 8)
]


def test_split_lookup_sort_items(oracle):
    text = "".join(l + "\n" for l in SORT_LINES)
    g, info = run(SORT_LINES, threads=256, split=True, dump_rows=2000)
    assert info.kernel_launches > info.n_groups
    o = oracle.run_text(text, dump=2000)
    assert_parity(g, o)
    for k in range(len(SORT_LINES)):  # the first 2000 sorted slots, element by element (as a set)
        gd = g.dump[k]
        gd = gd[~np.all(gd == 0, axis=1)]
        n_l = int(SORT_LINES[k].split("-l ")[1].split()[0])
        assert len(gd) == min(2000, n_l)
        # every dumped (energy, material) row is one of the oracle's lookups with its exact results
        od = oracle.run_text(SORT_LINES[k] + "\n", dump=n_l).dumps[0]
        keys = {(r[0], r[1]): r for r in od}
        for r in gd:
            assert np.array_equal(np.asarray(keys[(r[0], r[1])]).view(np.uint64), r.view(np.uint64))


def test_split_largest_chunk(oracle):
    # xs_split_ok's limit: 2^22 lookups (64 count / scatter items, kb = 18: coarse 8 + fine 10
    # energy bits) is split; one more lookup runs fused over two sorted chunks
    lines = ["xsbench -s small -g 200 -l 4194304 -G hash -h 100 -r 41",
             "xsbench -s small -g 200 -l 4194305 -G hash -h 100 -r 42"]
    g, info = run(lines, threads=512)
    assert info.kernel_launches > info.n_groups  # the first instance's phase-2 kernel ran
    o = oracle.run_text("".join(l + "\n" for l in lines))
    assert_parity(g, o)


def test_split_column_paths(oracle):
    # phase 1b's hash column: shared-memory histogram (bins < 65536 and it fits), the global-column
    # path (bins >= 65536), and the arena-scratch sort (n_gp > 16384) with each
    lines = ["xsbench -s small -g 3000 -l 20000 -G hash -h 70000 -r 51",
             "xsbench -s small -g 18000 -l 20000 -G hash -h 70000 -r 52",
             "xsbench -s small -g 18000 -l 20000 -G hash -h 5000 -r 53",
             "xsbench -s small -g 4000 -l 20000 -G hash -h 3 -r 54",
             "xsbench -s small -g 2 -l 5000 -G hash -h 1000 -r 55"]
    text = "".join(l + "\n" for l in lines)
    g, info = run(lines, threads=256, split=True, dump_rows=20000)
    assert info.kernel_launches > info.n_groups
    o = oracle.run_text(text, dump=20000)
    assert_parity(g, o)
    for k in range(len(lines)):
        gd = g.dump[k]
        gd = gd[~np.all(gd == 0, axis=1)]
        gs, os_ = gd[np.lexsort((gd[:, 1], gd[:, 0]))], o.dumps[k][np.lexsort((o.dumps[k][:, 1], o.dumps[k][:, 0]))]
        assert gs.shape == os_.shape and np.array_equal(gs.view(np.uint64), os_.view(np.uint64)), lines[k]


def test_split_above_resident_ctas_parity(oracle):
    # the policy's any-N splits (RS groups; XS hash groups of non-small instances) against the
    # oracle, with more instances than resident CTAs, next to a small-hash group that stays fused
    lines = ([f"xsbench -s large -g 2000 -l 20000 -G hash -h 1500 -r {200 + i}" for i in range(160)] +
             [f"rsbench -s small -l 600 -p 40 -w 8 {'-d ' if i % 4 == 0 else ''}-r {300 + i}" for i in range(300)] +
             [f"xsbench -s small -g 300 -l 2000 -G hash -h 100 -r {700 + i}" for i in range(200)])
    g, info = run(lines, threads=512)
    assert info.kernel_launches >= 5  # XS: ensemble + init items + hash items; RS: ensemble + items
    o = oracle.run_text("".join(l + "\n" for l in lines))
    assert_parity(g, o)
