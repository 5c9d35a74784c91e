"""GPU ensemble semantics and fault paths (Fig. 4; §3.2).

Invariants: instance i inside an ensemble == a solo launch of line i; N
copies of one line give N identical records; permuting the lines permutes
the records; sharded launches (first, stride) reproduce the full launch.
Faults: bad flags -> exit 1 + usage text; arena too small -> exit 12 +
NOMEM; stdout buffer too small -> STDOUT_TRUNC; n = 0; ids beyond the file.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

from parity import assert_parity  # noqa: E402

LINES = [
    "xsbench -s small -g 64 -l 900 -r 1",
    "rsbench -s small -l 300 -p 30 -w 6 -r 2",
    "amgmk -x 6 -y 5 -z 4 -i 3 -r 9",
    "echo hello world",
    "xsbench -s small -g 40 -l 300 -G hash -h 30 -r 3",
    "xsbench -g 1",
    "nosuchapp -x",
]
FIELDS = ["instance", "exit_code", "app", "flags", "vhash", "bitsum", "fsum", "fabs", "work", "stdout_len"]


def ens():
    from paper_conf_icppw_tiancd23_b200 import ensemble
    return ensemble


def text(lines):
    return "".join(l + "\n" for l in lines)


def test_fig5_loader_on_device(oracle):
    """Fig. 5: 4 lines, -n 4 -t 128, argv[0] of the loader first."""
    import os
    t = open(os.path.join(os.path.dirname(__file__), "golden", "fig5_arguments.txt")).read()
    g = ens().run_text(t, app="echo", argv0="./user_app_gpu", threads=128)
    o = oracle.run_text(t, app=oracle.APP_ECHO, argv0="./user_app_gpu")
    assert_parity(g, o)
    assert list(g.records["exit_code"]) == [6, 6, 6, 6]


def same(a, b, f):
    """Exact fields bit-for-bit; fsum / fabs within 1e-12 (their reduction tree
    depends on the team size, which the auto scheduler picks per ensemble)."""
    if f in ("fsum", "fabs"):
        return abs(float(a) - float(b)) <= 1e-12 * max(abs(float(a)), 1e-300)
    return a == b


def test_solo_equals_ensemble():
    full = ens().run_text(text(LINES))
    for i, l in enumerate(LINES):
        solo = ens().run_text(text([l]))
        for f in FIELDS[1:]:
            assert same(solo.records[0][f], full.records[i][f], f), (i, f)
        assert solo.stdout[0] == full.stdout[i]
        assert np.array_equal(solo.tallies[0], full.tallies[i])


def test_copies_and_permutation():
    r = ens().run_text(text([LINES[0]] * 37))
    for f in FIELDS[1:]:
        assert all(same(x, r.records[f][0], f) for x in r.records[f])
    perm = [3, 0, 6, 2, 5, 1, 4]
    a = ens().run_text(text(LINES))
    b = ens().run_text(text([LINES[p] for p in perm]))
    for j, p in enumerate(perm):
        for f in FIELDS[1:]:
            assert same(a.records[p][f], b.records[j][f], f)


def test_sharded_launches_match_full():
    from paper_conf_icppw_tiancd23_b200 import Args
    full = ens().run_text(text(LINES))
    G = 3
    for rank in range(G):
        e = ens().Ensemble(Args.parse(text(LINES)), app="auto", first=rank, stride=G).launch()
        r = e.collect()
        for k in range(e.n):
            i = rank + k * G
            for f in FIELDS:
                assert same(r.records[k][f], full.records[i][f], f)
            assert r.stdout[k] == full.stdout[i]
        e.close()


def test_arena_too_small_is_nomem():
    r = ens().run_text(text(["xsbench -s small -g 100 -l 10", "echo x"]), arena_bytes=4096)
    assert r.records[0]["exit_code"] == 12 and r.records[0]["flags"] & 2
    assert r.records[1]["exit_code"] == 2


def test_stdout_truncation_flag():
    r = ens().run_text(text(["echo " + " ".join(["abcdefgh"] * 20)]), stdout_bytes=64)
    assert r.records[0]["flags"] & 1
    assert r.records[0]["exit_code"] == 21
    assert r.stdout[0].startswith(b"argc=21\n")


def test_empty_and_range():
    from paper_conf_icppw_tiancd23_b200 import Args, EnsError
    r = ens().run_text("", app="echo")
    assert len(r.records) == 0
    with pytest.raises(EnsError):
        ens().Ensemble(Args.parse("a\nb\n"), app="echo", n=3).launch()


def test_timestamps_and_smid():
    r = ens().run_text(text([LINES[0]] * 300), timestamps=True)
    assert np.all(r.records["t_end_ns"] >= r.records["t_start_ns"])
    assert np.all(r.records["t_start_ns"] > 0)
    assert len(set(r.records["smid"].tolist())) > 16


def test_runs_in_flight_on_one_stream():
    """Two launches queued on one stream with their own workspaces: collecting the first
    waits for its own run only (end event), while the second is still queued or running;
    both equal a solo sequential run, and collect is idempotent (second call = cached)."""
    import torch
    from paper_conf_icppw_tiancd23_b200 import Args, _ens
    lines = LINES[:5] * 6
    args = Args.parse(text(lines))
    cfg = _ens.make_cfg(len(lines))
    ws = _ens.workspace_bytes("auto", args, cfg)
    bufs = [torch.empty(ws, dtype=torch.uint8, device="cuda") for _ in range(2)]
    stream = torch.cuda.current_stream().cuda_stream
    want = ens().run_text(text(lines))
    runs = [_ens.Run.launch("auto", args, cfg, b.data_ptr(), ws, stream, keep=b) for b in bufs]
    for run in runs:
        for _ in range(2):
            got = run.collect()
            for f in FIELDS:
                assert all(same(got.records[k][f], want.records[k][f], f) for k in range(len(lines))), f
            assert got.stdout == want.stdout
            assert np.array_equal(got.tallies, want.tallies)
        run.close()


def test_concurrent_groups_equal_serial():
    """A mixed-app ensemble runs its per-app kernels concurrently on forked streams, each
    with its own arena region; ENS_F_SERIAL runs them one after another on one shared
    arena: the records, tallies and stdout are the same."""
    lines = LINES * 9
    a = ens().run_text(text(lines))
    b = ens().run_text(text(lines), serial=True)
    for f in FIELDS:
        assert all(same(a.records[k][f], b.records[k][f], f) for k in range(len(lines))), f
    assert a.stdout == b.stdout
    assert np.array_equal(a.tallies, b.tallies)
