"""Ensemble-semantics pins on the oracle (Fig. 4).

An ensemble run is the sequential loop over lines: instance i in an ensemble
equals a solo run of line i; N copies give N identical records; permuting
lines permutes records; the mixed-app (argv[0]) form equals per-app runs.
"""
import numpy as np

FIELDS = ["exit_code", "app", "vhash", "bitsum", "fsum", "fabs", "work", "stdout_len"]

LINES = [
    "xsbench -s small -g 50 -l 300 -r 1",
    "rsbench -s small -l 100 -p 20 -w 4 -r 2",
    "amgmk -x 4 -y 3 -z 5 -i 3 -r 9",
    "echo hello world",
    "xsbench -s small -g 40 -l 200 -G hash -h 30 -r 3",
    "xsbench -g 1",
    "nosuchapp -x",
]


def same(a, b):
    return all(a[k] == b[k] for k in FIELDS)


def test_solo_equals_ensemble(oracle):
    ens = oracle.run_text("\n".join(LINES) + "\n")
    for i, line in enumerate(LINES):
        solo = oracle.run_text(line + "\n", jobs=1)
        assert same(solo.records[0], ens.records[i])
        assert solo.stdout[0] == ens.stdout[i]
        assert np.array_equal(solo.tallies[0], ens.tallies[i])


def test_copies_identical_and_permutation(oracle):
    text = "\n".join([LINES[0]] * 5) + "\n"
    r = oracle.run_text(text)
    for i in range(1, 5):
        assert same(r.records[0], r.records[i]) and r.stdout[i] == r.stdout[0]
    perm = [3, 0, 6, 2, 5, 1, 4]
    a = oracle.run_text("\n".join(LINES) + "\n")
    b = oracle.run_text("\n".join(LINES[p] for p in perm) + "\n")
    for j, p in enumerate(perm):
        assert same(a.records[p], b.records[j]) and a.stdout[p] == b.stdout[j]


def test_unknown_app_and_usage(oracle):
    r = oracle.run_text("\n".join(LINES) + "\n")
    assert r.records[6]["exit_code"] == 127 and r.stdout[6] == b"nosuchapp: command not found\n"
    assert r.records[5]["exit_code"] == 1
    assert r.records[3]["exit_code"] == 3 and r.stdout[3] == b"argc=3\nargv[0]=echo\nargv[1]=hello\nargv[2]=world\n"
