"""Oracle loader pins: the paper's Fig. 5 worked example and the Q1-Q4 readings.

Fig. 4: argv of instance I = [argv[0] of the loader] + line I
split on ' '; Argc[I] = len(argv).  Fig. 5 is the worked example.
"""
import json
import os

import pytest

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_fig5_worked_example(oracle):
    text = open(os.path.join(GOLD, "fig5_arguments.txt")).read()
    exp = json.load(open(os.path.join(GOLD, "fig5_expected.json")))
    assert oracle.args_lines(text) == exp["n"]
    for i in range(exp["n"]):
        argv = oracle.args_argv(text, i, exp["argv0"])
        assert argv == exp["argv"][i]
        assert len(argv) == exp["argc"][i]


def test_fig5_equivalence_echo(oracle):
    """Fig. 5a == 5c: the ensemble equals one host run per line."""
    text = open(os.path.join(GOLD, "fig5_arguments.txt")).read()
    ens = oracle.run_text(text, app=oracle.APP_ECHO, argv0="./user_app_gpu")
    for i, line in enumerate(text.splitlines()):
        solo = oracle.run_text(line + "\n", app=oracle.APP_ECHO, argv0="./user_app_gpu")
        assert solo.stdout[0] == ens.stdout[i]
        assert solo.records[0]["exit_code"] == ens.records[i]["exit_code"] == 6
    assert ens.stdout[0] == (b"argc=6\nargv[0]=./user_app_gpu\nargv[1]=-a\nargv[2]=1\n"
                             b"argv[3]=-b\nargv[4]=-c\nargv[5]=data-1.bin\n")


@pytest.mark.parametrize("text,lines", [
    ("", []),
    ("\n", [[]]),
    ("a b\n", [["a", "b"]]),
    ("a b", [["a", "b"]]),
    ("a  \t b\r\n\nc\n", [["a", "b"], [], ["c"]]),
    ("  lead\ttrail  \n", [["lead", "trail"]]),
    ("x\n\n", [["x"], []]),
])
def test_split_readings(oracle, text, lines):
    """Readings Q1 (runs of ' '/'\\t', strip '\\r') and Q2 (every '\\n'-terminated line is an instance)."""
    assert oracle.args_lines(text) == len(lines)
    for i, toks in enumerate(lines):
        assert oracle.args_argv(text, i, "P") == ["P"] + toks


def test_argv0_from_first_token(oracle):
    """Reading Q3: without a loader argv0 the first token is argv[0]."""
    assert oracle.args_argv("echo 1 2\n", 0, None) == ["echo", "1", "2"]


def test_n_larger_than_lines_is_error(oracle):
    """Reading Q4: n > lines is an error, n < lines takes the first n."""
    with pytest.raises(ValueError):
        oracle.run_text("a\nb\n", app=oracle.APP_ECHO, n=3)
    r = oracle.run_text("a\nb\n", app=oracle.APP_ECHO, n=1)
    assert len(r.records) == 1
