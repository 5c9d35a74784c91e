"""CPU tests of the C ABI (no GPU compute): libens.so loads, exports every
symbol include/ens.h declares, and its host-side loader (S1) and stdout
formatter (S10) behave as the paper's loader and the readings say.

The loader is checked against the paper's Fig. 5 worked example
(tests/golden/fig5_*) and against the oracle's independent loader on
edge-case texts; the formatter against printf-formatted expectations.
"""
import ctypes
import json
import os
import re
import struct

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLD = os.path.join(ROOT, "tests", "golden")


def header_symbols():
    src = open(os.path.join(ROOT, "include", "ens.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ens_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    from paper_conf_icppw_tiancd23_b200 import _ens
    syms = header_symbols()
    assert len(syms) >= 16
    for s in syms:
        assert hasattr(_ens.lib, s), s
    assert set(syms) == set(_ens.EXPORTED)


def test_record_layout_matches_header():
    from paper_conf_icppw_tiancd23_b200 import RECORD_DTYPE
    assert RECORD_DTYPE.itemsize == 80
    assert list(RECORD_DTYPE.names)[:4] == ["instance", "exit_code", "app", "flags"]


def test_fig5_loader():
    from paper_conf_icppw_tiancd23_b200 import Args
    exp = json.load(open(os.path.join(GOLD, "fig5_expected.json")))
    a = Args.load(os.path.join(GOLD, "fig5_arguments.txt"), argv0=exp["argv0"])
    assert len(a) == exp["n"]
    assert [a.argv(i) for i in range(len(a))] == exp["argv"]


TEXTS = ["", "\n", "a b\n", "a b", "a  \t b\r\n\nc\n", "  lead\ttrail  \n", "x\n\n", "p q r\n\n\n s \n"]


@pytest.mark.parametrize("text", TEXTS)
@pytest.mark.parametrize("argv0", ["prog", None])
def test_loader_matches_oracle(oracle, text, argv0):
    from paper_conf_icppw_tiancd23_b200 import Args
    a = Args.parse(text, argv0=argv0)
    assert len(a) == oracle.args_lines(text)
    for i in range(len(a)):
        assert a.argv(i) == oracle.args_argv(text, i, argv0)


def test_loader_errors():
    from paper_conf_icppw_tiancd23_b200 import Args, EnsError
    from paper_conf_icppw_tiancd23_b200 import _ens
    with pytest.raises(EnsError) as e:
        Args.load("/nonexistent/args.txt")
    assert e.value.code == _ens.ENS_ENOENT
    with pytest.raises(EnsError) as e:
        Args.parse("x " * 200 + "\n", argv0="p")  # more than ENS_MAX_ARGC
    assert e.value.code == _ens.ENS_EINVAL
    with pytest.raises(EnsError) as e:
        Args.parse(b"a\x00b\n")
    assert e.value.code == _ens.ENS_EPARSE
    with pytest.raises(EnsError) as e:
        Args.parse("a\n").argv(1)
    assert e.value.code == _ens.ENS_ERANGE


def rec(fmt, *args):
    """Raw device stdout record: {u32 fmt, u32 payload}, 8-B slots, strings = len + bytes."""
    slots = b""
    for a in args:
        if isinstance(a, str):
            b = a.encode()
            slots += struct.pack("<Q", len(b)) + b + b"\0" * ((8 - len(b) % 8) % 8)
        elif isinstance(a, float):
            slots += struct.pack("<d", a)
        else:
            slots += struct.pack("<q", a)
    return struct.pack("<II", fmt, len(slots)) + slots


def test_stdout_formatter():
    from paper_conf_icppw_tiancd23_b200 import format_stdout
    raw = rec(5, 3) + rec(6, 0, "echo") + rec(6, 1, "héllo world, a long string of 32+ bytes")
    assert format_stdout(1, raw) == ("argc=3\nargv[0]=echo\nargv[1]=héllo world, a long string of 32+ bytes\n").encode()
    raw = rec(7, "small", 68, 1000, "unionized", 10000, 1070) + rec(8, 945990)
    assert format_stdout(2, raw) == (b"XSBench-style HM=small n_iso=68 n_gp=1000 grid=unionized L=10000 seed=1070\n"
                                     b"Verification checksum: 945990\n")
    raw = rec(10, 32768, 223232, 20, 0.1 + 0.2)
    assert format_stdout(4, raw) == b"AMGmk-style n=32768 nnz=223232 iters=20 maxerr=%.17g\n" % (0.1 + 0.2)
    raw = rec(4, "nosuchapp")
    assert format_stdout(0, raw) == b"nosuchapp: command not found\n"


def test_stdout_formatter_rejects_garbage():
    from paper_conf_icppw_tiancd23_b200 import EnsError, format_stdout
    with pytest.raises(EnsError):
        format_stdout(1, struct.pack("<II", 99, 0))
    with pytest.raises(EnsError):
        format_stdout(1, struct.pack("<II", 5, 64))


def py_expand(n, tpl):
    """Independent reference for @repeat: Python eval of {expr} with C integer semantics."""
    import re as _re

    def cdiv(a, b):
        q = abs(a) // abs(b)
        return q if (a >= 0) == (b >= 0) else -q

    out = []
    for i in range(n):
        def sub(mo):
            body = mo.group(1)
            if "|" in body:
                alts = body.split("|")
                return alts[i % len(alts)]
            expr = body.replace("i", str(i))
            expr = _re.sub(r"(\d+)\s*/\s*(\d+)", lambda m: str(cdiv(int(m.group(1)), int(m.group(2)))), expr)
            return str(eval(expr))
        out.append(_re.sub(r"\{([^}]*)\}", sub, tpl))
    return "".join(l + "\n" for l in out)


@pytest.mark.parametrize("n,tpl", [
    (4, "xsbench -s small -r {1070+i}"),
    (5, "rsbench -l {10000*(1+i%3)} -p {500|1000|2000} -w {50|100|200}{ -d|||}"),
    (3, "amgmk -x {32} -y {i*8+24} -z {(i+1)*(i+2)}"),
    (0, "echo {i}"),
])
def test_repeat_templates(n, tpl):
    from paper_conf_icppw_tiancd23_b200 import Args, _ens
    text = f"echo first\n@repeat {n} {tpl}\necho last\n"
    exp = "echo first\n" + py_expand(n, tpl) + "echo last\n"
    assert _ens.expand_args(text) == exp
    a = Args.parse(text)
    assert len(a) == n + 2
    ref = Args.parse(exp)
    assert [a.argv(k) for k in range(len(a))] == [ref.argv(k) for k in range(len(ref))]


@pytest.mark.parametrize("bad", ["@repeat x echo", "@repeat 3 echo {i", "@repeat 2 echo {i/0}", "@repeat 2 echo {j}"])
def test_repeat_errors(bad):
    from paper_conf_icppw_tiancd23_b200 import Args, EnsError
    with pytest.raises(EnsError):
        Args.parse(bad + "\n")
