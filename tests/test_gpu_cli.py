"""The C++ loader CLI `ens_run` (SURVEY.md §8(b) CLI, Fig. 5c): its stdout and its
--json records equal the oracle's, on one GPU and sharded over --gpus G (the GPUs this box has)."""
import json
import os
import subprocess

import numpy as np
import pytest

import oracle_lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ENS_RUN = os.path.join(ROOT, "paper_conf_icppw_tiancd23_b200", "ens_run")

TEXT = ("xsbench -s small -g 150 -l 2000 -G unionized -r 11\n"
        "rsbench -s small -l 300 -p 12 -w 3 -r 5\n"
        "amgmk -x 6 -y 5 -z 4 -i 3 -r 2\n"
        "xsbench -s small -g 120 -l 1500 -G hash -h 40 -r 12\n"
        "echo one two\n"
        "nosuch arg\n"
        "xsbench -s small -g 1 -l 10\n")


def _gpus():
    import torch
    return torch.cuda.device_count() if torch.cuda.is_available() else 0


@pytest.mark.gpu
@pytest.mark.parametrize("gpus", [1, 2])
def test_ens_run_cli_matches_oracle(tmp_path, gpus):
    if gpus > _gpus():
        pytest.skip(f"{gpus} GPUs not visible")
    f = tmp_path / "args.txt"
    f.write_text(TEXT)
    out = tmp_path / "run.json"
    p = subprocess.run([ENS_RUN, "-f", str(f), "-t", "128", "--gpus", str(gpus), "--json", str(out)],
                       capture_output=True, timeout=300)
    assert p.returncode == 0, p.stderr
    o = oracle_lib.run_text(TEXT)
    assert p.stdout == b"".join(o.stdout)
    d = json.loads(out.read_text())
    assert d["instances"] == len(o.records) and d["gpus"] == gpus
    for k, r in enumerate(d["records"]):
        b = o.records[k]
        assert r["instance"] == int(b["instance"]) and r["gpu"] == k % gpus
        for key in ("exit_code", "app", "flags", "vhash", "bitsum", "work"):
            assert r[key] == int(b[key]), (k, key, r[key], b[key])
        tol = 1e-12 * max(abs(float(b["fabs"])), 1e-300)
        assert abs(r["fsum"] - float(b["fsum"])) <= tol and abs(r["fabs"] - float(b["fabs"])) <= tol
        assert r["stdout"].encode() == o.stdout[k]
    assert np.count_nonzero([r["exit_code"] for r in d["records"]]) == d["nonzero_exit"]
