"""S11 on the device: the NCCL path of dist.gather_ensemble / run.py, world size 1 on one B200
(the multi-rank host logic is covered by tests/test_dist_gloo.py with gloo, world 2), and the
multi-GPU loader run through torch.distributed.run."""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LINES = ["xsbench -s small -g 200 -l 3000 -G unionized -r 1070",
         "rsbench -s small -l 500 -p 40 -w 8 -r 3",
         "amgmk -x 8 -y 8 -z 8 -i 5 -r 4",
         "echo hello nccl",
         "xsbench -s small -g 150 -l 2000 -G hash -h 50 -r 1071"]


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_gather_ensemble_nccl_world1(oracle):
    import torch
    import torch.distributed as dist
    from paper_conf_icppw_tiancd23_b200 import Args, dist as D
    from paper_conf_icppw_tiancd23_b200.ensemble import Ensemble
    from paper_conf_icppw_tiancd23_b200 import _ens
    from parity import assert_parity
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(free_port()))
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        assert dist.get_backend() == "nccl"
        text = "".join(l + "\n" for l in LINES)
        ens = Ensemble(Args.parse(text), app="auto", threads=256).launch()
        torch.cuda.synchronize()
        R, T, raw = D.gather_ensemble(ens, len(LINES))
        local = ens.collect()
        ens.close()
    finally:
        dist.destroy_process_group()
    # device records carry the RAW stdout length (the {fmt, args} records); ens_collect reports
    # the formatted length — every other field is the same bytes
    for f in R.dtype.names:
        if f != "stdout_len":
            assert np.array_equal(R[f], local.records[f]), f
    assert np.array_equal(T, local.tallies)
    outs = [_ens.format_stdout(int(R[k]["app"]), raw[k][:int(R[k]["stdout_len"])].tobytes()) for k in range(len(LINES))]
    assert outs == local.stdout
    o = oracle.run_text(text)

    class G:
        pass
    g = G()
    g.records, g.tallies, g.stdout = local.records, local.tallies, outs
    assert_parity(g, o)


def test_run_loader_torchrun(tmp_path, oracle):
    f = tmp_path / "args.txt"
    f.write_text("".join(l + "\n" for l in LINES))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "1",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()),
           "-m", "paper_conf_icppw_tiancd23_b200.run", "-f", str(f), "-t", "256"]
    env = dict(os.environ, NCCL_DEBUG="WARN", PYTHONPATH=ROOT)
    p = subprocess.run(cmd, cwd=ROOT, capture_output=True, timeout=600, env=env)
    assert p.returncode == 0, p.stderr.decode()[-2000:]
    o = oracle.run_text(f.read_text())
    assert p.stdout == b"".join(o.stdout)


def test_bench_strong_mode_runs():
    """bench.py --strong (C5: 4096 lines over the ranks) at --gpus 1: one JSON line, strong scaling,
    every instance exited 0 and the oracle sample matched."""
    import json
    p = subprocess.run([sys.executable, "bench.py", "--strong", "--steps", "2", "--warmup", "3", "--no-extras"],
                       cwd=ROOT, capture_output=True, timeout=900)
    assert p.returncode == 0, p.stderr.decode()[-2000:]
    d = json.loads(p.stdout.decode().strip().splitlines()[-1])
    assert d["scaling"] == "strong" and d["config"]["instances_total"] == 4096
    assert d["all_exit_ok"] and d["parity_sample_ok"]
