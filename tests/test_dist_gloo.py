"""S11 host logic with world_size 2 over gloo on CPU.

Each rank produces the records of its shard {i : i mod G == rank} — here from
the oracle, standing in for the device path (host records only) — and the
package's dist.gather_ensemble all-gathers records, tallies and raw stdout
rows and reorders them to instance order.  Rank 0's gathered result must
equal a single-process run of all lines, bit for bit.
"""
import os
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)

LINES = [
    "xsbench -s small -g 30 -l 200 -r 1",
    "rsbench -s small -l 50 -p 10 -w 3 -r 2",
    "amgmk -x 3 -y 4 -z 5 -i 2 -r 3",
    "echo a b",
    "xsbench -s small -g 20 -l 100 -G hash -h 9 -r 4",
    "nosuchapp",
    "amgmk -x 2 -y 2 -z 2 -i 1",
]


class FakeShard:
    """Duck-types Ensemble.device_records/_tallies/_stdout with host tensors."""

    def __init__(self, recs, tallies, outs, cap=256):
        self.recs = torch.from_numpy(recs.view(np.uint8).reshape(len(recs), 80).copy())
        self.tal = torch.from_numpy(tallies.view(np.uint8).reshape(len(recs), 128).copy())
        raw = np.zeros((len(recs), cap), dtype=np.uint8)
        for k, o in enumerate(outs):
            raw[k, :len(o)] = np.frombuffer(o, dtype=np.uint8)
        self.raw = torch.from_numpy(raw)

    def device_records(self):
        return self.recs

    def device_tallies(self):
        return self.tal

    def device_stdout(self):
        return self.raw


def _worker(rank, world, port, n_total, q):
    sys.path.insert(0, ROOT)
    sys.path.insert(0, HERE)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle_lib
        from paper_conf_icppw_tiancd23_b200 import dist as D
        ids = D.shard_ids(n_total, rank, world)
        assert len(ids) == D.shard_count(n_total, rank, world)
        text = "".join(LINES[i] + "\n" for i in ids)
        r = oracle_lib.run_text(text, jobs=1) if ids else None
        if r is None:
            recs = np.zeros(0, dtype=oracle_lib.RECORD_DTYPE)
            tal = np.zeros((0, 32), dtype=np.uint32)
            outs = []
        else:
            recs, tal, outs = r.records.copy(), r.tallies, r.stdout
            recs["instance"] = np.array(ids, dtype=np.uint32)
        R, T, raw = D.gather_ensemble(FakeShard(recs, tal, outs), n_total)
        if rank == 0:
            q.put((R.tobytes(), T.tobytes(), [bytes(raw[k][:int(R[k]["stdout_len"])]) for k in range(n_total)]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n_total", [7, 6, 1])
def test_gather_equals_single_process(oracle, n_total):
    world = 2
    port = 29600 + n_total
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n_total, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    full = oracle.run_text("".join(l + "\n" for l in LINES[:n_total]), jobs=1)
    R = np.frombuffer(got[0], dtype=oracle.RECORD_DTYPE)
    T = np.frombuffer(got[1], dtype=np.uint32).reshape(n_total, 32)
    assert R.tobytes() == full.records.tobytes()
    assert np.array_equal(T, full.tallies)
    assert got[2] == full.stdout


def test_shard_arithmetic():
    sys.path.insert(0, ROOT)
    from paper_conf_icppw_tiancd23_b200 import dist as D
    for n in range(0, 40):
        for g in (1, 2, 3, 4, 8):
            ids = [D.shard_ids(n, r, g) for r in range(g)]
            assert sorted(sum(ids, [])) == list(range(n))
            assert [len(x) for x in ids] == [D.shard_count(n, r, g) for r in range(g)]
            assert max([len(x) for x in ids] + [0]) == D.padded_count(n, g) or n == 0
    # reorder maps rank-major rows back to instance order
    g, n = 3, 8
    rows = D.padded_count(n, g)
    gathered = torch.full((g * rows, 1), -1, dtype=torch.int64)
    for r in range(g):
        for k, i in enumerate(D.shard_ids(n, r, g)):
            gathered[r * rows + k, 0] = i
    assert D.reorder(gathered, n, g)[:, 0].tolist() == list(range(n))
