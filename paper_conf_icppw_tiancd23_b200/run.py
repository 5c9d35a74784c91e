"""Multi-GPU ensemble launcher (the paper's loader, one process per GPU).

    python -m torch.distributed.run --nproc-per-node G --master-addr 127.0.0.1 \\
        -m paper_conf_icppw_tiancd23_b200.run -f args.txt [-n N] [-t T] [-a auto|xsbench|...]

Rank r runs instances {i < N : i mod G == r} as one ensemble on its GPU
(ens_launch(first = r, stride = G)); no communication during compute; one
NCCL all-gather of the 80-byte records, tallies and raw stdout buffers
(SURVEY.md §8(e)); rank 0 prints every instance's stdout in instance order and
a summary on stderr.  Without torchrun it runs on the current GPU alone.
"""
import argparse
import os
import sys

import torch
import torch.distributed as dist

from . import _ens
from . import dist as D
from ._ens import Args
from .ensemble import Ensemble


def main(argv=None):
    ap = argparse.ArgumentParser(prog="ens_run")
    ap.add_argument("-f", required=True, help="arguments file: one instance command line per line")
    ap.add_argument("-n", type=int, default=None, help="number of instances (default: all lines)")
    ap.add_argument("-t", type=int, default=256, help="thread limit per instance (an upper bound)")
    ap.add_argument("-a", default="auto", help="app: auto (argv[0] of each line), echo, xsbench, rsbench, amgmk, pagerank")
    ap.add_argument("-M", type=int, default=0, help="instances per CTA, the (N/M, M, 1) block mapping (P:393-404)")
    ap.add_argument("--argv0", default=None)
    ap.add_argument("-q", action="store_true", help="do not print the instances' stdout")
    a = ap.parse_args(argv)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    argv0 = a.argv0 if a.argv0 is not None else (None if a.a == "auto" else a.a)
    args = Args.load(a.f, argv0=argv0)
    n_total = len(args) if a.n is None else a.n
    if n_total > len(args):
        print(f"ens_run: -n {n_total} > {len(args)} lines", file=sys.stderr)
        return 2
    n_local = D.shard_count(n_total, rank, world)
    ens = Ensemble(args, app=a.a, n=n_local, first=rank, stride=world, threads=a.t,
                   instances_per_cta=a.M).launch()
    torch.cuda.synchronize()
    ms = ens.elapsed_ms() if n_local else 0.0
    if world > 1:
        recs, _, raw = D.gather_ensemble(ens, n_total)
        t = torch.tensor([ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        outs = []
        for k in range(n_total):
            ln = int(recs[k]["stdout_len"])
            outs.append(_ens.format_stdout(int(recs[k]["app"]), raw[k][:ln].tobytes()) if ln else b"")
    else:
        c = ens.collect()
        recs, outs = c.records, c.stdout
    if rank == 0:
        if not a.q:
            for o in outs:
                sys.stdout.buffer.write(o)
            sys.stdout.flush()
        nz = int((recs["exit_code"] != 0).sum())
        print(f"ens_run: {n_total} instances on {world} GPU(s), {ms:.3f} ms (max over ranks), "
              f"{n_total / (ms * 1e-3) if ms > 0 else 0:.1f} instances/s, {nz} nonzero exit", file=sys.stderr)
    ens.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
