"""S11: one process per GPU, instances sharded by id, one all-gather at the end.

Instances are independent (Fig. 4), so rank r of G runs instances
{i : i mod G == r} (round-robin balances mixed lines) with
ens_launch(first=r, stride=G) and no communication during compute.  The only
collective is an all-gather of the fixed 80-byte records (and the tallies and
raw stdout buffers) over NCCL — NVLink5 / NVSwitch on a B200 box — after
which every rank holds the whole ensemble's results in instance order.

The host-side logic (shard sizes, padding, reordering) is plain functions
here so it can be exercised with the gloo backend on CPU tensors.
"""
import numpy as np
import torch
import torch.distributed as dist

from ._ens import RECORD_DTYPE, ENS_RF_NOT_RUN, ENS_TALLIES


def shard_count(n_total, rank, world):
    """Number of instances rank `rank` runs: |{i < n_total : i mod world == rank}|."""
    return max(0, (n_total - rank + world - 1) // world)


def shard_ids(n_total, rank, world):
    return list(range(rank, n_total, world))


def padded_count(n_total, world):
    return shard_count(n_total, 0, world)


def pad_rows(t, rows):
    """Pad a [n, w] uint8 tensor to [rows, w] with zero rows (NOT_RUN records)."""
    if t.shape[0] == rows:
        return t.contiguous()
    out = torch.zeros((rows, t.shape[1]), dtype=t.dtype, device=t.device)
    out[: t.shape[0]] = t
    return out


def all_gather_rows(t, rows, group=None):
    """All-gather a per-rank [n_r, w] uint8 tensor padded to `rows` -> [world*rows, w]."""
    world = dist.get_world_size(group)
    src = pad_rows(t, rows)
    out = torch.empty((world * rows, t.shape[1]), dtype=t.dtype, device=t.device)
    dist.all_gather_into_tensor(out, src, group=group)
    return out


def reorder(gathered, n_total, world):
    """Rows gathered rank-major ([rank][k]) -> instance order i = rank + k*world."""
    rows = padded_count(n_total, world)
    g = gathered.reshape(world, rows, -1)
    idx = torch.arange(n_total, device=gathered.device)
    return g[idx % world, idx // world]


def records_from_bytes(b):
    """uint8 [n, 80] (host or device tensor) -> structured numpy records."""
    a = b.detach().cpu().contiguous().numpy()
    return a.view(RECORD_DTYPE).reshape(-1)


def gather_ensemble(ens, n_total, group=None):
    """All-gather one rank's device results into instance order on every rank.

    Returns (records [n_total] structured, tallies [n_total, 32] uint32,
    raw stdout uint8 [n_total, stdout_bytes]) as host arrays; records of
    instances that never ran carry ENS_RF_NOT_RUN.
    """
    world = dist.get_world_size(group)
    rows = padded_count(n_total, world)
    recs = reorder(all_gather_rows(ens.device_records(), rows, group), n_total, world)
    tal = reorder(all_gather_rows(ens.device_tallies(), rows, group), n_total, world)
    out = reorder(all_gather_rows(ens.device_stdout(), rows, group), n_total, world)
    R = records_from_bytes(recs).copy()
    missing = (R["flags"] & 8) == 0  # no ENS_RF_DONE
    R["flags"][missing] |= ENS_RF_NOT_RUN
    T = tal.detach().cpu().contiguous().numpy().view(np.uint32).reshape(n_total, ENS_TALLIES)
    return R, T, out.detach().cpu().numpy()
