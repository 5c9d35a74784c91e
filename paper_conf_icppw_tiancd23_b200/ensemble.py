"""N4: the Python face of ensemble execution, with PyTorch as plumbing only.

torch provides the device workspace (a uint8 tensor handed to ens_launch as a
plain pointer) and the CUDA stream; everything else happens in libens.so.

    ens = Ensemble(Args.parse(text, argv0=None), app="auto", threads=256)
    ens.launch()                 # one H2D copy + one persistent launch per app
    out = ens.collect()          # records, tallies, stdout (instance order)
"""
import torch

from . import _ens
from ._ens import Args, make_cfg


def _require_cuda():
    if not torch.cuda.is_available():
        raise RuntimeError("ensemble execution needs a CUDA device (no CPU fallback)")


class Ensemble:
    """One ensemble: instances first + k*stride (k < n) of `args` on one GPU."""

    def __init__(self, args, app="auto", n=None, first=0, stride=1, threads=256, grid=0, arena_bytes=0,
                 stdout_bytes=0, timestamps=False, device=None, stream=None, team_ctas=0, phases=False,
                 instances_per_cta=0, generic=False, serial=False, dump_rows=0, fused=False, split=False, clc=False):
        _require_cuda()
        self.args = args
        self.app = app
        total = len(args)
        if n is None:
            n = max(0, (total - first + stride - 1) // stride) if stride > 0 else 0
        self.cfg = make_cfg(n, first=first, stride=stride, grid=grid, threads=threads, arena_bytes=arena_bytes,
                            stdout_bytes=stdout_bytes,
                            flags=(_ens.ENS_F_TIMESTAMPS if timestamps else 0) | (_ens.ENS_F_PHASES if phases else 0)
                            | (_ens.ENS_F_GENERIC if generic else 0) | (_ens.ENS_F_SERIAL if serial else 0)
                            | (_ens.ENS_F_FUSED if fused else 0) | (_ens.ENS_F_SPLIT_PHASES if split else 0)
                            | (_ens.ENS_F_CLC if clc else 0),
                            team_ctas=team_ctas, instances_per_cta=instances_per_cta, dump_rows=dump_rows)
        self.n = n
        self.device = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        self.stream = stream
        self.run = None
        self.workspace = None

    def _stream_ptr(self):
        s = self.stream if self.stream is not None else torch.cuda.current_stream(self.device)
        return s.cuda_stream

    def launch(self):
        """Size and allocate the workspace, marshal the args, enqueue."""
        with torch.cuda.device(self.device):
            if self.run is not None:
                self.run.close()
            ws = _ens.workspace_bytes(self.app, self.args, self.cfg)
            if self.workspace is None or self.workspace.numel() < ws:
                self.workspace = torch.empty(max(ws, 1), dtype=torch.uint8, device=self.device)
            self.run = _ens.Run.launch(self.app, self.args, self.cfg, self.workspace.data_ptr(), ws,
                                       self._stream_ptr(), keep=self.workspace)
        return self

    def relaunch(self):
        """Re-run with the arguments already resident on the device."""
        with torch.cuda.device(self.device):
            self.run.relaunch(self._stream_ptr())
        return self

    def collect(self, tallies=True, stdout=True):
        out = self.run.collect(tallies=tallies, stdout=stdout)
        out.dump = self.run.collect_dump(self.cfg.dump_rows) if self.cfg.dump_rows else None
        return out

    def elapsed_ms(self):
        return self.run.elapsed_ms()

    def info(self):
        return self.run.info()

    def device_records(self):
        """The records as a uint8 view [n, 80] of the workspace (for NCCL)."""
        i = self.run.info()
        off = int(i.records_offset)
        return self.workspace[off:off + 80 * self.n].view(self.n, 80)

    def device_stdout(self):
        """Raw per-instance stdout buffers [n, stdout_bytes] (device view)."""
        i = self.run.info()
        off, cap = int(i.stdout_offset), int(i.stdout_bytes)
        return self.workspace[off:off + cap * self.n].view(self.n, cap)

    def device_tallies(self):
        i = self.run.info()
        off = int(i.tallies_offset)
        return self.workspace[off:off + 4 * _ens.ENS_TALLIES * self.n].view(self.n, 4 * _ens.ENS_TALLIES)

    def close(self):
        if self.run is not None:
            self.run.close()
            self.run = None
        big = self.workspace is not None and self.workspace.numel() > (8 << 30)
        self.workspace = None
        if big:  # hand a large workspace back to the device (ens_workspace_bytes sizes by free memory)
            torch.cuda.empty_cache()


def run_text(text, app="auto", argv0=None, **kw):
    """Parse `text`, run it as one ensemble, collect."""
    ens = Ensemble(Args.parse(text, argv0=argv0), app=app, **kw).launch()
    out = ens.collect()
    ens.close()
    return out
