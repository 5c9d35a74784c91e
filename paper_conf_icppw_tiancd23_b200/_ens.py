"""N4: thin ctypes binding over libens.so (include/ens.h), same names.

Argument marshalling only: every step of the hot path (loader, marshalling,
scheduling, instance bodies, reductions, stdout records) runs in libens.so and
its sm_100a kernels.  There is no CPU fallback: if the shared library is
missing this module raises on import.
"""
import ctypes
import os

import numpy as np

PKG_DIR = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("ENS_LIB_PATH") or os.path.join(PKG_DIR, "libens.so")  # override: A/B builds

ENS_OK, ENS_EINVAL, ENS_ENOENT, ENS_ENOMEM, ENS_ECUDA, ENS_ERANGE, ENS_EBUSY, ENS_EPARSE = 0, -1, -2, -3, -4, -5, -6, -7
ENS_EXIT_USAGE, ENS_EXIT_NOMEM, ENS_EXIT_NOTFOUND = 1, 12, 127
ENS_RF_STDOUT_TRUNC, ENS_RF_NOMEM, ENS_RF_NOT_RUN, ENS_RF_DONE = 1, 2, 4, 8
ENS_F_TIMESTAMPS, ENS_F_PHASES, ENS_F_GENERIC, ENS_F_SERIAL, ENS_F_FUSED, ENS_F_SPLIT_PHASES, ENS_F_CLC = \
    1, 2, 4, 8, 16, 32, 64
ENS_PHASES = 16
ENS_APP_BY_ARGV0, ENS_APP_ECHO, ENS_APP_XSBENCH, ENS_APP_RSBENCH, ENS_APP_AMGMK, ENS_APP_PAGERANK = 0, 1, 2, 3, 4, 5
ENS_N_APPS = 6
APP_IDS = {"auto": 0, "echo": 1, "xsbench": 2, "rsbench": 3, "amgmk": 4, "pagerank": 5}
ENS_TALLIES = 32
ENS_MAX_ARGC = 128

RECORD_DTYPE = np.dtype([
    ("instance", "<u4"), ("exit_code", "<i4"), ("app", "<u4"), ("flags", "<u4"),
    ("vhash", "<u8"), ("bitsum", "<u8"), ("fsum", "<f8"), ("fabs", "<f8"),
    ("work", "<u8"), ("stdout_len", "<u4"), ("smid", "<u4"),
    ("t_start_ns", "<u8"), ("t_end_ns", "<u8"),
])
assert RECORD_DTYPE.itemsize == 80


class EnsError(RuntimeError):
    def __init__(self, where, code, detail):
        super().__init__(f"{where}: {code} ({detail})")
        self.code = code


class LaunchCfg(ctypes.Structure):
    _fields_ = [("first", ctypes.c_int32), ("n_instances", ctypes.c_int32), ("stride", ctypes.c_int32),
                ("grid_blocks", ctypes.c_int32), ("block_threads", ctypes.c_int32),
                ("arena_bytes", ctypes.c_uint64), ("stdout_bytes", ctypes.c_uint32), ("flags", ctypes.c_uint32),
                ("team_ctas", ctypes.c_int32), ("instances_per_cta", ctypes.c_int32),
                ("dump_rows", ctypes.c_uint32)]


class KernelTime(ctypes.Structure):
    _fields_ = [("app", ctypes.c_int32), ("phase", ctypes.c_int32), ("kind", ctypes.c_int32),
                ("grid_ctas", ctypes.c_int32), ("block_threads", ctypes.c_int32), ("ms", ctypes.c_float)]


class RunInfo(ctypes.Structure):
    _fields_ = [("n_instances", ctypes.c_int32), ("n_groups", ctypes.c_int32),
                ("grid_blocks", ctypes.c_int32 * ENS_N_APPS), ("block_threads", ctypes.c_int32 * ENS_N_APPS),
                ("kernel_launches", ctypes.c_int32), ("arena_bytes", ctypes.c_uint64),
                ("ws_bytes", ctypes.c_uint64), ("records_offset", ctypes.c_uint64),
                ("tallies_offset", ctypes.c_uint64), ("stdout_offset", ctypes.c_uint64),
                ("stdout_bytes", ctypes.c_uint32), ("h2d_bytes", ctypes.c_uint64),
                ("d2h_bytes", ctypes.c_uint64), ("team_ctas", ctypes.c_int32 * ENS_N_APPS),
                ("instances_per_cta", ctypes.c_int32 * ENS_N_APPS)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it first (python -c 'import __graft_entry__ as g; g.build()' "
                          f"or make -C paper_conf_icppw_tiancd23_b200/csrc). There is no CPU fallback.")
    L = ctypes.CDLL(LIB_PATH)
    p, i, sz, u32, u64 = ctypes.c_void_p, ctypes.c_int, ctypes.c_size_t, ctypes.c_uint32, ctypes.c_uint64
    pp = ctypes.POINTER(ctypes.c_void_p)
    sigs = {
        "ens_load_args": (i, [ctypes.c_char_p, ctypes.c_char_p, pp]),
        "ens_parse_args": (i, [ctypes.c_char_p, sz, ctypes.c_char_p, pp]),
        "ens_args_count": (i, [p]),
        "ens_expand_args": (ctypes.c_long, [ctypes.c_char_p, sz, p, sz]),
        "ens_args_get": (i, [p, i, ctypes.POINTER(ctypes.c_int), ctypes.POINTER(ctypes.POINTER(ctypes.c_char_p))]),
        "ens_args_free": (None, [p]),
        "ens_workspace_bytes": (i, [i, p, ctypes.POINTER(LaunchCfg), ctypes.POINTER(sz)]),
        "ens_launch": (i, [i, p, ctypes.POINTER(LaunchCfg), p, sz, p, pp]),
        "ens_run_relaunch": (i, [p, p]),
        "ens_collect": (i, [p, p, p, p, sz, p]),
        "ens_collect_dump": (i, [p, p, sz]),
        "ens_run_elapsed_ms": (i, [p, ctypes.POINTER(ctypes.c_float)]),
        "ens_run_phases": (i, [p, ctypes.POINTER(ctypes.c_uint64)]),
        "ens_run_kernel_times": (i, [p, ctypes.POINTER(KernelTime), i]),
        "ens_run_get_info": (i, [p, ctypes.POINTER(RunInfo)]),
        "ens_format_stdout": (ctypes.c_long, [u32, p, sz, p, sz]),
        "ens_run_free": (None, [p]),
        "ens_strerror": (ctypes.c_char_p, [i]),
        "ens_last_error": (ctypes.c_char_p, []),
        "ens_version": (ctypes.c_char_p, []),
    }
    for name, (res, args) in sigs.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    return L


lib = _load()
EXPORTED = ["ens_load_args", "ens_parse_args", "ens_expand_args", "ens_args_count", "ens_args_get", "ens_args_free",
            "ens_workspace_bytes", "ens_launch", "ens_run_relaunch", "ens_collect", "ens_collect_dump",
            "ens_run_elapsed_ms",
            "ens_run_phases", "ens_run_kernel_times",
            "ens_run_get_info", "ens_format_stdout", "ens_run_free", "ens_strerror", "ens_last_error",
            "ens_version"]


def _check(where, rc):
    if rc != ENS_OK:
        raise EnsError(where, rc, (lib.ens_last_error() or b"").decode(errors="replace"))
    return rc


def _app_id(app):
    return APP_IDS[app] if isinstance(app, str) else int(app)


class Args:
    """ens_args: the parsed args file (one instance per line)."""

    def __init__(self, handle):
        self._h = handle

    @classmethod
    def load(cls, path, argv0=None):
        h = ctypes.c_void_p()
        _check("ens_load_args", lib.ens_load_args(os.fsencode(path), argv0.encode() if argv0 else None,
                                                  ctypes.byref(h)))
        return cls(h)

    @classmethod
    def parse(cls, text, argv0=None):
        if isinstance(text, str):
            text = text.encode()
        h = ctypes.c_void_p()
        _check("ens_parse_args", lib.ens_parse_args(text, len(text), argv0.encode() if argv0 else None,
                                                    ctypes.byref(h)))
        return cls(h)

    def __len__(self):
        return lib.ens_args_count(self._h)

    def argv(self, i):
        argc = ctypes.c_int()
        argv = ctypes.POINTER(ctypes.c_char_p)()
        _check("ens_args_get", lib.ens_args_get(self._h, i, ctypes.byref(argc), ctypes.byref(argv)))
        return [argv[k].decode() for k in range(argc.value)]

    @property
    def handle(self):
        return self._h

    def close(self):
        if self._h:
            lib.ens_args_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def make_cfg(n, first=0, stride=1, grid=0, threads=0, arena_bytes=0, stdout_bytes=0, flags=0, team_ctas=0,
             instances_per_cta=0, dump_rows=0):
    return LaunchCfg(first, n, stride, grid, threads, arena_bytes, stdout_bytes, flags, team_ctas,
                     instances_per_cta, dump_rows)


def workspace_bytes(app, args, cfg):
    b = ctypes.c_size_t()
    _check("ens_workspace_bytes", lib.ens_workspace_bytes(_app_id(app), args.handle, ctypes.byref(cfg),
                                                          ctypes.byref(b)))
    return b.value


class Collected:
    def __init__(self, records, tallies, stdout):
        self.records, self.tallies, self.stdout = records, tallies, stdout


class Run:
    """ens_run: one enqueued ensemble (keeps its workspace tensor alive)."""

    def __init__(self, handle, n, keep):
        self._h, self.n, self._keep = handle, n, keep

    @classmethod
    def launch(cls, app, args, cfg, workspace_ptr=None, ws_bytes=0, stream=None, keep=None):
        h = ctypes.c_void_p()
        _check("ens_launch", lib.ens_launch(_app_id(app), args.handle, ctypes.byref(cfg),
                                            ctypes.c_void_p(workspace_ptr) if workspace_ptr else None, ws_bytes,
                                            ctypes.c_void_p(stream) if stream else None, ctypes.byref(h)))
        return cls(h, cfg.n_instances, (args, keep))

    def relaunch(self, stream=None):
        _check("ens_run_relaunch", lib.ens_run_relaunch(self._h, ctypes.c_void_p(stream) if stream else None))

    def collect(self, tallies=True, stdout=True):
        n = self.n
        recs = np.zeros(n, dtype=RECORD_DTYPE)
        tal = np.zeros((n, ENS_TALLIES), dtype=np.uint32) if tallies else None
        off = np.zeros(n + 1, dtype=np.uint64)
        rp = recs.ctypes.data_as(ctypes.c_void_p) if n else None
        tp = tal.ctypes.data_as(ctypes.c_void_p) if (tallies and n) else None
        op = off.ctypes.data_as(ctypes.c_void_p)
        outs = None
        if stdout:
            _check("ens_collect", lib.ens_collect(self._h, rp, tp, None, 0, op))
            total = int(off[n])
            buf = ctypes.create_string_buffer(total + 1)
            _check("ens_collect", lib.ens_collect(self._h, rp, tp, buf, total + 1, op))
            raw = buf.raw
            outs = [raw[int(off[k]):int(off[k + 1])] for k in range(n)]
        else:
            _check("ens_collect", lib.ens_collect(self._h, rp, tp, None, 0, op))
        return Collected(recs, tal, outs)

    def collect_dump(self, dump_rows):
        """Element-wise result rows [n, dump_rows, 8] (launched with dump_rows > 0)."""
        d = np.zeros((self.n, dump_rows, 8))
        _check("ens_collect_dump", lib.ens_collect_dump(self._h, d.ctypes.data_as(ctypes.c_void_p) if d.size else None,
                                                        d.size))
        return d

    def elapsed_ms(self):
        ms = ctypes.c_float()
        _check("ens_run_elapsed_ms", lib.ens_run_elapsed_ms(self._h, ctypes.byref(ms)))
        return ms.value

    def kernel_times(self):
        """[(app, phase, kind, grid_ctas, block_threads, ms)] of the last (re)launch's kernels."""
        a = (KernelTime * 16)()
        n = lib.ens_run_kernel_times(self._h, a, 16)
        if n < 0:
            _check("ens_run_kernel_times", n)
        return [(a[q].app, a[q].phase, a[q].kind, a[q].grid_ctas, a[q].block_threads, a[q].ms) for q in range(n)]

    def phases_ns(self):
        """Per-phase device time summed over instances (launched with ENS_F_PHASES)."""
        a = (ctypes.c_uint64 * ENS_PHASES)()
        _check("ens_run_phases", lib.ens_run_phases(self._h, a))
        return list(a)

    def info(self):
        i = RunInfo()
        _check("ens_run_get_info", lib.ens_run_get_info(self._h, ctypes.byref(i)))
        return i

    def close(self):
        if self._h:
            lib.ens_run_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def format_stdout(app, raw):
    raw = bytes(raw)
    n = lib.ens_format_stdout(_app_id(app), raw, len(raw), None, 0)
    if n < 0:
        raise EnsError("ens_format_stdout", n, (lib.ens_last_error() or b"").decode())
    buf = ctypes.create_string_buffer(n + 1)
    lib.ens_format_stdout(_app_id(app), raw, len(raw), buf, n + 1)
    return buf.raw[:n]


def version():
    return lib.ens_version().decode()


def expand_args(text):
    """Expand "@repeat N <template>" lines (the args-file script language)."""
    if isinstance(text, str):
        text = text.encode()
    n = lib.ens_expand_args(text, len(text), None, 0)
    if n < 0:
        raise EnsError("ens_expand_args", n, "malformed @repeat template")
    buf = ctypes.create_string_buffer(n + 1)
    lib.ens_expand_args(text, len(text), buf, n + 1)
    return buf.raw[:n].decode()
