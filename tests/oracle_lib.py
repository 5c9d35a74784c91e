"""ctypes wrapper over oracle/liboracle.so — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this module (the oracle is the CPU definition the
CUDA path is checked against; see oracle/oracle.hpp).
"""
import ctypes
import os
import subprocess
import threading

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ORACLE_DIR = os.path.join(ROOT, "oracle")
LIB_PATH = os.path.join(ORACLE_DIR, "liboracle.so")
BIN_PATH = os.path.join(ORACLE_DIR, "ens_oracle")

APP_BY_ARGV0, APP_ECHO, APP_XSBENCH, APP_RSBENCH, APP_AMGMK, APP_PAGERANK = 0, 1, 2, 3, 4, 5
APP_NAMES = {APP_ECHO: "echo", APP_XSBENCH: "xsbench", APP_RSBENCH: "rsbench", APP_AMGMK: "amgmk",
             APP_PAGERANK: "pagerank"}
N_TALLIES = 32

RECORD_DTYPE = np.dtype([
    ("instance", "<u4"), ("exit_code", "<i4"), ("app", "<u4"), ("flags", "<u4"),
    ("vhash", "<u8"), ("bitsum", "<u8"), ("fsum", "<f8"), ("fabs", "<f8"),
    ("work", "<u8"), ("stdout_len", "<u4"), ("smid", "<u4"),
    ("t_start_ns", "<u8"), ("t_end_ns", "<u8"),
])
assert RECORD_DTYPE.itemsize == 80

_lock = threading.Lock()
_lib = None


def build():
    """make -C oracle (idempotent)."""
    subprocess.run(["make", "-s", "-C", ORACLE_DIR, "-j8"], check=True)


def lib():
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                build()
            L = ctypes.CDLL(LIB_PATH)
            c_p, c_sz, c_l, c_i, c_u32, c_u64, c_d = (ctypes.c_void_p, ctypes.c_size_t, ctypes.c_long,
                                                       ctypes.c_int, ctypes.c_uint32, ctypes.c_uint64,
                                                       ctypes.c_double)
            sig = {
                "oracle_run": (c_p, [ctypes.c_char_p, c_sz, ctypes.c_char_p, c_u32, c_l, c_i]),
                "oracle_count": (c_l, [c_p]),
                "oracle_run_dump": (c_p, [ctypes.c_char_p, c_sz, ctypes.c_char_p, c_u32, c_l, c_i, c_l]),
                "oracle_dump": (c_l, [c_p, c_l, c_p]),
                "oracle_margin": (c_d, [c_p, c_l]),
                "oracle_records": (None, [c_p, c_p]),
                "oracle_tallies": (None, [c_p, c_p]),
                "oracle_stdout_len": (c_sz, [c_p, c_l]),
                "oracle_stdout": (None, [c_p, c_l, c_p]),
                "oracle_free": (None, [c_p]),
                "oracle_args_lines": (c_l, [ctypes.c_char_p, c_sz]),
                "oracle_args_argv": (c_i, [ctypes.c_char_p, c_sz, ctypes.c_char_p, c_l, c_p, c_sz]),
                "oracle_lcg_step": (c_u64, [c_u64]),
                "oracle_lcg_ff": (c_u64, [c_u64, c_u64]),
                "oracle_lcg_double": (c_d, [ctypes.POINTER(c_u64)]),
                "oracle_pick_mat": (c_i, [ctypes.POINTER(c_u64)]),
                "oracle_grid_search": (c_l, [c_p, c_d, c_l, c_l]),
                "oracle_xs_build": (c_p, [c_i, c_l, c_i, c_l, c_u64]),
                "oracle_xs_energies": (None, [c_p, c_p]),
                "oracle_xs_union": (None, [c_p, c_p]),
                "oracle_xs_index_len": (c_sz, [c_p]),
                "oracle_xs_index": (None, [c_p, c_p]),
                "oracle_xs_bracket": (c_l, [c_p, c_i, c_d]),
                "oracle_xs_free": (None, [c_p]),
                "oracle_xs_materials": (c_i, [c_i, c_p, c_p, c_p]),
                "oracle_xs_set_conc_seed": (None, [c_u64]),
                "oracle_rs_fast_w": (None, [c_d, c_d, c_p, c_p]),
                "oracle_rs_trig": (None, [c_i, c_l, c_p, c_p]),
                "oracle_rs_tables": (c_i, [c_i, c_i, c_i, c_u64, c_p, c_p, c_p, c_p, c_i]),
                "oracle_rs_micro": (c_i, [c_i, c_i, c_i, c_u64, c_i, c_i, c_p, c_p, c_p, c_p, c_l, c_p, c_l,
                                          c_p, c_l]),
                "oracle_amg_nnz": (c_l, [c_l, c_l, c_l]),
                "oracle_amg_csr": (None, [c_l, c_l, c_l, c_p, c_p, c_p]),
                "oracle_amg_sweeps": (None, [c_l, c_l, c_l, c_l, c_p]),
                "oracle_amg_apply": (None, [c_l, c_l, c_l, c_p, c_p]),
                "oracle_pr_graph": (c_l, [c_l, c_l, c_u64, c_p, c_p, c_p]),
            }
            for name, (res, args) in sig.items():
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


class OracleRun:
    """Result of oracle_run: records (structured array), tallies [n,32], stdout list."""

    def __init__(self, records, tallies, stdout):
        self.records = records
        self.tallies = tallies
        self.stdout = stdout


def run_text(text, app=APP_BY_ARGV0, argv0=None, n=-1, jobs=None, dump=0):
    """Run the ensemble defined by args-file `text` on the CPU oracle.  dump > 0 also
    returns, per instance, its first `dump` result rows (8 doubles: key, material,
    v[0..4], argmax; see oracle.hpp Instance) in .dumps and the minimum relative
    argmax margin in .margins."""
    L = lib()
    if isinstance(text, str):
        text = text.encode()
    if argv0 is None and app != APP_BY_ARGV0:
        argv0 = APP_NAMES[app]
    a0 = argv0.encode() if argv0 else None
    if jobs is None:
        jobs = os.cpu_count() or 1
    h = L.oracle_run_dump(text, len(text), a0, app, n, jobs, dump) if dump else L.oracle_run(text, len(text), a0, app, n, jobs)
    if not h:
        raise ValueError("oracle_run: n larger than the number of lines")
    try:
        cnt = L.oracle_count(h)
        recs = np.zeros(cnt, dtype=RECORD_DTYPE)
        tal = np.zeros((cnt, N_TALLIES), dtype=np.uint32)
        if cnt:
            L.oracle_records(h, _ptr(recs))
            L.oracle_tallies(h, _ptr(tal))
        outs = []
        for i in range(cnt):
            ln = L.oracle_stdout_len(h, i)
            b = ctypes.create_string_buffer(ln + 1)
            L.oracle_stdout(h, i, b)
            outs.append(b.raw[:ln])
        run = OracleRun(recs, tal, outs)
        if dump:
            run.dumps, run.margins = [], np.zeros(cnt)
            for i in range(cnt):
                k = L.oracle_dump(h, i, None)
                d = np.zeros((k, 8))
                if k:
                    L.oracle_dump(h, i, _ptr(d))
                run.dumps.append(d)
                run.margins[i] = L.oracle_margin(h, i)
        return run
    finally:
        L.oracle_free(h)


def args_argv(text, i, argv0="prog"):
    L = lib()
    if isinstance(text, str):
        text = text.encode()
    buf = ctypes.create_string_buffer(1 << 16)
    argc = L.oracle_args_argv(text, len(text), argv0.encode() if argv0 else None, i, buf, len(buf))
    if argc < 0:
        raise IndexError(i)
    s = buf.value.decode()
    return s.split("\x1f") if argc > 0 else []


def args_lines(text):
    if isinstance(text, str):
        text = text.encode()
    return lib().oracle_args_lines(text, len(text))


def lcg_ff(s, n):
    return lib().oracle_lcg_ff(s, n)


def lcg_step(s):
    return lib().oracle_lcg_step(s)


def lcg_double(s):
    st = ctypes.c_uint64(s)
    d = lib().oracle_lcg_double(ctypes.byref(st))
    return d, st.value


def pick_mat(s):
    st = ctypes.c_uint64(s)
    m = lib().oracle_pick_mat(ctypes.byref(st))
    return m, st.value


def grid_search(A, q, lo, hi):
    A = np.ascontiguousarray(A, dtype=np.float64)
    return lib().oracle_grid_search(_ptr(A), q, lo, hi)


class XsTiny:
    """Tiny XS nuclide grid + acceleration structure built by the oracle."""

    def __init__(self, n_iso, n_gp, grid, bins=16, gseed=42):
        L = lib()
        self.n_iso, self.n_gp, self.grid, self.bins = n_iso, n_gp, grid, bins
        self.h = L.oracle_xs_build(n_iso, n_gp, grid, bins, gseed)
        self.energies = np.zeros(n_iso * n_gp)
        L.oracle_xs_energies(self.h, _ptr(self.energies))
        self.energies = self.energies.reshape(n_iso, n_gp)
        self.union = np.zeros(n_iso * n_gp) if grid == 0 else None
        if grid == 0:
            L.oracle_xs_union(self.h, _ptr(self.union))
        k = L.oracle_xs_index_len(self.h)
        self.index = np.zeros(k, dtype=np.int32)
        if k:
            L.oracle_xs_index(self.h, _ptr(self.index))

    def bracket(self, nuc, p):
        return lib().oracle_xs_bracket(self.h, nuc, p)

    def __del__(self):
        try:
            lib().oracle_xs_free(self.h)
        except Exception:
            pass


def xs_materials(n_iso):
    num = np.zeros(12, dtype=np.int32)
    mx = np.zeros(1, dtype=np.int32)
    k = lib().oracle_xs_materials(n_iso, _ptr(num), None, _ptr(mx))
    mats = np.zeros(k, dtype=np.int32)
    lib().oracle_xs_materials(n_iso, _ptr(num), _ptr(mats), _ptr(mx))
    return num, mats.reshape(12, int(mx[0]))


def xs_set_conc_seed(s):
    lib().oracle_xs_set_conc_seed(s)


def rs_fast_w(z):
    wr, wi = ctypes.c_double(), ctypes.c_double()
    lib().oracle_rs_fast_w(z.real, z.imag, ctypes.byref(wr), ctypes.byref(wi))
    return complex(wr.value, wi.value)


def rs_trig(kind, x):
    """RS-3's sin / cos / atan (kind 'sin' | 'cos' | 'atan'; reading R-rs-trig) at the points x."""
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.zeros_like(x)
    lib().oracle_rs_trig({"sin": 0, "cos": 1, "atan": 2}[kind], x.size, _ptr(x), _ptr(y))
    return y


def rs_tables(small, avg_poles, avg_windows, iseed=42):
    n_nuc = 68 if small else 355
    npol = np.zeros(n_nuc, dtype=np.int32)
    nwin = np.zeros(n_nuc, dtype=np.int32)
    cap = avg_windows * n_nuc + 16
    ws = np.zeros(cap, dtype=np.int32)
    we = np.zeros(cap, dtype=np.int32)
    k = lib().oracle_rs_tables(1 if small else 0, avg_poles, avg_windows, iseed, _ptr(npol), _ptr(nwin),
                               _ptr(ws), _ptr(we), cap)
    assert k >= 0
    return npol, nwin, ws[:k], we[:k]


def rs_micro(small, avg_poles, avg_windows, doppler, nucs, Es, iseed=42):
    """RS-3 micro xs (sigT, sigA, sigF, sigE) at (nucs[k], Es[k]) and the tables
    (poles: n x 9 = EA, RT, RA, RF as (re, im), l; windows: m x 3 = T, A, F;
    K0RS: n_nuc x 4), all from one RS-2 init."""
    n_nuc = 68 if small else 355
    nucs = np.ascontiguousarray(nucs, dtype=np.int32)
    Es = np.ascontiguousarray(Es, dtype=np.float64)
    micro = np.zeros((len(nucs), 4))
    poles = np.zeros((avg_poles * n_nuc, 9))
    wins = np.zeros((avg_windows * n_nuc, 3))
    k0 = np.zeros((n_nuc, 4))
    rc = lib().oracle_rs_micro(1 if small else 0, avg_poles, avg_windows, iseed, doppler, len(nucs), _ptr(nucs),
                               _ptr(Es), _ptr(micro), _ptr(poles), poles.size, _ptr(wins), wins.size, _ptr(k0),
                               k0.size)
    assert rc == 0
    return micro, poles, wins, k0


def amg_csr(nx, ny, nz):
    n = nx * ny * nz
    nnz = lib().oracle_amg_nnz(nx, ny, nz)
    rp = np.zeros(n + 1, dtype=np.int32)
    col = np.zeros(nnz, dtype=np.int32)
    val = np.zeros(nnz, dtype=np.float64)
    lib().oracle_amg_csr(nx, ny, nz, _ptr(rp), _ptr(col), _ptr(val))
    return rp, col, val


def amg_sweeps(nx, ny, nz, iters, u):
    u = np.array(u, dtype=np.float64, copy=True)
    lib().oracle_amg_sweeps(nx, ny, nz, iters, _ptr(u))
    return u


def pr_graph(n, avg, gseed=42):
    """PR-2 graph: out-degrees, in-edge CSR (ptr, src) in (source, edge) order."""
    e = lib().oracle_pr_graph(n, avg, gseed, None, None, None)
    deg = np.zeros(n, dtype=np.int64)
    ptr = np.zeros(n + 1, dtype=np.int64)
    src = np.zeros(max(e, 1), dtype=np.int64)
    lib().oracle_pr_graph(n, avg, gseed, _ptr(deg), _ptr(ptr), _ptr(src))
    return deg, ptr, src[:e]


def amg_apply(nx, ny, nz, u):
    u = np.ascontiguousarray(u, dtype=np.float64)
    y = np.zeros_like(u)
    lib().oracle_amg_apply(nx, ny, nz, _ptr(u), _ptr(y))
    return y
