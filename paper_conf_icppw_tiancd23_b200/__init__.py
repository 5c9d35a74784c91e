"""B200-native ensemble execution (Tian, Chapman, Doerfert, ICPP-W 2023).

N independent invocations of a CPU-style application, each with its own
command line, run as the thread blocks of one sm_100a kernel launch.  The
product is libens.so (C ABI, include/ens.h); this package is its thin binding
(_ens), the torch-plumbed single-GPU front end (ensemble) and the
one-process-per-GPU sharding + NCCL all-gather (dist).
"""
from ._ens import (APP_IDS, ENS_APP_AMGMK, ENS_APP_BY_ARGV0, ENS_APP_ECHO, ENS_APP_RSBENCH, ENS_APP_XSBENCH,
                   ENS_RF_DONE, ENS_RF_NOMEM, ENS_RF_NOT_RUN, ENS_RF_STDOUT_TRUNC, ENS_TALLIES, RECORD_DTYPE, Args,
                   EnsError, Run, format_stdout, make_cfg, version, workspace_bytes)

__all__ = ["APP_IDS", "ENS_APP_AMGMK", "ENS_APP_BY_ARGV0", "ENS_APP_ECHO", "ENS_APP_RSBENCH", "ENS_APP_XSBENCH",
           "ENS_RF_DONE", "ENS_RF_NOMEM", "ENS_RF_NOT_RUN", "ENS_RF_STDOUT_TRUNC", "ENS_TALLIES", "RECORD_DTYPE",
           "Args", "EnsError", "Run", "format_stdout", "make_cfg", "version", "workspace_bytes"]
