"""Launch one tile kernel via stf_bench_kernel (for ncu captures).
usage: python tools/prof_kernel.py KIND M N K REPS"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_augonnetasg24_b200 import _abi  # noqa: E402

kind, M, N, K, reps = (int(x) for x in sys.argv[1:6])
import os
if os.environ.get("STF_DATAFLOW") == "0":
    _abi.stf_set_option(b"dataflow", 0)
if os.environ.get("STF_TRSM"):
    _abi.stf_set_option(b"trsm", int(os.environ["STF_TRSM"]))
ms = ctypes.c_double()
rc = _abi.stf_bench_kernel(kind, M, N, K, reps, ctypes.byref(ms))
print("rc", rc, "avg_ms", ms.value, _abi.stf_last_error())
