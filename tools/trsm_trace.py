"""Timeline of the resident-panel TRSM kernel (CTA 0), one launch.
usage: python tools/trsm_trace.py [M] [n]"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_augonnetasg24_b200 import _abi  # noqa: E402

M = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
g = torch.Generator().manual_seed(0)
L = torch.tril(torch.randn(n, n, generator=g, dtype=torch.float64)) * 0.1 + torch.diag(1 + torch.rand(n, generator=g, dtype=torch.float64))
B = torch.randn(n, M, generator=g, dtype=torch.float64)  # column-major M x n == row-major n x M
dL = L.t().contiguous().cuda()  # column-major L
T = n // 64
for rep in range(3):
    dB = B.clone().cuda()
    tr = (ctypes.c_int64 * (6 * T))()
    cnt = _abi.stf_debug_trsm_trace(M, n, dL.data_ptr(), n, dB.data_ptr(), M, tr, 6 * T)
    assert cnt > 0, _abi.stf_last_error()
t0 = tr[0]
print("kb  mma_start  wait_solved  solved  ready  solve_start  solve_end   (us from start)")
for kb in range(T):
    ev = [tr[5 * kb + e] for e in range(5)] + [tr[5 * T + kb]]
    print("%2d " % kb + " ".join("%10.2f" % ((x - t0) / 1e3) if x else "%10s" % "-" for x in ev))
