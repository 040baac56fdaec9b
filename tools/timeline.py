"""Task timeline of one stf_potrf (STF_DEBUG_TRACE=1): per-kind busy time, the
start of the first / end of the last task of each kind, and a coarse profile of
how many compute tasks were running in each time bin.
usage: STF_DEBUG_TRACE=1 python tools/timeline.py N NB [host] [bins]"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["STF_DEBUG_TRACE"] = "1"
import torch  # noqa: E402

import paper_conf_sc_augonnetasg24_b200 as stf  # noqa: E402
from paper_conf_sc_augonnetasg24_b200 import _abi  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
host = len(sys.argv) > 3 and sys.argv[3] == "host"
bins = int(sys.argv[4]) if len(sys.argv) > 4 else 40
stf.init(1, [0])
if host:
    A = torch.empty((n, n), dtype=torch.float64, pin_memory=True)
    dev = torch.empty((n, n), dtype=torch.float64, device="cuda:0")
    for it in range(2):
        assert _abi.stf_fill_spd_block(dev.data_ptr(), n, n, 0, 0, n, n, 1) == 0
        A.copy_(dev)
        torch.cuda.synchronize()
        assert stf.potrf_colmajor(A.data_ptr(), n, n, nb, "L", None, 1) == 0
else:
    M = stf.TiledMatrix(n, nb, 1, 1, devices=[0])
    for it in range(2):
        M.fill_spd(1)
        assert M.potrf() == 0
ms = stf.last_stats()["device_ms"]
cnt = _abi.stf_debug_last_trace(None, 0)
buf = (ctypes.c_int64 * (7 * cnt))()
_abi.stf_debug_last_trace(buf, cnt)
R = np.frombuffer(buf, dtype=np.int64).reshape(cnt, 7)
t0 = R[R[:, 5] >= 0, 5].min()
R = R.copy()
R[:, 5:] -= t0
names = ["POTRF", "TRSM", "SYRK", "GEMM", "COPY", "LOAD", "STORE", "FENCE"]
print("n=%d nb=%d %s: device %.1f ms, traced span %.1f ms, %d tasks" % (n, nb, "HOST" if host else "TILED", ms,
                                                                         R[:, 6].max() / 1e6, cnt))
for k, nm in enumerate(names):
    sel = R[R[:, 0] == k]
    if len(sel):
        d = (sel[:, 6] - sel[:, 5]) / 1e3
        print("%-6s %5d tasks  first start %8.2f ms  last end %8.2f ms  mean %8.1f us  sum %9.1f ms" % (
            nm, len(sel), sel[:, 5].min() / 1e6, sel[:, 6].max() / 1e6, d.mean(), d.sum() / 1e3))
# critical panel: end of POTRF(k)
po = R[R[:, 0] == 0]
print("POTRF(k) end ms:", " ".join("%d:%.1f" % (r[3], r[6] / 1e6) for r in po[:: max(1, len(po) // 16)]))
if host:
    ld = R[R[:, 0] == 5]
    print("LOAD end ms by column:", " ".join("%d:%.1f" % (j, ld[ld[:, 2] == j][:, 6].max() / 1e6)
                                            for j in range(0, n // nb, max(1, n // nb // 16))))
# the critical chain POTRF(k) -> TRSM(k+1,k) -> SYRK(k+1,k) -> POTRF(k+1): start / end (ms)
if n // nb <= 32:
    def find(kind, i, j, k):
        sel = R[(R[:, 0] == kind) & (R[:, 1] == i) & (R[:, 2] == j) & (R[:, 3] == k)]
        return (sel[0, 5] / 1e6, sel[0, 6] / 1e6) if len(sel) else (float("nan"),) * 2
    for k in range(min(n // nb, 12)):
        p_ = find(0, k, k, k)
        t_ = find(1, k + 1, k, k)
        s_ = find(2, k + 1, k + 1, k)
        g_ = find(3, k + 1, k, k - 1)
        print("k=%2d POTRF %.3f-%.3f  TRSM(k+1) %.3f-%.3f  SYRK(k+1) %.3f-%.3f  GEMM(k+1,k,k-1) %.3f-%.3f" % (
            k, *p_, *t_, *s_, *g_))
# flop-weighted activity profile: GEMM/SYRK/TRSM flops completed per bin (task flops spread over its span)
span = R[:, 6].max()
edges = np.linspace(0, span, bins + 1)
fl = np.zeros(bins)
w = {0: nb ** 3 / 3, 1: nb ** 3, 2: nb ** 3, 3: 2 * nb ** 3}
for r in R:
    if r[0] in w and r[6] > r[5]:
        a, b = r[5], r[6]
        lo, hi = np.searchsorted(edges, a, "right") - 1, np.searchsorted(edges, b, "right") - 1
        for bi in range(max(lo, 0), min(hi, bins - 1) + 1):
            ov = min(b, edges[bi + 1]) - max(a, edges[bi])
            if ov > 0:
                fl[bi] += w[r[0]] * ov / (b - a)
tf = fl / ((edges[1] - edges[0]) * 1e-9) / 1e12
print("TFLOP/s per %.1f ms bin:" % ((edges[1] - edges[0]) / 1e6), " ".join("%.1f" % x for x in tf))
stf.finalize()
