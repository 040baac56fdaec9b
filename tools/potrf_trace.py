"""Timeline of the dataflow POTRF tile kernel (stf_debug_potrf_trace): critical
chain phases per 64-block step and bulk task occupancy.  usage: potrf_trace.py n ctas"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_augonnetasg24_b200 import _abi  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
ctas = int(sys.argv[2]) if len(sys.argv) > 2 else 0
T = (n + 63) // 64
A = torch.zeros((n, n), dtype=torch.float64, device="cuda")
_abi.stf_fill_spd_block(A.data_ptr(), n, n, 0, 0, n, n, 1)
cap = 6 * T + 3 * T ** 3
tr = (ctypes.c_int64 * cap)()
for rep in range(3):  # warm-up then the measured one
    _abi.stf_fill_spd_block(A.data_ptr(), n, n, 0, 0, n, n, 1)
    cnt = _abi.stf_debug_potrf_trace(n, A.data_ptr(), n, ctas, tr, cap)
t = np.array(tr[:cnt], dtype=np.int64)
chain = t[:6 * T].reshape(T, 6)
bulk = t[6 * T:].reshape(-1, 3)
bulk = bulk[bulk[:, 0] > 0]
t0 = min(chain[0, 0], bulk[:, 0].min() if len(bulk) else chain[0, 0])
print("n=%d ctas=%d total %.1f us, bulk tasks %d" % (n, ctas, (max(chain.max(), bulk.max() if len(bulk) else 0) - t0) / 1e3, len(bulk)))
print("step  P_us  S_in_ready  S_done  U_wait_us  U_us   (chain CTA; times from the step's P start; P and S overlap)")
for kb in range(T):
    c = chain[kb]
    if c[1] <= 0:
        continue
    f = lambda e: (c[e] - c[0]) / 1e3 if c[e] > 0 else float("nan")
    if kb + 1 < T:
        print("%3d %6.1f %10.1f %7.1f %9.1f %6.1f" % (kb, f(1), f(2), f(3), (c[4] - max(c[1], c[3])) / 1e3,
                                                   (c[5] - c[4]) / 1e3))
    else:
        print("%3d %6.1f" % (kb, f(1)))
if len(bulk):
    w = (bulk[:, 1] - bulk[:, 0]) / 1e3
    d = (bulk[:, 2] - bulk[:, 1]) / 1e3
    print("bulk: wait mean %.1f us (max %.1f), run mean %.1f us (max %.1f), busy sum %.1f us" % (
        w.mean(), w.max(), d.mean(), d.max(), d.sum()))

# ---- the bulk tasks that feed the chain's S input X(kb+1, kb): S(kb+1, kb-1) and U(kb+1, kb, kb-1)
def tasks_order(T):  # replica of dataflow.cu build_tasks(potrf, crit) ticket order
    t = [("P", 0, 0, 0)] + [("S", i, 0, 0) for i in range(1, T)] + [("U", i, 1, 0) for i in range(1, T)]
    for kb in range(T - 1):
        t.append(("P", kb + 1, kb + 1, kb + 1))
        t += [("S", i, kb + 1, kb + 1) for i in range(kb + 2, T)]
        if kb + 2 < T:
            t += [("U", i, kb + 2, kb) for i in range(kb + 2, T)]
            t += [("U", i, kb + 2, kb + 1) for i in range(kb + 2, T)]
        t += [("U", i, j, kb) for j in range(kb + 3, T) for i in range(j, T)]

    def chain(x):
        ty, i, j, k = x
        return ty == "P" or (ty == "S" and i == k + 1) or (ty == "U" and i == k + 1 and j == k + 1)
    return [x for x in t if not chain(x)]


order = tasks_order(T)
raw = t[6 * T:].reshape(-1, 3)
pos = {x: n for n, x in enumerate(order)}
print("feeders of X(kb+1,kb) (us from the chain's P(kb-1) start): S(kb+1,kb-1) claim/ready/done, "
      "U(kb+1,kb,kb-1) claim/ready/done; chain S(kb,kb-1) done")
for kb in range(2, T - 1):
    s0 = chain[kb - 1, 0]
    a = pos.get(("S", kb + 1, kb - 1, kb - 1))
    b = pos.get(("U", kb + 1, kb, kb - 1))
    f = lambda x: "%6.1f" % ((x - s0) / 1e3) if x > 0 else "   nan"
    if a is None or b is None or a >= len(raw) or b >= len(raw):
        continue
    print("%3d  S: %s %s %s   U: %s %s %s   chainS: %s" % (kb, f(raw[a, 0]), f(raw[a, 1]), f(raw[a, 2]),
                                                       f(raw[b, 0]), f(raw[b, 1]), f(raw[b, 2]), f(chain[kb - 1, 3])))
