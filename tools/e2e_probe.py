"""Time stf_potrf on a pinned HOST_COLMAJOR matrix (the bench's e2e call) under
the current environment (STF_DEBUG_SKIP, STF_LOAD_ORDER, ...), device ms per call.
usage: python tools/e2e_probe.py [N] [NB] [REPS]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_augonnetasg24_b200 as stf  # noqa: E402
from paper_conf_sc_augonnetasg24_b200 import _abi  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
stf.init(1, [0])
A = torch.empty((n, n), dtype=torch.float64, pin_memory=True)
dev = torch.empty((n, n), dtype=torch.float64, device="cuda:0")
ms = []
for it in range(reps + 1):
    assert _abi.stf_fill_spd_block(dev.data_ptr(), n, n, 0, 0, n, n, 1) == 0
    A.copy_(dev)
    torch.cuda.synchronize()
    stf.potrf_colmajor(A.data_ptr(), n, n, nb, "L", None, 1)
    if it:
        ms.append(stf.last_stats()["device_ms"])
print("%s skip=%s: e2e device ms %s -> %.1f GFLOP/s" % (
    os.environ.get("TAG", ""), os.environ.get("STF_DEBUG_SKIP", "none"), ["%.1f" % x for x in ms],
    n ** 3 / 3 / (min(ms) * 1e-3) / 1e9))
stf.finalize()
