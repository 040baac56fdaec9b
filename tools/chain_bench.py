"""Critical-chain step POTRF(k) -> TRSM(k+1,k) -> SYRK(k+1,k) alone (stf_bench_kernel
kind 4: one stream, one graph, event nodes around the chain), with and without the
programmatic TRSM launch, over the POTRF's trigger lead.  usage: chain_bench.py [nb ...]"""
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_augonnetasg24_b200 as stf  # noqa: E402
from paper_conf_sc_augonnetasg24_b200 import _abi  # noqa: E402

stf.init(1, [0])
for nb in [int(a) for a in sys.argv[1:]] or [1024, 512]:
    nbk = nb // 64
    rows = []
    for pdl, lead in [(0, 0)] + [(1, ld) for ld in sorted({nbk, 12, 10, 8, 6, 4, 2, 0}) if ld <= nbk]:
        stf.set_option("pdl", pdl)
        stf.set_option("pdl_lead", lead)
        ms = ctypes.c_double()
        rc = _abi.stf_bench_kernel(4, nb, nb, nb, 20, ctypes.byref(ms))
        rows.append({"nb": nb, "pdl": pdl, "lead": lead, "us": round(ms.value * 1e3, 1), "rc": rc})
        print(json.dumps(rows[-1]), flush=True)
stf.finalize()
