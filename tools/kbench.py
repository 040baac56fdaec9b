"""Kernels alone (stf_bench_kernel, CUDA events on the launching stream): the
critical-chain kernels and the GEMM tile at a tile size, plus small full
factorisations (n = 8192 / 16384).  usage: python tools/kbench.py [nb]"""
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_augonnetasg24_b200 as stf  # noqa: E402
from paper_conf_sc_augonnetasg24_b200 import _abi  # noqa: E402

nb = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
for kv in filter(None, os.environ.get("KB_OPT", "").split(",")):  # e.g. KB_OPT=trsm_res_split=4
    k, v = kv.split("=")
    stf.set_option(k, int(v))
PEAK = 37.09
out = {}
for name, kind, M, N, K in (("gemm_tile", 0, nb, nb, nb), ("syrk_tile", 1, nb, nb, nb), ("trsm_tile", 2, nb, nb, 0),
                            ("potrf_tile", 3, nb, nb, nb)):
    ms = ctypes.c_double()
    rc = _abi.stf_bench_kernel(kind, M, N, K, 20, ctypes.byref(ms))
    fl = {0: 2.0 * M * N * K, 1: 1.0 * M * M * K, 2: 1.0 * M * N * N, 3: M ** 3 / 3.0}[kind]
    out[name] = {"us": round(ms.value * 1e3, 1), "tflops": round(fl / (ms.value * 1e-3) / 1e12, 2), "rc": rc}
print(json.dumps(out), flush=True)
if os.environ.get("KB_FULL", "1") == "1":
    stf.init(1, [0])
    for kv in filter(None, os.environ.get("KB_OPT", "").split(",")):
        k, v = kv.split("=")
        stf.set_option(k, int(v))
    for n, b in ((8192, 1024), (8192, 512), (16384, 1024), (32768, 1024)):
        M = stf.TiledMatrix(n, b)
        ts = []
        for it in range(4):
            M.fill_spd(1)
            assert M.potrf() == 0
            ts.append(stf.last_stats()["device_ms"])
        t = min(ts[1:])
        print(json.dumps({"n": n, "nb": b, "ms": round(t, 3), "tflops": round(n ** 3 / 3 / t / 1e9, 2),
                          "frac": round(n ** 3 / 3 / t / 1e9 / PEAK, 4)}), flush=True)
        del M
    stf.finalize()
