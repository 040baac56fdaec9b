"""Out-of-core (NEXT-4) measurement: stf_potrf on a pinned HOST column-major
matrix with a cap on device tile frames.  Reports GFLOP/s (n^3/3), the tiles
moved each way and the implied PCIe traffic against the in-core call.

usage: python tools/ooc_bench.py [n] [nb] [cap,cap,...] [reps]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_augonnetasg24_b200 as stf  # noqa: E402
from paper_conf_sc_augonnetasg24_b200 import _abi  # noqa: E402


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
    nb = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
    caps = [int(c) for c in sys.argv[3].split(",")] if len(sys.argv) > 3 else [0, 264, 132, 66, 33]
    reps = int(sys.argv[4]) if len(sys.argv) > 4 else 2
    T = n // nb
    NT = T * (T + 1) // 2
    stf.init(1)
    A = torch.empty((n, n), dtype=torch.float64, pin_memory=True)
    dev = torch.empty((n, n), dtype=torch.float64, device="cuda:0")
    tile_b = nb * nb * 8
    # PCIe roofline: pinned host <-> device copy bandwidth of this box (1 GiB, best of 3)
    h = torch.empty(1 << 27, dtype=torch.float64, pin_memory=True)
    d = torch.empty(1 << 27, dtype=torch.float64, device="cuda:0")
    bw = {}
    for name, (dst, src) in (("h2d", (d, h)), ("d2h", (h, d))):
        best = 1e9
        for _ in range(3):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            dst.copy_(src, non_blocking=True)
            e1.record()
            e1.synchronize()
            best = min(best, e0.elapsed_time(e1))
        bw[name] = (1 << 30) / (best * 1e-3) / 1e9
    del h, d
    print(json.dumps({"pcie_h2d_GBps": round(bw["h2d"], 1), "pcie_d2h_GBps": round(bw["d2h"], 1)}), flush=True)
    out = []
    for cap in caps:
        stf.set_option("mem_cap_tiles", cap)
        res = []
        for r in range(reps + 1):
            assert _abi.stf_fill_spd_block(dev.data_ptr(), n, n, 0, 0, n, n, 1) == 0
            A.copy_(dev)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            info = stf.potrf_colmajor(A.data_ptr(), n, n, nb, "L", None, 1)
            wall = time.perf_counter() - t0
            assert info == 0
            st = stf.last_stats()
            if r:
                res.append((st["device_ms"], wall * 1e3, st))
        ms = min(x[0] for x in res)
        st = res[-1][2]
        line = {"n": n, "nb": nb, "cap_tiles": cap, "frames": st["frames"], "tiles": NT,
                "device_GB": round((cap or NT) * tile_b / 1e9, 2),
                "gflops": round(n ** 3 / 3 / (ms * 1e-3) / 1e9, 1), "ms": round(ms, 2),
                "host_loads": st["host_loads"], "host_stores": st["host_stores"],
                "h2d_GB": round(st["host_loads"] * tile_b / 1e9, 2), "d2h_GB": round(st["host_stores"] * tile_b / 1e9, 2),
                "h2d_GBps_avg": round(st["host_loads"] * tile_b / (ms * 1e-3) / 1e9, 1),
                "pcie_bound_ms": round(max(st["host_loads"] * tile_b / bw["h2d"], st["host_stores"] * tile_b / bw["d2h"]) / 1e6, 1),
                "graph_nodes": st["graph_nodes"], "build_ms": round(res[0][2]["build_ms"], 1)}
        print(json.dumps(line), flush=True)
        out.append(line)
    stf.set_option("mem_cap_tiles", 0)
    stf.finalize()


if __name__ == "__main__":
    main()
