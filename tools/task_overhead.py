"""Table I-style scheduler cost of our STF runtime: per task,
(a) host plan build (DAG by the STF rule + placement + stream assignment +
events + graph capture and instantiation) on a cold call, (b) device time of the
whole-DAG graph with every kernel skipped (debug_skip: dependencies, event and
empty-node overhead only), (c) host submission of the eager backend (graph=0)
with every kernel skipped.  usage: python tools/task_overhead.py"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_augonnetasg24_b200 as stf  # noqa: E402

SKIP_ALL = 0x1F  # potrf, trsm, syrk, gemm, copy
res = []
stf.init(1, [0])
for n, nb in ((8192, 256), (32768, 1024), (65536, 1024)):
    M = stf.TiledMatrix(n, nb)
    M.fill_spd(1)
    row = {"n": n, "nb": nb}
    for graph in (1, 0):
        stf.set_option("graph", graph)
        stf.set_option("debug_skip", SKIP_ALL)
        t0 = time.perf_counter()
        M.potrf()
        cold = (time.perf_counter() - t0) * 1e3
        st = stf.last_stats()
        walls, devs = [], []
        for _ in range(5):
            t0 = time.perf_counter()
            M.potrf()
            walls.append((time.perf_counter() - t0) * 1e3)
            devs.append(stf.last_stats()["device_ms"])
        tasks = st["dag_tasks"]
        key = "graph" if graph else "eager"
        row[key] = {"dag_tasks": tasks, "build_ms": round(st["build_ms"], 2), "cold_call_ms": round(cold, 2),
                    "build_us_per_task": round(1e3 * st["build_ms"] / tasks, 3),
                    "empty_device_us_per_task": round(1e3 * min(devs) / tasks, 3),
                    "empty_wall_us_per_task": round(1e3 * min(walls) / tasks, 3)}
        stf.set_option("debug_skip", 0)
    stf.set_option("graph", 1)
    del M
    res.append(row)
    print(json.dumps(row), flush=True)
stf.finalize()
