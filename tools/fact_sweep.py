"""Whole factorisations on device tiles under option variants (one process; the
plan memo is keyed on the options).  usage:
  fact_sweep.py "n:nb,n:nb" 'name=opt=v,opt=v;name=opt=v' [reps]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_augonnetasg24_b200 as stf  # noqa: E402

PEAK = 37.09
cfgs = [tuple(int(x) for x in c.split(":")) for c in sys.argv[1].split(",")]
variants = []
for v in sys.argv[2].split(";"):
    name, _, opts = v.partition("=")
    variants.append((name, [(kv.split("=")[0], int(kv.split("=")[1])) for kv in opts.split(",") if kv]))
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
stf.init(1, [0])
defaults = {}
for n, nb in cfgs:
    M = stf.TiledMatrix(n, nb)
    for name, opts in variants:
        for k, v in opts:
            if k not in defaults:
                defaults[k] = stf.get_option(k)
            stf.set_option(k, v)
        ts = []
        for it in range(reps + 1):
            M.fill_spd(1)
            info = M.potrf()
            ts.append(stf.last_stats()["device_ms"])
        t = min(ts[1:])
        print(json.dumps({"n": n, "nb": nb, "variant": name, "ms": round(t, 3), "tflops": round(n ** 3 / 3 / t / 1e9, 2),
                          "frac": round(n ** 3 / 3 / t / 1e9 / PEAK, 4), "info": info}), flush=True)
        for k, v in opts:
            stf.set_option(k, defaults[k])
    del M
stf.finalize()
