"""NEXT-1 ablations on our own path, reproducing the
paper's only Cholesky claims as B200 measurements:
stream pool vs one stream, look-ahead vs a per-step fence, graph vs eager
lowering, plus our own kernel variants.  Runs bench.py once per variant (a
fresh process, so environment options apply at init) and prints a table and
one JSON object.

usage: python tools/ablations.py [--n 32768 --nb 1024] [--steps 2 --warmup 1]
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

VARIANTS = [
    ("default (pool 4 crit + 8 bulk streams, graded priorities, graph, look-ahead)", {}),
    ("single stream (STF_SERIAL=1)  [paper: -5% on 1 GPU]", {"STF_SERIAL": "1"}),
    ("2 bulk streams", {"STF_STREAMS": "2"}),
    ("16 bulk streams", {"STF_STREAMS": "16"}),
    ("no priorities (STF_PRIO=0)", {"STF_PRIO": "0"}),
    ("no look-ahead: fence per panel step (STF_LOOKAHEAD=0)", {"STF_LOOKAHEAD": "0"}),
    ("eager streams+events, no graph (STF_GRAPH=0)", {"STF_GRAPH": "0"}),
    ("TRSM dataflow kernel (STF_TRSM=1)", {"STF_TRSM": "1"}),
    ("TRSM one panel launch, no GEMM split (STF_TRSM_SPLIT=1)", {"STF_TRSM_SPLIT": "1"}),
    ("TRSM split in 2 column blocks (STF_TRSM_SPLIT=2)", {"STF_TRSM_SPLIT": "2"}),
    ("TRSM split in 8 column blocks (STF_TRSM_SPLIT=8)", {"STF_TRSM_SPLIT": "8"}),
    ("TRSM row panel 32 rows (STF_TRSM_ROWS=32)", {"STF_TRSM_ROWS": "32"}),
    ("TRSM + POTRF recursive (STF_TRSM=0 STF_DATAFLOW=0)", {"STF_TRSM": "0", "STF_DATAFLOW": "0"}),
    ("GEMM 16 warps 32x32 (STF_GEMM_WARPS=16)", {"STF_GEMM_WARPS": "16"}),
    ("GEMM BK=16 x 4 stages (STF_GEMM_BK=16)", {"STF_GEMM_BK": "16"}),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=32768)
    ap.add_argument("--nb", type=int, default=1024)
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--warmup", type=int, default=1)
    ap.add_argument("--only", default="", help="comma-separated variant indices")
    a = ap.parse_args()
    only = {int(x) for x in a.only.split(",") if x}
    out = []
    base = None
    for idx, (name, env) in enumerate(VARIANTS):
        if only and idx not in only:
            continue
        e = dict(os.environ)
        e.update(env)
        cmd = [sys.executable, "bench.py", "--n", str(a.n), "--nb", str(a.nb), "--steps", str(a.steps),
               "--warmup", str(a.warmup), "--no-e2e", "--no-cpu"]
        r = subprocess.run(cmd, cwd=ROOT, env=e, capture_output=True, text=True, timeout=1200)
        line = [l for l in r.stdout.splitlines() if l.startswith("{")]
        if r.returncode != 0 or not line:
            out.append({"variant": name, "env": env, "error": r.stderr[-400:]})
            print("%-70s  FAILED" % name, flush=True)
            continue
        d = json.loads(line[-1])
        v = d["value"]
        base = base if base is not None else v
        out.append({"variant": name, "env": env, "gflops": v, "ms_per_step": d["ms_per_step"],
                    "frac_of_peak": d["roofline"]["frac"], "vs_default": round(v / base - 1, 4)})
        print("%-70s %10.1f GFLOP/s  %8.2f ms  %+6.1f%%" % (name, v, d["ms_per_step"], 100 * (v / base - 1)),
              flush=True)
    print(json.dumps({"n": a.n, "nb": a.nb, "results": out}))


if __name__ == "__main__":
    main()
