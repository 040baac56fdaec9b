"""NEXT-1 ablations on our own path, reproducing the
paper's Cholesky claims as B200 measurements:
  * stream pool vs "1 compute + 1 copy stream" vs a single stream;
  * look-ahead (pure STF DAG) vs a fence per panel step;
  * 2D block-cyclic vs 1D column block-cyclic + fence, the paper's explanation of
    cuSolverMg's gap, on 8 virtual GPU slots of one B200 (the
    distribution, replica copies and scheduling run; the NVLink hop does not);
  * graph vs eager lowering; COPY tasks vs fused push.
Runs bench.py once per variant (fresh process; options from the environment at
init) and prints a table and one JSON object.  Every variant's result is
checked bit-exact against the closed form by tests/test_gpu_potrf.py
(test_schedule_variants_p2_exact, test_virtual_grids_p2_exact).

usage: python tools/ablations.py [--n 32768 --nb 1024] [--steps 3 --warmup 2] [--only 0,3]
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

ONE = []  # 1 GPU slot
VIRT = ["--gpus", "8", "--virtual-slots", "1"]
VARIANTS = [
    ("1 GPU: default (6 high-priority + 32 bulk + 2 copy streams, graph, look-ahead)", {}, ONE),
    ("1 GPU: 1 compute + 1 copy stream (stream_pool=1)  [paper: pool +5% on 1 GPU]", {"STF_STREAM_POOL": "1"}, ONE),
    ("1 GPU: single stream for everything (stream_pool=2)", {"STF_STREAM_POOL": "2"}, ONE),
    ("1 GPU: 2 bulk streams", {"STF_STREAMS": "2"}, ONE),
    ("1 GPU: no priorities (priority=0)", {"STF_PRIO": "0"}, ONE),
    ("1 GPU: no look-ahead, fence per panel step (lookahead=0)", {"STF_LOOKAHEAD": "0"}, ONE),
    ("1 GPU: eager streams + events, no graph (graph=0)", {"STF_GRAPH": "0"}, ONE),
    ("1 GPU: panel chain with full-completion edges (pdl=0)", {"STF_PDL": "0"}, ONE),
    ("1 GPU: POTRF tile as one launch (potrf_split=0)", {"STF_POTRF_SPLIT": "0"}, ONE),
    ("8 virtual slots: 2D block-cyclic 2x4 (default)", {}, VIRT + ["--grid", "2x4"]),
    ("8 virtual slots: 1D column block-cyclic 1x8", {}, VIRT + ["--grid", "1x8"]),
    ("8 virtual slots: 1D column block-cyclic 1x8 + fence per step (cuSolverMg model)", {"STF_LOOKAHEAD": "0"},
     VIRT + ["--grid", "1x8"]),
    ("8 virtual slots: 2D 2x4 + fence per step", {"STF_LOOKAHEAD": "0"}, VIRT + ["--grid", "2x4"]),
    ("8 virtual slots: 2D 2x4, 1 compute + 1 copy stream per slot", {"STF_STREAM_POOL": "1"}, VIRT + ["--grid", "2x4"]),
    ("8 virtual slots: 2D 2x4, fused push (push=1)", {"STF_PUSH": "1"}, VIRT + ["--grid", "2x4"]),
    ("8 virtual slots: 2D 2x4, eager (graph=0)", {"STF_GRAPH": "0"}, VIRT + ["--grid", "2x4"]),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=32768)
    ap.add_argument("--nb", type=int, default=1024)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--only", default="", help="comma-separated variant indices")
    a = ap.parse_args()
    only = {int(x) for x in a.only.split(",") if x}
    out = []
    base = {}
    for idx, (name, env, extra) in enumerate(VARIANTS):
        if only and idx not in only:
            continue
        e = dict(os.environ)
        e.update(env)
        cmd = [sys.executable, "bench.py", "--n", str(a.n), "--nb", str(a.nb), "--steps", str(a.steps),
               "--warmup", str(a.warmup), "--no-e2e", "--no-cpu", "--no-check"] + extra
        r = subprocess.run(cmd, cwd=ROOT, env=e, capture_output=True, text=True, timeout=1800)
        line = [l for l in r.stdout.splitlines() if l.startswith("{")]
        if r.returncode != 0 or not line:
            out.append({"variant": name, "env": env, "args": extra, "error": r.stderr[-400:]})
            print("%-86s  FAILED %s" % (name, r.stderr[-300:]), flush=True)
            continue
        d = json.loads(line[-1])
        v = d["value"]
        key = "virt" if extra else "one"
        base.setdefault(key, v)
        out.append({"variant": name, "env": env, "args": extra, "gflops": v, "ms_per_step": d["ms_per_step"],
                    "step_ms": d["step_ms"], "graph": d["config"]["graph"], "plan": d["plan"],
                    "vs_first_of_group": round(v / base[key] - 1, 4)})
        print("%-86s %10.1f GFLOP/s  %8.2f ms  %+6.1f%%" % (name, v, d["ms_per_step"], 100 * (v / base[key] - 1)),
              flush=True)
    print(json.dumps({"n": a.n, "nb": a.nb, "results": out}))


if __name__ == "__main__":
    main()
