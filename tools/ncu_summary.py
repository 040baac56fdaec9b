"""Summarise an ncu report (one or more launches) into the JSON kept under profiles/.

usage: python tools/ncu_summary.py REPORT.ncu-rep [LABEL]
Prints per launch: duration, tensor/fp64 pipe activity, DRAM bytes, registers,
grid, shared memory, warp stalls per issue, and the instructions carrying the
largest share of stall samples (source page; needs -lineinfo builds).
"""
import csv
import io
import json
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "lts__t_bytes.sum",
    "launch__registers_per_thread",
    "launch__grid_size",
    "launch__block_size",
    "launch__shared_mem_per_block_dynamic",
    "launch__occupancy_limit_registers",
    "smsp__inst_executed.sum",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
]
STALL = "smsp__average_warps_issue_stalled_"


def ncu(args):
    return subprocess.run(["ncu"] + args, capture_output=True, text=True, check=True).stdout


def rows(text):
    lines = [l for l in text.splitlines() if l.startswith('"')]
    return list(csv.reader(io.StringIO("\n".join(lines))))


def raw(rep):
    r = rows(ncu(["-i", rep, "--page", "raw", "--csv"]))
    head, units, data = r[0], r[1], r[2:]
    out = []
    for d in data:
        rec = {"kernel": d[head.index("Kernel Name")][:120]}
        for k in KEYS:
            if k in head:
                i = head.index(k)
                rec[k] = (d[i] + " " + units[i]).strip()
        st = {}
        for i, h in enumerate(head):
            if h.startswith(STALL) and h.endswith("_per_issue_active.ratio"):
                name = h[len(STALL):-len("_per_issue_active.ratio")]
                try:
                    v = float(d[i].replace(",", ""))
                except ValueError:
                    continue
                if v >= 0.1:
                    st[name] = round(v, 3)
        rec["stalls_per_issue"] = dict(sorted(st.items(), key=lambda kv: -kv[1]))
        out.append(rec)
    return out


def sass_top(rep, n=10):
    try:
        txt = ncu(["-i", rep, "--page", "source", "--csv", "--print-source", "sass"])
    except subprocess.CalledProcessError:
        return []
    r = rows(txt)
    r = r[[i for i, x in enumerate(r) if x and x[0] == "Address"][0]:] if any(x and x[0] == "Address" for x in r) else []
    if not r:
        return []
    head = r[0]
    try:
        si = head.index("Source")
        wi = [i for i, h in enumerate(head) if h.startswith("Warp Stall Sampling (All")][0]
    except (ValueError, IndexError):
        return []
    acc = {}
    tot = 0.0
    for d in r[1:]:
        try:
            v = float(d[wi])
        except (ValueError, IndexError):
            continue
        op = d[si].strip().split(" ")[0] if d[si].strip() else "?"
        if op.startswith("@"):
            op = d[si].strip().split(" ")[1]
        acc[op] = acc.get(op, 0.0) + v
        tot += v
    if tot == 0:
        return []
    return [[k, round(100 * v / tot, 1)] for k, v in sorted(acc.items(), key=lambda kv: -kv[1])[:n]]


if __name__ == "__main__":
    rep = sys.argv[1]
    label = sys.argv[2] if len(sys.argv) > 2 else rep
    recs = raw(rep)
    top = sass_top(rep)
    for r in recs:
        r["sass_stall_share_top"] = top
    print("==", label)
    print(json.dumps(recs if len(recs) > 1 else recs[0], indent=1))


def line_top(rep, n=15):
    """CUDA source lines carrying the largest share of warp stall samples."""
    try:
        txt = ncu(["-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"])
    except subprocess.CalledProcessError:
        return []
    out, fname, wi, tot = [], "", None, 0.0
    for row in csv.reader(io.StringIO(txt)):
        if not row:
            continue
        if row[0] == "File Path":
            fname = row[1].split("/")[-1]
        elif row[0] == "Line No":
            wi = [i for i, h in enumerate(row) if h.startswith("Warp Stall Sampling (All")][0]
        elif wi is not None and row[0].isdigit():
            try:
                v = float(row[wi])
            except (ValueError, IndexError):
                continue
            if v > 0:
                out.append((v, "%s:%s" % (fname, row[0]), row[1].strip()[:80]))
                tot += v
    out.sort(key=lambda x: -x[0])
    return [[loc, round(100 * v / tot, 1), src] for v, loc, src in out[:n]] if tot else []


if __name__ == "__main__" and "--lines" in sys.argv:
    for r in line_top(sys.argv[1]):
        print(r)
