#!/bin/bash
# ncu launch list of the bench's timed step (NVTX range "bench_step": every kernel of one
# factorisation, serialised, cold cache) + summary by kernel.
# usage (under gpurun): bash tools/launchlist.sh [bench args]
mkdir -p gpurun_out
ncu --nvtx --nvtx-include "bench_step/" --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-check "$@" > gpurun_out/launches_bench.json 2> gpurun_out/launches_bench.err
echo "ncu rc=$?"
python tools/summarize_launches.py gpurun_out/launches.csv > gpurun_out/launches_summary.txt
cat gpurun_out/launches_summary.txt
gzip -kf gpurun_out/launches.csv
