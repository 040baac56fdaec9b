#!/bin/bash
# Whole-graph DRAM traffic / tensor-pipe activity of one timed factorisation (under gpurun).
mkdir -p gpurun_out
for cfg in "$@"; do
  set -- $(echo $cfg | tr ':' ' ')
  timeout 1500 ncu --graph-profiling graph --nvtx --nvtx-include "stf_potrf/" --clock-control none \
    --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed \
    --csv --log-file gpurun_out/graph_traffic_n$1.csv python tools/graph_traffic.py $1 $2 > gpurun_out/graph_traffic_n$1.log 2>&1
  echo "graph n=$1 rc=$?"
done
