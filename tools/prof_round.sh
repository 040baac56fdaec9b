#!/bin/bash
# ncu --set full of each tile kernel (one warm launch each) + whole-graph DRAM traffic at the bench sizes.
# usage (under gpurun): bash tools/prof_round.sh   -> gpurun_out/prof_*.ncu-rep, graph_traffic_*.csv, ncu_summaries.txt
mkdir -p gpurun_out
prof() {  # name regex skip count kind M N K
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$2 -s $3 -c $4 -f \
    -o gpurun_out/prof_$1 python tools/prof_kernel.py $5 $6 $7 $8 1 > gpurun_out/prof_$1.log 2>&1
  echo "$1 rc=$?"
}
prof gemm_tile gemm_nt 1 1 0 1024 1024 1024
prof gemm_full gemm_nt 1 1 0 8192 8192 1024
prof syrk_tile gemm_nt 1 1 1 1024 1024 1024
prof trsm_tile "trsm_res|gemm_nt" 3 3 2 1024 1024 0
prof potrf_tile "dataflow|bulk" 2 2 3 1024 1024 0
for cfg in "65536 1024" "32768 1024"; do
  set -- $cfg
  timeout 1500 ncu --graph-profiling graph --nvtx --nvtx-include "stf_potrf/" --clock-control none \
    --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed \
    --csv --log-file gpurun_out/graph_traffic_n$1.csv python tools/graph_traffic.py $1 $2 > gpurun_out/graph_traffic_n$1.log 2>&1
  echo "graph n=$1 rc=$?"
  tail -4 gpurun_out/graph_traffic_n$1.csv
done
for r in gemm_tile gemm_full syrk_tile trsm_tile potrf_tile; do
  echo "== $r"; python tools/ncu_summary.py gpurun_out/prof_$r.ncu-rep $r 2>&1 | head -60
done > gpurun_out/ncu_summaries.txt
echo done
