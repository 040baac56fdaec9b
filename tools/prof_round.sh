#!/bin/bash
# ncu --set full of each tile kernel (one warm launch each) + whole-graph DRAM traffic at the bench size.
mkdir -p gpurun_out
prof() {  # name regex kind M N K [env]
  env $7 timeout 600 ncu --set full --clock-control none --import-source on -k regex:$2 -s 1 -c 1 -f \
    -o gpurun_out/prof_$1 python tools/prof_kernel.py $3 $4 $5 $6 1 > gpurun_out/prof_$1.log 2>&1
  echo "$1 rc=$?"
}
prof gemm_tile gemm_nt 0 1024 1024 1024
prof gemm_full gemm_nt 0 8192 8192 1024
prof syrk_tile gemm_nt 1 1024 1024 1024
prof trsm_res_tile trsm_res 2 1024 1024 0
prof trsm_panel_tile trsm_panel 2 1024 1024 0 "STF_TRSM=2 STF_TRSM_ROWS=128"
prof trsm_w256 trsm_panel 2 1024 256 0 "STF_TRSM=2 STF_TRSM_ROWS=128"
prof potrf_tile dataflow 3 1024 1024 0
timeout 900 ncu --graph-profiling graph --nvtx --nvtx-include "stf_potrf/" --clock-control none \
  --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed \
  --csv --log-file gpurun_out/graph_traffic.csv python tools/graph_traffic.py ${1:-32768} ${2:-1024} > gpurun_out/graph_traffic.log 2>&1
echo "graph rc=$?"
tail -3 gpurun_out/graph_traffic.log; cat gpurun_out/graph_traffic.csv | tail -8
