#!/bin/bash
# kernel timings (stf_bench_kernel): GEMM variants, SYRK, TRSM/POTRF dataflow vs recursive
for v in 8 16; do
  for s in "0 8192 8192 1024" "0 1024 1024 1024" "0 16384 16384 1024" "1 1024 1024 1024"; do
    echo -n "warps=$v kind/shape=$s : "; STF_GEMM_WARPS=$v python tools/prof_kernel.py $s 10
  done
done
for df in 1 0; do
  for s in "2 1024 1024 0" "3 1024 1024 0" "2 512 512 0" "3 512 512 0" "3 2048 2048 0"; do
    echo -n "dataflow=$df kind/shape=$s : "; STF_DATAFLOW=$df python tools/prof_kernel.py $s 5
  done
done
