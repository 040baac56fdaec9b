#!/bin/bash
# kernel timings (stf_bench_kernel): GEMM, SYRK, TRSM variants, POTRF variants
for s in "0 8192 8192 1024" "0 1024 1024 1024" "1 1024 1024 1024"; do
  echo -n "gemm kind/shape=$s : "; python tools/prof_kernel.py $s 10
done
for tr in 2 1 0; do for s in "2 1024 1024 0" "2 512 512 0" "2 2048 2048 0"; do
  echo -n "trsm=$tr kind/shape=$s : "; STF_TRSM=$tr python tools/prof_kernel.py $s 5
done; done
for c in 8 16 32; do for s in "3 1024 1024 0" "3 512 512 0" "3 2048 2048 0"; do
  echo -n "potrf dataflow ctas=$c kind/shape=$s : "; STF_DF_CTAS=$c python tools/prof_kernel.py $s 5
done; done
for bk in 16 32; do for w in 16 8; do
  echo -n "gemm bk=$bk warps=$w 8192x8192x1024: "; STF_GEMM_BK=$bk STF_GEMM_WARPS=$w python tools/prof_kernel.py 0 8192 8192 1024 10
  echo -n "gemm bk=$bk warps=$w 1024^3: "; STF_GEMM_BK=$bk STF_GEMM_WARPS=$w python tools/prof_kernel.py 0 1024 1024 1024 10
done; done
