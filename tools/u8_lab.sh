#!/bin/bash
# Fast U on all warps + TRSM split sweep at small n (run under gpurun).
mkdir -p gpurun_out
{
echo "== potrf_trace 1024"; timeout 120 python tools/potrf_trace.py 1024 2>&1 | head -20
echo "== kbench (kernels)"; KB_FULL=0 timeout 300 python tools/kbench.py 1024
echo "== chain_bench"; timeout 300 python tools/chain_bench.py 1024 | grep -E '"lead": (0|8)'
echo "== fact_sweep"; timeout 900 python tools/fact_sweep.py "8192:1024,16384:1024,32768:1024" "base=pdl=1;split8=trsm_split=8;split2=trsm_split=2;rows64=trsm_rows=64;whatif_trsm_half_gemm=debug_skip=131072" 3
echo "== GPU tests"; timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
} > gpurun_out/u8_lab.txt 2>&1
cat gpurun_out/u8_lab.txt
