#!/bin/bash
mkdir -p gpurun_out
{
for sp in 1 0; do
echo "== STF_POTRF_SPLIT=$sp"
STF_POTRF_SPLIT=$sp timeout 120 python tools/potrf_trace.py 1024 2>&1 | head -6
STF_POTRF_SPLIT=$sp KB_FULL=0 timeout 300 python tools/kbench.py 1024
STF_POTRF_SPLIT=$sp timeout 300 python tools/chain_bench.py 1024 | grep -E '"lead": (0|8|16)'
STF_POTRF_SPLIT=$sp timeout 600 python tools/fact_sweep.py "8192:1024,8192:512,16384:1024,32768:1024" "base=pdl=1" 3
done
echo "== tests (split)"
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_potrf.py -m gpu -x -q 2>&1 | tail -15
} > gpurun_out/split_lab.txt 2>&1
cat gpurun_out/split_lab.txt
