#!/bin/bash
mkdir -p gpurun_out
{
echo "== potrf_trace 1024"; timeout 120 python tools/potrf_trace.py 1024 2>&1 | head -20
echo "== kbench (kernels)"; KB_FULL=0 timeout 300 python tools/kbench.py 1024
echo "== chain_bench"; timeout 300 python tools/chain_bench.py 1024 | tail -3
echo "== pytest potrf kernels"; timeout 900 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -k "potrf" 2>&1 | tail -2
echo "== pytest P2 potrf"; timeout 900 python -m pytest tests/test_gpu_potrf.py -m gpu -x -q 2>&1 | tail -2
} > gpurun_out/potrf_quick.txt 2>&1
cat gpurun_out/potrf_quick.txt
