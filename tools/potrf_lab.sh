#!/bin/bash
# POTRF tile iteration (run under gpurun): reciprocal check, P lab, tile timeline, chain kernels, parity.
mkdir -p gpurun_out
{
echo "== check_rcp"; timeout 120 ./tools/check_rcp
echo "== p_lab"; timeout 60 ./tools/p_lab
echo "== potrf_trace 1024"; timeout 120 python tools/potrf_trace.py 1024 | head -22
echo "== kbench (kernels)"; KB_FULL=0 timeout 300 python tools/kbench.py 1024
echo "== chain_bench"; timeout 300 python tools/chain_bench.py 1024
echo "== pytest potrf kernels + P2"; timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_potrf.py -m gpu -x -q 2>&1 | tail -4
} > gpurun_out/potrf_lab.txt 2>&1
cat gpurun_out/potrf_lab.txt
