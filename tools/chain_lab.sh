#!/bin/bash
# Critical-chain diagnostics (run under gpurun): FP64 op latencies, the P(kb) lab,
# the POTRF / TRSM tile timelines and the chain kernels alone.
mkdir -p gpurun_out
{
echo "== fp64_latency"; ./tools/fp64_latency
echo "== dmma_latency"; ./tools/dmma_latency
echo "== p_lab"; ./tools/p_lab
echo "== chol_lab"; timeout 120 ./tools/chol_lab
echo "== potrf_trace 1024"; timeout 120 python tools/potrf_trace.py 1024
echo "== trsm_trace 1024 1024"; timeout 120 python tools/trsm_trace.py 1024 1024
echo "== kbench 1024 (kernels only)"; KB_FULL=0 timeout 300 python tools/kbench.py 1024
} > gpurun_out/chain_lab.txt 2>&1
tail -60 gpurun_out/chain_lab.txt
