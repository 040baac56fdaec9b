#!/bin/bash
# Branch-free pivot sqrt/reciprocal, heavy+light POTRF launches (run under gpurun).
mkdir -p gpurun_out
{
echo "== serialised launches: ncu on the POTRF tile (must not hang)"
timeout 300 ncu --metrics gpu__time_duration.sum -k regex:"dataflow|bulk" -c 4 python tools/prof_kernel.py 3 1024 1024 0 1 2>&1 | grep -E "dataflow|bulk|gpu__time|rc " | head -12; echo "ncu rc=$?"
echo "== CUDA_LAUNCH_BLOCKING=1, eager: potrf tests"
CUDA_LAUNCH_BLOCKING=1 STF_GRAPH=0 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -k "potrf" 2>&1 | tail -2
echo "== check_rcp"; timeout 300 ./tools/check_rcp
echo "== p_lab"; timeout 60 ./tools/p_lab
echo "== potrf_trace 1024"; timeout 120 python tools/potrf_trace.py 1024 2>&1 | head -20
echo "== kbench (kernels)"; KB_FULL=0 timeout 300 python tools/kbench.py 1024
echo "== chain_bench"; timeout 300 python tools/chain_bench.py 1024 512 | grep -E '"lead": (0|8)'
echo "== fact_sweep"; timeout 900 python tools/fact_sweep.py "8192:1024,8192:512,16384:1024,32768:1024" "base=pdl=1" 3
echo "== GPU tests"; timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
} > gpurun_out/pivot_lab.txt 2>&1
cat gpurun_out/pivot_lab.txt
