#!/bin/bash
# PDL chain lab (run under gpurun): chain step alone, full factorisations, parity with pdl=1.
mkdir -p gpurun_out
{
echo "== chain_bench"; timeout 300 python tools/chain_bench.py 1024 512
echo "== fact_sweep"; timeout 600 python tools/fact_sweep.py "8192:1024,8192:512,16384:1024,32768:1024" "base=pdl=0;pdl4=pdl=1,pdl_lead=4;pdl6=pdl=1,pdl_lead=6;pdl10=pdl=1,pdl_lead=10" 3
echo "== pytest STF_PDL=1"; STF_PDL=1 timeout 900 python -m pytest tests/test_gpu_potrf.py tests/test_gpu_fullsize.py tests/test_gpu_kernels.py -m gpu -x -q 2>&1 | tail -5
} > gpurun_out/pdl_lab.txt 2>&1
cat gpurun_out/pdl_lab.txt
