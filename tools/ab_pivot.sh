#!/bin/bash
# A/B of the POTRF chain's pivot forms in one call (STF_DF_DBG: 1 library sqrt/1-over-x in P, 2 S warps' own reciprocals)
mkdir -p gpurun_out
{
for rep in 1 2; do
for dbg in 0 1 2 3; do
  echo "== STF_DF_DBG=$dbg rep $rep"
  STF_DF_DBG=$dbg KB_FULL=0 timeout 300 python tools/kbench.py 1024 | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('potrf_tile us', d['potrf_tile']['us'])"
  STF_DF_DBG=$dbg timeout 120 python tools/potrf_trace.py 1024 2>&1 | sed -n 2p
done
done
for dbg in 0 3; do echo "== fact STF_DF_DBG=$dbg"; STF_DF_DBG=$dbg timeout 600 python tools/fact_sweep.py "8192:1024,16384:1024" "base=pdl=1" 3; done
} > gpurun_out/ab_pivot.txt 2>&1
cat gpurun_out/ab_pivot.txt
