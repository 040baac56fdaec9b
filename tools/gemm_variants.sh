#!/bin/bash
# GEMM tile-kernel variants: alone (8192^2 x 1024, 1024^3) and in the whole factorisation (n = 32768, 65536).
for v in "STF_GEMM_NARROW=2" "STF_GEMM_NARROW=1" "STF_GEMM_NARROW=0"; do
  env $v KB_FULL=0 python tools/kbench.py 1024 | head -1
  env $v python tools/prof_kernel.py 0 8192 8192 1024 5
  for n in 32768 65536; do
    r=$(env $v python bench.py --n $n --steps 3 --warmup 2 --no-e2e --no-cpu --no-check 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print(d['value'], d['ms_per_step'])")
    echo "$v n=$n -> $r"
  done
done
