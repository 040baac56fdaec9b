#!/bin/bash
# gemm_merge distance D in the whole factorisation (bench.py with its on-box P2 check)
for n in 32768 65536; do
  for d in 0 1 2 3 5; do
    r=$(STF_GEMM_MERGE=$d python bench.py --n $n --steps 3 --warmup 2 --no-e2e --no-cpu 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['check']['bit_exact'], d['plan']['merged_gemms'], d['plan']['tasks'])")
    echo "n=$n gemm_merge=$d -> $r"
  done
done
