#!/bin/bash
# gemm_merge distance D x gemm_group G in the whole factorisation (bench.py with its on-box P2 check)
for n in 65536 32768; do
  for dg in "0 2" "2 2" "1 3" "2 3" "1 4" "2 4" "3 4"; do
    set -- $dg
    r=$(STF_GEMM_MERGE=$1 STF_GEMM_GROUP=$2 python bench.py --n $n --steps 3 --warmup 2 --no-e2e --no-cpu 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['check']['bit_exact'], d['plan']['merged_gemms'], d['plan']['tasks'])")
    echo "n=$n gemm_merge=$1 gemm_group=$2 -> $r"
  done
done
