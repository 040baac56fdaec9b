#!/bin/bash
# Non-critical TRSM variants in the whole factorisation (bench.py, device time), n = 32768 and 65536.
for n in 32768 65536; do
  for v in "" "STF_TRSM_RES_TAIL=1000000" "STF_TRSM_SPLIT=2" "STF_TRSM_SPLIT=8" "STF_TRSM_RES_SPLIT=1"; do
    r=$(env $v python bench.py --n $n --steps 3 --warmup 2 --no-e2e --no-cpu --no-check 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print(d['value'], d['ms_per_step'])")
    echo "n=$n ${v:-default} -> $r"
  done
done
