#!/bin/bash
for v in "0 0" "2 1" "2 0" "0 1"; do set -- $v
  TAG="load_order=$1 col_updates=$2" STF_LOAD_ORDER=$1 STF_COL_UPDATES=$2 timeout 300 python tools/e2e_probe.py 32768 1024 2
done
STF_LOAD_ORDER=2 STF_COL_UPDATES=1 timeout 300 python tools/timeline.py 32768 1024 host 40 | grep -v "^TRSM\|^SYRK"
for c in 0 1 0 1; do echo -n "device col_updates=$c: "; STF_COL_UPDATES=$c timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; done
