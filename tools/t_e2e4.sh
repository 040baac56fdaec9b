#!/bin/bash
p() { timeout 300 python tools/e2e_probe.py 32768 1024 2; }
TAG=base p
TAG=store_early STF_STORE_EARLY=1 p
TAG=store_early+lazy+col STF_STORE_EARLY=1 STF_LOAD_ORDER=2 STF_COL_UPDATES=1 p
TAG=asap STF_ORDER_ASAP=1 p
TAG=asap+store_early+lazy STF_ORDER_ASAP=1 STF_STORE_EARLY=1 STF_LOAD_ORDER=2 p
STF_ORDER_ASAP=1 timeout 300 python tools/timeline.py 32768 1024 host 40 | grep -v "^TRSM\|^SYRK"
for a in 1 0 1; do echo -n "device asap=$a: "; STF_ORDER_ASAP=$a timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; done
for a in 1 0; do echo -n "device 8192 asap=$a: "; STF_ORDER_ASAP=$a timeout 300 python bench.py --order 8192 --tile 512 --steps 5 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; done
