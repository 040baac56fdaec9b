#!/bin/bash
for sk in none potrf,trsm,syrk,gemm potrf,trsm gemm; do
  STF_DEBUG_SKIP=$sk timeout 300 python tools/e2e_probe.py 32768 1024 2
done
TAG=load_row STF_LOAD_ORDER=1 timeout 300 python tools/e2e_probe.py 32768 1024 2
TAG=same_stream STF_STORE_STREAM=0 STF_DEBUG_SKIP=potrf,trsm,syrk,gemm timeout 300 python tools/e2e_probe.py 32768 1024 2
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('bench', d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
