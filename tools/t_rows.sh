#!/bin/bash
# 128-row TRSM panel: tests, panel throughput/latency, bench with 64 vs 128 rows; e2e with the new load order
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_kernels.py -x -q -k "trsm" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_potrf.py -x -q -k "rows_same_bits or trsm_variants" 2>&1 | tail -2
for r in 64 128; do for s in "2 1024 256 0" "2 37888 256 0" "2 37888 1024 0"; do
  echo -n "rows=$r $s: "; STF_TRSM=2 STF_TRSM_ROWS=$r python tools/prof_kernel.py $s 10; done; done
for r in 64 128 64 128; do
  echo -n "bench rows=$r: "; STF_TRSM_ROWS=$r timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"
done
bash tools/e2e_check.sh
