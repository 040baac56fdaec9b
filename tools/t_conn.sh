#!/bin/bash
# hardware work queues (CUDA_DEVICE_MAX_CONNECTIONS) x bulk streams, n=32768 and the small configs
mkdir -p gpurun_out
b() { timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --no-e2e | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; }
for conn in 8 32; do for st in 8 16 32; do for cfg in "32768 1024" "8192 1024" "8192 512" "8192 256"; do set -- $cfg
  echo -n "conn=$conn streams=$st n=$1 nb=$2: "; CUDA_DEVICE_MAX_CONNECTIONS=$conn STF_STREAMS=$st STF_TRSM_ROWS=128 b $1 $2
done; done; done
