#!/bin/bash
# A/B: library build in ab/libstf_old.so against the in-tree one, interleaved runs.
for c in "8192 1024" "8192 512" "32768 1024"; do
  set -- $c
  for rep in 1 2; do
    for lib in ab/libstf_old.so ""; do
      v=$(STF_LIB_PATH=$lib timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-e2e --no-cpu 2>/dev/null | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])")
      echo "n=$1 nb=$2 ${lib:-new} $v"
    done
  done
done
