#!/bin/bash
# A/B: library builds under ab/ against the in-tree one, interleaved runs.
# usage: tools/ab.sh "8192 1024;32768 1024" ab/libstf_old.so [ab/libstf_x.so ...]
cfgs=${1:-"8192 1024;8192 512;32768 1024"}; shift
libs="$@ in-tree"
IFS=';' read -ra C <<< "$cfgs"
for c in "${C[@]}"; do
  set -- $c
  for rep in 1 2; do
    for lib in $libs; do
      L=$lib; [ "$lib" = in-tree ] && L=""
      v=$(STF_LIB_PATH=$L timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-e2e --no-cpu 2>/dev/null | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])")
      echo "n=$1 nb=$2 $lib $v"
    done
  done
done
