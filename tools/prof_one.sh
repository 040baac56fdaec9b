#!/bin/bash
# usage: tools/prof_one.sh NAME REGEX KIND M N K  -> gpurun_out/prof_NAME.ncu-rep (ncu --set full, one warm launch)
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$2 -s 1 -c 1 -f \
  -o gpurun_out/prof_$1 python tools/prof_kernel.py $3 $4 $5 $6 1 > gpurun_out/prof_$1.log 2>&1
echo "$1 rc=$?"
