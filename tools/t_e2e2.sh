#!/bin/bash
./tools/h2d_bw 32768 1024 | grep -i "busy\|streams=1"
TAG=graph STF_GRAPH=1 timeout 300 python tools/e2e_probe.py 32768 1024 2
TAG=eager STF_GRAPH=0 timeout 300 python tools/e2e_probe.py 32768 1024 2
TAG=eager_copyonly STF_GRAPH=0 STF_DEBUG_SKIP=potrf,trsm,syrk,gemm timeout 300 python tools/e2e_probe.py 32768 1024 2
