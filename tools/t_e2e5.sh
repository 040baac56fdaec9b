#!/bin/bash
p() { timeout 300 python tools/e2e_probe.py 32768 1024 2; }
for c in 8 32; do for a in 0 1; do for g in 1 0; do
  TAG="conn=$c asap=$a graph=$g" CUDA_DEVICE_MAX_CONNECTIONS=$c STF_ORDER_ASAP=$a STF_GRAPH=$g p
done; done; done
TAG="conn=32 asap=1 graph=0 lazy store_early" CUDA_DEVICE_MAX_CONNECTIONS=32 STF_ORDER_ASAP=1 STF_GRAPH=0 STF_LOAD_ORDER=2 STF_STORE_EARLY=1 p
