#!/bin/bash
# quick loop: kernel tests, TRSM/POTRF timings, short bench
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x 2>&1 | tail -2
for s in "2 1024 1024 0" "2 512 512 0" "2 2048 2048 0" "3 1024 1024 0"; do echo -n "$s: "; python tools/prof_kernel.py $s 5; done
timeout 400 python bench.py --steps 3 --warmup 2 --no-e2e --no-cpu
