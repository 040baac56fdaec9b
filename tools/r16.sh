timeout 600 python -m pytest tests/test_gpu_potrf.py -x -q -k "early_start or colmajor" > gpurun_out/pytest_host.log 2>&1; tail -2 gpurun_out/pytest_host.log
for k in 256 512 1024 2048 4096; do echo -n "gemm 8192x8192x$k: "; python tools/prof_kernel.py 0 8192 8192 $k 5; done
