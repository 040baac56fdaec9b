./tools/h2d_bw 32768 1024 > gpurun_out/h2d_bw.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
bash tools/t_conn.sh > gpurun_out/t_conn.log 2>&1
