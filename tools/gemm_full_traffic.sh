#!/bin/bash
# DRAM traffic and time of the 8192^2 x 1024 GEMM kernel alone (bench's gemm_full) under ncu.
mkdir -p gpurun_out
cat > /tmp/gf.py <<'PY'
import ctypes, sys, os
sys.path.insert(0, os.getcwd())
from paper_conf_sc_augonnetasg24_b200 import _abi
ms = ctypes.c_double()
assert _abi.stf_bench_kernel(0, 8192, 8192, 1024, 3, ctypes.byref(ms)) == 0
print("gemm_full alone %.4f ms, %.2f TFLOP/s" % (ms.value, 2 * 8192 * 8192 * 1024 / ms.value / 1e9))
PY
python /tmp/gf.py
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum --clock-control none \
    -k regex:gemm_nt_dmma --launch-skip 1 --launch-count 1 python /tmp/gf.py 2>&1 | grep -E "dram__|gpu__time|lts__t_bytes|gemm_nt"
