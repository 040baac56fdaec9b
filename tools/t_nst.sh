timeout 300 python -m pytest tests/test_gpu_kernels.py -x -q -k "trsm" 2>&1 | tail -1
STF_TRSM_DBG=0 timeout 60 python tools/trsm_trace.py 1024 1024 | tail -3
echo -n "kernel 1024x1024: "; timeout 60 python tools/prof_kernel.py 2 1024 1024 0 10
echo -n "kernel 16384x1024: "; timeout 60 python tools/prof_kernel.py 2 16384 1024 0 10
for R in 4 8 16 64; do
for cfg in "32768 1024" "8192 1024" "8192 512" "8192 256" "16384 512" "16384 1024"; do set -- $cfg
  STF_TRSM_RES_TAIL=$R timeout 300 python bench.py --order $1 --tile $2 --steps 4 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('R=$R $1 $2', d['value'], d['ms_per_step'])"
done; done
