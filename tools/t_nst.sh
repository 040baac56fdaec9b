timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k "trsm" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_potrf.py -x -q 2>&1 | tail -1
for s in "2 1024 256 0" "2 1024 1024 0" "2 16384 1024 0"; do echo -n "rowpanel $s: "; STF_TRSM=2 python tools/prof_kernel.py $s 10; done
for cfg in "32768 1024" "8192 1024" "8192 512"; do set -- $cfg
  timeout 300 python bench.py --order $1 --tile $2 --steps 4 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$1 $2', d['value'], d['ms_per_step'])"
done
