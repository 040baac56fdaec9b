timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k "potrf" 2>&1 | tail -2
timeout 600 python -m pytest tests/test_gpu_potrf.py -x -q -k "bit or pin or p1 or p2 or p3 or exact" 2>&1 | tail -2
python tools/potrf_trace.py 1024 | head -6
for s in "3 1024 1024 0" "3 512 512 0" "3 256 256 0"; do echo -n "potrf $s: "; python tools/prof_kernel.py $s 10; done
for cfg in "8192 1024" "8192 512" "1024 256"; do set -- $cfg
  timeout 300 python bench.py --order $1 --tile $2 --steps 4 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$1 $2', d['value'], d['ms_per_step'])"
done
