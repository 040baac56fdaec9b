for t in 1 2; do
  echo "== TPC=$t"
  STF_GEMM_TPC=$t timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k gemm 2>&1 | tail -1
  for s in "0 8192 8192 1024" "0 1024 1024 1024" "0 8192 8192 2048"; do echo -n "  gemm $s: "; STF_GEMM_TPC=$t python tools/prof_kernel.py $s 5; done
done
for t in 2 1 2 1; do echo -n "bench TPC=$t: "; STF_GEMM_TPC=$t timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; done
STF_GEMM_TPC=2 timeout 600 python -m pytest tests/test_gpu_potrf.py -x -q 2>&1 | tail -1
