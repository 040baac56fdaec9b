timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for cfg in "8192 1024" "8192 512" "8192 256" "1024 256"; do set -- $cfg
  timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --e2e-steps 3 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$1 $2', d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
done > gpurun_out/small_cfgs.log 2>&1
