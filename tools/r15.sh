for cfg in "8192 256" "8192 512" "8192 1024" "16384 512" "16384 1024"; do set -- $cfg
  timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --e2e-steps 3 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$1 $2', d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
done > gpurun_out/small_cfgs3.log 2>&1
timeout 900 python bench.py --order 65536 --tile 1024 --steps 2 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/bench_65536.json 2>gpurun_out/bench_65536.err
timeout 600 python bench.py --virtual-slots 1 --gpus 8 --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_virtual24.json 2>gpurun_out/bench_virtual24.err
