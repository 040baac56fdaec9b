for cfg in "8192 256" "8192 512" "16384 512" "16384 1024"; do set -- $cfg
  timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --e2e-steps 3 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$1 $2', d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
done > gpurun_out/small_cfgs2.log 2>&1
STF_HOST_GRAPH=1 timeout 300 python bench.py --order 8192 --tile 512 --steps 5 --warmup 3 --no-cpu --e2e-steps 3 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('graph 8192 512', d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])" >> gpurun_out/small_cfgs2.log 2>&1
