timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
python -c "import json; d=json.load(open('gpurun_out/bench_default.json')); print('bench', d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
for cfg in "8192 1024" "8192 512" "8192 256" "16384 1024" "16384 512" "1024 256"; do set -- $cfg
  timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --e2e-steps 3 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$1 $2', d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
done
