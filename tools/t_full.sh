timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
timeout 500 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -2 gpurun_out/bench.err; python -c "import json; d=json.load(open('gpurun_out/bench.json')); print(d['value'], d['roofline']['frac'], d['roofline']['traffic'], d['e2e']['value'], d['cpu_baseline']['value'], d['clocks'])"
for cfg in "8192 1024" "8192 512" "8192 256" "1024 256" "65536 1024"; do set -- $cfg
  timeout 300 python bench.py --order $1 --tile $2 --steps 3 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$1 $2', d['value'], d['ms_per_step'])"
done
