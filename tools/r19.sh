timeout 300 python tools/timeline.py 8192 1024 dev 20 | grep "^k=\|device"
for cfg in "8192 1024" "8192 512" "8192 256" "16384 1024" "32768 1024" "32768 1024"; do set -- $cfg
  timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --no-e2e | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$1 $2', d['value'], d['ms_per_step'])"
done
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
