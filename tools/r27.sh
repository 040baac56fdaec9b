b() { timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --no-e2e | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; }
for rep in 1 2; do
for v in "0 0" "2 8" "2 16" "2 12"; do set -- $v
  echo -n "n=32768 mode=$1 tail=$2: "; STF_ORDER_MODE=$1 STF_ORDER_TAIL=$2 b 32768 1024
done; done
for v in "0 0" "2 16"; do set -- $v; echo -n "n=65536 mode=$1 tail=$2: "; STF_ORDER_MODE=$1 STF_ORDER_TAIL=$2 timeout 600 python bench.py --order 65536 --tile 1024 --steps 2 --warmup 3 --no-cpu --no-e2e | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; done
