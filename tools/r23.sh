p() { timeout 300 python tools/e2e_probe.py $1 $2 2; }
TAG="e2e asap" p 32768 1024
TAG="e2e list" STF_ORDER_MODE=2 STF_ORDER_ASAP=0 p 32768 1024
TAG="e2e list+graph" STF_HOST_GRAPH=1 STF_ORDER_MODE=2 STF_ORDER_ASAP=0 p 32768 1024
TAG="e2e asap" p 8192 1024
TAG="e2e list" STF_ORDER_MODE=2 STF_ORDER_ASAP=0 p 8192 1024
TAG="e2e prog" p 8192 512
TAG="e2e list graph" STF_ORDER_MODE=2 p 8192 512
b() { timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --no-e2e | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; }
for cfg in "8192 1024" "8192 512" "8192 256" "32768 1024"; do set -- $cfg; echo -n "default n=$1 nb=$2: "; b $1 $2; done
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
