p() { timeout 300 python tools/e2e_probe.py $1 $2 2; }
TAG="e2e list(new model)" p 32768 1024
TAG="e2e list(new model)" p 16384 512
TAG="e2e list(new model)" p 8192 512
TAG="e2e prog" STF_ORDER_MODE=0 p 16384 512
b() { timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --no-e2e | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; }
for cfg in "8192 1024" "8192 512" "16384 1024" "16384 512" "32768 1024"; do set -- $cfg; echo -n "device n=$1 nb=$2: "; b $1 $2; done
