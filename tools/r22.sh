STF_ORDER_MODE=2 timeout 300 python tools/timeline.py 8192 1024 dev 20 | grep "^k=\|device"
b() { timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --no-e2e | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; }
for cfg in "8192 1024" "8192 512" "8192 256" "16384 1024" "32768 1024"; do set -- $cfg
  for m in 0 2; do echo -n "mode=$m n=$1 nb=$2: "; STF_ORDER_MODE=$m b $1 $2; done
done
for w in 2 4 6; do echo -n "mode=2 width=$w n=8192 nb=1024: "; STF_ORDER_MODE=2 STF_SCHED_WIDTH=$w b 8192 1024; done
echo -n "mode=2 width=4 n=32768: "; STF_ORDER_MODE=2 STF_SCHED_WIDTH=4 b 32768 1024
