#!/bin/bash
# e2e (HOST_COLMAJOR) vs device-resident at the bench size, plus the small configs
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/bench_e2e.json 2> gpurun_out/bench_e2e.err
python - <<'PY'
import json
d = json.load(open("gpurun_out/bench_e2e.json"))
print("value", d["value"], "ms", d["ms_per_step"], "e2e", d["e2e"]["value"], d["e2e"]["ms_per_step"])
PY
for cfg in "8192 1024" "8192 512" "8192 256" "1024 256"; do set -- $cfg
  timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --e2e-steps 3 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$1 $2', d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
done
