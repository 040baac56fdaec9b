#!/bin/bash
# (1) FP64 latencies, (2) e2e load order x store stream, (3) fast division (STF_DIV_EXACT=0) build: pins, kernels, bench
mkdir -p gpurun_out
./tools/fp64_latency
e2e() { python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"; }
for lo in 0 1; do for ss in 0 1; do
  echo -n "load_order=$lo store_own_stream=$ss: "
  STF_LOAD_ORDER=$lo STF_STORE_STREAM=$ss timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 2 | e2e
done; done
kt() { for s in "2 1024 256 0" "2 1024 1024 0" "3 1024 1024 0"; do echo -n "  $1 $s: "; env $2 python tools/prof_kernel.py $s 10; done; }
kt exact "STF_TRSM=2 STF_TRSM_ROWS=128"
kt exact_res "STF_TRSM=3"
STF_NVCC_DEFS="-DSTF_DIV_EXACT=0" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_fast.log 2>&1; echo "fast build rc=$?"
kt fast "STF_TRSM=2 STF_TRSM_ROWS=128"
kt fast_res "STF_TRSM=3"
timeout 1200 python -m pytest tests/test_gpu_potrf.py tests/test_gpu_kernels.py -x -q 2>&1 | tail -3
for r in 64 128; do
  echo -n "fast bench rows=$r: "; STF_TRSM_ROWS=$r timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"
done
for cfg in "8192 1024" "8192 512" "8192 256"; do set -- $cfg
  echo -n "fast $1 $2 rows=128: "; STF_TRSM_ROWS=128 timeout 300 python bench.py --order $1 --tile $2 --steps 5 --warmup 3 --no-cpu --no-e2e | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"
done
