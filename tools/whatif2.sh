for sk in none potrf trsm trsm_as_half_gemm "potrf,trsm"; do
  if [ "$sk" = none ]; then unset STF_DEBUG_SKIP; else export STF_DEBUG_SKIP=$sk; fi
  for cfg in "32768 1024" "8192 1024"; do set -- $cfg
  v=$(timeout 300 python bench.py --order $1 --tile $2 --steps 4 --warmup 3 --no-e2e --no-cpu 2>/dev/null | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])")
  echo "n=$1 nb=$2 skip=$sk -> $v"
  done
done
