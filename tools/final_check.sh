#!/bin/bash
# Round-end evidence at HEAD (under gpurun): sanitizers on smoke(), the 8-process bench on virtual
# slots, ncu summaries of the tile kernels, kernels alone / small configs, GPU tests, default bench.
mkdir -p gpurun_out
timeout 600 compute-sanitizer --tool memcheck --leak-check no python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_memcheck.txt 2>&1; tail -1 gpurun_out/sanitize_memcheck.txt
timeout 600 compute-sanitizer --tool synccheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_synccheck.txt 2>&1; tail -1 gpurun_out/sanitize_synccheck.txt
timeout 900 compute-sanitizer --tool racecheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_racecheck.txt 2>&1; tail -1 gpurun_out/sanitize_racecheck.txt
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node=8 --master-addr 127.0.0.1 --master-port 29801 \
  bench.py --gpus 8 --virtual-slots 1 --order 16384 --tile 1024 --steps 3 --warmup 2 --no-e2e --no-cpu \
  > gpurun_out/bench_mp8_virtual.json 2> gpurun_out/bench_mp8_virtual.err; echo "mp8 rc=$?"; cut -c1-300 gpurun_out/bench_mp8_virtual.json
python tools/kbench.py 1024 > gpurun_out/kbench.txt 2>&1; cat gpurun_out/kbench.txt
bash tools/prof_round.sh > gpurun_out/prof_round.log 2>&1; tail -3 gpurun_out/prof_round.log
bash tools/round_check.sh
