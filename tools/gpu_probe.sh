set -x
nvidia-smi -L
nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/mc_probe tools/mc_probe.cu -lcuda && /tmp/mc_probe > gpurun_out/mc_probe.txt 2>&1; cat gpurun_out/mc_probe.txt
timeout 600 compute-sanitizer --tool memcheck --leak-check no python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_memcheck.txt 2>&1; echo memcheck rc=$? ; tail -5 gpurun_out/sanitize_memcheck.txt
timeout 900 compute-sanitizer --tool racecheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_racecheck.txt 2>&1; echo racecheck rc=$?; tail -5 gpurun_out/sanitize_racecheck.txt
timeout 600 compute-sanitizer --tool synccheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_synccheck.txt 2>&1; echo synccheck rc=$?; tail -5 gpurun_out/sanitize_synccheck.txt
